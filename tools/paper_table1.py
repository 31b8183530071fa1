#!/usr/bin/env python
"""The paper's own experiment on one B200, as context for Table 1.

Setup as in P:L285: n = 5000 particles, d = 200, 2000 iterations, w = 0.9,
c1 = c2 = 2, each result the mean of 10 runs; Sphere (+-5.12), Griewank
(+-600) and Easom (+-2 pi).  A "run" is what a user of the library does:
pso_create (swarm initialisation on the device, Alg. 1 lines 1-3) +
pso_step(2000) + pso_get_gbest (fitness, index and the d-float position to
the host), timed on the host around the whole sequence.  The paper's V100
times (Table 1) are printed beside it: other hardware, other implementation --
context, not a target.

    python tools/paper_table1.py > profiles/r02_paper_table1_context.txt
"""
from __future__ import annotations

import math
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import paper_conf_icpp_liuwc21_b200 as fp  # noqa: E402
from synth import EASOM, GRIEWANK, SPHERE  # noqa: E402

PAPER_V100_S = {SPHERE: 0.67, GRIEWANK: 0.66, EASOM: 0.87}  # Table 1, fastpso
NAMES = {SPHERE: "Sphere", GRIEWANK: "Griewank", EASOM: "Easom"}
DOM = {SPHERE: (-5.12, 5.12), GRIEWANK: (-600.0, 600.0), EASOM: (-2 * math.pi, 2 * math.pi)}
N, D, T, RUNS = 5000, 200, 2000, 10


def one_run(obj, seed):
    import torch
    lo, hi = DOM[obj]
    pos = np.empty(D, np.float32)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    s = fp.Swarm(N, D, 0.9, 2.0, 2.0, lo, hi, obj, seed, device=0)
    s.step(T)
    f, i, _ = s.gbest(out=pos)
    dt = time.perf_counter() - t0
    info = s.info()
    s.close()
    return dt, f, info


def main():
    print(f"# The paper's default experiment (P:L285) on one B200: n={N}, d={D}, T={T}, "
          f"w=0.9, c1=c2=2, mean of {RUNS} runs")
    print("# run = pso_create + pso_step(2000) + pso_get_gbest(position), host wall time")
    one_run(SPHERE, 1)  # warm-up: module load, CUDA context, kernel images
    for obj in (SPHERE, GRIEWANK, EASOM):
        times, fits = [], []
        info = None
        for r in range(RUNS):
            dt, f, info = one_run(obj, 2021 + r)
            times.append(dt)
            fits.append(f)
        m = statistics.mean(times)
        path = ["streaming", "cta-resident", "grid-resident", "persistent-streaming"][info["resident"]]
        print(f"{NAMES[obj]:9s} {m * 1e3:8.2f} ms  ({N * D * T / m:.3e} updates/s; path {path}; "
              f"min {min(times) * 1e3:.2f} ms)  mean gbest {statistics.mean(fits):.6g}  |  "
              f"paper, V100: {PAPER_V100_S[obj]:.2f} s ({N * D * T / PAPER_V100_S[obj]:.3e} updates/s)"
              f" -> {PAPER_V100_S[obj] / m:.0f}x")


if __name__ == "__main__":
    main()
