"""Seeded synthetic workloads shared by the tests, smoke() and bench.py.

This module holds configuration and seeded input generators only — none of
the method's arithmetic.  Both the CUDA path and the oracle consume what it
produces; neither is imported here.

Workload shapes follow BASELINE.json ``configs`` (C1-C5) and the north_star
target (Rastrigin 100k x 2000, 1 GPU).  PSO parameters are the paper's
defaults (omega = 0.9, c1 = c2 = 2); domains are P:L291 (Sphere,
+-5.12), P:L299 (Griewank, +-600), P:L305 (Easom, +-2pi) and the standard
[20] domains for Rastrigin (+-5.12), Rosenbrock (+-2.048) and
Ackley (+-32.768).  The velocity bound is the reading-3 default |v| <= 1
unless a config says otherwise.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, replace

import numpy as np

# Objective ids: interface values of include/fastpso.h (PSO_OBJ_*).
SPHERE, RASTRIGIN, ROSENBROCK, GRIEWANK, ACKLEY, EASOM = 1, 2, 3, 4, 5, 6
OBJ_NAMES = {SPHERE: "sphere", RASTRIGIN: "rastrigin", ROSENBROCK: "rosenbrock",
             GRIEWANK: "griewank", ACKLEY: "ackley", EASOM: "easom"}
DOMAINS = {
    SPHERE: (-5.12, 5.12),
    RASTRIGIN: (-5.12, 5.12),
    ROSENBROCK: (-2.048, 2.048),
    GRIEWANK: (-600.0, 600.0),
    ACKLEY: (-32.768, 32.768),
    EASOM: (-2.0 * math.pi, 2.0 * math.pi),
}

PAPER_W, PAPER_C1, PAPER_C2 = 0.9, 2.0, 2.0
DEFAULT_SEED = 2021


@dataclass(frozen=True)
class Workload:
    name: str
    objective: int
    n: int
    d: int
    iters: int
    gpus: tuple = (1,)
    w: float = PAPER_W
    c1: float = PAPER_C1
    c2: float = PAPER_C2
    seed: int = DEFAULT_SEED
    vmax: float = 0.0  # 0 -> library default 1.0 (reading 3)

    @property
    def lo(self) -> float:
        return DOMAINS[self.objective][0]

    @property
    def hi(self) -> float:
        return DOMAINS[self.objective][1]

    @property
    def elements(self) -> int:
        return self.n * self.d

    def with_(self, **kw) -> "Workload":
        return replace(self, **kw)


WORKLOADS = {
    # BASELINE.json configs[0..4]
    "C1": Workload("C1-sphere-32x10", SPHERE, 32, 10, 100),
    "C2": Workload("C2-rastrigin-1024x1000", RASTRIGIN, 1024, 1000, 1000),
    "C3": Workload("C3-rosenbrock-10000x1000", ROSENBROCK, 10_000, 1000, 1000),
    "C4": Workload("C4-griewank-100000x2000", GRIEWANK, 100_000, 2000, 500, gpus=(1, 2, 4, 8)),
    "C5": Workload("C5-ackley-1000000x4096", ACKLEY, 1_000_000, 4096, 200, gpus=(8,)),
    # north_star target: >= 70% of HBM bandwidth on Rastrigin 100k x 2000 at 1 GPU
    "NS": Workload("northstar-rastrigin-100000x2000", RASTRIGIN, 100_000, 2000, 500,
                   gpus=(1, 2, 4, 8)),
    # NEXT-3: rows wider than one CTA (d > 8192), split over a thread-block cluster
    "W64K": Workload("wide-rastrigin-4096x65536", RASTRIGIN, 4096, 65536, 200),
    "W16K": Workload("wide-griewank-16384x16384", GRIEWANK, 16384, 16384, 200),
    # NEXT-3 beyond one cluster's row (d > 65536): the column split on one GPU
    "W256K": Workload("wide-rastrigin-1024x262144", RASTRIGIN, 1024, 262144, 200),
    # one rank's shard of NS at 2 / 4 / 8 GPUs (rows floor(n r / k) ..), to time the
    # per-rank step on one GPU (with PSO_FORCE_EXCHANGE=1: the exchange path too)
    "NS_R2": Workload("northstar-shard-of-2-rastrigin-50000x2000", RASTRIGIN, 50_000, 2000, 500),
    "NS_R4": Workload("northstar-shard-of-4-rastrigin-25000x2000", RASTRIGIN, 25_000, 2000, 500),
    "NS_R8": Workload("northstar-shard-of-8-rastrigin-12500x2000", RASTRIGIN, 12_500, 2000, 500),
    # C5's optional HBM-capacity sweep: n doubled until the state nears ~80 % of
    # the 180 GB of one B200 (12 B per element: X, V, PB; 2.9M x 4096 = 142.5 GB)
    "C5_2M": Workload("C5-ackley-2000000x4096", ACKLEY, 2_000_000, 4096, 200),
    "C5_2900K": Workload("C5-ackley-2900000x4096", ACKLEY, 2_900_000, 4096, 200),
    # reading 3 (vmax = 1) made visible: the survey's C4 velocity bound (vmax = 600, the
    # domain half-width) and the north-star swarm at vmax = 5.12 (its domain half-width)
    "C4_V600": Workload("C4-griewank-100000x2000-vmax600", GRIEWANK, 100_000, 2000, 500, vmax=600.0),
    "NS_V512": Workload("northstar-rastrigin-100000x2000-vmax5.12", RASTRIGIN, 100_000, 2000, 500,
                        vmax=5.12),
    # the paper's own default experiment, for the Table 2 plausibility band
    "PAPER": Workload("paper-default-5000x200", SPHERE, 5000, 200, 2000),
}


def row_range(n: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous particle shard of `rank`: [floor(n r/k), floor(n (r+1)/k))."""
    return (n * rank) // world, (n * (rank + 1)) // world


def random_state(n: int, d: int, lo: float, hi: float, vmax: float, seed: int,
                 pf_mode: str = "inf"):
    """A seeded swarm state to inject through set_state (numpy float32, dense n x d).

    X ~ U[lo, hi], V ~ U[-vmax, vmax], PB ~ U[lo, hi].  pf is +inf ("inf":
    every row improves on the first step), or large finite values drawn
    per row ("rand"), so both branches of the pbest compare are exercised.
    """
    rng = np.random.default_rng(seed)
    X = rng.uniform(lo, hi, size=(n, d)).astype(np.float32)
    V = rng.uniform(-vmax, vmax, size=(n, d)).astype(np.float32)
    PB = rng.uniform(lo, hi, size=(n, d)).astype(np.float32)
    if pf_mode == "inf":
        pf = np.full(n, np.inf, np.float32)
    elif pf_mode == "zero":
        pf = np.zeros(n, np.float32)
    else:
        pf = rng.uniform(0.0, 1.0, size=n).astype(np.float32)
    return X, V, PB, pf


def sample_rows(n: int, k: int, seed: int) -> np.ndarray:
    """Sorted sample of k distinct row indices, always including the first and last row."""
    rng = np.random.default_rng(seed)
    k = min(k, n)
    idx = set(rng.choice(n, size=max(k - 2, 0), replace=False).tolist())
    idx.update({0, n - 1})
    return np.array(sorted(idx), dtype=np.int64)
