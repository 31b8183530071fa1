"""Small runs of every kernel variant, for compute-sanitizer (memcheck/racecheck/synccheck)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_liuwc21_b200 as fp  # noqa: E402
from synth import DOMAINS  # noqa: E402

for kernel in ("reg", "tma"):
    os.environ["PSO_KERNEL"] = kernel
    for obj, n, d in ((2, 40, 1000), (3, 33, 999), (4, 20, 2000), (5, 7, 4096), (1, 5, 13)):
        lo, hi = DOMAINS[obj]
        s = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 7, device=0)
        s.step(3)
        f, i, _ = s.gbest()
        info = s.info()
        print(kernel, obj, n, d, "tma" if info["tma_pipeline"] else "reg", f, i, flush=True)
        s.close()
