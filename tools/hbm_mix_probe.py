#!/usr/bin/env python
"""HBM bandwidth by read:write mix on one B200 (context for roofline.peak).

MEASURED_PEAKS.json's hbm_gbs is a 1:1 copy (b.copy_(a)).  The streaming step
kernel's traffic is read-heavy (NS: 11.6 B read, 8.4 B written per update,
58:42), so it can run above that figure.  This probe times torch kernels of
other mixes over 4 GiB operands (CUDA events, best of 10, warm):
  copy      b.copy_(a)             1 R : 1 W
  add       torch.add(a, b, out=c) 2 R : 1 W
  add3      a + b + c -> d (fused by torch.addcmul(a, b, c, value=1) with out) 3 R : 1 W
  read      torch.amax(a)          read only (a 4-byte result)
  write     a.fill_(1)             write only

    python tools/hbm_mix_probe.py > profiles/r02_hbm_mix_probe.json
"""
import json

import torch


def best_ms(fn, reps=10):
    fn()
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best


def main():
    n = 1 << 30  # fp32 elements: 4 GiB per operand
    a = torch.rand(n, device="cuda")
    b = torch.rand(n, device="cuda")
    c = torch.rand(n, device="cuda")
    d = torch.empty(n, device="cuda")
    B = 4 * n
    cases = {
        "copy_1r1w": (lambda: b.copy_(a), 2 * B, 0.5),
        "add_2r1w": (lambda: torch.add(a, b, out=d), 3 * B, 2 / 3),
        "addcmul_3r1w": (lambda: torch.addcmul(a, b, c, value=1.0, out=d), 4 * B, 0.75),
        "read_only": (lambda: torch.amax(a), B, 1.0),
        "write_only": (lambda: d.fill_(1.0), B, 0.0),
    }
    out = {"gpu": torch.cuda.get_device_name(), "operand_bytes": B, "reps": 10, "cases": {}}
    for k, (fn, nbytes, rfrac) in cases.items():
        ms = best_ms(fn)
        out["cases"][k] = {"read_fraction": round(rfrac, 4), "ms": round(ms, 4),
                           "GBps": round(nbytes / ms / 1e6, 1)}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
