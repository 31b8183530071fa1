#!/usr/bin/env python
"""Per-kernel SASS summary of the built library (no GPU needed).

For every kernel in libfastpso.so: registers, local memory (spill) bytes,
static shared memory, and the count of the opcodes that prove the design runs
on the sm_100a data-movement engines -- UBLKCP (cp.async.bulk, the TMA bulk
copy engine), UBLKPF (cp.async.bulk.prefetch.L2), SYNCS (mbarrier
arrive/wait/expect_tx), plus LDG/STG (plain global loads / stores), LDS/STS,
MUFU and IMAD.WIDE (the Philox multiplies).  Writes a fixed-width table.

    python tools/sass_summary.py [lib] > profiles/r02_sass_summary.txt
"""
from __future__ import annotations

import collections
import re
import subprocess
import sys

LIB = sys.argv[1] if len(sys.argv) > 1 else "paper_conf_icpp_liuwc21_b200/libfastpso.so"
OPS = ["UBLKCP", "UBLKPF", "SYNCS", "LDG", "STG", "LDS", "STS", "MUFU", "IMAD.WIDE", "ATOMG", "RED"]


def demangle(names):
    out = subprocess.run(["c++filt"], input="\n".join(names), capture_output=True, text=True).stdout
    return out.splitlines()


def short(name: str) -> str:
    name = re.sub(r"\(anonymous namespace\)::", "", name)
    name = name.replace("fastpso::", "").replace("user::", "")
    name = re.sub(r"\(.*\)$", "", name)
    return name


def main():
    res = subprocess.run(["cuobjdump", "-res-usage", LIB], capture_output=True, text=True).stdout
    usage = {}
    fn = None
    for line in res.splitlines():
        m = re.match(r"\s*Function (\S+):", line)
        if m:
            fn = m.group(1)
            continue
        m = re.search(r"REG:(\d+) STACK:(\d+) SHARED:(\d+) LOCAL:(\d+)", line)
        if m and fn:
            usage[fn] = tuple(int(x) for x in m.groups())
            fn = None
    sass = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True).stdout
    counts = collections.defaultdict(collections.Counter)
    fn = None
    for line in sass.splitlines():
        m = re.match(r"\s*Function : (\S+)", line)
        if m:
            fn = m.group(1)
            continue
        m = re.match(r"\s*/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]*)", line)
        if m and fn:
            op = m.group(1)
            for o in OPS:
                if op == o or op.startswith(o + "."):
                    counts[fn][o] += 1
    names = sorted(set(usage) | set(counts))
    pretty = dict(zip(names, demangle(names)))
    rows = []
    for n in names:
        r, stack, shared, local = usage.get(n, (0, 0, 0, 0))
        c = counts[n]
        rows.append((short(pretty[n]), r, local, stack, shared, *[c[o] for o in OPS]))
    rows.sort()
    hdr = ("kernel", "regs", "spill(local)B", "stackB", "static smemB", *OPS)
    w = max(len(r[0]) for r in rows)
    print(f"# SASS summary of {LIB} (cuobjdump -res-usage / -sass; sm_100a)")
    print(f"# {len(rows)} kernels; spills: {sum(1 for r in rows if r[2])} kernels with local memory")
    print(f"{hdr[0]:<{w}}  " + "  ".join(f"{h:>7}" for h in hdr[1:]))
    for r in rows:
        print(f"{r[0]:<{w}}  " + "  ".join(f"{v:>7}" for v in r[1:]))


if __name__ == "__main__":
    main()
