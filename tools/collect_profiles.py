"""Copy a tools/profile_round.sh refresh (gpurun_out/prof/) into profiles/ under the round's
names, and rewrite profiles/ncu_traffic.json from the ncu summaries (no GPU needed):
    python tools/collect_profiles.py [--round r02] [--src gpurun_out/prof]"""
import argparse
import json
import os
import re
import shutil
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from synth import WORKLOADS  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--round", default="r02")
ap.add_argument("--src", default=os.path.join(ROOT, "gpurun_out", "prof"))
args = ap.parse_args()
src, dst, rn = args.src, os.path.join(ROOT, "profiles"), args.round


def copy(name, out):
    p = os.path.join(src, name)
    if os.path.exists(p) and os.path.getsize(p) > 0:
        shutil.copyfile(p, os.path.join(dst, out))
        print(f"{name} -> profiles/{out}")


copy("bench_default.json", f"{rn}_bench_default_northstar.json")
copy("bench_reference.json", f"{rn}_bench_reference_oracle.json")
copy("hbm_mix_probe.json", f"{rn}_hbm_mix_probe.json")
copy("launches_northstar.csv", f"{rn}_launches_northstar.csv")
for f in sorted(os.listdir(src)):
    m = re.match(r"sweep_(\w+)\.json$", f)
    if m:
        copy(f, f"{rn}_bench_sweep_{m.group(1)}.json")

traffic = {}
for f in sorted(os.listdir(src)):
    m = re.match(r"ncu_summary_(\w+)\.txt$", f)
    if not m:
        continue
    w = m.group(1)
    txt = open(os.path.join(src, f)).read()
    k = re.search(r"kernel: .*?(k_\w+)<(\w+)", txt)
    kernel = k.group(1) if k else "kernel"
    if kernel == "k_step_tma" and "512>" in txt.splitlines()[0]:
        kernel = "k_step_tma_wide"
    copy(f, f"{rn}_ncu_full_{kernel}_{w}.txt")
    rd = re.search(r"dram__bytes_read\.sum\s+([\d.]+) (\w)byte", txt)
    wr = re.search(r"dram__bytes_write\.sum\s+([\d.]+) (\w)byte", txt)
    scale = {"G": 1e9, "M": 1e6, "K": 1e3}
    if rd and wr and w in WORKLOADS:
        traffic[WORKLOADS[w].name] = int(round(float(rd.group(1)) * scale[rd.group(2)] +
                                               float(wr.group(1)) * scale[wr.group(2)]))
if traffic:
    out = {"_source": f"round {rn[1:]} (final code): ncu --set full --metrics lts__t_bytes.sum,"
                      "lts__t_sector_hit_rate.pct --clock-control none -k regex:'k_step|k_col_step' "
                      f"-s 8 -c 1 (profiles/{rn}_ncu_full_*.txt): dram__bytes_read.sum + "
                      "dram__bytes_write.sum of one step-kernel launch, bytes (early iterations: "
                      "pbest improvement rates differ from a long run)"}
    out.update(traffic)
    with open(os.path.join(dst, "ncu_traffic.json"), "w") as fh:
        json.dump(out, fh, indent=1)
        fh.write("\n")
    print("profiles/ncu_traffic.json:", traffic)
