# Round 2 profile refresh (tools/profile_round.sh) + compute-sanitizer over every kernel path.
exec > gpurun_out/r2prof.log 2>&1
WORKLOADS="C1 C2 C3 C4 NS C5 W16K W64K W256K NS_R8 C4_V600 NS_V512" NCU_WORKLOADS="NS C4 C3 W16K W64K" bash tools/profile_round.sh
bash tools/gpu_sanitize.sh
