# Bounds-checked run (compute-sanitizer is closed on this GPU pool): build the library with
# -DPSO_DEVICE_CHECKS (row / tile indices, ring extents against %dynamic_smem_size, global
# offsets; a failed check prints and traps), run every kernel path (tools/sanitize_run.py)
# and the GPU tests of the streaming, cluster and column-split kernels, then rebuild the
# product library.  Output: gpurun_out/devchk/.
mkdir -p gpurun_out/devchk
exec > gpurun_out/devchk/log.txt 2>&1
set -x
make lib -j32 EXTRA=-DPSO_DEVICE_CHECKS -B > gpurun_out/devchk/build.txt 2>&1
echo "traps in the checked build: $(cuobjdump -sass paper_conf_icpp_liuwc21_b200/libfastpso.so | grep -c BPT.TRAP)"
timeout 900 python tools/sanitize_run.py 2>&1 | tail -30
timeout 2400 python -m pytest tests -m gpu -q -k "column or cluster or wide or tma or lazy or edge or multirank or full_size or row_order or slots or persistent" 2>&1 | tail -5
grep -h "PSO_DCHECK" gpurun_out/devchk/log.txt | grep -v "grep" | head -5
make lib -j32 -B > /dev/null 2>&1
echo "traps in the product build: $(cuobjdump -sass paper_conf_icpp_liuwc21_b200/libfastpso.so | grep -c BPT.TRAP)"
