set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 1500 python -m pytest tests/test_gpu_edge_cases.py tests/test_gpu_multirank.py tests/test_bench_contract.py -m gpu -q -k "not async" 2>&1 | tail -60 > gpurun_out/t1.log
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "iteration_counter or sharing_a_kernel or switch_to_nvlink or exchange_path or nvlink_peer" 2>&1 | tail -30 > gpurun_out/t2.log
cat gpurun_out/t1.log gpurun_out/t2.log | tail -80
