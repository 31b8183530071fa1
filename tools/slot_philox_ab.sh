# A/B: row-invariant Philox rounds in the 256-thread TMA kernel (PSO_SLOT_PHILOX_NARROW).
exec > gpurun_out/exp2.log 2>&1
echo "== default"; WORKLOADS="C4 NS C4 NS" STEPS=500 bash tools/bench_sweep.sh
make lib -j16 EXTRA=-DPSO_SLOT_PHILOX_NARROW=1 -B > /dev/null 2>&1
grep -A3 "obj_griewank.*k_step_tmaINS_8GriewankELi2ELb0ELi256" paper_conf_icpp_liuwc21_b200/build.log | grep Used
grep -A3 "obj_rastrigin.*k_step_tmaINS_9RastriginELi2ELb0ELi256" paper_conf_icpp_liuwc21_b200/build.log | grep Used
echo "== narrow slot philox"; WORKLOADS="C4 NS C4 NS" STEPS=500 bash tools/bench_sweep.sh
