# End-of-round sweep of the tree: every GPU test, smoke, a bench line per
# workload (BASELINE.json's + the NEXT-row f1 workloads), the reference arm,
# Table-4 operator bandwidth, and ncu captures of the kernels changed since
# the last sweep (induce with dynamic claims, PinSAGE).
O=gpurun_out/final2; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > $O/gpu.txt
timeout 2400 python -m pytest tests -m gpu -q -rf > $O/pytest_gpu_all.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 600 python bench.py > $O/bench_default.log 2>&1; echo "rc=$?" >> $O/bench_default.log
for w in kgcn_pd pass_pd shadow_pd ladies_lj fastgcn_lj ares_pp deepwalk_fs node2vec_fs saint_pd pinsage_pd; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_$w.log 2>&1; echo "rc=$?" >> $O/bench_$w.log
done
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_reference.log 2>&1
timeout 600 python tools/ops_bench.py > $O/ops_bench.log 2>&1
for w in saint_pd shadow_pd pinsage_pd; do
  timeout 600 ncu --kernel-name-base demangled -k regex:gsb:: --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $O/launches_$w.csv python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline > $O/b_ncu_$w.log 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:shadow_induce -s 1 -c 1 -o $O/prof_saint_pd python tools/run_once.py saint_pd 2 > $O/ncu_saint.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:shadow_induce -s 1 -c 1 -o $O/prof_shadow_pd python tools/run_once.py shadow_pd 2 > $O/ncu_shadow.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pinsage_kernel -s 1 -c 1 -o $O/prof_pinsage_pd python tools/run_once.py pinsage_pd 2 > $O/ncu_pinsage.log 2>&1
