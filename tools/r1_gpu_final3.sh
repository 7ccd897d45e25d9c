# End-of-round check of the final tree: every GPU test, smoke, the default bench
# line (cpu_baseline on), a bench line per other workload, the reference arm.
O=gpurun_out/final3; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > $O/gpu.txt
timeout 2400 python -m pytest tests -m gpu -q -rf > $O/pytest_gpu_all.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 600 python bench.py > $O/bench_default.log 2>&1; echo "rc=$?" >> $O/bench_default.log
for w in kgcn_pd pass_pd shadow_pd ladies_lj fastgcn_lj ares_pp deepwalk_fs node2vec_fs saint_pd pinsage_pd pass_full_pd; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_$w.log 2>&1; echo "rc=$?" >> $O/bench_$w.log
done
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_reference.log 2>&1
timeout 600 python tools/ops_bench.py > $O/ops_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:walk_kernel -s 1 -c 1 -o $O/prof_node2vec_fs python tools/run_once.py node2vec_fs 2 > $O/ncu_n2v.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pass_att_kernel -s 1 -c 1 -o $O/prof_pass_full_pd python tools/run_once.py pass_full_pd 2 > $O/ncu_pass.log 2>&1
