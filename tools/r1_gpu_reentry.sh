# Re-entry check of the restored tree: every GPU test, smoke, and a bench line per
# workload with the roofline line model (cpu_baseline on for the default workload).
O=gpurun_out/reentry; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > $O/gpu.txt
timeout 2400 python -m pytest tests -m gpu -q -rf > $O/pytest_gpu_all.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 600 python bench.py > $O/bench_default.log 2>&1; echo "rc=$?" >> $O/bench_default.log
for w in kgcn_pd pass_pd shadow_pd ladies_lj fastgcn_lj ares_pp deepwalk_fs node2vec_fs; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_$w.log 2>&1; echo "rc=$?" >> $O/bench_$w.log
done
