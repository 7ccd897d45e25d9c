# Round-1 GPU sweep of the current kernels: all GPU tests, smoke, a bench line per
# workload, a launch list per workload and one ncu --set full capture of each dominant kernel.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu_all.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "rc=$?" >> gpurun_out/smoke.log
for w in graphsage_pd kgcn_pd pass_pd shadow_pd ladies_lj fastgcn_lj ares_pp deepwalk_fs node2vec_fs; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 > gpurun_out/bench_$w.log 2>&1; echo "rc=$?" >> gpurun_out/bench_$w.log
done
for w in graphsage_pd ladies_lj deepwalk_fs; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:gsb -c 200 --csv --log-file gpurun_out/launches_$w.csv python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/b_ncu_$w.log 2>&1
done
for w in graphsage_pd:nodewise_wave pass_pd:nodewise_wave shadow_pd:shadow_induce ladies_lj:layerwise_kernel fastgcn_lj:layerwise_kernel ares_pp:nodewise_wave deepwalk_fs:walk_kernel node2vec_fs:walk_kernel; do
  wl=${w%%:*}; k=${w##*:}
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 -o gpurun_out/prof_$wl python tools/run_once.py $wl 2 > gpurun_out/ncu_$wl.log 2>&1
done
