# Round-1 sweep of the kernels in the tree: every GPU test, smoke, a bench line per
# workload (cpu_baseline on), launch lists (demangled gsb:: kernels) and one ncu
# --set full capture of each dominant kernel.
mkdir -p gpurun_out/final
O=gpurun_out/final
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > $O/gpu.txt
timeout 2400 python -m pytest tests -m gpu -q -rf > $O/pytest_gpu_all.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
for w in graphsage_pd kgcn_pd pass_pd shadow_pd ladies_lj fastgcn_lj ares_pp deepwalk_fs node2vec_fs; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 > $O/bench_$w.log 2>&1; echo "rc=$?" >> $O/bench_$w.log
done
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_reference_graphsage_pd.log 2>&1
for w in graphsage_pd ladies_lj fastgcn_lj shadow_pd deepwalk_fs; do
  timeout 600 ncu --kernel-name-base demangled -k regex:gsb:: --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $O/launches_$w.csv python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline > $O/b_ncu_$w.log 2>&1
done
for w in graphsage_pd:nodewise_wave pass_pd:nodewise_wave shadow_pd:shadow_induce ladies_lj:layerwise_kernel fastgcn_lj:layerwise_bm ares_pp:nodewise_wave deepwalk_fs:walk_kernel node2vec_fs:walk_kernel kgcn_pd:nodewise_wave; do
  wl=${w%%:*}; k=${w##*:}
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 -o $O/prof_$wl python tools/run_once.py $wl 2 > $O/ncu_$wl.log 2>&1
done
