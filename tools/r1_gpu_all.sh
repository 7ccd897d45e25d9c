# Round-1 GPU sweep: all GPU tests, a bench line per workload, launch list + ncu of each kernel.
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu_all.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_all.log
for w in graphsage_pd kgcn_pd pass_pd shadow_pd ladies_lj fastgcn_lj ares_pp deepwalk_fs node2vec_fs; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 > gpurun_out/bench_$w.log 2>&1; echo "rc=$?" >> gpurun_out/bench_$w.log
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:gsb -c 200 --csv --log-file gpurun_out/launches_graphsage_pd.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/b_ncu.log 2>&1
for w in ladies_lj fastgcn_lj; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:layerwise_kernel -s 1 -c 1 -o gpurun_out/prof_$w python tools/run_once.py $w 2 > gpurun_out/ncu_$w.log 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:walk_kernel -s 1 -c 1 -o gpurun_out/prof_deepwalk_fs python tools/run_once.py deepwalk_fs 2 > gpurun_out/ncu_deepwalk.log 2>&1
