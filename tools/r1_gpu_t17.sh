mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_layerwise.py tests/test_gpu_nodewise.py -m gpu -q -x -rf > gpurun_out/pytest_t17.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t17.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k "layerwise or shadow" > gpurun_out/pytest_t17_full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t17_full.log
timeout 600 python bench.py --workload fastgcn_lj > gpurun_out/bench_t17_fastgcn.log 2>&1
timeout 600 python bench.py --workload shadow_pd > gpurun_out/bench_t17_shadow.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:layerwise_bm -s 1 -c 1 -o gpurun_out/prof_fastgcn_t17 python tools/run_once.py fastgcn_lj 2 > gpurun_out/ncu_fg_t17.log 2>&1
