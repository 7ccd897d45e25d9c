mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_layerwise.py -m gpu -q -x -rf > gpurun_out/pytest_t3.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t3.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k "not walks and not ares" > gpurun_out/pytest_t3_full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t3_full.log
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_t3_gs.log 2>&1
timeout 600 python bench.py --workload fastgcn_lj --steps 3 --no-cpu-baseline > gpurun_out/bench_t3_fastgcn.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:layerwise_bm -s 1 -c 1 -o gpurun_out/prof_fastgcn_bm2 python tools/run_once.py fastgcn_lj 2 > gpurun_out/ncu_fastgcn_bm2.log 2>&1
