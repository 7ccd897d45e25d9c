mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_layerwise.py -m gpu -q -x -rf > gpurun_out/pytest_t18.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t18.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k "layerwise" > gpurun_out/pytest_t18_full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t18_full.log
timeout 600 python bench.py --workload ladies_lj > gpurun_out/bench_t18_ladies.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:layerwise_kernel -s 1 -c 1 -o gpurun_out/prof_ladies_t18 python tools/run_once.py ladies_lj 2 > gpurun_out/ncu_ladies_t18.log 2>&1
