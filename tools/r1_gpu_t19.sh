mkdir -p gpurun_out
export GS_LIB_PATH=$PWD/tools/exp_libs/libM.so
timeout 900 python -m pytest tests/test_gpu_layerwise.py -m gpu -q -x -rf > gpurun_out/pytest_t19.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t19.log
timeout 600 python bench.py --workload ladies_lj --no-cpu-baseline > gpurun_out/bench_t19_ladiesM.log 2>&1
unset GS_LIB_PATH
timeout 600 python bench.py --workload ladies_lj --no-cpu-baseline > gpurun_out/bench_t19_ladies_cur.log 2>&1
