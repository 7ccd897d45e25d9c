mkdir -p gpurun_out
export GS_LIB_PATH=$PWD/tools/exp_libs/libH.so
timeout 900 python -m pytest tests/test_gpu_layerwise.py -m gpu -q -x -rf > gpurun_out/pytest_t12.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t12.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k "layerwise" > gpurun_out/pytest_t12_full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t12_full.log
for rep in 1 2; do timeout 600 python bench.py --workload ladies_lj --no-cpu-baseline > gpurun_out/bench_t12_ladies_H$rep.log 2>&1; done
unset GS_LIB_PATH
timeout 600 python bench.py --workload ladies_lj --no-cpu-baseline > gpurun_out/bench_t12_ladies_cur.log 2>&1
