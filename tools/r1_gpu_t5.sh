mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_nodewise.py -m gpu -q -x -rf > gpurun_out/pytest_t5.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t5.log
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k "not walks and not layerwise" > gpurun_out/pytest_t5_full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t5_full.log
for w in graphsage_pd kgcn_pd pass_pd ares_pp; do timeout 600 python bench.py --workload $w --no-cpu-baseline > gpurun_out/bench_t5_$w.log 2>&1; done
GS_LIB_PATH=$PWD/tools/exp_libs/libE.so timeout 600 python bench.py --workload ares_pp --no-cpu-baseline > gpurun_out/bench_t5_ares_E.log 2>&1
GS_LIB_PATH=$PWD/tools/exp_libs/libE.so timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k "ares" > gpurun_out/pytest_t5_E.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t5_E.log
