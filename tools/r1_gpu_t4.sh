mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_layerwise.py -m gpu -q -x -rf > gpurun_out/pytest_t4.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t4.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k "shadow or layerwise" > gpurun_out/pytest_t4_full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t4_full.log
timeout 600 python bench.py --workload fastgcn_lj --steps 3 --no-cpu-baseline > gpurun_out/bench_t4_fastgcn.log 2>&1
timeout 600 python bench.py --workload shadow_pd --no-cpu-baseline > gpurun_out/bench_t4_shadow.log 2>&1
for v in D; do GS_LIB_PATH=$PWD/tools/exp_libs/lib$v.so; for wv in 32 48 64; do GS_LIB_PATH=$PWD/tools/exp_libs/libD.so GS_WAVE=$wv timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_t4_D$wv.log 2>&1; done; done
