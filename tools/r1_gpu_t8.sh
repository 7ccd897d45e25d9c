mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_layerwise.py -m gpu -q -x -rf > gpurun_out/pytest_t8.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t8.log
for w in graphsage_pd kgcn_pd shadow_pd; do GS_VERBOSE=1 timeout 600 python bench.py --workload $w --no-cpu-baseline > gpurun_out/bench_t8_$w.log 2>&1; done
