mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_nodewise.py -m gpu -q -x -rf > gpurun_out/pytest_t6.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t6.log
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k "not walks and not layerwise" > gpurun_out/pytest_t6_full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t6_full.log
for w in ares_pp pass_pd shadow_pd graphsage_pd; do timeout 600 python bench.py --workload $w --no-cpu-baseline > gpurun_out/bench_t6_$w.log 2>&1; done
