mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_layerwise.py -m gpu -q -x -rf > gpurun_out/pytest_t10.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t10.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k layerwise > gpurun_out/pytest_t10_full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t10_full.log
for w in ladies_lj fastgcn_lj; do timeout 600 python bench.py --workload $w --steps 5 --no-cpu-baseline > gpurun_out/bench_t10_$w.log 2>&1; done
