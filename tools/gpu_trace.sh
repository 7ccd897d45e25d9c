mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_layerwise.py tests/test_gpu_fullsize.py -m gpu -q -k "layerwise or ladies or fastgcn" > gpurun_out/pytest_lw.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_lw.log
for w in ladies_lj fastgcn_lj; do timeout 900 python bench.py --workload $w --steps 5 --no-cpu-baseline > gpurun_out/bench_$w.log 2>&1; done
