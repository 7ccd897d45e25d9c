mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_fullsize.py -m gpu -q -x > gpurun_out/pytest_wave.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_wave.log
timeout 300 python bench.py --workload shadow_pd --steps 5 --no-cpu-baseline > gpurun_out/bench_shadow.log 2>&1
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_sage.log 2>&1
