mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_fullsize.py -m gpu -q > gpurun_out/pytest_wave.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_wave.log
GS_VERBOSE=1 timeout 600 python bench.py --workload pass_pd --steps 5 --no-cpu-baseline > gpurun_out/bench_pass_pd.log 2>&1
GS_VERBOSE=1 timeout 600 python bench.py --workload ares_pp --steps 3 --no-cpu-baseline > gpurun_out/bench_ares_pp.log 2>&1
