mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_fullsize.py -m gpu -q -x -k "not shadow" > gpurun_out/pytest_wave.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_wave.log
GS_WAVE=8 GS_TRACE=gpurun_out/wave_trace_8.txt timeout 300 python tools/run_once.py graphsage_pd 1 > gpurun_out/trace_8.log 2>&1
for wv in 4 8 16 32; do GS_WAVE=$wv timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_wave$wv.log 2>&1; done
