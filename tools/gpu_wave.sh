mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_fullsize.py -m gpu -q -x -k "not shadow" > gpurun_out/pytest_wave.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_wave.log
for wv in 8 16 32 64; do GS_WAVE=$wv timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_wave$wv.log 2>&1; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nodewise_wave -s 1 -c 1 -o gpurun_out/prof_wave python tools/run_once.py graphsage_pd 2 > gpurun_out/ncu_wave.log 2>&1
