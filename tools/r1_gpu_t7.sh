mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_nodewise.py -m gpu -q -x -rf > gpurun_out/pytest_t7.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t7.log
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k "pass or ares" > gpurun_out/pytest_t7_full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t7_full.log
for w in ares_pp pass_pd graphsage_pd kgcn_pd; do GS_VERBOSE=1 timeout 600 python bench.py --workload $w --no-cpu-baseline > gpurun_out/bench_t7_$w.log 2>&1; done
rm -f gpurun_out/wave_trace.txt*
GS_TRACE=gpurun_out/wave_trace.txt timeout 300 python tools/run_once.py graphsage_pd 3 > gpurun_out/trace_run.log 2>&1
python tools/wave_trace.py gpurun_out/wave_trace.txt > gpurun_out/wave_trace_summary.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nodewise_wave -s 1 -c 1 -o gpurun_out/prof_gs_t7 python tools/run_once.py graphsage_pd 2 > gpurun_out/ncu_gs_t7.log 2>&1
