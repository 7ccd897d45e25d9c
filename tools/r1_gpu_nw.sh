mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_fullsize.py -m gpu -q -x -rf -k "not layerwise and not walks" > gpurun_out/pytest_nw.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_nw.log
for wv in 8 16 32; do GS_WAVE=$wv timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_wave$wv.log 2>&1; done
timeout 300 python bench.py --workload kgcn_pd --no-cpu-baseline > gpurun_out/bench_kgcn.log 2>&1
timeout 300 python bench.py --workload pass_pd --no-cpu-baseline > gpurun_out/bench_pass.log 2>&1
timeout 300 python bench.py --workload shadow_pd --no-cpu-baseline > gpurun_out/bench_shadow.log 2>&1
rm -f gpurun_out/wave_trace.txt*
GS_TRACE=gpurun_out/wave_trace.txt timeout 300 python tools/run_once.py graphsage_pd 3 > gpurun_out/trace_run.log 2>&1
python tools/wave_trace.py gpurun_out/wave_trace.txt > gpurun_out/wave_trace_summary.txt 2>&1
