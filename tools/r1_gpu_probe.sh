# L2 fetch-granularity probe + launch lists (demangled names) + wave-kernel step trace.
mkdir -p gpurun_out
timeout 300 ./tools/microbench_l2fetch > gpurun_out/mb_l2fetch.txt 2>&1
timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none --csv ./tools/microbench_l2fetch > gpurun_out/mb_l2fetch_ncu.csv 2>&1
for w in graphsage_pd ladies_lj deepwalk_fs; do
  timeout 600 ncu --kernel-name-base demangled -k regex:gsb:: --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_$w.csv python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/b_ncu_$w.log 2>&1
done
rm -f gpurun_out/wave_trace.txt*
GS_TRACE=gpurun_out/wave_trace.txt timeout 300 python tools/run_once.py graphsage_pd 3 > gpurun_out/trace_run.log 2>&1
python tools/wave_trace.py gpurun_out/wave_trace.txt > gpurun_out/wave_trace_summary.txt 2>&1
