mkdir -p gpurun_out
for m in 0 1; do GS_VERBOSE=1 GS_NW_MAP=$m timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_map$m.log 2>&1; done
for c in 37 74 148; do GS_LW_CTAS=$c timeout 600 python bench.py --workload fastgcn_lj --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_fastgcn_ctas$c.log 2>&1; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:layerwise_bm -s 1 -c 1 -o gpurun_out/prof_fastgcn_bm python tools/run_once.py fastgcn_lj 2 > gpurun_out/ncu_fastgcn_bm.log 2>&1
