mkdir -p gpurun_out
for rep in 1 2; do
  timeout 300 python bench.py --no-cpu-baseline --steps 20 > gpurun_out/bench_t9_bal_$rep.log 2>&1
  GS_WAVE=64 timeout 300 python bench.py --no-cpu-baseline --steps 20 > gpurun_out/bench_t9_w64_$rep.log 2>&1
done
timeout 600 python bench.py --workload ladies_lj --no-cpu-baseline > gpurun_out/bench_t9_ladies.log 2>&1
timeout 600 python bench.py --workload shadow_pd --no-cpu-baseline > gpurun_out/bench_t9_shadow.log 2>&1
