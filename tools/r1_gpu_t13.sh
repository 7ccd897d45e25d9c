mkdir -p gpurun_out
for rep in 1 2; do
  GS_LIB_PATH=$PWD/tools/exp_libs/libI.so timeout 300 python bench.py --no-cpu-baseline --steps 20 > gpurun_out/bench_t13_gsI$rep.log 2>&1
  timeout 300 python bench.py --no-cpu-baseline --steps 20 > gpurun_out/bench_t13_gscur$rep.log 2>&1
done
GS_LIB_PATH=$PWD/tools/exp_libs/libI.so timeout 600 python bench.py --workload ares_pp --no-cpu-baseline > gpurun_out/bench_t13_aresI.log 2>&1
timeout 600 python bench.py --workload ares_pp --no-cpu-baseline > gpurun_out/bench_t13_arescur.log 2>&1
GS_LIB_PATH=$PWD/tools/exp_libs/libI.so timeout 600 python bench.py --workload shadow_pd --no-cpu-baseline > gpurun_out/bench_t13_shI.log 2>&1
