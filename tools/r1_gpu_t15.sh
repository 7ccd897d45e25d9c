mkdir -p gpurun_out
for rep in 1 2; do
  GS_LIB_PATH=$PWD/tools/exp_libs/libK.so timeout 300 python bench.py --no-cpu-baseline --steps 20 > gpurun_out/bench_t15_K$rep.log 2>&1
  timeout 300 python bench.py --no-cpu-baseline --steps 20 > gpurun_out/bench_t15_cur$rep.log 2>&1
done
GS_LIB_PATH=$PWD/tools/exp_libs/libK.so timeout 600 python bench.py --workload ares_pp --no-cpu-baseline > gpurun_out/bench_t15_aresK.log 2>&1
