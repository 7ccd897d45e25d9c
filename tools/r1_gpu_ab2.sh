mkdir -p gpurun_out
for v in A B C new A; do
  if [ $v = new ]; then unset GS_LIB_PATH; else export GS_LIB_PATH=$PWD/tools/exp_libs/lib$v.so; fi
  timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_var$v.log 2>&1
done
export GS_LIB_PATH=$PWD/tools/exp_libs/libC.so
timeout 900 python -m pytest tests/test_gpu_nodewise.py -m gpu -q -x > gpurun_out/pytest_varC.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_varC.log
