# PinSAGE knobs: 96 KB chunk tables, 4 walks per thread, 1024-thread CTAs (tree: 48 KB, 2, 512).
O=gpurun_out/t40; mkdir -p $O
for v in ps_smem96 ps_ilp4 ps_thr1024; do
  GS_LIB_PATH=$PWD/tools/exp_libs/lib$v.so timeout 600 python -m pytest tests/test_gpu_pinsage.py -m gpu -q -x -k "tiny or medium" > $O/pytest_$v.log 2>&1; echo "rc=$?" >> $O/pytest_$v.log
  GS_LIB_PATH=$PWD/tools/exp_libs/lib$v.so timeout 600 python bench.py --workload pinsage_pd --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_$v.log 2>&1
done
