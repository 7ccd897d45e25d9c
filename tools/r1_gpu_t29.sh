# Node2Vec interpolation depth sweep (WALK_INTERP = 1 / 3 (tree) / 6 / 12).
O=gpurun_out/t29; mkdir -p $O
for v in interp1 interp6 interp12; do
  GS_LIB_PATH=$PWD/tools/exp_libs/lib$v.so timeout 900 python bench.py --workload node2vec_fs --steps 3 --warmup 3 --no-cpu-baseline > $O/bench_$v.log 2>&1
done
timeout 900 python bench.py --workload node2vec_fs --steps 3 --warmup 3 --no-cpu-baseline > $O/bench_interp3.log 2>&1
