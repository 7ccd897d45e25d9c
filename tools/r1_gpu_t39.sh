# induce knobs: claim granularity 1 / 16 (tree 4), loads in flight 16 (tree 8).
O=gpurun_out/t39; mkdir -p $O
for v in claim1 claim16 ilp16; do
  for w in saint_pd shadow_pd; do
    GS_LIB_PATH=$PWD/tools/exp_libs/lib$v.so timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_${v}_$w.log 2>&1
  done
done
