O=gpurun_out/r2af; mkdir -p $O
for f in 1 0; do
GS_ARES_SPLIT=$f GS_HOP_TIMING=1 timeout 900 python bench.py --no-cpu-baseline --steps 3 --workload ares_pp > $O/pp_$f.log 2>&1
done
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 --workload pass_pd > $O/pass.log 2>&1
