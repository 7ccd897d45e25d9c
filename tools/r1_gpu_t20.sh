mkdir -p gpurun_out
for w in graphsage_pd deepwalk_fs ladies_lj; do timeout 600 python bench.py --workload $w --no-cpu-baseline --steps 3 > gpurun_out/bench_t20_$w.log 2>&1; done
