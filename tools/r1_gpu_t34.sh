# induce staging stores with L2 evict_last vs the tree (SAINT, ShaDow).
O=gpurun_out/t34; mkdir -p $O
export GS_LIB_PATH=$PWD/tools/exp_libs/libshstage.so
timeout 900 python -m pytest tests/test_gpu_saint.py -m gpu -q -rf -x > $O/pytest_var.log 2>&1; echo "rc=$?" >> $O/pytest_var.log
for w in saint_pd shadow_pd; do timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_var_$w.log 2>&1; done
unset GS_LIB_PATH
for w in saint_pd shadow_pd; do timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_tree_$w.log 2>&1; done
