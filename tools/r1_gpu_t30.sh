# PASS SDDMM with L2 policies (projected rows evict_last, streamed arrays evict_first) vs the tree.
O=gpurun_out/t30; mkdir -p $O
export GS_LIB_PATH=$PWD/tools/exp_libs/libpahint.so
timeout 900 python -m pytest tests/test_gpu_pass_full.py -m gpu -q -rf > $O/pytest_pahint.log 2>&1; echo "rc=$?" >> $O/pytest_pahint.log
timeout 900 python bench.py --workload pass_full_pd --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_pahint.log 2>&1
unset GS_LIB_PATH
timeout 900 python bench.py --workload pass_full_pd --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_tree.log 2>&1
