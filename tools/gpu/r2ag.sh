O=gpurun_out/r2ag; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_pass_full.py tests/test_gpu_ragged_induce.py -x -q -m gpu > $O/pytest.log 2>&1
for f in 1 0; do
GS_ARES_SPLIT=$f GS_HOP_TIMING=1 timeout 900 python bench.py --no-cpu-baseline --steps 3 --workload ares_pp > $O/pp_$f.log 2>&1
done
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 --workload pass_pd > $O/pass.log 2>&1
