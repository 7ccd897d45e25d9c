O=gpurun_out/r2w; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_pass_full.py tests/test_gpu_ragged_induce.py -m gpu -q -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "pass_and or ares or shadow" > $O/pytest_full.log 2>&1; echo "rc=$?" >> $O/pytest_full.log
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 --workload pass_pd > $O/timing_pass.log 2>&1
GS_HOP_TIMING=1 timeout 900 python bench.py --no-cpu-baseline --steps 3 --workload ares_pp > $O/timing_pp.log 2>&1
