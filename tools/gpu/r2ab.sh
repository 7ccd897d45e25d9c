O=gpurun_out/r2ab; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_pass_full.py tests/test_gpu_uva.py -x -q -m gpu > $O/pytest.log 2>&1
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 --workload pass_pd > $O/pass.log 2>&1
GS_HOP_TIMING=1 timeout 900 python bench.py --no-cpu-baseline --steps 3 --workload ares_pp > $O/pp.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --steps 3 --workload graphsage_pd_uva > $O/uva.log 2>&1
