O=gpurun_out/r2j; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_saint.py -m gpu -q -x > $O/pytest_nw.log 2>&1; echo "rc=$?" >> $O/pytest_nw.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "graphsage or pass_and or shadow or ares" > $O/pytest_full.log 2>&1; echo "rc=$?" >> $O/pytest_full.log
GS_VERBOSE=1 GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing.log 2>&1
GS_HOP_FIN=g GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing_g.log 2>&1
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 --workload kgcn_pd > $O/timing_kgcn.log 2>&1
timeout 300 python bench.py --no-cpu-baseline > $O/bench.log 2>&1
