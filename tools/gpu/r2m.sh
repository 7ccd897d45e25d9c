O=gpurun_out/r2m; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_saint.py -m gpu -q -x > $O/pytest_nw.log 2>&1; echo "rc=$?" >> $O/pytest_nw.log
GS_HOP_FUSE=1 timeout 600 python -m pytest tests/test_gpu_nodewise.py -m gpu -q -x > $O/pytest_nw_fuse.log 2>&1; echo "rc=$?" >> $O/pytest_nw_fuse.log
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing.log 2>&1
GS_HOP_FUSE=1 GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing_fuse.log 2>&1
GS_SEL_CTAS=3 GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing_c3.log 2>&1
GS_SEL_CTAS=2 GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing_c2.log 2>&1
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 --workload kgcn_pd > $O/timing_kgcn.log 2>&1
timeout 300 python bench.py --no-cpu-baseline > $O/bench.log 2>&1
