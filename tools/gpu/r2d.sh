O=gpurun_out/r2d; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_saint.py -m gpu -q -x > $O/pytest_nw.log 2>&1; echo "rc=$?" >> $O/pytest_nw.log
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "graphsage or pass_and or shadow or ares" > $O/pytest_full.log 2>&1; echo "rc=$?" >> $O/pytest_full.log
for mb in 64 128; do GS_HOP_L2MB=$mb timeout 600 python bench.py --no-cpu-baseline > $O/bench_hop_l2_$mb.log 2>&1; done
GS_HOP_TIMING=1 GS_HOP_L2MB=128 timeout 600 python bench.py --no-cpu-baseline --steps 3 > $O/timing128.log 2>&1
GS_HOP_TIMING=1 GS_HOP_L2MB=64 timeout 600 python bench.py --no-cpu-baseline --steps 3 > $O/timing64.log 2>&1
GS_HOP_TIMING=1 timeout 600 python bench.py --no-cpu-baseline --steps 3 --workload ares_pp > $O/timing_pp.log 2>&1
