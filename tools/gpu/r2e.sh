O=gpurun_out/r2e; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_saint.py -m gpu -q -x > $O/pytest_nw.log 2>&1; echo "rc=$?" >> $O/pytest_nw.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "graphsage or pass_and or shadow or ares" > $O/pytest_full.log 2>&1; echo "rc=$?" >> $O/pytest_full.log
for mb in 64 128; do GS_HOP_L2MB=$mb timeout 300 python bench.py --no-cpu-baseline > $O/bench_hop_l2_$mb.log 2>&1; done
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing.log 2>&1
GS_VERBOSE=1 GS_HOP_TIMING=1 timeout 600 python bench.py --no-cpu-baseline --steps 3 --workload ares_pp > $O/timing_pp.log 2>&1
for w in kgcn_pd pass_pd; do timeout 300 python bench.py --no-cpu-baseline --workload $w > $O/bench_hop_$w.log 2>&1; done
