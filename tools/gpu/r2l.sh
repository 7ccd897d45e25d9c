O=gpurun_out/r2l; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_saint.py -m gpu -q -x > $O/pytest_nw.log 2>&1; echo "rc=$?" >> $O/pytest_nw.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "graphsage or pass_and or shadow or ares" > $O/pytest_full.log 2>&1; echo "rc=$?" >> $O/pytest_full.log
GS_VERBOSE=1 GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing.log 2>&1
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 --workload kgcn_pd > $O/timing_kgcn.log 2>&1
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 --workload pass_pd > $O/timing_pass.log 2>&1
GS_HOP_TIMING=1 timeout 600 python bench.py --no-cpu-baseline --steps 3 --workload ares_pp > $O/timing_pp.log 2>&1
timeout 300 python bench.py --no-cpu-baseline > $O/bench.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:hop_rows --launch-skip 4 --launch-count 1 -o $O/ncu_rows python bench.py --steps 1 --warmup 3 --no-cpu-baseline > $O/ncu_rows.log 2>&1
