O=gpurun_out/r2i; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_nodewise.py -m gpu -q -x > $O/pytest_nw.log 2>&1; echo "rc=$?" >> $O/pytest_nw.log
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing.log 2>&1
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 --workload kgcn_pd > $O/timing_kgcn.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:hop_select --launch-skip 5 --launch-count 1 -o $O/ncu_sel python bench.py --steps 1 --warmup 3 --no-cpu-baseline > $O/ncu_sel.log 2>&1
