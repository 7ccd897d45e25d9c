O=gpurun_out/r2f; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_nodewise.py -m gpu -q -x > $O/pytest_nw.log 2>&1; echo "rc=$?" >> $O/pytest_nw.log
timeout 300 python bench.py --no-cpu-baseline > $O/bench.log 2>&1
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing.log 2>&1
for k in hop_select hop_rows hop_relabel; do
timeout 600 ncu --set full --import-source on --clock-control none -k regex:$k --launch-skip 5 --launch-count 1 -o $O/ncu_$k python bench.py --steps 1 --warmup 3 --no-cpu-baseline > $O/ncu_$k.log 2>&1
done
