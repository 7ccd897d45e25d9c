O=gpurun_out/r2q; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_saint.py -m gpu -q -x > $O/pytest_nw.log 2>&1; echo "rc=$?" >> $O/pytest_nw.log
GS_HOP_L2MB=64 timeout 600 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "graphsage or pass_and or shadow or ares" > $O/pytest_full.log 2>&1; echo "rc=$?" >> $O/pytest_full.log
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing.log 2>&1
for mb in 128 64 32; do for ns in 1 2; do
GS_HOP_L2MB=$mb GS_HOP_STREAMS=$ns timeout 300 python bench.py --no-cpu-baseline > $O/bench_${mb}_$ns.log 2>&1
done; done
