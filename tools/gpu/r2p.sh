O=gpurun_out/r2p; mkdir -p $O
GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing.log 2>&1
GS_SEL_CTAS=2 GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing_c2.log 2>&1
GS_SEL_NQ=1 GS_SEL_CLAIM=4 GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing_q1.log 2>&1
