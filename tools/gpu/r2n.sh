O=gpurun_out/r2n; mkdir -p $O
for v in "32 2" "1 4" "8 4" "32 4" "4 2"; do set -- $v
GS_SEL_NQ=$1 GS_SEL_CLAIM=$2 GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing_$1_$2.log 2>&1
done
GS_SEL_NQ=1 GS_SEL_CLAIM=4 timeout 600 ncu --set full --import-source on --clock-control none -k regex:hop_select --launch-skip 5 --launch-count 1 -o $O/ncu_sel_1 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > $O/ncu_sel.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:hop_select --launch-skip 5 --launch-count 1 -o $O/ncu_sel_32 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > $O/ncu_sel.log 2>&1
