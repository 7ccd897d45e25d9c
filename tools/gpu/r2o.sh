O=gpurun_out/r2o; mkdir -p $O
for v in "0 -1" "1 -1" "2 -1" "0 100" "1 100"; do set -- $v
if [ "$2" = "-1" ]; then unset GS_SEL_CARVE; else export GS_SEL_CARVE=$2; fi
GS_SEL_LD=$1 GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 > $O/timing_$1_$2.log 2>&1
done
