O=gpurun_out/r2aa; mkdir -p $O
for v in "32 2" "1 4" "1 1"; do set -- $v
GS_SEL_NQ=$1 GS_SEL_CLAIM=$2 GS_HOP_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --steps 3 --workload pass_pd > $O/pass_$1_$2.log 2>&1
done
GS_VERBOSE=1 GS_HOP_TIMING=1 timeout 900 python bench.py --no-cpu-baseline --steps 3 --workload ares_pp > $O/pp_32_2.log 2>&1
GS_SEL_NQ=1 GS_SEL_CLAIM=4 GS_HOP_TIMING=1 timeout 900 python bench.py --no-cpu-baseline --steps 3 --workload ares_pp > $O/pp_1_4.log 2>&1
GS_NODEWISE=wave timeout 900 python bench.py --no-cpu-baseline --steps 3 --workload ares_pp > $O/pp_wave.log 2>&1
