O=gpurun_out/r2ae; mkdir -p $O
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:hop_select --launch-skip 2 --launch-count 1 -o $O/ncu_pp_select2 python bench.py --workload ares_pp --steps 1 --warmup 1 --no-cpu-baseline --no-graph > $O/b_ncu.log 2>&1
GS_ARES_FLAT=0 timeout 1500 ncu --set full --import-source on --clock-control none -k regex:hop_select --launch-skip 2 --launch-count 1 -o $O/ncu_pp_select2_f0 python bench.py --workload ares_pp --steps 1 --warmup 1 --no-cpu-baseline --no-graph > $O/b_ncu0.log 2>&1
