O=gpurun_out/r2ah; mkdir -p $O
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:"hop_ares_big|hop_select" --launch-skip 4 --launch-count 2 -o $O/ncu_pp_big python bench.py --workload ares_pp --steps 1 --warmup 1 --no-cpu-baseline --no-graph > $O/b_ncu.log 2>&1
