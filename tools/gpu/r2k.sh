O=gpurun_out/r2k; mkdir -p $O
timeout 600 ncu --set full --import-source on --clock-control none -k regex:hop_fin --launch-skip 5 --launch-count 1 -o $O/ncu_fin python bench.py --steps 1 --warmup 3 --no-cpu-baseline > $O/ncu_fin.log 2>&1
