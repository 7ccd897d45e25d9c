mkdir -p gpurun_out
for lim in 32 64 0; do timeout 120 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum --clock-control none -c 2 --csv ./tools/microbench_l2fetch3 $lim > gpurun_out/mb3_$lim.csv 2>&1; done
