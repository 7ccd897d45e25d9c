mkdir -p gpurun_out
timeout 300 ./tools/microbench_l2fetch2 > gpurun_out/mb_l2fetch2.txt 2>&1
timeout 600 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_requests_srcunit_tex_op_read.sum --clock-control none -c 8 --csv ./tools/microbench_l2fetch2 > gpurun_out/mb_l2fetch2_ncu.csv 2>&1
