# ncu --set full of the current PinSAGE kernel and the Table-4 operator kernels.
O=gpurun_out/t35; mkdir -p $O
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pinsage_kernel -s 1 -c 1 -o $O/prof_pinsage_pd python tools/run_once.py pinsage_pd 2 > $O/ncu_pinsage.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"col_copy_kernel|map_kernel|col_sum_kernel" -s 3 -c 3 -o $O/prof_ops python tools/ops_bench.py > $O/ncu_ops.log 2>&1
