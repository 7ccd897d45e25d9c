mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_nodewise.py -m gpu -q -x -rf > gpurun_out/pytest_t14.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t14.log
timeout 1500 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k "not walks and not layerwise" > gpurun_out/pytest_t14_full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t14_full.log
for w in graphsage_pd ares_pp pass_pd kgcn_pd shadow_pd; do timeout 600 python bench.py --workload $w > gpurun_out/bench_t14_$w.log 2>&1; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:walk_kernel -s 1 -c 1 -o gpurun_out/prof_node2vec_idx python tools/run_once.py node2vec_fs 2 > gpurun_out/ncu_n2v_idx.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nodewise_wave -s 1 -c 1 -o gpurun_out/prof_ares_t14 python tools/run_once.py ares_pp 2 > gpurun_out/ncu_ares_t14.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nodewise_wave -s 1 -c 1 -o gpurun_out/prof_gs_t14 python tools/run_once.py graphsage_pd 2 > gpurun_out/ncu_gs_t14.log 2>&1
