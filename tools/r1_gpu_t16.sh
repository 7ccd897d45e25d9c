mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_nodewise.py -m gpu -q -x -rf -k shadow > gpurun_out/pytest_t16.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t16.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k shadow > gpurun_out/pytest_t16_full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t16_full.log
timeout 600 python bench.py --workload shadow_pd > gpurun_out/bench_t16_shadow.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:shadow_induce -s 1 -c 1 -o gpurun_out/prof_shadow_t16 python tools/run_once.py shadow_pd 2 > gpurun_out/ncu_sh_t16.log 2>&1
