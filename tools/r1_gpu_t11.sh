mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_walk.py -m gpu -q -x -rf > gpurun_out/pytest_t11.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t11.log
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k walks > gpurun_out/pytest_t11_full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t11_full.log
for w in deepwalk_fs node2vec_fs; do timeout 900 python bench.py --workload $w --steps 3 --no-cpu-baseline > gpurun_out/bench_t11_$w.log 2>&1; done
for v in F G; do
  for rep in 1 2; do GS_LIB_PATH=$PWD/tools/exp_libs/lib$v.so timeout 300 python bench.py --no-cpu-baseline --steps 20 > gpurun_out/bench_t11_$v$rep.log 2>&1; done
done
for rep in 1 2; do timeout 300 python bench.py --no-cpu-baseline --steps 20 > gpurun_out/bench_t11_cur$rep.log 2>&1; done
GS_LIB_PATH=$PWD/tools/exp_libs/libG.so timeout 900 python -m pytest tests/test_gpu_nodewise.py -m gpu -q -x > gpurun_out/pytest_t11_G.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_t11_G.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:walk_kernel -s 1 -c 1 -o gpurun_out/prof_deepwalk_idx python tools/run_once.py deepwalk_fs 2 > gpurun_out/ncu_dw_idx.log 2>&1
