O=gpurun_out/r2v; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_layerwise.py -m gpu -q -x > $O/pytest_lw.log 2>&1; echo "rc=$?" >> $O/pytest_lw.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "layerwise" > $O/pytest_full.log 2>&1; echo "rc=$?" >> $O/pytest_full.log
GS_VERBOSE=1 timeout 600 python bench.py --workload ladies_lj --no-cpu-baseline > $O/bench_ladies.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:layerwise_sm --launch-skip 2 --launch-count 1 -o $O/ncu_lsm python bench.py --workload ladies_lj --steps 1 --warmup 1 --no-cpu-baseline --no-graph > $O/ncu.log 2>&1
