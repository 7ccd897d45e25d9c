mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_layerwise.py -m gpu -q -x -rf > gpurun_out/pytest_lw.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_lw.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -rf -k layerwise > gpurun_out/pytest_lw_full.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_lw_full.log
for w in fastgcn_lj ladies_lj; do
  for p in bm old; do GS_LW_PATH=$p timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${w}_$p.log 2>&1; done
done
