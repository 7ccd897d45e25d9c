# PinSAGE 2-walk ILP + 4-word rank prefix; induce kernel with cluster-wide dynamic column claims.
O=gpurun_out/t21; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_pinsage.py tests/test_gpu_saint.py -m gpu -q -rf -x > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
timeout 1200 python -m pytest tests/test_gpu_nodewise.py tests/test_gpu_fullsize.py -m gpu -q -rf -x -k "shadow" > $O/pytest_shadow.log 2>&1; echo "pytest rc=$?" >> $O/pytest_shadow.log
for w in pinsage_pd saint_pd shadow_pd; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_$w.log 2>&1; echo "rc=$?" >> $O/bench_$w.log
done
