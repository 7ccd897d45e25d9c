# PinSAGE walks through the walk index (one 16-byte record per step).
O=gpurun_out/t33; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_pinsage.py tests/test_gpu_uva.py -m gpu -q -rf > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
timeout 900 python bench.py --workload pinsage_pd --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_pinsage_pd.log 2>&1; echo "rc=$?" >> $O/bench_pinsage_pd.log
