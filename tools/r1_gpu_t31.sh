# UVA (host-mapped CSC) parity + bench line.
O=gpurun_out/t31; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_uva.py tests/test_gpu_ops.py -m gpu -q -rf > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
timeout 900 python bench.py --workload graphsage_pd_uva --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_uva.log 2>&1; echo "rc=$?" >> $O/bench_uva.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_default.log 2>&1; echo "rc=$?" >> $O/bench_default.log
