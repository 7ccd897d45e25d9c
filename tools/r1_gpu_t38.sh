O=gpurun_out/t38; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_ops.py -m gpu -q -rf > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
timeout 600 python tools/ops_bench.py > $O/ops_bench.log 2>&1
