# Table-4 operator layer (ops.cu): GPU parity + kernel bandwidth.
O=gpurun_out/t24; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_ops.py -m gpu -q -rf > $O/pytest_ops.log 2>&1; echo "pytest rc=$?" >> $O/pytest_ops.log
timeout 600 python tools/ops_bench.py > $O/ops_bench.log 2>&1; echo "rc=$?" >> $O/ops_bench.log
