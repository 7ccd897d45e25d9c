O=gpurun_out/r2z; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_ops.py -m gpu -q -x > $O/pytest_ops.log 2>&1; echo "rc=$?" >> $O/pytest_ops.log
