O=gpurun_out/t32; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_pass_full.py -m gpu -q -rf > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
