O=gpurun_out/r2y; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_nodewise.py -m gpu -q -x -k pack > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 300 python bench.py --no-cpu-baseline > $O/bench.log 2>&1
