O=gpurun_out/r2ac; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_nodewise.py -x -q -m gpu -k weighted > $O/pytest.log 2>&1
timeout 900 compute-sanitizer --print-limit 5 python -m pytest tests/test_gpu_nodewise.py -x -q -m gpu -k "weighted and 1" > $O/san.log 2>&1
