set -x
O=gpurun_out/r2a; mkdir -p $O
nvidia-smi -L > $O/smi.txt
timeout 900 python -m pytest tests/test_gpu_nodewise.py tests/test_c_abi.py tests/test_gpu_saint.py -m gpu -q -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 600 python bench.py --no-cpu-baseline > $O/bench.log 2>&1; echo "rc=$?" >> $O/bench.log
