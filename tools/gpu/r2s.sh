O=gpurun_out/r2s; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_strong_split.py tests/test_gpu_ragged_induce.py tests/test_c_abi.py -m gpu -q -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 600 python bench.py > $O/bench_default.log 2>&1; echo "rc=$?" >> $O/bench_default.log
timeout 600 python bench.py --no-graph --no-cpu-baseline > $O/bench_nograph.log 2>&1
GS_BENCH_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 3 --warmup 3 > $O/bench_gloo2.log 2>&1; echo "rc=$?" >> $O/bench_gloo2.log
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_reference.log 2>&1; echo "rc=$?" >> $O/bench_reference.log
