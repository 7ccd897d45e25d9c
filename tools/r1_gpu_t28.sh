# Node2Vec membership by interpolation search (3 probes, then bisection).
O=gpurun_out/t28; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_walk.py tests/test_gpu_fullsize.py -m gpu -q -rf -k "walk or node2vec or deepwalk or fs" > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
timeout 900 python bench.py --workload node2vec_fs --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_node2vec_fs.log 2>&1; echo "rc=$?" >> $O/bench_node2vec_fs.log
