# SDDMM kernel: 8 lanes per edge, 4 edge steps in flight (vs lane per edge: 15 ms); ops empty-output fix.
O=gpurun_out/t27; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_pass_full.py tests/test_gpu_ops.py -m gpu -q -rf > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
timeout 900 python bench.py --workload pass_full_pd --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_pass_full_pd.log 2>&1; echo "rc=$?" >> $O/bench_pass_full_pd.log
timeout 600 ncu --kernel-name-base demangled -k regex:"gsb::|nvjet|gemm" --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file $O/launches_pass_full_pd.csv python bench.py --workload pass_full_pd --steps 3 --warmup 3 --no-cpu-baseline > $O/b_ncu.log 2>&1
