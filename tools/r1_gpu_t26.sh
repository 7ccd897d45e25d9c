# PASS full parity after the fp32-W3 oracle fix; bench lines (default, pinsage, pass_full) after the bench.py fix.
O=gpurun_out/t26; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_pass_full.py tests/test_gpu_pinsage.py tests/test_gpu_ops.py -m gpu -q -rf > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
timeout 600 python bench.py > $O/bench_default.log 2>&1; echo "rc=$?" >> $O/bench_default.log
for w in pinsage_pd pass_full_pd; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_$w.log 2>&1; echo "rc=$?" >> $O/bench_$w.log
done
timeout 600 ncu --kernel-name-base demangled -k regex:"gsb::|gemm|Gemm|sm100" --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file $O/launches_pass_full_pd.csv python bench.py --workload pass_full_pd --steps 3 --warmup 3 --no-cpu-baseline > $O/b_ncu.log 2>&1
