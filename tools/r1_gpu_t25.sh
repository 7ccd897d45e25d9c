# PASS full (f2): attention parity + sampling parity, bench line, launch list, ncu of the SDDMM kernel;
# PinSAGE flat relabel re-measured.
O=gpurun_out/t25; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_pass_full.py tests/test_gpu_pinsage.py -m gpu -q -rf > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
timeout 900 python bench.py --workload pass_full_pd --steps 5 --warmup 3 > $O/bench_pass_full_pd.log 2>&1; echo "rc=$?" >> $O/bench_pass_full_pd.log
timeout 900 python bench.py --workload pinsage_pd --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_pinsage_pd.log 2>&1; echo "rc=$?" >> $O/bench_pinsage_pd.log
timeout 600 ncu --kernel-name-base demangled --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file $O/launches_pass_full_pd.csv python bench.py --workload pass_full_pd --steps 3 --warmup 3 > $O/b_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pass_att_kernel -s 1 -c 1 -o $O/prof_pass_full_pd python tools/run_once.py pass_full_pd 2 > $O/ncu_pass.log 2>&1
