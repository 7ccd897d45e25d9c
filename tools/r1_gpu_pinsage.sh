# PinSAGE-style: GPU parity tests, bench line, launch list, ncu --set full of the kernel.
O=gpurun_out/pinsage; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_pinsage.py -m gpu -q -rf -x > $O/pytest_pinsage.log 2>&1; echo "pytest rc=$?" >> $O/pytest_pinsage.log
timeout 900 python bench.py --workload pinsage_pd --steps 5 --warmup 3 > $O/bench_pinsage_pd.log 2>&1; echo "rc=$?" >> $O/bench_pinsage_pd.log
timeout 600 ncu --kernel-name-base demangled -k regex:gsb:: --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $O/launches_pinsage_pd.csv python bench.py --workload pinsage_pd --steps 3 --warmup 3 --no-cpu-baseline > $O/b_ncu_pinsage.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pinsage_kernel -s 1 -c 1 -o $O/prof_pinsage_pd python tools/run_once.py pinsage_pd 2 > $O/ncu_pinsage.log 2>&1
