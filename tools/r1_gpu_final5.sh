# Last check of the final tree: every GPU test, smoke, the default bench line (cpu_baseline on), reference arm.
O=gpurun_out/final5; mkdir -p $O
timeout 2400 python -m pytest tests -m gpu -q -rf > $O/pytest_gpu_all.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 600 python bench.py > $O/bench_default.log 2>&1; echo "rc=$?" >> $O/bench_default.log
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_reference.log 2>&1; echo "rc=$?" >> $O/bench_reference.log
timeout 600 ncu --kernel-name-base demangled -k regex:gsb:: --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $O/launches_graphsage_pd.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $O/b_ncu.log 2>&1
