# GraphSAINT-RW: GPU parity tests, smoke, a bench line (cpu_baseline on), the
# launch list and one ncu --set full capture of the induce kernel.
O=gpurun_out/saint; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_saint.py -m gpu -q -rf > $O/pytest_saint.log 2>&1; echo "pytest rc=$?" >> $O/pytest_saint.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 900 python bench.py --workload saint_pd --steps 5 --warmup 3 > $O/bench_saint_pd.log 2>&1; echo "rc=$?" >> $O/bench_saint_pd.log
timeout 600 python bench.py --impl reference --workload saint_pd --steps 2 --warmup 1 > $O/bench_reference_saint_pd.log 2>&1
timeout 600 ncu --kernel-name-base demangled -k regex:gsb:: --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $O/launches_saint_pd.csv python bench.py --workload saint_pd --steps 3 --warmup 3 --no-cpu-baseline > $O/b_ncu_saint.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:shadow_induce -s 1 -c 1 -o $O/prof_saint_pd python tools/run_once.py saint_pd 2 > $O/ncu_saint.log 2>&1
