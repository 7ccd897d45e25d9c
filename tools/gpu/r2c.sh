O=gpurun_out/r2c; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_nodewise.py tests/test_c_abi.py tests/test_gpu_saint.py tests/test_gpu_uva.py -m gpu -q -x > $O/pytest_nw.log 2>&1; echo "rc=$?" >> $O/pytest_nw.log
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "graphsage or pass_and or shadow or ares" > $O/pytest_full.log 2>&1; echo "rc=$?" >> $O/pytest_full.log
for mb in 64 128; do GS_VERBOSE=1 GS_HOP_L2MB=$mb timeout 600 python bench.py --no-cpu-baseline > $O/bench_hop_l2_$mb.log 2>&1; done
for w in kgcn_pd pass_pd; do timeout 600 python bench.py --no-cpu-baseline --workload $w > $O/bench_hop_$w.log 2>&1; done
timeout 600 ncu --kernel-name-base demangled -k regex:hop_ --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file $O/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $O/b_ncu.log 2>&1
