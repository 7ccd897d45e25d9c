# induce count pass with 16-byte index vectors (SH_V = 4 per lane in flight).
O=gpurun_out/t22; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_saint.py tests/test_gpu_nodewise.py tests/test_gpu_fullsize.py -m gpu -q -rf -x -k "saint or shadow" > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
for w in saint_pd shadow_pd; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_$w.log 2>&1; echo "rc=$?" >> $O/bench_$w.log
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:shadow_induce -s 1 -c 1 -o $O/prof_saint_pd python tools/run_once.py saint_pd 2 > $O/ncu_saint.log 2>&1
