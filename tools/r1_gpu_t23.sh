# PinSAGE warp-bitonic top-k; induce back to scalar loads (+ dynamic claims).
O=gpurun_out/t23; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_pinsage.py tests/test_gpu_saint.py -m gpu -q -rf -x > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
for w in pinsage_pd saint_pd; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 > $O/bench_$w.log 2>&1; echo "rc=$?" >> $O/bench_$w.log
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pinsage_kernel -s 1 -c 1 -o $O/prof_pinsage_pd python tools/run_once.py pinsage_pd 2 > $O/ncu_pinsage.log 2>&1
