# Round-2 evidence (final session): full GPU tests, smoke, the default bench
# line (+ reference arm), a sweep of every workload, the launch list and an
# ncu --set full capture of the default workload's hop kernels.
O=gpurun_out/ev12; mkdir -p $O
timeout 2400 python -m pytest tests -m gpu -q -rf > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 600 python bench.py > $O/bench_default.log 2>&1; echo "rc=$?" >> $O/bench_default.log
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_reference.log 2>&1
for w in kgcn_pd pass_pd shadow_pd saint_pd pinsage_pd pass_full_pd ladies_lj fastgcn_lj ares_pp deepwalk_fs node2vec_fs graphsage_pd_uva graphsage_pd_uva_cache; do
  timeout 900 python bench.py --workload $w --no-cpu-baseline --steps 5 >> $O/bench_sweep.jsonl 2> $O/bench_$w.err
done
timeout 300 python tools/strong_probe.py > $O/strong_probe.txt 2>&1
timeout 600 ncu --kernel-name-base demangled -k regex:"hop_|bptr_" --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file $O/launches_graphsage_pd.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-graph > $O/b_ncu1.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"hop_select|hop_rows|hop_relabel|hop_nprep" --launch-skip 10 --launch-count 8 -o $O/ncu_graphsage_pd python bench.py --steps 1 --warmup 2 --no-cpu-baseline --no-graph > $O/b_ncu2.log 2>&1
