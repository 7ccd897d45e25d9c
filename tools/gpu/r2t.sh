O=gpurun_out/r2t; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_pass_full.py -m gpu -q -x > $O/pytest_pass.log 2>&1; echo "rc=$?" >> $O/pytest_pass.log
timeout 600 python bench.py --workload pass_full_pd --no-cpu-baseline > $O/bench_passfull.log 2>&1
GS_PASS_GEMM=cublas timeout 600 python bench.py --workload pass_full_pd --no-cpu-baseline > $O/bench_passfull_cublas.log 2>&1
timeout 600 ncu --kernel-name-base demangled -k regex:"proj_gemm|gemm|Kernel|pass_att" --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 20 --csv --log-file $O/launches_gemm.csv python bench.py --workload pass_full_pd --steps 1 --warmup 1 --no-cpu-baseline --no-graph > $O/b_ncu.log 2>&1
GS_PASS_GEMM=cublas timeout 600 ncu --kernel-name-base demangled -k regex:"gemm|Kernel|pass_att" --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 20 --csv --log-file $O/launches_cublas.csv python bench.py --workload pass_full_pd --steps 1 --warmup 1 --no-cpu-baseline --no-graph > $O/b_ncu2.log 2>&1
