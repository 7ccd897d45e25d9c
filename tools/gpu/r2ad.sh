O=gpurun_out/r2ad; mkdir -p $O
timeout 900 python tools/ppstats.py PP > $O/pp.txt 2>&1
timeout 300 python tools/ppstats.py PDw > $O/pd.txt 2>&1
