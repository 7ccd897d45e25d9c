mkdir -p gpurun_out
GS_WAVE=16 timeout 600 ncu --set full --clock-control none --import-source on -k regex:nodewise_wave -s 1 -c 1 -o gpurun_out/prof_wave python tools/run_once.py graphsage_pd 2 > gpurun_out/ncu_wave.log 2>&1
