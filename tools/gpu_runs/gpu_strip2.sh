python tools/phase_time.py --config C3 --scale 0.5 > gpurun_out/phase_C3.txt 2>&1; cat gpurun_out/phase_C3.txt
ncu --set full --clock-control none --import-source on -k regex:strip_kernel -c 1 -o gpurun_out/prof_strip_C3 python tools/prof_one.py --config C3 --scale 0.5 --reps 1 > gpurun_out/ncu_strip.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:panel_win -c 1 -o gpurun_out/prof_pwin_C3 python tools/prof_one.py --config C3 --scale 0.5 --reps 1 > gpurun_out/ncu_pwin.log 2>&1
tail -2 gpurun_out/ncu_strip.log
