ncu --set full --clock-control none --import-source on -k regex:getrs_strip -c 1 -o gpurun_out/prof_getrs_C4 python tools/prof_one.py --config C4 --reps 1 > gpurun_out/ncu_getrs.log 2>&1
tail -2 gpurun_out/ncu_getrs.log
