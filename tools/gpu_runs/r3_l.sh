# ncu of the a5.2 strip kernel (getrs_strip_kernel) on C4
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3l; mkdir -p $O
timeout 900 ncu --set full --clock-control none --import-source on -k regex:getrs_strip -c 1 -o $O/prof_getrs_C4 python tools/prof_one.py --config C4 --reps 1 > $O/ncu.log 2>&1; echo ncu rc $?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C4.csv python tools/prof_one.py --config C4 --reps 1 > /dev/null 2>&1; echo launches rc $?
