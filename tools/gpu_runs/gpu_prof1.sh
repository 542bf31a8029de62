set -x
ncu --set full --clock-control none --import-source on -k regex:lu_l1 -c 1 -o gpurun_out/prof_l1_C2 python tools/prof_one.py --config C2 --reps 1 > gpurun_out/ncu_l1.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:lu_small -c 1 -o gpurun_out/prof_small_C1big python tools/prof_one.py --config C1big --scale 0.25 --reps 1 > gpurun_out/ncu_small.log 2>&1
ls -la gpurun_out
