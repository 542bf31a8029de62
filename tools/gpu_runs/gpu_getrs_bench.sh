python -m paper_conf_sc_abdelfattahgbtld22_b200.build > gpurun_out/build.log 2>&1
for args in "" "--nrhs 1" "--nrhs 16" "--batch 2000 --n-max 1024" "--batch 2000 --n-max 1024 --nrhs 1"; do timeout 300 python tools/bench_getrs.py $args >> gpurun_out/bench_getrs.jsonl 2>> gpurun_out/bench_getrs.err; done; cat gpurun_out/bench_getrs.jsonl; tail -3 gpurun_out/bench_getrs.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_getrs.csv python tools/bench_getrs.py --reps 2 > gpurun_out/ncu_getrs_launch.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:getrs -c 1 -o gpurun_out/prof_getrs python tools/bench_getrs.py --reps 1 > gpurun_out/ncu_getrs.log 2>&1; tail -1 gpurun_out/ncu_getrs.log
