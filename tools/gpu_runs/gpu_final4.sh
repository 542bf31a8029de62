timeout 900 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc $?; tail -2 gpurun_out/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; python tools/summ.py gpurun_out/bench_default.json
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
for c in C1big C3 C4; do timeout 600 python bench.py --config $c > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; python tools/summ.py gpurun_out/bench_$c.json; done
timeout 900 python bench.py --config C5 --steps 3 --no-cpu-baseline > gpurun_out/bench_C5.json 2> gpurun_out/bench_C5.err; python -c "import json; d=json.load(open('gpurun_out/bench_C5.json')); print('C5', d['ms_per_step'], d['value'])"
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_C2.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"lu_l1|lu_mid|lu_small" -c 8 -o gpurun_out/prof_full_C2 python tools/prof_one.py --config C2 --reps 1 > gpurun_out/ncu_full.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"strip_kernel|panel_win" -c 2 -o gpurun_out/prof_strip_C3 python tools/prof_one.py --config C3 --scale 0.5 --reps 1 > gpurun_out/ncu_strip.log 2>&1
ls gpurun_out
