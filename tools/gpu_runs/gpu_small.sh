timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc $?; tail -3 gpurun_out/pytest_gpu.log
for c in C1big C2; do timeout 300 python bench.py --config $c --no-cpu-baseline --no-e2e > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; tail -2 gpurun_out/bench_$c.err
python -c "import json; d=json.load(open('gpurun_out/bench_$c.json')); print('$c', round(d['ms_per_step'],3), round(d['value'],1), {k:round(v,3) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3), d['clocks'])"; done
ncu --set full --clock-control none --import-source on -k regex:lu_small -c 1 -o gpurun_out/prof_small_C1big python tools/prof_one.py --config C1big --reps 1 > gpurun_out/ncu_small.log 2>&1
