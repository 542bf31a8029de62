export PATH=/usr/local/cuda/bin:$PATH
timeout 900 python -m pytest tests -q -m "gpu and not full" -x -p no:randomly > gpurun_out/pytest_gpu_g.log 2>&1; echo pytest rc $?; tail -3 gpurun_out/pytest_gpu_g.log; grep -E "^FAILED|^ERROR" gpurun_out/pytest_gpu_g.log | head
run() { c=$1; shift; timeout 400 python bench.py --config $c --no-cpu-baseline --no-e2e "$@" > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
cp /tmp/b.json gpurun_out/bench_${c}_$(echo "$*" | tr -c 'a-z0-9\n' '_').json
python -c "import json,sys; d=json.load(open('/tmp/b.json')); print('$c $*', round(d['ms_per_step'],3), round(d['value'],1), {k:round(v,3) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"; }
run C1big
run C2
run C3
run C5 --steps 3
timeout 900 ncu --set full --clock-control none --import-source on -k regex:xgemm_sched -s 2 -c 1 -o gpurun_out/prof_xgemm2_C3 python bench.py --config C3 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_xgemm2.log 2>&1; echo ncu $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lu_small -s 3 -c 1 -o gpurun_out/prof_small2_C1big python bench.py --config C1big --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_small2.log 2>&1; echo ncu $?
