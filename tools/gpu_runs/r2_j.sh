# outer_swap_trsm2 (outer_kernel=1) A/B + fused LAPACK-style partial
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 python -m pytest tests/test_gpu_getrf.py tests/test_gpu_partial.py -q -m "gpu and not full" -x -p no:randomly > gpurun_out/pytest_gpu_j.log 2>&1; echo pytest rc $?; tail -3 gpurun_out/pytest_gpu_j.log; grep -E "^FAILED|^ERROR" gpurun_out/pytest_gpu_j.log | head
run() { c=$1; shift; timeout 400 python bench.py --config $c --no-cpu-baseline --no-e2e "$@" > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
cp /tmp/b.json gpurun_out/bench_${c}_$(echo "$*" | tr -c 'a-z0-9\n' '_').json
python -c "import json,sys; d=json.load(open('/tmp/b.json')); print('$c $*', round(d['ms_per_step'],3), round(d['value'],1), {k:round(v,3) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"; }
run C3 --tune outer_kernel=1
run C3
run C5 --steps 3 --tune outer_kernel=1
timeout 600 python tools/bench_next.py --what lapack --reps 3 2>&1 | tail -3
timeout 900 ncu --set full --clock-control none --import-source on -k regex:outer_swap_trsm2 -s 3 -c 1 -o gpurun_out/prof_outer2_C5 python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --tune outer_kernel=1 > gpurun_out/ncu_outer2.log 2>&1; echo ncu rc $?
