# row-major grid tier (rm_grid=1): parity + A/B
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 python -m pytest tests/test_gpu_getrf.py -q -m "gpu and not full" -p no:randomly -k "row_major or two_level or outer" > gpurun_out/pytest_gpu_m2.log 2>&1; echo pytest rc $?; tail -3 gpurun_out/pytest_gpu_m2.log; grep -E "^FAILED|^ERROR|^E  " gpurun_out/pytest_gpu_m2.log | head -20
run() { c=$1; shift; timeout 400 python bench.py --config $c --no-cpu-baseline --no-e2e "$@" > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
cp /tmp/b.json gpurun_out/bench_${c}_$(echo "$*" | tr -c 'a-z0-9\n' '_').json
python -c "import json,sys; d=json.load(open('/tmp/b.json')); print('$c $*', round(d['ms_per_step'],3), round(d['value'],1), {k:round(v,3) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"; }
run C3 --tune rm_grid=1
run C3
run C5 --steps 3 --tune rm_grid=1
run C5 --steps 3
