timeout 900 python -m pytest tests -q -m "gpu and not full" -x -p no:randomly > gpurun_out/pytest_gpu_i.log 2>&1; echo pytest rc $?; tail -3 gpurun_out/pytest_gpu_i.log; grep -E "^FAILED|^ERROR" gpurun_out/pytest_gpu_i.log | head
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_i.log 2>&1; tail -1 gpurun_out/smoke_i.log
run() { c=$1; shift; timeout 400 python bench.py --config $c --no-cpu-baseline --no-e2e "$@" > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
cp /tmp/b.json gpurun_out/bench_${c}_$(echo "$*" | tr -c 'a-z0-9\n' '_').json
python -c "import json,sys; d=json.load(open('/tmp/b.json')); print('$c $*', round(d['ms_per_step'],3), round(d['value'],1), {k:round(v,3) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"; }
run C2
run C3
run C4 --steps 3
run C5 --steps 3
