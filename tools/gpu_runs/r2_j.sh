timeout 600 python -m pytest tests/test_gpu_getrf.py -q -x -p no:randomly -k "two_parts or two_level" > gpurun_out/pytest_gpu_j.log 2>&1; echo pytest rc $?; tail -3 gpurun_out/pytest_gpu_j.log
run() { c=$1; shift; timeout 400 python bench.py --config $c --no-cpu-baseline --no-e2e "$@" > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
cp /tmp/b.json gpurun_out/bench_${c}_$(echo "$*" | tr -c 'a-z0-9\n' '_').json
python -c "import json,sys; d=json.load(open('/tmp/b.json')); print('$c $*', round(d['ms_per_step'],3), round(d['value'],1), {k:round(v,3) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"; }
run C3 --tune parts=2
run C3 --tune parts=2 --tune part_grid=2
run C5 --steps 3 --tune parts=2
run C5 --steps 3 --tune parts=2 --tune part_grid=2
run C4 --steps 3 --tune parts=2
