timeout 900 python -m pytest tests/test_gpu_getrf.py -x -q > gpurun_out/pytest_getrf.log 2>&1; echo rc $?; tail -2 gpurun_out/pytest_getrf.log
for t in "nb=32" "nb=64" "nb=48" "nb=64 --tune dmma=0"; do
timeout 300 python bench.py --config C3 --no-cpu-baseline --no-e2e --steps 3 --tune $t > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
python -c "import json; d=json.load(open('/tmp/b.json')); print('C3 $t', round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"
done
timeout 300 python bench.py --config C2 --no-cpu-baseline --no-e2e > /tmp/b.json 2>/tmp/b.err
python -c "import json; d=json.load(open('/tmp/b.json')); print('C2', round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"
