timeout 600 python -m pytest tests/test_gpu_getrf.py -x -q -k "pipelined or status" > gpurun_out/pytest_e2e.log 2>&1; echo rc $?; tail -3 gpurun_out/pytest_e2e.log
for ch in 16 8 32; do timeout 300 python bench.py --no-cpu-baseline --e2e-chunks $ch > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
python -c "import json; d=json.load(open('/tmp/b.json')); print('C2 chunks $ch', round(d['ms_per_step'],3), round(d['value'],1), 'e2e', round(d['e2e']['value'],1), round(d['e2e']['ms_per_step'],2))"; done
timeout 300 python bench.py --config C4 --no-cpu-baseline --e2e-chunks 16 > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
python -c "import json; d=json.load(open('/tmp/b.json')); print('C4', round(d['ms_per_step'],3), round(d['value'],1), 'e2e', round(d['e2e']['value'],1), round(d['e2e']['ms_per_step'],2))"
