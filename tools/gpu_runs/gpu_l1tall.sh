timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo rc $?; tail -3 gpurun_out/pytest_gpu.log
for c in C3 C2 C4; do for r in 1024 256; do
timeout 300 python bench.py --config $c --no-cpu-baseline --no-e2e --steps 5 --tune l1_rows=$r > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
python -c "import json; d=json.load(open('/tmp/b.json')); print('$c l1_rows=$r', round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"
done; done
