timeout 900 python -m pytest tests/test_gpu_blocks.py tests/test_gpu_partial.py tests/test_gpu_getrs.py -x -q > gpurun_out/pytest_x.log 2>&1; echo rc $?; tail -2 gpurun_out/pytest_x.log
timeout 400 python bench.py --config C4 --no-cpu-baseline --no-e2e > /tmp/b.json 2>/tmp/b.err; tail -1 /tmp/b.err
python -c "import json; d=json.load(open('/tmp/b.json')); print('C4', round(d['ms_per_step'],3), round(d['value'],1), {k:round(v,3) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"
cp /tmp/b.json gpurun_out/bench_C4_x.json
