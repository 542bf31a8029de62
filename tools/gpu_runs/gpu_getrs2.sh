timeout 600 python -m pytest tests/test_gpu_partial.py -x -q > gpurun_out/pytest_partial.log 2>&1; echo rc $?; tail -2 gpurun_out/pytest_partial.log
timeout 300 python bench.py --config C4 --no-cpu-baseline --no-e2e --steps 5 > /tmp/b.json 2>/tmp/b.err; tail -3 /tmp/b.err
python -c "import json; d=json.load(open('/tmp/b.json')); print(d['ms_per_step'], {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['frac'])"
ncu --set full --clock-control none -k regex:getrs_strip -c 1 -o gpurun_out/prof_getrs_C4b python tools/prof_one.py --config C4 --reps 1 > /dev/null 2>&1
