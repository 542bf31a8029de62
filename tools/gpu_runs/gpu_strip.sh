python tools/phase_time.py --config C3 --scale 0.5
timeout 300 python bench.py --config C2 --no-cpu-baseline --no-e2e > /tmp/b.json 2>/tmp/b.err
python -c "import json; d=json.load(open('/tmp/b.json')); print('C2', round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"
ncu --set full --clock-control none --import-source on -k regex:strip_kernel -s 2 -c 1 -o gpurun_out/prof_strip_C3 python tools/prof_one.py --config C3 --scale 0.5 --reps 1 > /dev/null 2>&1
