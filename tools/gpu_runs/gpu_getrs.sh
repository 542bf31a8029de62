timeout 600 python -m pytest tests/test_gpu_partial.py tests/test_gpu_blocks.py -x -q > gpurun_out/pytest_partial.log 2>&1; echo rc $?; tail -15 gpurun_out/pytest_partial.log
for t in "getrs_fused=1" "getrs_fused=0"; do
timeout 300 python bench.py --config C4 --no-cpu-baseline --no-e2e --steps 5 --tune $t > /tmp/b.json 2>/tmp/b.err; tail -3 /tmp/b.err
python -c "import json; d=json.load(open('/tmp/b.json')); print('$t', d['ms_per_step'], {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()}, d['roofline'])"
done
