timeout 600 python -m pytest tests/test_gpu_getrf.py -x -q > gpurun_out/pytest_getrf.log 2>&1; echo rc $?; tail -2 gpurun_out/pytest_getrf.log
for t in "l1_rowmap=1" "l1_rowmap=1 --tune l1_dmma=1" "l1_rowmap=0"; do
echo "== $t"
python tools/phase_time.py --config C2 --tune $t --tune tier_m_max=0 --tune concurrent=0
timeout 300 python bench.py --config C2 --no-cpu-baseline --no-e2e --tune $t > /tmp/b.json
python -c "import json; d=json.load(open('/tmp/b.json')); print('$t', d['ms_per_step'], d['kernel_ms_per_step'], d['roofline']['frac'])"
done
