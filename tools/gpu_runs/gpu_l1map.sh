set -x
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo rc $?
tail -5 gpurun_out/pytest_gpu.log
for rm in 0 1; do
python tools/phase_time.py --config C2 --tune l1_rowmap=$rm --tune tier_m_max=0 --tune concurrent=0
timeout 300 python bench.py --config C2 --no-cpu-baseline --no-e2e --tune l1_rowmap=$rm > gpurun_out/bench_C2_rm$rm.json
python -c "import json; d=json.load(open('gpurun_out/bench_C2_rm$rm.json')); print('rowmap $rm', d['ms_per_step'], d['kernel_ms_per_step'], d['roofline']['frac'])"
done
timeout 300 python bench.py --config C2 --no-cpu-baseline --no-e2e --tune l1_dmma=1 > gpurun_out/bench_C2_dmma.json
python -c "import json; d=json.load(open('gpurun_out/bench_C2_dmma.json')); print('rowmap dmma', d['ms_per_step'], d['kernel_ms_per_step'], d['roofline']['frac'])"
