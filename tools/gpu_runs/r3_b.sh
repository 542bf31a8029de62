# grouped tier S (tier_s = 2) + branch-free multiplier: tests, C1big A/B, L1 ncu (the m<=256 variant)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r3b
timeout 900 python -m pytest tests/test_gpu_getrf.py -x -q > gpurun_out/r3b/pytest_getrf.log 2>&1; echo pytest rc $?; tail -3 gpurun_out/r3b/pytest_getrf.log
for ts in 2 1; do timeout 300 python bench.py --config C1big --no-cpu-baseline --no-e2e --tune tier_s=$ts > gpurun_out/r3b/bench_C1big_ts$ts.json 2> gpurun_out/r3b/bench_C1big_ts$ts.err; echo "ts=$ts rc $?"; python -c "import json; d=json.load(open('gpurun_out/r3b/bench_C1big_ts$ts.json')); print('C1big ts=$ts', round(d['ms_per_step'],3), round(d['roofline']['frac'],3), d['kernel_ms_per_step'])"; done
timeout 300 python bench.py --config C2 --no-cpu-baseline --no-e2e > gpurun_out/r3b/bench_C2.json 2> gpurun_out/r3b/bench_C2.err; python -c "import json; d=json.load(open('gpurun_out/r3b/bench_C2.json')); print('C2', round(d['ms_per_step'],3), d['kernel_ms_per_step'])"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lu_group_kernel -c 2 -o gpurun_out/r3b/prof_group_C1big python tools/prof_one.py --config C1big --reps 1 > gpurun_out/r3b/ncu_group.log 2>&1; echo ncu1 rc $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lu_l1_kernel -s 1 -c 1 -o gpurun_out/r3b/prof_l1_C2 python tools/prof_one.py --config C2 --reps 1 > gpurun_out/r3b/ncu_l1.log 2>&1; echo ncu2 rc $?
