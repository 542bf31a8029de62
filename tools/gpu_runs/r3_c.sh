# pair kernel (tier_s = 3) for the widest tier-S class
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r3c
timeout 900 python -m pytest tests/test_gpu_getrf.py -x -q -k "grouped or c1_parity or edge or g1 or singular or closed or leading" > gpurun_out/r3c/pytest.log 2>&1; echo pytest rc $?; tail -3 gpurun_out/r3c/pytest.log
for ts in 3 2; do timeout 300 python bench.py --config C1big --no-cpu-baseline --no-e2e --tune tier_s=$ts > gpurun_out/r3c/bench_C1big_ts$ts.json 2> gpurun_out/r3c/bench_C1big_ts$ts.err; echo "ts=$ts rc $?"; python -c "import json; d=json.load(open('gpurun_out/r3c/bench_C1big_ts$ts.json')); print('C1big ts=$ts', round(d['ms_per_step'],3), round(d['roofline']['frac'],3), d['kernel_ms_per_step'])"; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lu_pair_kernel -c 1 -o gpurun_out/r3c/prof_pair_C1big python tools/prof_one.py --config C1big --reps 1 --tune tier_s=3 > gpurun_out/r3c/ncu_pair.log 2>&1; echo ncu1 rc $?
