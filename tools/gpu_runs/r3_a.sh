# session 2 of round 2: baseline re-check + ncu source-level of tier S (C1big) and lu_l1 (C2)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r3a
nvidia-smi --query-gpu=name,driver_version,clocks.max.sm --format=csv > gpurun_out/r3a/smi.txt
timeout 600 python -m pytest tests/test_gpu_getrf.py -x -q > gpurun_out/r3a/pytest_getrf.log 2>&1; echo pytest rc $?; tail -1 gpurun_out/r3a/pytest_getrf.log
for c in C1big C2; do timeout 300 python bench.py --config $c --no-cpu-baseline --no-e2e > gpurun_out/r3a/bench_$c.json 2> gpurun_out/r3a/bench_$c.err; echo "$c rc $?"; python -c "import json; d=json.load(open('gpurun_out/r3a/bench_$c.json')); print('$c', round(d['ms_per_step'],3), d['kernel_ms_per_step'])"; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lu_small_kernel -c 3 -o gpurun_out/r3a/prof_small_C1big python tools/prof_one.py --config C1big --reps 1 > gpurun_out/r3a/ncu_small.log 2>&1; echo ncu1 rc $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lu_l1_kernel -c 1 -o gpurun_out/r3a/prof_l1_C2 python tools/prof_one.py --config C2 --reps 1 > gpurun_out/r3a/ncu_l1.log 2>&1; echo ncu2 rc $?
