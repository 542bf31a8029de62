# ws xgemm with the setmaxnreg budget fixed (56 / 216); tier-S load/store cleanup
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r3f
timeout 240 python -m pytest tests/test_gpu_blocks.py -x -q -k "gemm_big" > gpurun_out/r3f/pytest_blocks.log 2>&1; echo pytest-blocks rc $?; tail -2 gpurun_out/r3f/pytest_blocks.log
timeout 400 python -m pytest tests/test_gpu_getrf.py -x -q -k "xgemm or grouped or c1_parity or edge or g1 or singular or closed or leading or two_level" > gpurun_out/r3f/pytest_getrf.log 2>&1; echo pytest-getrf rc $?; tail -2 gpurun_out/r3f/pytest_getrf.log
timeout 200 python bench.py --config C1big --no-cpu-baseline --no-e2e > gpurun_out/r3f/bench_C1big.json 2> gpurun_out/r3f/bench_C1big.err; python -c "import json; d=json.load(open('gpurun_out/r3f/bench_C1big.json')); print('C1big', round(d['ms_per_step'],3), round(d['roofline']['frac'],3), d['kernel_ms_per_step'])"
for w in 9 8; do
timeout 200 python bench.py --config C3 --no-cpu-baseline --no-e2e --tune xgemm_warps=$w > gpurun_out/r3f/bench_C3_w$w.json 2> gpurun_out/r3f/bench_C3_w$w.err; python -c "import json; d=json.load(open('gpurun_out/r3f/bench_C3_w$w.json')); print('C3 w=$w', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
done
timeout 300 python bench.py --config C4 --steps 3 --no-cpu-baseline --no-e2e --tune xgemm_warps=9 > gpurun_out/r3f/bench_C4_w9.json 2> gpurun_out/r3f/bench_C4_w9.err; python -c "import json; d=json.load(open('gpurun_out/r3f/bench_C4_w9.json')); print('C4 w=9', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
timeout 500 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e --tune xgemm_warps=9 > gpurun_out/r3f/bench_C5_w9.json 2> gpurun_out/r3f/bench_C5_w9.err; python -c "import json; d=json.load(open('gpurun_out/r3f/bench_C5_w9.json')); print('C5 w=9', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:xgemm_ws -s 3 -c 1 -o gpurun_out/r3f/prof_xws_C3 python tools/prof_one.py --config C3 --reps 1 --tune xgemm_warps=9 > gpurun_out/r3f/ncu.log 2>&1; echo ncu rc $?
