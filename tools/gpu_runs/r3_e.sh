# warp-specialised xgemm (xgemm_warps = 9): tests, C3 / C4 / C5 A/B
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r3e
timeout 900 python -m pytest tests/test_gpu_blocks.py tests/test_gpu_getrf.py -x -q -k "gemm or xgemm or two_level or outer" > gpurun_out/r3e/pytest.log 2>&1; echo pytest rc $?; tail -3 gpurun_out/r3e/pytest.log
for w in 9 8; do
timeout 300 python bench.py --config C3 --no-cpu-baseline --no-e2e --tune xgemm_warps=$w > gpurun_out/r3e/bench_C3_w$w.json 2> gpurun_out/r3e/bench_C3_w$w.err; python -c "import json; d=json.load(open('gpurun_out/r3e/bench_C3_w$w.json')); print('C3 w=$w', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
done
timeout 600 python bench.py --config C4 --steps 3 --no-cpu-baseline --no-e2e --tune xgemm_warps=9 > gpurun_out/r3e/bench_C4_w9.json 2> gpurun_out/r3e/bench_C4_w9.err; python -c "import json; d=json.load(open('gpurun_out/r3e/bench_C4_w9.json')); print('C4 w=9', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
timeout 900 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e --tune xgemm_warps=9 > gpurun_out/r3e/bench_C5_w9.json 2> gpurun_out/r3e/bench_C5_w9.err; python -c "import json; d=json.load(open('gpurun_out/r3e/bench_C5_w9.json')); print('C5 w=9', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:xgemm_ws -s 3 -c 1 -o gpurun_out/r3e/prof_xws_C3 python tools/prof_one.py --config C3 --reps 1 --tune xgemm_warps=9 > gpurun_out/r3e/ncu.log 2>&1; echo ncu rc $?
