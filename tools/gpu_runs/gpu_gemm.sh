set -x
timeout 600 python -m pytest tests/test_gpu_blocks.py tests/test_gpu_partial.py -x -q > gpurun_out/pytest_blocks.log 2>&1; echo rc $?
tail -3 gpurun_out/pytest_blocks.log
for gb in 0 1; do
timeout 120 python tools/gemm_bench.py --tune gemm_big=$gb
timeout 120 python tools/gemm_bench.py --tune gemm_big=$gb --m 512 --n 512 --k 512 --batch 256
timeout 120 python tools/gemm_bench.py --tune gemm_big=$gb --m 1024 --n 1024 --k 256 --batch 64
done
timeout 600 python bench.py --config C4 --no-cpu-baseline --no-e2e --steps 5 > gpurun_out/bench_C4_big.json 2>gpurun_out/bench_C4_big.err
python -c "import json; d=json.load(open('gpurun_out/bench_C4_big.json')); print(d['ms_per_step'], d['kernel_ms_per_step'])"
