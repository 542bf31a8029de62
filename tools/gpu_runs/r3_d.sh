# xgemm: next tile's prologue overlapped with the current epilogue
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r3d
timeout 900 python -m pytest tests/test_gpu_getrf.py tests/test_gpu_partial.py tests/test_gpu_blocks.py -x -q > gpurun_out/r3d/pytest.log 2>&1; echo pytest rc $?; tail -3 gpurun_out/r3d/pytest.log
timeout 300 python bench.py --config C3 --no-cpu-baseline --no-e2e > gpurun_out/r3d/bench_C3.json 2> gpurun_out/r3d/bench_C3.err; python -c "import json; d=json.load(open('gpurun_out/r3d/bench_C3.json')); print('C3', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
timeout 600 python bench.py --config C4 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/r3d/bench_C4.json 2> gpurun_out/r3d/bench_C4.err; python -c "import json; d=json.load(open('gpurun_out/r3d/bench_C4.json')); print('C4', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
timeout 900 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/r3d/bench_C5.json 2> gpurun_out/r3d/bench_C5.err; python -c "import json; d=json.load(open('gpurun_out/r3d/bench_C5.json')); print('C5', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
