# a5.2 strip kernel 128 columns wide (64 x 128 DMMA tile, 32 x 32 warp tiles, 3-deep ring): tests + C4 A/B vs 64
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3m; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_partial.py tests/test_gpu_getrs.py tests/test_gpu_tree.py -x -q > $O/pytest.log 2>&1; echo pytest rc $?; tail -1 $O/pytest.log
timeout 300 python bench.py --config C4 --steps 3 --no-cpu-baseline --no-e2e > $O/bench_C4_sw128.json 2> $O/bench_C4_sw128.err; python -c "import json; d=json.load(open('$O/bench_C4_sw128.json')); print('C4 sw128', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
timeout 600 python tools/bench_getrs.py > $O/bench_getrs_sw128.jsonl 2> $O/bench_getrs_sw128.err; echo getrs rc $?; tail -4 $O/bench_getrs_sw128.jsonl
IRR_NVCC_EXTRA="-DIRR_GS_SW=64" timeout 600 python -m paper_conf_sc_abdelfattahgbtld22_b200.build --force > /dev/null 2>&1; echo build64 rc $?
timeout 300 python bench.py --config C4 --steps 3 --no-cpu-baseline --no-e2e > $O/bench_C4_sw64.json 2> $O/bench_C4_sw64.err; python -c "import json; d=json.load(open('$O/bench_C4_sw64.json')); print('C4 sw64', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
timeout 600 python tools/bench_getrs.py > $O/bench_getrs_sw64.jsonl 2> $O/bench_getrs_sw64.err; echo getrs rc $?; tail -4 $O/bench_getrs_sw64.jsonl
