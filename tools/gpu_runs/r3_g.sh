# tier S: n <= 24 width class (NC = 24, 5 or 6 CTAs/SM)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r3g
timeout 300 python -m pytest tests/test_gpu_getrf.py -x -q -k "grouped or c1_parity or edge or g1 or singular or closed or leading" > gpurun_out/r3g/pytest.log 2>&1; echo pytest rc $?; tail -2 gpurun_out/r3g/pytest.log
timeout 200 python bench.py --config C1big --no-cpu-baseline --no-e2e > gpurun_out/r3g/bench_C1big_c5.json 2> gpurun_out/r3g/bench_C1big_c5.err; python -c "import json; d=json.load(open('gpurun_out/r3g/bench_C1big_c5.json')); print('C1big ctas5', round(d['ms_per_step'],3), round(d['roofline']['frac'],3), d['kernel_ms_per_step'])"
IRR_NVCC_EXTRA="-DIRR_S24_CTAS=6" timeout 600 python -m paper_conf_sc_abdelfattahgbtld22_b200.build --force > /dev/null 2>&1
timeout 200 python bench.py --config C1big --no-cpu-baseline --no-e2e > gpurun_out/r3g/bench_C1big_c6.json 2> gpurun_out/r3g/bench_C1big_c6.err; python -c "import json; d=json.load(open('gpurun_out/r3g/bench_C1big_c6.json')); print('C1big ctas6', round(d['ms_per_step'],3), round(d['roofline']['frac'],3), d['kernel_ms_per_step'])"
