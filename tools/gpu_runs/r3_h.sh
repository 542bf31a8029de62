# TMA (cp.async.bulk) A operand in the warp-specialised trailing GEMM: tests + A/B; tier-S narrow classes on a second stream
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3h; mkdir -p $O
timeout 300 python -m pytest tests/test_gpu_blocks.py -x -q -k "gemm_big" > $O/pytest_blocks.log 2>&1; echo pytest-blocks rc $?; tail -1 $O/pytest_blocks.log
timeout 500 python -m pytest tests/test_gpu_getrf.py -x -q -k "xgemm or two_level or grouped or c1_parity or edge or g1 or outer" > $O/pytest_getrf.log 2>&1; echo pytest-getrf rc $?; tail -1 $O/pytest_getrf.log
timeout 200 python bench.py --config C1big --no-cpu-baseline --no-e2e > $O/bench_C1big.json 2> $O/bench_C1big.err; python -c "import json; d=json.load(open('$O/bench_C1big.json')); print('C1big', round(d['ms_per_step'],3), round(d['roofline']['frac'],3), d['kernel_ms_per_step'])"
timeout 200 python bench.py --config C1big --no-cpu-baseline --no-e2e --tune concurrent=0 > $O/bench_C1big_nc.json 2> $O/bench_C1big_nc.err; python -c "import json; d=json.load(open('$O/bench_C1big_nc.json')); print('C1big one stream', round(d['ms_per_step'],3), round(d['roofline']['frac'],3), d['kernel_ms_per_step'])"
for t in 1 0; do
timeout 200 python bench.py --config C3 --no-cpu-baseline --no-e2e --tune xgemm_tma=$t > $O/bench_C3_tma$t.json 2> $O/bench_C3_tma$t.err; python -c "import json; d=json.load(open('$O/bench_C3_tma$t.json')); print('C3 tma=$t', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
timeout 500 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e --tune xgemm_tma=$t > $O/bench_C5_tma$t.json 2> $O/bench_C5_tma$t.err; python -c "import json; d=json.load(open('$O/bench_C5_tma$t.json')); print('C5 tma=$t', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:xgemm_ws -s 3 -c 1 -o $O/prof_xws_tma_C3 python tools/prof_one.py --config C3 --reps 1 --tune xgemm_tma=1 > $O/ncu.log 2>&1; echo ncu rc $?
# ring depth / K chunk of the xgemm (compile-time): 5 x 16, 3 x 32
for v in "-DXGEMM_ST=5" "-DXGEMM_BK=32 -DXGEMM_ST=3"; do
  IRR_NVCC_EXTRA="$v" timeout 600 python -m paper_conf_sc_abdelfattahgbtld22_b200.build --force > /dev/null 2>&1; echo "build [$v] rc $?"
  tag=$(echo "$v" | tr -d ' =-')
  timeout 200 python bench.py --config C3 --no-cpu-baseline --no-e2e > $O/bench_C3_$tag.json 2> $O/bench_C3_$tag.err; python -c "import json; d=json.load(open('$O/bench_C3_$tag.json')); print('C3 $tag', round(d['ms_per_step'],3), round(d['kernel_ms_per_step']['gemm_trailing'],2))"
  timeout 500 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e > $O/bench_C5_$tag.json 2> $O/bench_C5_$tag.err; python -c "import json; d=json.load(open('$O/bench_C5_$tag.json')); print('C5 $tag', round(d['ms_per_step'],3), round(d['kernel_ms_per_step']['gemm_trailing'],2))"
done
