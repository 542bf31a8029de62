# tier S: L2 prefetch distance 1 vs 2 items (build switch IRR_S_PF)
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3w; mkdir -p $O
timeout 200 python bench.py --config C1big --no-cpu-baseline --no-e2e > $O/bench_C1big_pf1.json 2> $O/bench_C1big_pf1.err; python -c "import json; d=json.load(open('$O/bench_C1big_pf1.json')); print('C1big pf1', round(d['ms_per_step'],3))"
IRR_NVCC_EXTRA="-DIRR_S_PF=2" timeout 600 python -m paper_conf_sc_abdelfattahgbtld22_b200.build --force > /dev/null 2>&1; echo build rc $?
timeout 200 python bench.py --config C1big --no-cpu-baseline --no-e2e > $O/bench_C1big_pf2.json 2> $O/bench_C1big_pf2.err; python -c "import json; d=json.load(open('$O/bench_C1big_pf2.json')); print('C1big pf2', round(d['ms_per_step'],3))"
IRR_NVCC_EXTRA="-DIRR_S_PF=3" timeout 600 python -m paper_conf_sc_abdelfattahgbtld22_b200.build --force > /dev/null 2>&1; echo build rc $?
timeout 200 python bench.py --config C1big --no-cpu-baseline --no-e2e > $O/bench_C1big_pf3.json 2> $O/bench_C1big_pf3.err; python -c "import json; d=json.load(open('$O/bench_C1big_pf3.json')); print('C1big pf3', round(d['ms_per_step'],3))"
