# C5 A/B of the TMA operand path, alternating runs on one box (decides the default)
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3p; mkdir -p $O
for rep in 1 2; do for t in 0 1; do
timeout 500 python bench.py --config C5 --steps 5 --no-cpu-baseline --no-e2e --tune xgemm_tma=$t > $O/bench_C5_tma${t}_r$rep.json 2> $O/bench_C5_tma${t}_r$rep.err; python -c "import json; d=json.load(open('$O/bench_C5_tma${t}_r$rep.json')); print('C5 tma=$t rep $rep', round(d['ms_per_step'],3), round(d['kernel_ms_per_step']['gemm_trailing'],2))"
done; done
# panel_win: tree reduction of the warp partials (NW <= 16): tests + C3 + few-large
timeout 900 python -m pytest tests/test_gpu_getrf.py tests/test_gpu_large.py -x -q -k "windowed or grid_panel or two_level or large_g1 or 8192 or c3_sample or g1_exact" > $O/pytest.log 2>&1; echo pytest rc $?; tail -1 $O/pytest.log
timeout 200 python bench.py --config C3 --no-cpu-baseline --no-e2e > $O/bench_C3.json 2> $O/bench_C3.err; python -c "import json; d=json.load(open('$O/bench_C3.json')); print('C3', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
timeout 900 python tools/bench_next.py --what large --reps 3 > $O/bench_large.jsonl 2> $O/bench_large.err; echo large rc $?; cut -c1-120 $O/bench_large.jsonl; grep -o '"nb_outer=128,split_strip=1": {"ms": [0-9.]*' $O/bench_large.jsonl
