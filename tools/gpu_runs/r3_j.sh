# branch-free multiplier in panel_regs / panel_win: tests + C2 / C3 / C4 / C5; A/B l1_rows 384 on C5
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3j; mkdir -p $O
timeout 900 python -m pytest tests -x -q -m "gpu and not full" > $O/pytest.log 2>&1; echo pytest rc $?; tail -1 $O/pytest.log
for c in C2 C3; do timeout 200 python bench.py --config $c --no-cpu-baseline --no-e2e > $O/bench_$c.json 2> $O/bench_$c.err; python -c "import json; d=json.load(open('$O/bench_$c.json')); print('$c', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"; done
timeout 300 python bench.py --config C4 --steps 3 --no-cpu-baseline --no-e2e > $O/bench_C4.json 2> $O/bench_C4.err; python -c "import json; d=json.load(open('$O/bench_C4.json')); print('C4', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
for r in 512 384; do
timeout 500 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e --tune l1_rows=$r > $O/bench_C5_l1r$r.json 2> $O/bench_C5_l1r$r.err; python -c "import json; d=json.load(open('$O/bench_C5_l1r$r.json')); print('C5 l1_rows=$r', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
done
