# defaults after TMA-on + S-only stream split: tests, C1big / C5 bench; A/B l1_rows 256 vs 512 on C3 / C5
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3i; mkdir -p $O
timeout 900 python -m pytest tests -x -q -m "gpu and not full" > $O/pytest.log 2>&1; echo pytest rc $?; tail -1 $O/pytest.log
timeout 200 python bench.py --config C1big --no-cpu-baseline --no-e2e > $O/bench_C1big.json 2> $O/bench_C1big.err; python -c "import json; d=json.load(open('$O/bench_C1big.json')); print('C1big', round(d['ms_per_step'],3), round(d['roofline']['frac'],3), d['kernel_ms_per_step'])"
for r in 256 512; do
timeout 200 python bench.py --config C3 --no-cpu-baseline --no-e2e --tune l1_rows=$r > $O/bench_C3_l1r$r.json 2> $O/bench_C3_l1r$r.err; python -c "import json; d=json.load(open('$O/bench_C3_l1r$r.json')); print('C3 l1_rows=$r', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
timeout 500 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e --tune l1_rows=$r > $O/bench_C5_l1r$r.json 2> $O/bench_C5_l1r$r.err; python -c "import json; d=json.load(open('$O/bench_C5_l1r$r.json')); print('C5 l1_rows=$r', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
done
