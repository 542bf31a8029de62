# bench accounting with per-class busy time (union of launch intervals): parts 1 / 2 on C3 / C5, C1big
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3s; mkdir -p $O
timeout 200 python bench.py --config C1big --no-cpu-baseline --no-e2e > $O/bench_C1big.json 2> $O/bench_C1big.err; python -c "import json; d=json.load(open('$O/bench_C1big.json')); print('C1big', round(d['ms_per_step'],3), d['roofline']['kernel'], round(d['roofline']['frac'],3), d['kernel_busy_ms_per_step'])"
for p in 1 2; do
timeout 200 python bench.py --config C3 --no-cpu-baseline --no-e2e --tune parts=$p > $O/bench_C3_p$p.json 2> $O/bench_C3_p$p.err; python -c "import json; d=json.load(open('$O/bench_C3_p$p.json')); print('C3 parts=$p', round(d['ms_per_step'],3), d['roofline']['kernel'], round(d['roofline']['frac'],3), {k:round(v,2) for k,v in d['kernel_busy_ms_per_step'].items()})"
timeout 500 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e --tune parts=$p > $O/bench_C5_p$p.json 2> $O/bench_C5_p$p.err; python -c "import json; d=json.load(open('$O/bench_C5_p$p.json')); print('C5 parts=$p', round(d['ms_per_step'],3), d['roofline']['kernel'], round(d['roofline']['frac'],3), {k:round(v,2) for k,v in d['kernel_busy_ms_per_step'].items()})"
done
