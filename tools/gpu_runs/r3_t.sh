# A/B: CTA-per-matrix tier residency (l1_ctas_per_sm 2 vs 3) on C2 / C5
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3t; mkdir -p $O
for c in 2 3; do
timeout 200 python bench.py --config C2 --no-cpu-baseline --no-e2e --tune l1_ctas_per_sm=$c > $O/bench_C2_c$c.json 2> $O/bench_C2_c$c.err; python -c "import json; d=json.load(open('$O/bench_C2_c$c.json')); print('C2 ctas=$c', round(d['ms_per_step'],3))"
timeout 500 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e --tune l1_ctas_per_sm=$c > $O/bench_C5_c$c.json 2> $O/bench_C5_c$c.err; python -c "import json; d=json.load(open('$O/bench_C5_c$c.json')); print('C5 ctas=$c', round(d['ms_per_step'],3), round(d['kernel_busy_ms_per_step']['lu_l1'],2))"
done
