# A/B: inner panel width nb (16 / 24 / 32) on C3 and C5
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3n; mkdir -p $O
for nb in 16 24 32; do
timeout 200 python bench.py --config C3 --no-cpu-baseline --no-e2e --tune nb=$nb > $O/bench_C3_nb$nb.json 2> $O/bench_C3_nb$nb.err; python -c "import json; d=json.load(open('$O/bench_C3_nb$nb.json')); print('C3 nb=$nb', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
timeout 500 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e --tune nb=$nb > $O/bench_C5_nb$nb.json 2> $O/bench_C5_nb$nb.err; python -c "import json; d=json.load(open('$O/bench_C5_nb$nb.json')); print('C5 nb=$nb', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
done
timeout 200 python bench.py --config C2 --no-cpu-baseline --no-e2e --tune nb=16 > $O/bench_C2_nb16.json 2> $O/bench_C2_nb16.err; python -c "import json; d=json.load(open('$O/bench_C2_nb16.json')); print('C2 nb=16', round(d['ms_per_step'],3))"
