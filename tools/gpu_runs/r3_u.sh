# C5 tuning re-check with the ws GEMM: outer_cols 32, nb_outer 96 / 64 (baseline in the same run)
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3u; mkdir -p $O
for v in "outer_cols=64" "outer_cols=32" "nb_outer=96" "nb_outer=64"; do
tag=$(echo $v | tr '=' '_')
timeout 500 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e --tune $v > $O/bench_C5_$tag.json 2> $O/bench_C5_$tag.err; python -c "import json; d=json.load(open('$O/bench_C5_$tag.json')); print('C5 $v', round(d['ms_per_step'],3), round(d['roofline']['frac'],3), {k:round(v,1) for k,v in d['kernel_busy_ms_per_step'].items()})"
done
