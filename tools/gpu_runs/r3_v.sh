# split_strip = 1 (inner trailing update as a grid-wide GEMM) on the large batches C3 / C5 / C4
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3v; mkdir -p $O
for v in 1 2; do
timeout 200 python bench.py --config C3 --no-cpu-baseline --no-e2e --tune split_strip=$v > $O/bench_C3_s$v.json 2> $O/bench_C3_s$v.err; python -c "import json; d=json.load(open('$O/bench_C3_s$v.json')); print('C3 split=$v', round(d['ms_per_step'],3), {k:round(v,1) for k,v in d['kernel_busy_ms_per_step'].items()})"
timeout 500 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e --tune split_strip=$v > $O/bench_C5_s$v.json 2> $O/bench_C5_s$v.err; python -c "import json; d=json.load(open('$O/bench_C5_s$v.json')); print('C5 split=$v', round(d['ms_per_step'],3), {k:round(v,1) for k,v in d['kernel_busy_ms_per_step'].items()})"
done
