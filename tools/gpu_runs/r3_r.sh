# A/B: two parts on two streams (parts = 2) with the warp-specialised GEMM
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3r; mkdir -p $O
for v in "1 1" "2 1" "2 2"; do set -- $v
timeout 200 python bench.py --config C3 --no-cpu-baseline --no-e2e --tune parts=$1 --tune part_grid=$2 > $O/bench_C3_p$1_g$2.json 2> $O/bench_C3_p$1_g$2.err; python -c "import json; d=json.load(open('$O/bench_C3_p$1_g$2.json')); print('C3 parts=$1 grid=$2', round(d['ms_per_step'],3))"
timeout 500 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e --tune parts=$1 --tune part_grid=$2 > $O/bench_C5_p$1_g$2.json 2> $O/bench_C5_p$1_g$2.err; python -c "import json; d=json.load(open('$O/bench_C5_p$1_g$2.json')); print('C5 parts=$1 grid=$2', round(d['ms_per_step'],3))"
done
