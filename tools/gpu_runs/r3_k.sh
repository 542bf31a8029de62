# tier M with the DMMA trailing update (mid_dmma) and larger tier-M bins: tests + A/B on C2 / C4 / C5
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/r3k; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_getrf.py -x -q -k "tier_m or g1_exact or c2_scaled or leading or edge" > $O/pytest.log 2>&1; echo pytest rc $?; tail -1 $O/pytest.log
for v in "0 6144" "1 6144" "1 12288" "1 24576" "0 24576"; do set -- $v
timeout 200 python bench.py --config C2 --no-cpu-baseline --no-e2e --tune mid_dmma=$1 --tune tier_m_max=$2 > $O/bench_C2_d$1_m$2.json 2> $O/bench_C2_d$1_m$2.err; python -c "import json; d=json.load(open('$O/bench_C2_d$1_m$2.json')); print('C2 dmma=$1 tmm=$2', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
done
for v in "1 12288" "1 24576" "0 6144"; do set -- $v
timeout 300 python bench.py --config C4 --steps 3 --no-cpu-baseline --no-e2e --tune mid_dmma=$1 --tune tier_m_max=$2 > $O/bench_C4_d$1_m$2.json 2> $O/bench_C4_d$1_m$2.err; python -c "import json; d=json.load(open('$O/bench_C4_d$1_m$2.json')); print('C4 dmma=$1 tmm=$2', round(d['ms_per_step'],3))"
timeout 500 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e --tune mid_dmma=$1 --tune tier_m_max=$2 > $O/bench_C5_d$1_m$2.json 2> $O/bench_C5_d$1_m$2.err; python -c "import json; d=json.load(open('$O/bench_C5_d$1_m$2.json')); print('C5 dmma=$1 tmm=$2', round(d['ms_per_step'],3), {k:round(v,2) for k,v in d['kernel_ms_per_step'].items()})"
done
