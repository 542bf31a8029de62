run() { c=$1; shift; timeout 400 python bench.py --config $c --no-cpu-baseline --no-e2e "$@" > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
cp /tmp/b.json gpurun_out/bench_${c}_$(echo "$*" | tr -c 'a-z0-9\n' '_').json
python -c "import json,sys; d=json.load(open('/tmp/b.json')); print('$c $*', round(d['ms_per_step'],3), round(d['value'],1), {k:round(v,3) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"; }
run C2
run C2 --tune concurrent=0
run C2 --tune tier_m_max=6144
run C2 --tune tier_m_max=0
run C1big
