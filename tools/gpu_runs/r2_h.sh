run() { c=$1; shift; timeout 400 python bench.py --config $c --no-cpu-baseline --no-e2e "$@" > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
cp /tmp/b.json gpurun_out/bench_${c}_$(echo "$*" | tr -c 'a-z0-9\n' '_').json
python -c "import json,sys; d=json.load(open('/tmp/b.json')); print('$c $*', round(d['ms_per_step'],3), round(d['value'],1), {k:round(v,3) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"; }
run C3 --tune xgemm_warps=16
run C3 --tune l1_rows=512
run C3 --tune l1_rows=1024
run C3 --tune l1_rows=1024 --tune l1_ctas_per_sm=2
run C5 --steps 3 --tune xgemm_warps=16
run C5 --steps 3 --tune l1_rows=512
