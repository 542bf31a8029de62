timeout 600 python -m pytest tests/test_gpu_getrf.py -q -x -p no:randomly -k "outer_strip or two_level or two_parts" > gpurun_out/pytest_gpu_l.log 2>&1; echo pytest rc $?; tail -2 gpurun_out/pytest_gpu_l.log
run() { c=$1; shift; timeout 400 python bench.py --config $c --no-cpu-baseline --no-e2e "$@" > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
cp /tmp/b.json gpurun_out/bench_${c}_$(echo "$*" | tr -c 'a-z0-9\n' '_').json
python -c "import json,sys; d=json.load(open('/tmp/b.json')); print('$c $*', round(d['ms_per_step'],3), round(d['value'],1), {k:round(v,3) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"; }
run C3 --tune outer_cols=32
run C5 --steps 3 --tune outer_cols=32
run C3 --tune nb=64
run C5 --steps 3 --tune nb=64
for v in "-DXGEMM_BK=32 -DXGEMM_ST=2" "-DXGEMM_BK=32 -DXGEMM_ST=3"; do
  IRR_NVCC_EXTRA="$v" python -m paper_conf_sc_abdelfattahgbtld22_b200.build --force > gpurun_out/build_var.log 2>&1 || { echo build failed; tail -5 gpurun_out/build_var.log; }
  echo "== $v"
  run C3
  run C5 --steps 3
done
python -m paper_conf_sc_abdelfattahgbtld22_b200.build --force > /dev/null 2>&1
