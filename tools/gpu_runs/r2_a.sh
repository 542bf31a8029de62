# round 2, first call: GPU suite incl. full-config parity, then bench A/Bs of the panel width
nvidia-smi --query-gpu=name,memory.total --format=csv > gpurun_out/smi.txt; nproc >> gpurun_out/smi.txt; free -g >> gpurun_out/smi.txt; lscpu | grep 'Model name' >> gpurun_out/smi.txt
timeout 1500 python -m pytest tests -q -m gpu -s -p no:randomly > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc $?; tail -3 gpurun_out/pytest_gpu.log; grep '\[parity' gpurun_out/pytest_gpu.log
run() { c=$1; shift; timeout 400 python bench.py --config $c --no-cpu-baseline --no-e2e "$@" > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
cp /tmp/b.json gpurun_out/bench_${c}_$(echo "$*" | tr -c 'a-z0-9\n' '_').json
python -c "import json,sys; d=json.load(open('/tmp/b.json')); print('$c $*', round(d['ms_per_step'],3), round(d['value'],1), {k:round(v,3) for k,v in d['kernel_ms_per_step'].items()}, d['roofline']['kernel'], round(d['roofline']['frac'],3))"; }
run C3
run C3 --tune nb=64
run C3 --tune nb=48
run C5 --steps 3
run C5 --steps 3 --tune nb=64
