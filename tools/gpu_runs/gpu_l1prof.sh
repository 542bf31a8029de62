python tools/phase_time.py --config C2 --tune tier_m_max=0 --tune concurrent=0 > gpurun_out/phase_C2.txt 2>&1
python tools/phase_time.py --config C2 --tune tier_m_max=0 --tune concurrent=0 --tune nb=16 > gpurun_out/phase_C2_nb16.txt 2>&1
cat gpurun_out/phase_C2.txt gpurun_out/phase_C2_nb16.txt
for t in "nb=16" "nb=24" "l1_ctas_per_sm=2"; do timeout 300 python bench.py --config C2 --no-cpu-baseline --no-e2e --tune $t > /tmp/b.json 2>/tmp/b.err; tail -2 /tmp/b.err
python -c "import json,sys; d=json.load(open('/tmp/b.json')); print('C2 $t', round(d['ms_per_step'],3), round(d['value'],1), {k:round(v,3) for k,v in d['kernel_ms_per_step'].items()})"; done
ncu --set full --clock-control none --import-source on -k regex:lu_l1_kernel -c 1 -o gpurun_out/prof_l1_C2 python tools/prof_one.py --config C2 --reps 1 > gpurun_out/ncu_l1.log 2>&1
