python tools/pcie_bw.py
for ch in 8 32 128; do timeout 600 python bench.py --config C1big --no-cpu-baseline --e2e-chunks $ch --steps 3 > /tmp/b.json 2>/tmp/b.err; tail -1 /tmp/b.err
python -c "import json; d=json.load(open('/tmp/b.json')); print('C1big chunks $ch', round(d['ms_per_step'],3), round(d['value'],1), 'e2e', round(d['e2e']['value'],1), round(d['e2e']['ms_per_step'],2))"; done
for ch in 8 32; do timeout 600 python bench.py --config C2 --no-cpu-baseline --e2e-chunks $ch > /tmp/b.json 2>/tmp/b.err; tail -1 /tmp/b.err
python -c "import json; d=json.load(open('/tmp/b.json')); print('C2 chunks $ch', round(d['ms_per_step'],3), round(d['value'],1), 'e2e', round(d['e2e']['value'],1), round(d['e2e']['ms_per_step'],2))"; done
