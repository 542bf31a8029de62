import json,sys
for f in sys.argv[1:]:
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, 'ERR', e); continue
    print(f, 'value %.1f Gflop/s ms/step %.3f'%(d['value'],d['ms_per_step']), 'launches',d.get('gpu_launches'))
    r=d['roofline']; print('  roof', r['kernel'], r['bound'], '%.1f %s frac %.3f share %.2f'%(r['achieved'],r['unit'],r['frac'],r['share_of_step']))
    print('  whole', {k:round(v,4) for k,v in d['whole_step'].items() if 'frac' in k})
    print('  kms', {k:round(v,4) for k,v in d['kernel_ms_per_step'].items()})
    if d.get('e2e'): print('  e2e %.1f'%d['e2e']['value'])
