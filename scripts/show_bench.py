import json, sys
for f in sys.argv[1:]:
    for ln in open(f):
        if ln.startswith('{'):
            d = json.loads(ln)
            print(f, 'value', round(d['value']), 'ms', round(d['ms_per_step'], 4),
                  'e2e', round(d['e2e']['value']) if d.get('e2e') else None,
                  'train', d['train'] and round(d['train']['value']),
                  'ev_ms', d.get('kernel_timing', {}).get('ms_per_step_with_events'))
            print('  kernels(ms/step)', {k: round(v, 4) for k, v in d['kernel_ms_per_step'].items()})
            if d.get('bf16'):
                bb = d['bf16']
                print('  bf16 value', round(bb['value']), 'ms', round(bb['ms_per_step'], 4),
                      {k: round(v, 4) for k, v in bb['kernel_ms_per_step'].items()})
            print('  roofline', {k: (round(v, 3) if isinstance(v, float) else v) for k, v in d['roofline'].items()})
            print('  agg GB/s', d['aggregation']['achieved'], 'clocks', d['clocks'])
            if d.get('train') and d['train'].get('kernel_ms_per_step'):
                print('  train ms', round(d['train']['ms_per_step'], 3), {k: round(v, 3) for k, v in sorted(d['train']['kernel_ms_per_step'].items(), key=lambda x: -x[1])})
        elif ln.startswith('==='):
            print(ln.strip())
        elif ln.strip():
            print('  ', ln.strip()[:200])
