import json, sys
for f in sys.argv[1:]:
    d = json.loads(open(f).read().strip().splitlines()[-1])
    print(f, d.get('sgemm_impl'), 'value', round(d['value']), 'ms', round(d['ms_per_step'], 3),
          'one_stream', round(d['one_stream']['value']), 'e2e', d['e2e'] and round(d['e2e']['value']))
    print(' roof', {k: (round(v, 3) if isinstance(v, float) else v) for k, v in d['roofline'].items() if k != 'peak_source'})
    for k, v in d['per_kernel'].items():
        print('  ', k, {kk: round(vv, 3) for kk, vv in v.items()})
    print(' serial', {k: round(v['value']) for k, v in d['serial'].items()}, 'speedup',
          {k: round(v, 2) for k, v in d['speedup_vs_serial'].items()}, 'hbm', round(d['hbm_gbs_membound']), d['clocks'])
