import json, sys
for f in sys.argv[1:]:
    for l in open(f):
        if l.startswith('{'):
            d = json.loads(l)
            print(f, 'value %.4g  ms/step %.1f  e2e %s' % (d['value'], d['ms_per_step'], ('%.4g' % d['e2e']['value']) if d.get('e2e') else None))
            print('  roof', {k: v for k, v in d['roofline'].items() if k in ('kernel', 'achieved', 'frac', 'kernel_ms')})
            print('  kern', {k: round(v, 2) for k, v in d['kernel_time_ms'].items()})
            print('  phase', {k: round(v, 1) for k, v in d['phase_ms_last_step'].items()})
            if d.get('cpu_baseline'): print('  cpu', d['cpu_baseline'])
            print('  clocks', d.get('clocks'))
        elif 'rc=' in l or 'Error' in l or 'error' in l: print(f, l.strip()[:300])
