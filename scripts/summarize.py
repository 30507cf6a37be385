import json, sys
for f in sys.argv[1:]:
    try:
        l = [x for x in open(f) if x.startswith('{')]
        d = json.loads(l[-1]); r = d['roofline']; h = d['roofline_secondary']
        print('%-34s value %.3e ms/step %.3f %s kernel_ms %.4f | %s %.1f %s frac %.3f | %s %.1f %s frac %.3f | e2e %s' % (
            f, d['value'], d['ms_per_step'], d['config'].get('kernel'), r['kernel_ms'], r['bound'], r['achieved'], r['unit'],
            r['frac'], h['bound'], h['achieved'], h['unit'], h['frac'], (d.get('e2e') or {}).get('value')))
    except Exception as e:
        print(f, 'ERR', e, open(f).read()[-600:])
