import json, sys
for f in sys.argv[1:]:
    try:
        l = [x for x in open(f) if x.startswith('{')]
        d = json.loads(l[-1]); r = d['roofline']; h = d['roofline_hbm']
        print('%-40s value %.3e ms/step %.3f variant %s kernel_ms %.4f %s frac %.3f ach %.1f %s | hbm %.0f GB/s (%.3f)' % (
            f, d['value'], d['ms_per_step'], d['config']['variant'], r['kernel_ms'], r['bound'], r['frac'], r['achieved'],
            r['unit'], h['achieved'], h['frac']))
    except Exception as e:
        print(f, 'ERR', e, open(f).read()[-600:])
