import json, sys
for fn in sys.argv[1:]:
    for l in open(fn):
        d = json.loads(l)
        print(d['matrix'], d['m'], d['nnz'], d['dtype'])
        for f, r in d['formats'].items():
            if isinstance(r, str):
                print('   ', f, r); continue
            print('   %-4s %8.1fMB hot %7.1fus %6.0fGB/s  cold %7.1fus %6.0fGB/s frac %.2f conv %.0fus v%d' % (
                f, r['bytes'] / 1e6, r['hot_us'], r['hot_gbs'], r.get('cold_us', 0), r.get('cold_gbs', 0),
                r.get('cold_frac', 0), r['convert_us_incl_features'], r['variant']))
