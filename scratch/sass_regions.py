# stall samples / instructions of a k_update_tc ncu capture summed by SASS index ranges (roles)
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]; data = [dict(zip(h, x)) for x in rows[2:] if len(x) == len(h)]
S = 'Warp Stall Sampling (All Samples)'
cols = [c for c in h if c.startswith('stall_') and 'Not Issued' not in c]
tot = sum(float(x[S] or 0) for x in data); itot = sum(float(x['Instructions Executed'] or 0) for x in data)
regions = [tuple(int(v) if v.isdigit() else v for v in r.split(':')) for r in sys.argv[2:]]
for name, a, b in regions:
    seg = data[a:b]
    s = sum(float(x[S] or 0) for x in seg); ins = sum(float(x['Instructions Executed'] or 0) for x in seg)
    st = sorted(((sum(float(x[c] or 0) for x in seg), c[6:]) for c in cols), reverse=True)[:5]
    print(f"{name:12s} samples {s/tot:.3f} inst {ins/itot:.3f} ({ins:.3g})  " + ' '.join(f"{c}={v/max(s,1):.2f}" for v, c in st))
