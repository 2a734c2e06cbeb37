# summarise an ncu launch list (gpu__time_duration per kernel): totals and the big launches in order
import csv, sys
from collections import defaultdict
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]; d = [dict(zip(h, r)) for r in rows[1:]]
agg = defaultdict(float); cnt = defaultdict(int); seq = []
for x in d:
    if x['Metric Name'] != 'gpu__time_duration.sum': continue
    v = float(x['Metric Value'].replace(',', ''))
    v *= {'nsecond': 1, 'ns': 1, 'usecond': 1e3, 'us': 1e3, 'msecond': 1e6, 'ms': 1e6}.get(x['Metric Unit'], 1)
    k = x['Kernel Name'][:60]
    agg[k] += v; cnt[k] += 1; seq.append((k, v))
tot = sum(agg.values())
for k, v in sorted(agg.items(), key=lambda t: -t[1])[:15]:
    print(f"{v/1e6:9.3f} ms {cnt[k]:4d} {v/tot:6.3f} {k}")
print("launches > 0.5 ms in order:", [(k[:24], round(v / 1e6, 2)) for k, v in seq if v > 5e5])
