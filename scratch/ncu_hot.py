import csv, subprocess, sys
rep = sys.argv[1]; frac = float(sys.argv[2]) if len(sys.argv) > 2 else 0.25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
blocks = []; cur = None
for r in rows:
    if r and r[0] == 'Kernel Name': cur = []; blocks.append(cur); continue
    if cur is not None: cur.append(r)
b = blocks[0]; h = b[0]; data = [dict(zip(h, r)) for r in b[1:] if len(r) == len(h)]
ie = [int(d['Instructions Executed'] or 0) for d in data]
st = [int(d['Warp Stall Sampling (All Samples)'] or 0) for d in data]
tot = sum(ie); mx = max(ie)
print("total warp-inst", tot, "max line count", mx)
for i, d in enumerate(data):
    if ie[i] >= frac * mx:
        print(f"{i:5d} {ie[i]/mx:5.2f} {st[i]:7d} {d['Source'][:95]}")
# group by execution count buckets (regions)
import collections
reg = collections.OrderedDict()
for i, d in enumerate(data):
    if ie[i] == 0: continue
    key = round(ie[i] / mx, 3)
    reg.setdefault(key, [0, 0, i, i])
    reg[key][0] += ie[i]; reg[key][1] += 1; reg[key][3] = i
print("---- regions by count (share of total inst) ----")
for k, (s, c, a, b_) in sorted(reg.items(), key=lambda x: -x[1][0])[:20]:
    print(f"count/max={k:6.3f} lines={c:4d} share={s/tot:5.3f} first={a} last={b_}  e.g. {data[a]['Source'][:60]}")
