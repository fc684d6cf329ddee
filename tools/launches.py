import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
hdr = None; seq = []
for r in rows:
    if r and r[0] == 'ID': hdr = r; continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d['Metric Name'] != 'gpu__time_duration.sum': continue
        v = float(d['Metric Value'].replace(',', ''))
        u = d['Metric Unit']
        v = v / 1000 if u == 'nsecond' else (v * 1000 if u == 'msecond' else v)
        seq.append((d['Kernel Name'].split('(')[0][:48], d['Grid Size'], v))
agg = collections.defaultdict(lambda: [0, 0.0])
for n, g, v in seq: agg[n][0] += 1; agg[n][1] += v
tot = sum(v for _, _, v in seq)
for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]): print(f"{t:10.1f} us {100*t/tot:5.1f}% {c:5d}  {k}")
if len(sys.argv) > 2:
    for n, g, v in seq[:int(sys.argv[2])]: print(f"{v:9.1f}  {g:>16}  {n}")
