"""Summarise an ncu launch list (gpu__time_duration.sum CSV) per kernel."""
import csv
import sys
from collections import defaultdict

path = sys.argv[1]
rows = list(csv.reader(open(path)))
hdr = [i for i, r in enumerate(rows) if 'Kernel Name' in r][0]
h = rows[hdr]
ki, vi, ui = h.index('Kernel Name'), h.index('Metric Value'), h.index('Metric Unit')
agg = defaultdict(list)
for r in rows[hdr + 1:]:
    if len(r) <= vi or not r[vi]:
        continue
    v = float(r[vi].replace(',', ''))
    u = r[ui]
    us = v / 1000.0 if u in ('nsecond', 'ns') else (v * 1000.0 if u in ('msecond', 'ms') else v)
    name = r[ki].split('(')[0].split('<')[0].split('::')[-1].strip()
    agg[name].append(us)
tot = sum(sum(v) for v in agg.values())
print('| kernel | launches | mean us | share of summed time |')
print('|---|---|---|---|')
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print(f'| {k} | {len(v)} | {sum(v)/len(v):.1f} | {100*sum(v)/tot:.1f}% |')
