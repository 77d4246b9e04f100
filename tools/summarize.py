import csv, glob, json
rows=list(csv.reader(open('gpurun_out/launches.csv')))
hdr=[i for i,r in enumerate(rows) if 'Kernel Name' in r][0]
h=rows[hdr]; ki=h.index('Kernel Name'); vi=h.index('Metric Value')
print([(r[ki].split('(')[0].split('::')[-1][:14], r[vi]) for r in rows[hdr+1:hdr+11]])
rows=[]
for l in open('gpurun_out/trace_c32.log'):
    if l.startswith('trace'):
        d=dict(kv.split('=') for kv in l.split()[1:]); rows.append({k:float(v) for k,v in d.items()})
if rows:
    dn=[r['done'] for r in rows]; lat=[r['done']-r['start'] for r in rows]
    print('trace period', (dn[-1]-dn[len(dn)//2])/(len(dn)-1-len(dn)//2), 'mean latency', sum(lat[len(lat)//2:])/len(lat[len(lat)//2:]))
print(open('gpurun_out/probe_host.log').read().strip())
for f in sorted(glob.glob('gpurun_out/bench_b*_s*.log')):
    for l in open(f):
        if l.startswith('{'):
            d=json.loads(l); print(f, round(d['value'],1), 'ms/step', round(d['ms_per_step'],4), 'e2e', round(d['e2e']['value'],1))
