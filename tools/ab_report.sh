# print A/B results: tools/ab_report.sh v1 v2 ...
for v in "$@"; do echo "== $v"; cat gpurun_out/ab_scan_$v.log 2>/dev/null; cat gpurun_out/ab_sha_$v.log 2>/dev/null; python -c "
import json,sys
for l in open('gpurun_out/ab_bench_$v.log'):
  if l.startswith('{'):
    d=json.loads(l); k=d['kernels']
    lat=k.get('stage_latency_ms_per_batch') or {a:b['ms_per_batch'] for a,b in k.items() if isinstance(b,dict) and 'ms_per_batch' in b}
    iso={a:round(k[a]['input_gbs'],1) for a in ('sha1','chunk_stage') if a in k and 'input_gbs' in k[a]}
    print('bench', round(d['value'],1), 'GB/s; e2e', round(d['e2e']['value'],1), '; isolated GB/s', iso, '; roofline frac', round(d['roofline']['frac'],3), '; stage ms:', {a:round(b,3) for a,b in lat.items()})
" 2>/dev/null; done
