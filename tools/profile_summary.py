"""Write profiles/<tag>_ncu_summary.md + profiles/ncu_traffic.json from
gpurun_out/bench_launches.csv and gpurun_out/prof_full.ncu-rep."""
import csv
import os
import re
import json
import subprocess
import sys
from collections import defaultdict

tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
BATCH = 64 << 20


def kname(full):
    s = re.sub(r'\(anonymous namespace\)::|<unnamed>::|^void ', '', full)
    return s.split('(')[0].split('<')[0].split('::')[-1].strip()


def launch_table(path):
    rows = list(csv.reader(open(path)))
    hdr = [i for i, r in enumerate(rows) if 'Kernel Name' in r][0]
    h = rows[hdr]
    ki, vi, ui = h.index('Kernel Name'), h.index('Metric Value'), h.index('Metric Unit')
    agg = defaultdict(list)
    for r in rows[hdr + 1:]:
        if len(r) <= vi or not r[vi]:
            continue
        v = float(r[vi].replace(',', ''))
        us = v / 1000.0 if r[ui] in ('nsecond', 'ns') else (v * 1000.0 if r[ui] in ('msecond', 'ms') else v)
        agg[kname(r[ki])].append(us)
    tot = sum(sum(v) for v in agg.values())
    out = ['| kernel | launches | mean us | share of summed time |', '|---|---|---|---|']
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        out.append(f'| {k} | {len(v)} | {sum(v)/len(v):.1f} | {100*sum(v)/tot:.1f}% |')
    return out


M = ['gpu__time_duration.sum', 'smsp__inst_executed.sum', 'sm__inst_executed.avg.per_cycle_active',
     'smsp__issue_active.avg.pct_of_peak_sustained_active', 'sm__warps_active.avg.pct_of_peak_sustained_active',
     'sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active',
     'sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active',
     'sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active',
     'smsp__thread_inst_executed_per_inst_executed.ratio', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
     'launch__registers_per_thread', 'launch__grid_size', 'launch__block_size', 'sm__cycles_active.avg',
     'sm__inst_executed_pipe_alu.sum', 'sm__inst_executed_pipe_fmaheavy.sum']


def full_table(rep):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv', '--print-units', 'base'],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h = rows[0]
    lines = ['| kernel | ' + ' | '.join(m.split('.')[0].replace('__', ' ') + ('' if '.sum' not in m else ' (sum)') for m in M) + ' | top stalls per issue |',
             '|---' * (len(M) + 2) + '|']
    traffic = {}
    for r in rows[2:]:
        name = kname(r[h.index('Kernel Name')])
        vals = [r[h.index(m)] if m in h else '' for m in M]
        st = [(k.split('issue_stalled_')[1].split('_per')[0], float(r[i])) for i, k in enumerate(h)
              if k.startswith('smsp__average_warps_issue_stalled_') and k.endswith('per_issue_active.ratio') and r[i]]
        st.sort(key=lambda x: -x[1])
        lines.append(f'| {name} | ' + ' | '.join(vals) + ' | ' + ', '.join(f'{a} {b:.2f}' for a, b in st[:4]) + ' |')
        rd = float(r[h.index('dram__bytes_read.sum')]) + float(r[h.index('dram__bytes_write.sum')])
        traffic[name] = rd
    return lines, traffic


lt = launch_table('gpurun_out/bench_launches.csv')
ft, traffic = full_table('gpurun_out/prof_full.ncu-rep')
md = [f'# {tag} profiles (B200, sm_100a)', '',
      'Commands (under gpurun, one GPU): `bash tools/gpu_profiles.sh`', '',
      '```', open('tools/gpu_profiles.sh').read().strip(), '```', '',
      '## Launch list of the bench step (`bench.py --step-only`: warm-up + timed steps; cold-cache, serialised by ncu: shares, not absolutes)', '']
md += lt
md += ['', '## ncu --set full, 64 MiB batches of C3 (tools/one_batch.py)', '',
       'Units: ns, instructions, %, bytes.  `dram` = DRAM bytes of the launch.', '']
md += ft
if os.path.exists('gpurun_out/prof_sha.ncu-rep'):
    sh, _ = full_table('gpurun_out/prof_sha.ncu-rep')
    md += ['', '## ncu --set full, the SHA-1 kernel alone on all 672 MiB of C3 chunks '
               '(tools/sha_sizes.py, one launch)', '']
    md += sh
if os.path.exists('gpurun_out/prof_roll.ncu-rep'):
    rl, _ = full_table('gpurun_out/prof_roll.ncu-rep')
    md += ['', '## ncu --set full, the roll and tile-selection kernels over all 672 MiB of C3 '
               '(tools/scan_sizes.py, one op_chunk launch: 512-byte lanes)', '']
    md += rl
if os.path.exists('gpurun_out/prof_fm.ncu-rep'):
    fm, fm_traffic = full_table('gpurun_out/prof_fm.ncu-rep')
    md += ['', '## ncu --set full, row NEXT-1 FindMatch, one 64 MiB batch of C2 (tools/fm_sizes.py)', '']
    md += fm
    traffic.update({'findmatch_' + k: v for k, v in fm_traffic.items()})
open(f'profiles/{tag}_ncu_summary.md', 'w').write('\n'.join(md) + '\n')
tj = {"_source": "ncu --set full, tools/one_batch.py (64 MiB batches of C3); DRAM read+write bytes per "
                 "launch; bench scales per input byte", "capture_batch_bytes": BATCH}
name_map = {'sha1_kernel': 'sha1', 'rabin_roll_kernel': 'rabin_roll', 'select_emit_ev_kernel': 'select_emit',
            'table_insert_kernel': 'table_insert'}
for k, v in traffic.items():
    tj[name_map.get(k, k)] = v
json.dump(tj, open('profiles/ncu_traffic.json', 'w'), indent=1)
print('\n'.join(md))
