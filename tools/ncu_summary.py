"""Key metrics of an ncu report (raw page) per kernel."""
import csv
import subprocess
import sys

KEYS = ['gpu__time_duration.sum', 'smsp__inst_executed.sum', 'sm__inst_executed.avg.per_cycle_active',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'sm__warps_active.avg.pct_of_peak_sustained_active',
        'sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active',
        'sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active',
        'sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active',
        'smsp__thread_inst_executed_per_inst_executed.ratio', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum', 'l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum',
        'l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum', 'launch__registers_per_thread', 'launch__grid_size',
        'launch__block_size', 'launch__occupancy_limit_registers', 'sm__cycles_active.avg']
out = subprocess.run(['ncu', '-i', sys.argv[1], '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h, u = rows[0], rows[1]
for r in rows[2:]:
    print('==', r[h.index('Kernel Name')][:60])
    for k in KEYS:
        if k in h:
            print(f'  {k} = {r[h.index(k)]} {u[h.index(k)]}')
    st = [(k.split('issue_stalled_')[1].split('_per')[0], float(r[i])) for i, k in enumerate(h)
          if k.startswith('smsp__average_warps_issue_stalled_') and k.endswith('per_issue_active.ratio') and r[i]]
    st.sort(key=lambda x: -x[1])
    print('  stalls/issue:', ', '.join(f'{a} {b:.2f}' for a, b in st[:8]))
