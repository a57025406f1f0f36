#!/usr/bin/env python
"""Key metrics per kernel from an `ncu --page raw --csv` export:
python scripts/ncu_brief.py raw.csv"""
import csv
import sys
rows = list(csv.reader(open(sys.argv[1])))
h, units, data = rows[0], rows[1], rows[2:]
col = {c: i for i, c in enumerate(h)}
want = ['gpu__time_duration.sum', 'sm__warps_active.avg.pct_of_peak_sustained_active',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'smsp__thread_inst_executed_per_inst_executed.ratio',
        'smsp__inst_executed.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum', 'lts__t_bytes.sum',
        'launch__occupancy_limit_shared_mem', 'launch__occupancy_limit_registers', 'launch__registers_per_thread',
        'launch__shared_mem_per_block_dynamic', 'launch__grid_size', 'launch__block_size',
        'l1tex__t_bytes_pipe_lsu_mem_local_op_ld.sum', 'l1tex__t_bytes_pipe_lsu_mem_local_op_st.sum']
for d in data:
    print('----', d[col['Kernel Name']][:70])
    for w in want:
        if w in col:
            print(f"  {w}: {d[col[w]]} {units[col[w]]}")
    st = []
    for c, i in col.items():
        if c.startswith('smsp__pcsamp_warps_issue_stalled') and not c.endswith('not_issued'):
            try:
                st.append((float(d[i].replace(',', '') or 0), c.replace('smsp__pcsamp_warps_issue_stalled_', '')))
            except ValueError:
                pass
    st.sort(reverse=True)
    tot = sum(v for v, _ in st) or 1
    print('  stalls %:', ', '.join(f"{c} {100 * v / tot:.1f}" for v, c in st[:8]))
