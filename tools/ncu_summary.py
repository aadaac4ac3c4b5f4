"""Summarise an .ncu-rep: per launch duration, throughput, occupancy, instr/issue, stalls."""
import csv, subprocess, sys, io
rep = sys.argv[1]
out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(out)))
hdr, units = r[0], r[1]
def g(row, name):
    try: return row[hdr.index(name)]
    except ValueError: return '?'
cols = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum', 'smsp__inst_executed.sum',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'smsp__issue_active.avg.pct_of_peak_sustained_active',
        'lts__t_sector_hit_rate.pct', 'l1tex__t_sector_hit_rate.pct', 'smsp__thread_inst_executed_per_inst_executed.ratio',
        'lts__t_sectors.sum', 'launch__registers_per_thread', 'launch__grid_size', 'launch__block_size']
for row in r[2:]:
    print('==', g(row, 'ID'), g(row, 'Kernel Name')[:60])
    for c in cols:
        print(f'    {c:60s} {g(row, c)} {units[hdr.index(c)] if c in hdr else ""}')
    st = {}
    for i, h in enumerate(hdr):
        if h.startswith('smsp__pcsamp_warps_issue_stalled_') and not h.endswith('not_issued'):
            try: st[h[len('smsp__pcsamp_warps_issue_stalled_'):]] = float(row[i])
            except: pass
    tot = sum(st.values()) or 1
    print('    stalls:', ', '.join(f'{k} {100*v/tot:.0f}%' for k, v in sorted(st.items(), key=lambda x: -x[1])[:6]))
