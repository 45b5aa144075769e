"""Key metrics + stall reasons from an ncu report."""
import csv, subprocess, sys, io
rep = sys.argv[1]
raw = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
hdr, units = r[0], r[1]
keys = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum', 'smsp__inst_executed.sum',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'smsp__issue_active.avg.pct_of_peak_sustained_active',
        'sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active', 'launch__registers_per_thread',
        'l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum', 'dram__throughput.avg.pct_of_peak_sustained_elapsed',
        'lts__t_bytes.sum', 'l1tex__t_bytes.sum', 'smsp__warps_eligible.avg.per_cycle_active',
        'smsp__warps_active.avg.per_cycle_active', 'launch__occupancy_limit_registers', 'launch__occupancy_limit_shared_mem']
for row in r[2:]:
    print(row[hdr.index('Kernel Name')][:60])
    for k in keys:
        if k in hdr:
            print('   %-70s %s %s' % (k, row[hdr.index(k)], units[hdr.index(k)]))
    st = []
    for h, v in zip(hdr, row):
        if h.startswith('smsp__pcsamp_warps_issue_stalled') and not h.endswith('not_issued'):
            try:
                st.append((float(v), h.replace('smsp__pcsamp_warps_issue_stalled_', '')))
            except ValueError:
                pass
    tot = sum(x for x, _ in st) or 1
    print('   stalls:', ', '.join('%s %.0f%%' % (h, 100 * x / tot) for x, h in sorted(st, reverse=True)[:9]))
