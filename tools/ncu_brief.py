"""Key metrics of one kernel from an ncu report.  Usage: python tools/ncu_brief.py rep [kernel-regex]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
args = ["ncu", "-i", rep, "--page", "raw", "--csv"]
if len(sys.argv) > 2:
    args += ["-k", "regex:" + sys.argv[2]]
rows = list(csv.reader(io.StringIO(subprocess.run(args, capture_output=True, text=True).stdout)))
h, units = rows[0], rows[1]
keys = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'smsp__inst_executed.sum',
        'sm__warps_active.avg.per_cycle_active', 'launch__registers_per_thread',
        'l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed',
        'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed',
        'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum', 'l1tex__data_pipe_lsu_wavefronts.sum',
        'smsp__thread_inst_executed_per_inst_executed.ratio', 'lts__t_sector_hit_rate.pct',
        'l1tex__t_sector_hit_rate.pct', 'lts__t_sectors_srcunit_tex_op_read.sum',
        'lts__t_sectors_srcunit_tex_op_red.sum', 'lts__throughput.avg.pct_of_peak_sustained_elapsed',
        'l1tex__throughput.avg.pct_of_peak_sustained_active', 'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed']
for v in rows[2:]:
    print('==', v[h.index('Kernel Name')][:70])
    for k in keys:
        if k in h:
            i = h.index(k)
            print(f'  {k:80s} {v[i]} {units[i]}')
    st = []
    for i, k in enumerate(h):
        if k.startswith('smsp__average_warp_latency_issue_stalled_') or k.startswith('smsp__average_warps_issue_stalled_'):
            if k.endswith('_per_issue_active.ratio'):
                try:
                    st.append((float(v[i]), k.split('stalled_')[1].replace('_per_issue_active.ratio', '')))
                except ValueError:
                    pass
    st.sort(reverse=True)
    print('  stalls/issue:', ', '.join(f'{n} {x:.2f}' for x, n in st[:8]))
