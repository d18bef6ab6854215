"""Brief of an ncu --set full report: SOL, memory, occupancy, scheduler, stall samples, smem conflicts."""
import csv, subprocess, sys
rep = sys.argv[1]
d = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(d.splitlines()))
h = r[0]
ki, si, mi, vi, ui = (h.index(x) for x in ('Kernel Name', 'Section Name', 'Metric Name', 'Metric Value', 'Metric Unit'))
keep = ('GPU Speed Of Light Throughput', 'Memory Workload Analysis', 'Occupancy', 'Warp State Statistics',
        'Scheduler Statistics')
for x in r[1:]:
    if x[si] in keep and not any(s in x[mi] for s in ('Cluster', 'Compression', 'Frequency', 'Block Limit')):
        print(f"{x[ki][:14]:14s} {x[mi]:45s} {x[vi]:>14s} {x[ui]}")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rr = list(csv.reader(raw.splitlines()))
hh, vv = rr[0], rr[2]
st = []
for i, n in enumerate(hh):
    if n.startswith('smsp__pcsamp_warps_issue_stalled_') and not n.endswith('not_issued'):
        try:
            v = float(vv[i].replace(',', ''))
        except ValueError:
            continue
        if v > 0:
            st.append((v, n.replace('smsp__pcsamp_warps_issue_stalled_', '')))
    if n in ('l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum', 'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum',
             'dram__bytes_read.sum', 'dram__bytes_write.sum', 'smsp__inst_executed.sum', 'lts__t_sectors.sum',
             'lts__t_sectors_srcunit_tex_op_read.sum', 'l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum',
             'l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum'):
        print(n, vv[i])
tot = sum(v for v, _ in st)
print("stalls:", ", ".join(f"{n} {v / tot * 100:.0f}%" for v, n in sorted(st, reverse=True)[:8]))
