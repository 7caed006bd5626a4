"""stall breakdown (warp cycles per issued instruction by reason) from ncu --page raw csv files"""
import csv, sys
tabs = []
for fn in sys.argv[1:]:
    rows = list(csv.reader(open(fn)))
    h, u, v = rows[0], rows[1], rows[2]
    tabs.append({a: b for a, b in zip(h, v)})
keys = [k for k in tabs[0] if k.startswith('smsp__average_warps_issue_stalled_') and k.endswith('_per_issue_active.ratio')]
keys.sort(key=lambda k: -float(tabs[0][k] or 0))
for k in keys:
    vals = [t.get(k, '-') for t in tabs]
    if max(float(x or 0) for x in vals) < 0.05: continue
    print(f"{k[len('smsp__average_warps_issue_stalled_'):-len('_per_issue_active.ratio')]:24s}", " ".join(f"{float(x):8.2f}" for x in vals))
for k in ['dram__bytes_read.sum', 'dram__bytes_write.sum', 'smsp__inst_executed.sum', 'lts__t_sectors_srcunit_tex_op_write.sum', 'lts__t_sectors_srcunit_tex_op_read.sum', 'l1tex__t_requests_pipe_lsu_mem_global_op_st.sum', 'l1tex__t_sectors_pipe_lsu_mem_global_op_st.sum']:
    print(k, [t.get(k) for t in tabs])
