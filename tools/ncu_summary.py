"""Summarise an .ncu-rep (raw metrics + top stall lines)."""
import csv, subprocess, sys
rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(raw.splitlines())); h = rows[0]; v = rows[2]
want = ['Kernel Name', 'gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 'sm__warps_active.avg.pct_of_peak_sustained_active',
        'launch__registers_per_thread', 'smsp__inst_executed.sum', 'launch__grid_size', 'launch__block_size',
        'l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum', 'l1tex__t_sectors_pipe_lsu_mem_global_op_st.sum',
        'l1tex__t_sectors_pipe_lsu_mem_local_op_st.sum', 'lts__t_sectors_srcunit_tex_op_read.sum']
for w in want:
    for i, n in enumerate(h):
        if n == w:
            print(f"  {w:55s} {v[i][:60]} {rows[1][i]}")
st = [(float(v[i]), h[i].replace('smsp__pcsamp_warps_issue_stalled_', '')) for i, n in enumerate(h)
      if 'pcsamp_warps_issue_stalled' in n and 'not_issued' not in n]
print("  stalls:", sorted(st, reverse=True)[:6])
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(src.splitlines()))
if len(rows) > 2:
    h = rows[1]; data = rows[2:]
    i_s = h.index("Warp Stall Sampling (All Samples)")
    tot = sum(int(r[i_s]) for r in data if r[i_s].isdigit())
    top = sorted(((int(r[i_s]), k, r[1]) for k, r in enumerate(data) if r[i_s].isdigit()), reverse=True)[:int(sys.argv[2]) if len(sys.argv) > 2 else 8]
    print("  samples", tot)
    for s_, k, t in top:
        print(f"   {s_:7d} {k:5d} {t.strip()[:70]}")
