"""Per-kernel shared-memory wavefronts / bank conflicts and pipe use from an ncu report."""
import csv, io, subprocess, sys
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[0]
want = ["gpu__time_duration.sum", "launch__grid_size", "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_issued.avg.pct_of_peak_sustained_active", "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"]
short = ["us", "grid", "lds_wf", "lds_conf", "sts_wf", "sts_conf", "fp64%", "issue%", "l1%", "dram%"]
for r in rows[2:]:
    vals = []
    for k in want:
        v = r[h.index(k)] if k in h else "-"
        vals.append(v)
    print(r[h.index("Kernel Name")][:34].ljust(34), " ".join(f"{s}={v}" for s, v in zip(short, vals)))
