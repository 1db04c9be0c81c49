"""Summarise an ncu --set full report: per launch duration, DRAM bytes, issue/pipe use, top stalls."""
import csv, subprocess, sys, io, json

def load(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    return hdr, data

KEYS = {"dur_us": "gpu__time_duration.sum", "dram_rd": "dram__bytes_read.sum", "dram_wr": "dram__bytes_write.sum",
        "issue_pct": "sm__inst_issued.avg.pct_of_peak_sustained_active",
        "fp64_pct": "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "fma_pct": "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "alu_pct": "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "lsu_pct": "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "dram_pct": "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "warps_active": "sm__warps_active.avg.pct_of_peak_sustained_active",
        "regs": "launch__registers_per_thread", "grid": "launch__grid_size",
        "tensor_pct": "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active"}

def main(rep):
    hdr, data = load(rep)
    ix = {h: i for i, h in enumerate(hdr)}
    res = []
    for row in data:
        d = {"kernel": row[ix["Kernel Name"]][:60]}
        for k, m in KEYS.items():
            if m in ix:
                v = row[ix[m]].replace(",", "")
                try: d[k] = float(v)
                except ValueError: d[k] = v
        stalls = {h.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(row[i].replace(",", "") or 0)
                  for h, i in ix.items() if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("not_issued")}
        tot = sum(stalls.values()) or 1
        d["top_stalls"] = {k: round(v / tot, 3) for k, v in sorted(stalls.items(), key=lambda x: -x[1])[:5]}
        res.append(d)
    return res

if __name__ == "__main__":
    for d in main(sys.argv[1]):
        print(json.dumps(d))
