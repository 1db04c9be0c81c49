"""Turn one gpu_evidence.sh run (gpurun_out/) into the committed profile summaries.

usage: python tools/make_profiles.py ROUND   (e.g. r01)

reads  gpurun_out/launches.csv      ncu --metrics gpu__time_duration.sum launch list
       gpurun_out/prof_top.ncu-rep  ncu --set full capture of the top kernels
       gpurun_out/bench_full.json   the bench.py JSON line of the same run
writes profiles/<ROUND>_ncu_launches.csv, <ROUND>_ncu_launches_summary.csv,
       <ROUND>_ncu_full_top_kernels.jsonl, <ROUND>_bench.json, ncu_traffic.json
"""
import csv
import json
import os
import shutil
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
import ncu_summary  # noqa: E402

LIMB = 65536 * 8


def launches(rnd, src, dst_dir):
    shutil.copy(src, os.path.join(dst_dir, f"{rnd}_ncu_launches.csv"))
    rows = list(csv.reader(open(src)))
    i = [k for k, r in enumerate(rows) if r and r[0] == "ID"][0]
    h, data = rows[i], rows[i + 1:]
    ik, iv = h.index("Kernel Name"), h.index("Metric Value")
    agg = defaultdict(lambda: [0, 0.0])
    for r in data:
        if len(r) <= iv:
            continue
        name = r[ik].split("(")[0]
        agg[name][0] += 1
        agg[name][1] += float(r[iv].replace(",", "")) / 1e3
    tot = sum(v[1] for v in agg.values())
    with open(os.path.join(dst_dir, f"{rnd}_ncu_launches_summary.csv"), "w") as f:
        f.write("# ncu launch list (gpu__time_duration.sum, --clock-control none) of "
                "bench.py --steps 2 --warmup 1 --graph 0 --streams 1 --no-hoisted\n")
        f.write("# cold-cache, serialised: compare SHARES with bench.py's breakdown, not absolutes\n")
        f.write(f"# {sum(v[0] for v in agg.values())} launches (warmup + 2 steps + profiled pass), "
                f"total {tot:.1f} us\n")
        f.write("kernel,launches,total_us,share\n")
        for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
            f.write(f"{k},{v[0]},{v[1]:.1f},{v[1] / tot:.4f}\n")


# algorithmic bytes of the captured launches (bench.bytes_model per launch), keyed by kernel
# template and launch shape: (regex on the kernel name, limbs read + written, description)
ALGO = [
    ("k_ntt_row<16, 1, 1, 4, 0>", 2 * 108, "ntt_row", "forward row pass over the 108 ModUp limbs (Set-B, l=35, B=1)"),
    ("k_ntt_col<16, 1, 1, 4>", 2 * 108, "ntt_col", "forward column pass over the 108 ModUp limbs (Set-B, l=35, B=1)"),
    ("k_keyip", None, "keyip", "KeyIP over 48 limbs x 3 digits x 2 (evk at 5 B/residue + dhat + acc)"),
]


def traffic(rnd, full):
    out = {"_note": f"DRAM bytes (dram__bytes_read.sum + dram__bytes_write.sum) of one launch from the {rnd} "
                    "ncu --set full capture (--clock-control none); writes still resident in L2 when the launch "
                    "ends are not counted. algo_bytes = read + write of the launch's limbs (8 B words)."}
    for pat, limbs, kind, desc in ALGO:
        hit = [d for d in full if pat in d["kernel"]]
        if not hit:
            continue
        d = hit[0]
        algo = limbs * LIMB if limbs else int((3 * 48 + 2 * 48) * LIMB + 2 * 3 * 48 * 65536 * 5)
        out[kind] = {"bytes_per_launch": int((d["dram_rd"] + d["dram_wr"]) * 1e6), "algo_bytes_per_launch": algo,
                     "launch": desc, "dram_read": int(d["dram_rd"] * 1e6), "dram_write": int(d["dram_wr"] * 1e6),
                     "dur_us_cold": d["dur_us"]}
    if "ntt_row" in out and "ntt_col" in out:        # the NTT as one kind (bench.py's roofline.traffic)
        r, c = out["ntt_row"], out["ntt_col"]
        out["ntt"] = {"bytes_per_launch": r["bytes_per_launch"] + c["bytes_per_launch"],
                      "algo_bytes_per_launch": 108 * 2 * LIMB,
                      "launch": "forward NTT of the 108 ModUp limbs (Set-B, l=35, B=1): column + row pass, FP64 form",
                      "dram_read": r["dram_read"] + c["dram_read"], "dram_write": r["dram_write"] + c["dram_write"],
                      "dur_us_cold": round(r["dur_us_cold"] + c["dur_us_cold"], 3),
                      "source": f"profiles/{rnd}_ncu_full_top_kernels.jsonl (ncu --set full, --clock-control none)"}
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:                                              # keep entries other tools added (warm-cache captures)
        old = json.load(open(path))
        for k, v in old.items():
            out.setdefault(k, v)
    except Exception:
        pass
    json.dump(out, open(path, "w"), indent=1)


def main():
    rnd = sys.argv[1]
    g = os.path.join(ROOT, "gpurun_out")
    dst = os.path.join(ROOT, "profiles")
    if os.path.exists(os.path.join(g, "launches.csv")):
        launches(rnd, os.path.join(g, "launches.csv"), dst)
    if os.path.exists(os.path.join(g, "prof_top.ncu-rep")):
        full = ncu_summary.main(os.path.join(g, "prof_top.ncu-rep"))
        with open(os.path.join(dst, f"{rnd}_ncu_full_top_kernels.jsonl"), "w") as f:
            for d in full:
                f.write(json.dumps(d) + "\n")
        traffic(rnd, full)
    if os.path.exists(os.path.join(g, "bench_full.json")):
        shutil.copy(os.path.join(g, "bench_full.json"), os.path.join(dst, f"{rnd}_bench.json"))


if __name__ == "__main__":
    main()
