"""Summarise an ncu --set full capture of the matching launches (profile_round.sh) into
profiles/ncu_full_summary.json (bench.py reads dram_bytes_per_launch from it).
    python scripts/ncu_summary.py gpurun_out/full_TAG.ncu-rep TAG q1,q2,...  (queries in launch order)"""
import csv, json, subprocess, sys

rep, tag, qs = sys.argv[1], sys.argv[2], sys.argv[3].split(",")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(raw.splitlines()))
hdr, units, data = rows[0], rows[1], rows[2:]
col = {h: i for i, h in enumerate(hdr)}
want = {"duration_s": ("gpu__time_duration.sum", 1e-9), "dram_read": ("dram__bytes_read.sum", 1),
        "dram_write": ("dram__bytes_write.sum", 1), "l2_hit_pct": ("lts__t_sector_hit_rate.pct", 1),
        "l1_hit_pct": ("l1tex__t_sector_hit_rate.pct", 1),
        "issue_active_pct": ("sm__inst_issued.avg.pct_of_peak_sustained_active", 1),
        "warps_active_pct": ("sm__warps_active.avg.pct_of_peak_sustained_active", 1),
        "inst_executed": ("smsp__inst_executed.sum", 1), "registers": ("launch__registers_per_thread", 1),
        "threads_per_inst": ("smsp__thread_inst_executed_per_inst_executed.ratio", 1)}
scale_units = {"ns": 1, "us": 1e3, "ms": 1e6, "s": 1e9, "byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
per = {}
for q, r in zip(qs, data):
    d = {}
    for k, (m, s) in want.items():
        if m not in col:
            continue
        v = float(r[col[m]].replace(",", ""))
        u = units[col[m]]
        if u in scale_units:
            v *= scale_units[u]
        d[k] = v * s
    d["dram_bytes"] = d.get("dram_read", 0) + d.get("dram_write", 0)
    per[q] = d
out = {"round": tag, "kernel": "tdfs_kernel<0,0> (count, no stats)",
       "source": "ncu --set full --clock-control none --import-source on, the 5 timed launches of bench.py --steps 1 (config 2)",
       "per_query": per,
       "dram_bytes_per_launch": sum(d["dram_bytes"] for d in per.values()) / max(1, len(per)),
       "note": "dram_bytes_per_launch = mean over the five query launches; the C2 CSR (32.5 MB) is L2-resident"}
json.dump(out, open("profiles/ncu_full_summary.json", "w"), indent=1)
for q, d in per.items():
    print(q, {k: round(v, 4) if isinstance(v, float) else v for k, v in d.items()})
