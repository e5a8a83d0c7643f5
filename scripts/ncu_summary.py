"""Summarise the per-query ncu --set full captures of profile_round.sh into
gpurun_out/ncu_full_summary_TAG.json (copy to profiles/ncu_full_summary.json to be read by
bench.py, which uses it only when its source_hash equals the current kernel sources).
    python scripts/ncu_summary.py TAG CONFIG q1,q2,..."""
import csv
import json
import os
import subprocess
import sys

sys.path.insert(0, os.getcwd())
from bench import kernel_source_hash  # noqa: E402

tag, cfg, qs = sys.argv[1], int(sys.argv[2]), sys.argv[3].split(",")
want = {"duration_ms": ("gpu__time_duration.sum", 1e-6), "dram_read": ("dram__bytes_read.sum", 1),
        "dram_write": ("dram__bytes_write.sum", 1), "lts_bytes": ("lts__t_bytes.sum", 1),
        "l2_hit": ("lts__t_sector_hit_rate.pct", 1), "l1_hit": ("l1tex__t_sector_hit_rate.pct", 1),
        "issue_active_pct": ("sm__inst_issued.avg.pct_of_peak_sustained_active", 1),
        "warps_active_pct": ("sm__warps_active.avg.pct_of_peak_sustained_active", 1),
        "inst_executed": ("smsp__inst_executed.sum", 1), "registers": ("launch__registers_per_thread", 1),
        "threads_per_inst": ("smsp__thread_inst_executed_per_inst_executed.ratio", 1),
        "local_load_sectors": ("l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum", 1),
        "local_store_sectors": ("l1tex__t_sectors_pipe_lsu_mem_local_op_st.sum", 1),
        "lts_sectors": ("lts__t_sectors.sum", 1),
        "lts_read_sectors_sm": ("lts__t_sectors_srcunit_tex_op_read.sum", 1),
        "lts_throughput_pct": ("lts__throughput.avg.pct_of_peak_sustained_elapsed", 1)}
scale_units = {"ns": 1, "us": 1e3, "ms": 1e6, "s": 1e9, "byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9,
               "Tbyte": 1e12}
per = {}
for q in qs:
    rep = f"gpurun_out/full_{tag}_{q}.ncu-rep"
    if not os.path.exists(rep):
        continue
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    if len(rows) < 3:
        continue
    hdr, units, r = rows[0], rows[1], rows[2]
    col = {h: i for i, h in enumerate(hdr)}
    d = {}
    for k, (m, sc) in want.items():
        if m not in col:
            continue
        try:
            v = float(r[col[m]].replace(",", ""))
        except ValueError:
            continue
        v *= scale_units.get(units[col[m]], 1)
        d[k] = v * sc
    d["dram_bytes"] = d.get("dram_read", 0) + d.get("dram_write", 0)
    if "lts_bytes" not in d and "lts_sectors" in d:
        d["lts_bytes"] = 32.0 * d["lts_sectors"]
    per[q] = d
l2, l2r = None, None
p = f"gpurun_out/l2_peak_{tag}.json"
if os.path.exists(p):
    lj = json.load(open(p))
    l2 = lj["l2_read_peak_gbs"]
    l2r = lj.get("l2_random_sectors_per_ns")
out = {"round": tag, "config": cfg, "source_hash": kernel_source_hash(), "kernel": "tdfs_kernel<0,0> (count, no stats)",
       "source": "ncu --set full --clock-control none --import-source on, one timed launch per query "
                 "(bench.py --steps 1 --warmup 0 --queries q; -s 1 skips the STATS launch)",
       "l2_peak_gbs": l2, "l2_random_sectors_per_ns": l2r, "per_query": per}
json.dump(out, open(f"gpurun_out/ncu_full_summary_{tag}.json", "w"), indent=1)
for q, d in per.items():
    print(q, {k: round(v, 4) if isinstance(v, float) else v for k, v in d.items()})
