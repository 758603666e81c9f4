#!/usr/bin/env python
"""Summarise ncu output brought back in gpurun_out/ into profiles/ (tracked).

    python scripts/ncu_summary.py --launches gpurun_out/launches_c3.csv \
        --rep gpurun_out/prof_c3.ncu-rep --key nw_n32768_p10/tile0 --tag r01

Writes profiles/<tag>_launches.csv (the per-launch device times, copied), a one-page text
summary profiles/<tag>_<key>.txt with the key metrics of the full capture, and updates
profiles/ncu_traffic.json[key] = dram read+write bytes per launch (bench.py `roofline.traffic`).
"""
import argparse
import csv
import io
import json
import os
import shutil
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PROF = os.path.join(ROOT, "profiles")

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "launch__shared_mem_per_block_dynamic", "launch__occupancy_limit_shared_mem",
    "sm__inst_executed.sum", "smsp__inst_executed.avg.per_cycle_active", "sm__cycles_elapsed.avg",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "lts__t_bytes.sum",
    "smsp__average_warp_latency_issue_stalled_barrier", "gpc__cycles_elapsed.max",
    "sm__cycles_active.avg", "smsp__cycles_active.avg", "dram__cycles_active.avg",
]


def raw_metrics(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return []
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        res.append({h: (v, u) for h, u, v in zip(hdr, units, r)})
    return res


def stall_reasons(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return {}
    hdr = rows[0]
    vals = rows[2]
    st = {}
    for h, v in zip(hdr, vals):
        if h.startswith("smsp__average_warp_latency_issue_stalled_") or h.startswith("smsp__pcsamp_warps_issue_stalled_"):
            try:
                st[h] = float(v.replace(",", ""))
            except ValueError:
                pass
    return dict(sorted(st.items(), key=lambda kv: -kv[1])[:14])


def to_float(v):
    try:
        return float(str(v).replace(",", ""))
    except ValueError:
        return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--launches")
    ap.add_argument("--rep")
    ap.add_argument("--key", required=True)
    ap.add_argument("--tag", default="r01")
    a = ap.parse_args()
    os.makedirs(PROF, exist_ok=True)
    safe = a.key.replace("/", "_")
    lines = [f"# ncu summary {a.tag} {a.key}", ""]
    if a.launches and os.path.exists(a.launches):
        shutil.copy(a.launches, os.path.join(PROF, f"{a.tag}_{safe}_launches.csv"))
        lines.append(f"launch list: {a.tag}_{safe}_launches.csv (ncu --metrics gpu__time_duration.sum "
                     "--clock-control none; cold-cache, serialised)")
    if a.rep and os.path.exists(a.rep):
        ms = raw_metrics(a.rep)
        for i, m in enumerate(ms):
            name = m.get("Kernel Name", ("?", ""))[0]
            lines.append(f"\n## launch {i}: {name}")
            for k in KEYS:
                if k in m:
                    lines.append(f"  {k:70s} {m[k][0]:>20s} {m[k][1]}")
            rd, wr = to_float(m.get("dram__bytes_read.sum", ("", ""))[0]), to_float(m.get("dram__bytes_write.sum", ("", ""))[0])
            if rd is not None and wr is not None:
                scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
                rd *= scale.get(m["dram__bytes_read.sum"][1], 1)
                wr *= scale.get(m["dram__bytes_write.sum"][1], 1)
                lines.append(f"  dram read+write bytes per launch: {rd + wr:.6e}")
                tj = os.path.join(PROF, "ncu_traffic.json")
                d = json.load(open(tj)) if os.path.exists(tj) else {}
                d[a.key] = rd + wr
                json.dump(d, open(tj, "w"), indent=1, sort_keys=True)
        sr = stall_reasons(a.rep)
        if sr:
            lines.append("\n## top stall reasons (launch 0)")
            for k, v in sr.items():
                lines.append(f"  {k:80s} {v:10.3f}")
    with open(os.path.join(PROF, f"{a.tag}_{safe}.txt"), "w") as f:
        f.write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
