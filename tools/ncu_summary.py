#!/usr/bin/env python
"""Summarise ncu outputs brought back in gpurun_out/ into profiles/ (tracked).

    python tools/ncu_summary.py --tag r01_cfg2 --launches gpurun_out/launches_cfg2.csv \
        --rep gpurun_out/prof_cfg2.ncu-rep --traffic-json profiles/traffic_cfg2.json
"""
import argparse
import csv
import io
import json
import os
import subprocess
from collections import defaultdict

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__bytes_read.sum.per_second", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__occupancy_limit_registers", "sm__inst_executed.sum",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fmaheavy.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.avg.per_cycle_active", "sm__instruction_throughput.avg.pct_of_peak_sustained_active",
        "l1tex__t_bytes.sum", "lts__t_bytes.sum", "launch__shared_mem_per_block_static",
        "smsp__average_warp_latency_issue_stalled", "sm__cycles_elapsed.avg.per_second"]


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hdr]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    d = defaultdict(list)
    for r in rows[hdr + 1:]:
        if len(r) > vi:
            v = float(r[vi].replace(",", ""))
            if r[ui] == "us":
                v *= 1e3
            elif r[ui] == "ms":
                v *= 1e6
            d[r[ki].split("(")[0][:60]].append(v)
    tot = sum(sum(v) for v in d.values())
    return [{"kernel": k, "launches": len(v), "avg_ns": sum(v) / len(v), "share": sum(v) / tot}
            for k, v in sorted(d.items(), key=lambda kv: -sum(kv[1]))]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        k = {"kernel": r[h.index("Kernel Name")][:60]}
        for key in KEYS:
            if key in h:
                i = h.index(key)
                k[key] = f"{r[i]} {units[i]}".strip()
        # warp-stall breakdown (cycles per issued instruction, by reason)
        stalls = {}
        for i, key in enumerate(h):
            if key.startswith("smsp__average_warps_issue_stalled_") and key.endswith("_per_issue_active.ratio"):
                try:
                    stalls[key[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]] = \
                        float(r[i].replace(",", ""))
                except ValueError:
                    pass
        if stalls:
            k["stall_cycles_per_issue"] = dict(sorted(stalls.items(), key=lambda kv: -kv[1])[:12])
        res.append(k)
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", required=True)
    ap.add_argument("--launches")
    ap.add_argument("--rep")
    ap.add_argument("--traffic-json", help="write the top kernel's DRAM bytes per launch here "
                    "(bench.py reads profiles/traffic/<workload key>.json)")
    ap.add_argument("--note", default="")
    a = ap.parse_args()
    os.makedirs("profiles", exist_ok=True)
    summ = {"tag": a.tag, "note": a.note}
    if a.launches:
        summ["launch_list"] = launches(a.launches)
    if a.rep:
        summ["full"] = raw(a.rep)
        if a.traffic_json and summ["full"]:
            f = summ["full"][0]
            def mb(key):
                v, u = f[key].split()
                v = float(v.replace(",", ""))
                return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[u]
            os.makedirs(os.path.dirname(a.traffic_json) or ".", exist_ok=True)
            json.dump({"kernel": f["kernel"], "dram_bytes_per_launch": mb("dram__bytes_read.sum") + mb("dram__bytes_write.sum"),
                       "source": f"profiles/{a.tag}.json (ncu --set full: {os.path.basename(a.rep)})", "tag": a.tag}, open(a.traffic_json, "w"), indent=1)
    os.makedirs(os.path.dirname(f"profiles/{a.tag}.json"), exist_ok=True)
    json.dump(summ, open(f"profiles/{a.tag}.json", "w"), indent=1)
    print(json.dumps(summ, indent=1)[:3000])


if __name__ == "__main__":
    main()
