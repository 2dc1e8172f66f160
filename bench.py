#!/usr/bin/env python
"""bench.py -- tuples/s for SELECT SUM(expr) over DECIMAL columns on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C] [--impl up|reference]

Default workload = BASELINE.json configs[1] (the paper's Fig. 1 high-p query):
SELECT SUM(c1+c2), 10M tuples per GPU, c1 DECIMAL(35,5), c2 DECIMAL(32,2).
A step = one pass of the whole hot path over the resident columns:
fused eval+SUM kernel (+ NCCL all-gather of the partials and the exact
combine kernel when N > 1).  Inputs are seeded synthetic columns (gen/),
larger than L2 (no flush needed).  For N > 1 rows are sharded (weak
scaling: every rank owns `rows` rows; typing uses the global row count).

Also reported: `e2e` (same metric through the C ABI from pinned HOST buffers,
H2D + ingestion + SUM + D2H of the result inside the timed region),
`roofline` (fused kernel's algorithmic bytes / kernel time vs the measured
HBM copy bandwidth), `cpu_baseline` (the CPU oracle, as it stands, timed on
the host cores on a bounded sample), clocks sampled with NVML during the
timed region, and `gpu_launches` (libup kernels launched in the timed region).
`--impl reference` times the CPU oracle instead (the reference arm).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "tuples/sec for SELECT SUM(expr) by DECIMAL precision at 1/2/4/8 B200; % HBM/INT peak"

CONFIGS = {
    1: dict(name="cfg1 SUM(c1+c2) DECIMAL(17,5)+DECIMAL(14,2)", expr="c1+c2", types=[(17, 5), (14, 2)],
            rows=1_000_000, bound="hbm"),
    2: dict(name="cfg2 SUM(c1+c2) DECIMAL(35,5)+DECIMAL(32,2) (Fig.1 high-p)", expr="c1+c2",
            types=[(35, 5), (32, 2)], rows=10_000_000, bound="hbm"),
    3: dict(name="cfg3 SUM(c1*c2 - c3/c4) DECIMAL(200,50)", expr="c1*c2 - c3/c4", types=[(200, 50)] * 4,
            rows=12_500_000, bound="alu", lead=(3,)),
}


def _peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


class ClockSampler:
    """NVML sampling of SM clock + throttle reasons during the timed region."""

    REASONS = {
        "gpu_idle": 0x1, "applications_clocks_setting": 0x2, "sw_power_cap": 0x4, "hw_slowdown": 0x8,
        "sync_boost": 0x10, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
        "hw_power_brake_slowdown": 0x80, "display_clock_setting": 0x100,
    }

    def __init__(self, index: int):
        self.samples, self.reasons = [], 0
        self.max_mhz = None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                self.reasons |= self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            except Exception:
                pass
            time.sleep(0.002)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.nv:
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unavailable"]}
        s = sorted(self.samples)
        names = [k for k, v in self.REASONS.items() if self.reasons & v and k != "gpu_idle"]
        return {"sm_mhz": s[len(s) // 2], "sm_max_mhz": self.max_mhz, "reasons": names, "samples": len(s)}


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def cpu_baseline(cfg, host_cols, budget_s=12.0):
    """The oracle (oracle/updec.c, as it stands) on a bounded row sample,
    all host cores (pthreads, static row blocks, exact combine)."""
    import oracle
    cores = len(os.sched_getaffinity(0))
    ocols = [oracle.Column(p, s, m, g) for (m, g), (p, s) in zip(host_cols, cfg["types"])]
    n_all = host_cols[0][0].shape[0]
    n = min(n_all, 20000)
    t0 = time.perf_counter()
    oracle.eval_sum(cfg["expr"], [c.head(n) for c in ocols], n=n, n_global=n_all, threads=cores)
    dt = time.perf_counter() - t0
    # scale the sample to ~budget_s of CPU work (bounded by the rows we have)
    n2 = int(min(n_all, max(n, n * budget_s / max(dt, 1e-3) * 0.8)))
    if n2 > n:
        t0 = time.perf_counter()
        oracle.eval_sum(cfg["expr"], [c.head(n2) for c in ocols], n=n2, n_global=n_all, threads=cores)
        dt = time.perf_counter() - t0
        n = n2
    return {"value": n / dt, "unit": "tuples/s", "cores": cores, "kind": "oracle",
            "sample": f"first {n} of {n_all} rows of the same seeded workload, SUM({cfg['expr']}), "
                      f"{cores} threads, {dt:.2f} s"}


def run_reference(args, cfg):
    """--impl reference: the CPU oracle as the reference arm (rank 0 only)."""
    ws, rank, _ = dist_env()
    if rank != 0:
        return 0
    import oracle
    from gen import synth
    cores = len(os.sched_getaffinity(0))
    rows = args.rows or cfg["rows"]
    sample = min(rows, args.ref_rows)
    host = []
    for k, (p, s) in enumerate(cfg["types"]):
        host.append(synth.uniform_decimal(sample, p, args.config, k + 1, nonzero_lead=(k in cfg.get("lead", ()))))
    ocols = [oracle.Column(p, s, m, g) for (m, g), (p, s) in zip(host, cfg["types"])]
    for _ in range(args.warmup):
        oracle.eval_sum(cfg["expr"], ocols, n_global=rows * ws, threads=cores)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.eval_sum(cfg["expr"], ocols, n_global=rows * ws, threads=cores)
    dt = (time.perf_counter() - t0) / args.steps
    val = sample / dt
    line = {
        "impl": "reference", "metric": METRIC, "value": val, "unit": "tuples/s", "n_gpus": ws,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": cfg["name"], "rows_per_step": sample, "rows_per_gpu_up_arm": rows},
        "cpu_baseline": {"value": val, "unit": "tuples/s", "cores": cores, "kind": "oracle",
                         "sample": f"first {sample} rows per step of the seeded workload, {cores} threads"},
        "e2e": {"value": val, "unit": "tuples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--rows", type=int, default=0, help="rows per GPU (default: the config's)")
    ap.add_argument("--impl", default="up", choices=["up", "reference"])
    ap.add_argument("--ref-rows", type=int, default=200_000)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=0)
    args = ap.parse_args()
    cfg = CONFIGS[args.config]
    if args.impl == "reference":
        return run_reference(args, cfg)

    import numpy as np
    import torch
    import torch.distributed as dist

    from gen import device as gdev
    from gen import synth
    from paper_conf_icde_lixylz24_b200 import up

    ws, rank, local = dist_env()
    torch.cuda.set_device(local)
    if ws > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    ctx = up.Context(local)
    stream = torch.cuda.current_stream()
    rows = args.rows or cfg["rows"]
    n_global = rows * ws
    row0 = rank * rows

    # ---- inputs: device generator (bit-identical to the host twin), resident in HBM
    gdev.build()
    cols, raw = [], []
    for k, (p, s) in enumerate(cfg["types"]):
        mag, neg = gdev.uniform_decimal(rows, p, args.config, k + 1, row0=row0,
                                        nonzero_lead=(k in cfg.get("lead", ())))
        raw.append((mag, neg))
        cols.append(ctx.column_from_device_bin(p, s, mag, neg))
    ctx.check()
    P, S, LA = ctx.sum_type(cfg["expr"], cols, n_global)
    partial = torch.empty(LA, dtype=torch.int32, device="cuda")
    gathered = torch.empty(LA * ws, dtype=torch.int32, device="cuda")
    total = torch.empty(LA, dtype=torch.int32, device="cuda")

    def step():
        ctx.sum_expr(cfg["expr"], cols, n_global, out=partial)
        if ws > 1:
            dist.all_gather_into_tensor(gathered, partial)
            ctx.sum_combine(gathered, LA, out=total)

    # warm-up (specialises + JIT-compiles the kernel: excluded from timing)
    for _ in range(max(3, args.warmup)):
        step()
    ctx.check()
    torch.cuda.synchronize()

    # ---- timed region: K steps, barrier + sync on both sides, CUDA events
    K = args.steps
    kev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    t_start, t_end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    l0 = ctx.launches
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        t_start.record(stream)
        for i in range(K):
            kev[i][0].record(stream)
            ctx.sum_expr(cfg["expr"], cols, n_global, out=partial)
            kev[i][1].record(stream)
            if ws > 1:
                dist.all_gather_into_tensor(gathered, partial)
                ctx.sum_combine(gathered, LA, out=total)
        t_end.record(stream)
        torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    launches = ctx.launches - l0
    ms = t_start.elapsed_time(t_end)
    kernel_ms = sum(a.elapsed_time(b) for a, b in kev) / K
    if ws > 1:
        t = torch.tensor([ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    ms_per_step = ms / K
    value = n_global / (ms_per_step / 1e3)
    ctx.check()
    result = up.result_to_string(total if ws > 1 else partial, S)

    # ---- roofline of the fused kernel (algorithmic bytes: the limb planes read)
    bytes_per_row = sum(4 * up.limbs(p) for p, s in cfg["types"])
    alg_bytes = bytes_per_row * rows
    peaks = _peaks()
    peak = peaks.get("hbm_gbs", 6650.0)
    achieved = alg_bytes / (kernel_ms / 1e3) / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", f"traffic_cfg{args.config}.json")
    if os.path.exists(tp):
        try:
            traffic = json.load(open(tp)).get("dram_bytes_per_launch")
        except Exception:
            traffic = None
    roofline = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                "frac": round(achieved / peak, 4), "traffic": traffic,
                "kernel_ms": round(kernel_ms, 5), "alg_bytes_per_launch": alg_bytes,
                "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy, burst)" if "hbm_gbs" in peaks else "fallback 6.65 TB/s"}

    # ---- e2e through the C ABI from pinned host buffers
    host = []
    for mag, neg in raw:
        hm = torch.empty(mag.shape, dtype=torch.int32, pin_memory=True)
        hn = torch.empty(neg.shape, dtype=torch.uint8, pin_memory=True)
        hm.copy_(mag)
        hn.copy_(neg)
        host.append((hm, hn))
    torch.cuda.synchronize()
    e2e_cols = [up.Column(p, s, rows) for p, s in cfg["types"]]
    res_host = torch.empty(LA, dtype=torch.int32, pin_memory=True)

    def e2e_step():
        for (hm, hn), (p, s), col in zip(host, cfg["types"], e2e_cols):
            ctx.column_from_host_bin(p, s, hm, hn, out=col)
        ctx.sum_expr(cfg["expr"], e2e_cols, n_global, out=partial)
        if ws > 1:
            dist.all_gather_into_tensor(gathered, partial)
            ctx.sum_combine(gathered, LA, out=total)
            res_host.copy_(total, non_blocking=True)
        else:
            res_host.copy_(partial, non_blocking=True)

    for _ in range(3):
        e2e_step()
    torch.cuda.synchronize()
    K2 = args.e2e_steps or max(3, min(K, 20))
    if ws > 1:
        dist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(stream)
    for _ in range(K2):
        e2e_step()
    e1.record(stream)
    torch.cuda.synchronize()
    ems = e0.elapsed_time(e1)
    if ws > 1:
        t = torch.tensor([ems], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ems = float(t.item())
    ctx.check()
    assert up.format_decimal(res_host.tolist(), S) == result, "e2e result differs from the device-resident run"
    h2d = sum(hm.numel() * 4 + hn.numel() for hm, hn in host)
    e2e = {"value": n_global / (ems / K2 / 1e3), "unit": "tuples/s", "h2d_bytes_per_step": h2d,
           "d2h_bytes_per_step": LA * 4, "ms_per_step": ems / K2}

    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        hc = [(m.cpu().numpy().view(np.uint32), g.cpu().numpy()) for m, g in raw]
        cpu = cpu_baseline(cfg, hc)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "tuples/s", "n_gpus": ws, "steps": K,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": cfg["name"], "expr": cfg["expr"], "types": cfg["types"],
                       "rows_per_gpu": rows, "global_rows": n_global, "sum_type": [P, S], "sum_limbs": LA,
                       "parallelism": f"rows sharded x{ws}, NCCL all-gather of partials" if ws > 1 else "1 GPU",
                       "l2": "inputs %.0f MB/GPU > 126 MB L2 (no flush)" % (alg_bytes / 1e6)},
            "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches,
            "clocks": clk.summary(), "result": result, "jit_ms": round(ctx.jit_ms, 1),
        }
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
