#!/usr/bin/env python
"""bench.py -- tuples/s for SELECT SUM(...) over DECIMAL columns on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C] [--impl up|reference]

Default workload = BASELINE.json configs[1] (the paper's Fig. 1 high-p query):
SELECT SUM(c1+c2), 10M tuples per GPU, c1 DECIMAL(35,5), c2 DECIMAL(32,2),
the columns resident in the paper's compact rows (29 B/row; --layout planes
for limb planes, 32 B/row).
Other configs (parity-test cases by default, bench lines on request):
  1  SUM(c1+c2) DECIMAL(17,5)+DECIMAL(14,2), 1M tuples (L2-resident: flushed)
  3  SUM(c1*c2 - c3/c4) DECIMAL(200,50) x4, 12.5M tuples/GPU (100M on 8)
  4  SUM(x^65537 mod N), 1024-bit N, 10M tuples (RSA, Query 4 generalised)
  5  SUM(sin_P(x)), P = 1000 digits, x ~ N(0.78, 0.01) DECIMAL(9,8), 1M tuples
A step = one pass of the whole hot path over the resident columns: the fused
kernel (+ NCCL all-gather of the partials and the exact combine kernel when
N > 1).  Inputs are seeded synthetic columns (gen/).  For N > 1 rows are
sharded (weak scaling: every rank owns `rows` rows; typing uses the global
row count).  Steps over resident columns are launched pipelined
(up_set_pipelined: programmatic dependent launch, each step's kernel may
start while the previous one finishes; --no-pipelined turns it off) and
timed with one event pair around the K steps (per step, with the L2 flush
outside, when the flush is needed).  Reported with it: `e2e` (same metric through the C ABI from
pinned HOST buffers in the paper's compact row format: H2D + ingestion + SUM
+ D2H of the result in the timed region), `roofline` of the fused kernel, `cpu_baseline` (the CPU oracle as it
stands on a bounded sample), NVML clocks during the timed region, and
`gpu_launches`.  `--impl reference` times the CPU oracle (the reference arm).
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

E2E_MAX_ROWS = 1 << 26
METRIC = "tuples/sec for SELECT SUM(expr) by DECIMAL precision at 1/2/4/8 B200; % HBM/INT peak"
# Integer roofline for the compute-bound configs, in 32x32->64 LIMB PRODUCTS/s.
# Every limb product needs one high-half multiply (IMAD.HI / the high half of
# IMAD.WIDE); tools/intpipe.cu measured IMAD.HI on this B200 at 31.75
# lanes/clk/SM (half the 60.85 of IMAD) = 9.23e12/s: the peak used below
# (profiles/intpipe_b200_r01.json).  Fallback if the file is missing: 32
# lanes/clk/SM x 148 SMs x 1.965 GHz.
def _product_peak():
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "intpipe_b200_r01.json")))
        return d["imad_hi"]["ops_per_s"], "measured IMAD.HI rate (tools/intpipe.cu, profiles/intpipe_b200_r01.json)"
    except Exception:
        return 32 * 148 * 1.965e9, "derived: 32 IMAD.HI lanes/clk/SM x 148 SMs x 1.965 GHz (fallback)"

CONFIGS = {
    1: dict(kind="expr", name="cfg1 SUM(c1+c2) DECIMAL(17,5)+DECIMAL(14,2)", expr="c1+c2",
            types=[(17, 5), (14, 2)], rows=1_000_000),
    2: dict(kind="expr", name="cfg2 SUM(c1+c2) DECIMAL(35,5)+DECIMAL(32,2) (Fig.1 high-p)", expr="c1+c2",
            types=[(35, 5), (32, 2)], rows=10_000_000),
    3: dict(kind="expr", name="cfg3 SUM(c1*c2 - c3/c4) DECIMAL(200,50)", expr="c1*c2 - c3/c4",
            types=[(200, 50)] * 4, rows=12_500_000, lead=(3,)),
    4: dict(kind="modexp", name="cfg4 SUM(x^65537 mod N) 1024-bit RSA", bits=1024, e=65537, rows=10_000_000),
    5: dict(kind="sin", name="cfg5 SUM(sin_P(x)) P=1000, x~N(0.78,0.01) DECIMAL(9,8)", P=1000, mu=0.78,
            rows=1_000_000),
}


def traffic_key(cfg, rows, layout="planes"):
    """profiles/traffic/<key>.json key: the workload name + rows per GPU
    (+ "_compact" for compact-resident columns: a different byte count)."""
    import re
    return re.sub(r"[^A-Za-z0-9]+", "_", cfg["name"]).strip("_") + f"_{rows}" + ("" if layout == "planes" else "_" + layout)


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


# --------------------------------------------------------------------------- workloads
class Workload:
    """Inputs (device-resident + pinned-host copies) and the step for one config."""

    def __init__(self, cfg, args, ctx, rows, n_global, row0):
        self.cfg, self.args, self.ctx = cfg, args, ctx
        self.rows, self.n_global, self.row0 = rows, n_global, row0
        # e2e (host buffers -> result) runs on at most E2E_MAX_ROWS of this
        # rank's rows: pinned host copies of 2^30-row columns would be 15-31 GB
        self.e2e_rows = min(rows, E2E_MAX_ROWS)


def _h2d_copy_gbs(nbytes, reps=5):
    """pinned host -> device copy bandwidth for nbytes (the e2e path's link)"""
    import torch
    nbytes = max(1 << 20, min(int(nbytes), 1 << 30))
    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    d.copy_(h, non_blocking=True)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        d.copy_(h, non_blocking=True)
    b.record()
    torch.cuda.synchronize()
    return round(nbytes * reps / (a.elapsed_time(b) / 1e3) / 1e9, 2)


def _col_bytes(p, layout):
    from paper_conf_icde_lixylz24_b200 import up
    return {"compact": up.compact_bytes(p), "quads": 16 * up.quads(p)}.get(layout, 4 * up.limbs(p))


class ExprWorkload(Workload):
    def setup(self):
        from gen import device as gdev
        from paper_conf_icde_lixylz24_b200 import up
        cfg, ctx = self.cfg, self.ctx
        self.raw, self.cols = [], []
        for k, (p, s) in enumerate(cfg["types"]):
            mag, neg = gdev.uniform_decimal(self.rows, p, self.args.config, k + 1, row0=self.row0,
                                            nonzero_lead=(k in cfg.get("lead", ())))
            self.raw.append((mag, neg))
            self.cols.append(ctx.column_from_device_bin(p, s, mag, neg, layout=self.col_layout(k)))
        ctx.check()
        self.P, self.S, self.LA = ctx.sum_type(cfg["expr"], self.cols, self.n_global)
        self.e2e_cols = [up.Column(p, s, self.e2e_rows, layout=self.col_layout(k)) for k, (p, s) in enumerate(cfg["types"])]
        # algorithmic bytes per row: the columns as stored -- limb planes (4 B per
        # limb), the paper's compact rows (Lb bytes) or limb quads
        # (16 B per quad, the sign-flag limb and padding included)
        self.bytes_per_row = sum(_col_bytes(p, self.col_layout(k)) for k, (p, s) in enumerate(cfg["types"]))

    def col_layout(self, k):
        """layout of column k: --layout, or for "mixed" (cfg3's default) limb quads
        for the product's columns c1, c2 (the tensor cores read them straight
        from TMA) and limb planes for the division's c3, c4 (fewer bytes beside
        the concurrent contraction)"""
        if self.args.layout == "mixed":
            return "quads" if k < 2 else "planes"
        return self.args.layout

    def kernel(self, out):
        self.ctx.sum_expr(self.cfg["expr"], self.cols, self.n_global, out=out)

    def e2e_host_buffers(self):
        """Pinned host copies of the inputs in the paper's compact row format
        (P:L843-873): Lb bytes per row, what a scan would hand to the GPU."""
        import numpy as np
        import torch
        from gen import synth
        bufs = []
        for (mag, neg), (p, s) in zip(self.raw, self.cfg["types"]):
            m, g = mag[: self.e2e_rows], neg[: self.e2e_rows]
            cb = synth.to_compact(m.cpu().numpy().view(np.uint32), g.cpu().numpy(), p)
            t = torch.empty(cb.shape, dtype=torch.uint8, pin_memory=True)
            t.copy_(torch.from_numpy(cb))
            bufs.append(t)
        return bufs

    def e2e_ingest(self, host):
        for hb, (p, s), col in zip(host, self.cfg["types"], self.e2e_cols):
            # compact layout: the host rows land in place (H2D + range check);
            # planes: H2D + in-kernel expand into limb planes
            self.ctx.column_from_compact(p, s, hb, n=self.e2e_rows, out=col)

    def e2e_kernel(self, out):
        self.ctx.sum_expr(self.cfg["expr"], self.e2e_cols, self.n_global, out=out)

    def roofline(self, kernel_ms, peaks):
        tc = not (os.environ.get("UP_NO_TC") or os.environ.get("UP_NO_SPLIT"))
        if self.cfg["types"][0][0] >= 100 and not tc:     # wide expressions on CUDA cores: integer-pipe bound
            return self._alu_roofline(kernel_ms, self.alg_products_per_row())
        # HBM roofline.  Wide expressions with the tensor-core split (default):
        # SUM(c1*c2) is an integer GEMM over the rows on tcgen05 (kind::i8,
        # contract_tc.cu) whose FLOPs are ~1/30 of the tensor peak, c3/c4 is
        # decided from the operands' top limbs -- what remains is moving the
        # columns; algorithmic bytes = every limb plane of every column
        alg = self.bytes_per_row * self.rows
        peak = peaks.get("hbm_gbs", 6650.0)
        ach = alg / (kernel_ms / 1e3) / 1e9
        r = {"bound": "hbm", "achieved": round(ach, 1), "peak": peak, "unit": "GB/s",
             "frac": round(ach / peak, 4), "kernel_ms": round(kernel_ms, 5), "alg_bytes_per_launch": alg,
             "alg_unit": f"{self.bytes_per_row} B/row ({self.args.layout} layout"
                         f" of all columns) x {self.rows} rows",
             "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy, burst)" if "hbm_gbs" in peaks
             else "fallback 6.65 TB/s"}
        if self.cfg["types"][0][0] >= 100:
            r = self._split_roofline(kernel_ms, peaks)
        return r

    def _time(self, fn, reps=5):
        import torch
        st = torch.cuda.current_stream()
        fn()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        for _ in range(reps):
            fn()
        b.record(st)
        torch.cuda.synchronize()
        return a.elapsed_time(b) / reps

    def _split_roofline(self, step_ms, peaks):
        """cfg3 with the tensor-core split: per-kernel fractions, each on what
        that kernel does.  SUM(c1*c2) alone launches the tcgen05 contraction
        (it reads c1, c2 whole: 2 x 4L B/row, HBM roofline); SUM(c3/c4) alone
        launches the fused rest kernel (top-limb division: reads a window of
        c3/c4's top limbs, integer roofline on the SURVEY's division count).
        The line's roofline is the dominant (contraction) kernel's."""
        import torch
        from paper_conf_icde_lixylz24_b200 import up
        p, s = self.cfg["types"][0]
        L = up.limbs(p)
        c1, c2, c3, c4 = self.cols
        out = torch.empty(self.LA, dtype=torch.int32, device="cuda")
        t_tc = self._time(lambda: self.ctx.sum_expr("c1*c2", [c1, c2], self.n_global, out=out))
        t_rest = self._time(lambda: self.ctx.sum_expr("c1/c2", [c3, c4], self.n_global, out=out))
        peak = peaks.get("hbm_gbs", 6650.0)
        tc_row = _col_bytes(p, self.col_layout(0))
        tc_bytes = 2 * tc_row * self.rows
        ach = tc_bytes / (t_tc / 1e3) / 1e9
        # the rest kernel's arithmetic: the top-limb decision per row (DESIGN §5,
        # up_dev.cuh div_top_decide): ah x C (T x NC limb products) and NQ quotient
        # limbs of T products each (3-by-2 step + multiply-subtract); NC = limbs of
        # C = 10^(s+4), NQ = limbs of the quotient type, T = max(NC, NQ) + 1 -- the
        # products the kernel performs, not the SURVEY's full-division count
        nc = ((10 ** (s + 4)).bit_length() + 31) // 32
        nq = up.limbs(max(s + 5, 1))
        T = max(nc, nq) + 1
        div_products = T * (nc + nq)
        pk, src = _product_peak()
        rest_ach = div_products * self.rows / (t_rest / 1e3)
        return {"bound": "hbm", "achieved": round(ach, 1), "peak": peak, "unit": "GB/s", "frac": round(ach / peak, 4),
                "kernel_ms": round(t_tc, 5), "alg_bytes_per_launch": tc_bytes,
                "alg_unit": f"contraction kernel: c1, c2 as stored ({self.col_layout(0)}) {2 * tc_row} B/row x {self.rows} rows",
                "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy, burst)" if "hbm_gbs" in peaks else "fallback 6.65 TB/s",
                "kernels": [
                    {"kernel": ("k_contract_tq" if self.col_layout(0) == "quads" else "k_contract_tc") +
                               " (SUM(c1*c2), tcgen05 kind::i8)", "ms": round(t_tc, 5), "bound": "hbm",
                     "alg_bytes": tc_bytes, "achieved_gbs": round(ach, 1), "frac": round(ach / peak, 4)},
                    {"kernel": "upk rest (SUM(-c3/c4), top-limb division)", "ms": round(t_rest, 5), "bound": "alu",
                     "alg_products": div_products * self.rows,
                     "alg_unit": f"{div_products} limb products/row (top-limb decision: T={T} limbs x (C {nc} + "
                                 f"quotient {nq} limbs))",
                     "achieved_T_products_s": round(rest_ach / 1e12, 4), "frac": round(rest_ach / pk, 4),
                     "peak_source": src}],
                "step_ms": round(step_ms, 5),
                "note": "step = contraction + rest + exact combine, back to back on one stream"}

    def alg_products_per_row(self):
        """limb products of c1*c2 - c3/c4 = x (L*L) + / prescale
        (L x limbs(10^(s+4))) + / (quotient limbs x L) + alignment of the
        quotient (limbs(q) x limbs(10^(2s-(s+4))))."""
        from paper_conf_icde_lixylz24_b200 import up
        p, s = self.cfg["types"][0]
        mag = lambda k: max(1, (10 ** k).bit_length() // 32 + 1)   # noqa: E731
        L = up.limbs(p)
        nu = mag(p + s + 4)
        return L * L + L * mag(s + 4) + (nu - L + 1) * L + up.limbs(s + 5) * mag(s - 4)

    def _alu_roofline(self, kernel_ms, products_per_row, note=""):
        peak, src = _product_peak()
        ops = products_per_row * self.rows
        ach = ops / (kernel_ms / 1e3)
        return {"bound": "alu", "achieved": round(ach / 1e12, 4), "peak": round(peak / 1e12, 4),
                "unit": "T limb-products/s", "frac": round(ach / peak, 4), "kernel_ms": round(kernel_ms, 4),
                "alg_ops_per_launch": ops,
                "alg_unit": f"{products_per_row} 32x32->64 limb products/row x {self.rows} rows" + note,
                "peak_source": src}

    def host_for_oracle(self, max_rows=1 << 25):
        """Host copies of (at most the first max_rows of) the inputs for the oracle."""
        import numpy as np
        import oracle
        k = min(self.rows, max_rows)
        return [oracle.Column(p, s, m[:k].cpu().numpy().view(np.uint32), g[:k].cpu().numpy())
                for (m, g), (p, s) in zip(self.raw, self.cfg["types"])]

    def oracle_sum(self, ocols, n, threads):
        import oracle
        return oracle.eval_sum(self.cfg["expr"], [c.head(n) for c in ocols], n=n, n_global=self.n_global,
                               threads=threads)[0]

    def workload_desc(self):
        return {"expr": self.cfg["expr"], "types": self.cfg["types"], "sum_type": [self.P, self.S],
                "sum_limbs": self.LA}


class ModexpWorkload(ExprWorkload):
    def setup(self):
        from gen import device as gdev
        from gen import synth
        from paper_conf_icde_lixylz24_b200 import up
        cfg, ctx = self.cfg, self.ctx
        self.N, _, _ = synth.rsa_modulus(cfg["bits"])
        self.e = cfg["e"]
        self.d = len(str(self.N))
        mag, neg = gdev.uniform_range(synth.SEED, synth.stream_id(4, 0), self.rows, 0, self.N - 1, signed=False,
                                      row0=self.row0)
        self.raw = [(mag, neg)]
        self.cols = [ctx.column_from_device_bin(self.d, 0, mag, neg)]
        ctx.check()
        self.P, self.LA = ctx.modexp_sum_type(self.N, self.n_global)
        self.S = 0
        self.e2e_cols = [up.Column(self.d, 0, self.e2e_rows)]
        self.cfg = dict(cfg, types=[(self.d, 0)])

    def kernel(self, out):
        self.ctx.modexp_sum(self.cols[0], self.e, self.N, self.n_global, out=out)

    # e2e streamed in row chunks (the public API composed): the ingestion of
    # chunk k+1 (its H2D copy on the ctx copy stream) runs while the modexp SUM
    # of chunk k computes; the chunk partials (typed with the global N) are
    # added by up_sum_combine.  The host link and the integer pipes overlap.
    E2E_CHUNKS = 8

    def e2e_ingest(self, host):
        self._e2e_host = host

    def e2e_kernel(self, out):
        import torch
        from paper_conf_icde_lixylz24_b200 import up
        hb, col = self._e2e_host[0], self.e2e_cols[0]
        Lb = up.compact_bytes(self.d)
        n, C = col.n, self.E2E_CHUNKS
        if getattr(self, "_parts", None) is None:
            self._parts = torch.empty((C, self.LA), dtype=torch.int32, device="cuda")
        for k in range(C):
            r0 = (n * k // C) & ~255
            r1 = n if k == C - 1 else (n * (k + 1) // C) & ~255
            view = col.rows(r0, r1)
            self.ctx.column_from_compact(self.d, 0, hb[r0 * Lb:r1 * Lb], n=r1 - r0, out=view)
            self.ctx.modexp_sum(view, self.e, self.N, self.n_global, out=self._parts[k])
        self.ctx.sum_combine(self._parts, self.LA, out=out)

    def roofline(self, kernel_ms, peaks):
        n = (self.N.bit_length() + 31) // 32
        montmuls = (self.e.bit_length() - 1) + bin(self.e).count("1") - 1 + 2   # squarings + multiplies + in/out
        note = f"; {montmuls} Montgomery products x (2n^2+n), n = {n} (SURVEY §8d count)"
        if self.e % 2 == 1 and self.e > 1 and n <= 64:
            note += ("; the radix-2^28 kernel performs up to two fewer: for odd e its last multiply takes the plain "
                     "base and leaves Montgomery form, and the base's zero upper chunk (x < R) needs no conversion product")
        return self._alu_roofline(kernel_ms, montmuls * (2 * n * n + n), note)

    def oracle_sum(self, ocols, n, threads):
        import oracle
        return oracle.modexp_sum(ocols[0].head(n), self.e, self.N, threads=threads)

    def workload_desc(self):
        return {"modulus_bits": self.N.bit_length(), "e": self.e, "base_type": [self.d, 0],
                "sum_type": [self.P, 0], "sum_limbs": self.LA}


class SinWorkload(ExprWorkload):
    def setup(self):
        import torch
        from gen import synth
        from paper_conf_icde_lixylz24_b200 import up
        cfg, ctx = self.cfg, self.ctx
        self.Pd = cfg["P"]
        mag, neg = synth.normal_decimal(self.rows, cfg["mu"], 0.01, 8, config=5, column=0, row0=self.row0)
        self.host_np = (mag, neg)
        tm = torch.from_numpy(mag.view("int32")).cuda()
        tn = torch.from_numpy(neg).cuda()
        self.raw = [(tm, tn)]
        self.cols = [ctx.column_from_device_bin(9, 8, tm, tn)]
        ctx.check()
        self.P = up.sum_precision(self.Pd + 1, self.n_global)
        self.S = self.Pd
        self.LA = up.limbs(self.P)
        self.e2e_cols = [up.Column(9, 8, self.e2e_rows)]
        self.cfg = dict(cfg, types=[(9, 8)])
        # active-limb sum per row, from a sample of rows
        import numpy as np
        acts = []
        for m in mag[: 128, 0].tolist():
            t, k, a = m * 10 ** (self.Pd - 8), 1, 0
            while t:
                a += (t.bit_length() + 31) // 32
                t = t * m * m // (10 ** 16 * (2 * k) * (2 * k + 1))
                k += 1
            acts.append(a)
        self.active_limb_terms = float(np.mean(acts))

    def kernel(self, out):
        self.ctx.sin_taylor_sum(self.cols[0], self.Pd, self.n_global, out=out)

    def e2e_kernel(self, out):
        self.ctx.sin_taylor_sum(self.e2e_cols[0], self.Pd, self.n_global, out=out)

    def roofline(self, kernel_ms, peaks):
        # per active limb-term: t x m_x^2 (2 limb products) + 3 short-division
        # steps (one 32x32->64 reciprocal product each) = 5 limb products
        per_row = int(round(self.active_limb_terms * 5))
        return self._alu_roofline(kernel_ms, per_row,
                                  f"; mean active-limb sum {self.active_limb_terms:.0f} per row x 5")

    def oracle_sum(self, ocols, n, threads):
        import oracle
        return oracle.sin_sum(ocols[0].head(n), self.Pd, threads=threads)

    def workload_desc(self):
        return {"P": self.Pd, "x_type": [9, 8], "mu": self.cfg["mu"], "sigma": 0.01, "sum_type": [self.P, self.S],
                "sum_limbs": self.LA}


KINDS = {"expr": ExprWorkload, "modexp": ModexpWorkload, "sin": SinWorkload}


def cpu_baseline(wl, budget_s=12.0):
    """The oracle (oracle/updec.c, as it stands) on a bounded row sample, all
    host cores (pthreads, static row blocks, exact combine)."""
    cores = len(os.sched_getaffinity(0))
    ocols = wl.host_for_oracle()
    n_all = ocols[0].n          # <= wl.rows (the copy is capped for 2^30-row columns)
    n = min(n_all, 64)
    t0 = time.perf_counter()
    val = wl.oracle_sum(ocols, n, cores)
    dt = time.perf_counter() - t0
    while dt < budget_s / 8 and n < n_all:
        n = int(min(n_all, n * max(2.0, budget_s / 2 / max(dt, 1e-4))))
        t0 = time.perf_counter()
        val = wl.oracle_sum(ocols, n, cores)
        dt = time.perf_counter() - t0
    out = {"value": n / dt, "unit": "tuples/s", "cores": cores, "kind": "oracle",
           "sample": f"first {n} of {n_all} rows of the same seeded workload ({wl.cfg['name']}), "
                     f"{cores} threads, {dt:.2f} s"}
    # the oracle's SUM over every row is the parity check of the bench's own result
    return out, (val if n == wl.rows else None)


def run_reference(args, cfg):
    """--impl reference: the CPU oracle as the reference arm (rank 0 only)."""
    ws, rank, _ = dist_env()
    if rank != 0:
        return 0
    import numpy as np
    import oracle
    from gen import synth
    cores = len(os.sched_getaffinity(0))
    rows = args.rows or cfg["rows"]
    sample = min(rows, args.ref_rows)
    if cfg["kind"] == "expr":
        host = [synth.uniform_decimal(sample, p, args.config, k + 1, nonzero_lead=(k in cfg.get("lead", ())))
                for k, (p, s) in enumerate(cfg["types"])]
        ocols = [oracle.Column(p, s, m, g) for (m, g), (p, s) in zip(host, cfg["types"])]
        fn = lambda: oracle.eval_sum(cfg["expr"], ocols, n_global=rows * ws, threads=cores)  # noqa: E731
    elif cfg["kind"] == "modexp":
        N, _, _ = synth.rsa_modulus(cfg["bits"])
        sample = min(sample, 2000)
        m, g = synth.rsa_messages(sample, N)
        col = oracle.Column(len(str(N)), 0, m, g)
        fn = lambda: oracle.modexp_sum(col, cfg["e"], N, threads=cores)  # noqa: E731
    else:
        sample = min(sample, 2000)
        m, g = synth.normal_decimal(sample, cfg["mu"], 0.01, 8, config=5, column=0)
        col = oracle.Column(9, 8, m, g)
        fn = lambda: oracle.sin_sum(col, cfg["P"], threads=cores)  # noqa: E731
    for _ in range(args.warmup):
        fn()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        fn()
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
    ap.add_argument("--steps", type=int, default=0, help="timed steps (default per config)")
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--rows", type=int, default=0, help="rows per GPU (default: the config's)")
    ap.add_argument("--global-rows", type=int, default=0, help="total rows, sharded over the GPUs (strong scaling)")
    ap.add_argument("--impl", default="up", choices=["up", "reference"])
    ap.add_argument("--layout", default=None, choices=["planes", "compact", "quads", "mixed"],
                    help="column storage for the expression configs (1-3): limb planes, the paper's compact rows or "
                         "limb quads, or mixed (cfg3: quads for the product's c1, c2, planes for c3, c4); default: "
                         "compact rows for 1-2, mixed for 3")
    ap.add_argument("--ref-rows", type=int, default=200_000)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-pipelined", action="store_true",
                    help="launch each step's SUM kernel without programmatic dependent launch")
    ap.add_argument("--e2e-steps", type=int, default=0)
    ap.add_argument("--P", type=int, default=0, help="cfg5 digits")
    ap.add_argument("--bits", type=int, default=0, help="cfg4 modulus bits")
    ap.add_argument("--e", type=int, default=0, help="cfg4 exponent")
    ap.add_argument("--p", type=int, default=0, help="cfg3 precision (scale from the config table)")
    args = ap.parse_args()
    cfg = dict(CONFIGS[args.config])
    if args.P:
        cfg["P"] = args.P
        cfg["name"] = cfg["name"].replace("P=1000", f"P={args.P}")
    if args.bits:
        cfg["bits"] = args.bits
        cfg["name"] = cfg["name"].replace("1024-bit", f"{args.bits}-bit")
    if args.e:
        cfg["e"] = args.e
        cfg["name"] = cfg["name"].replace("65537", str(args.e))
    if args.p:
        s = {200: 50, 500: 75, 1000: 100}.get(args.p, args.p // 4)
        cfg["types"] = [(args.p, s)] * 4
        cfg["name"] = f"cfg3 SUM(c1*c2 - c3/c4) DECIMAL({args.p},{s})"
    if args.layout is None:
        # expression configs: the paper's compact rows for the narrow columns
        # (cDecimal, P:L843-873 -- fewer bytes per row than limb planes, read in
        # place by the fused kernel); for cfg3 limb quads for the product's
        # columns (the tensor cores' operand layout) and limb planes for the
        # division's; modexp / sine read limb planes
        if cfg["kind"] != "expr":
            args.layout = "planes"
        else:
            args.layout = "mixed" if cfg["types"][0][0] >= 100 else "compact"
    if not args.steps:
        args.steps = {"expr": 200, "modexp": 5, "sin": 3}[cfg["kind"]] if cfg["kind"] != "expr" or \
            cfg["types"][0][0] < 100 else 5
    if args.impl == "reference":
        return run_reference(args, cfg)

    import torch
    import torch.distributed as dist

    from gen import device as gdev
    from paper_conf_icde_lixylz24_b200 import up
    from paper_conf_icde_lixylz24_b200.dist import ShardedSum, shard_range

    ws, rank, local = dist_env()
    torch.cuda.set_device(local)
    if ws > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    ctx = up.Context(local)
    stream = torch.cuda.current_stream()
    # Row sharding (rows a13/e).  N = 1: the config's rows (configs[1]:
    # 10M).  N > 1, memory-bound configs 1/2: STRONG scaling of 2^30-row columns
    # (SURVEY §8e), so the all-gather + combine stays a small part of the step;
    # compute-bound configs 3-5: weak scaling (the config's rows per GPU).
    # --global-rows / --rows override.
    if args.global_rows:
        n_global, scaling = args.global_rows, "strong"
    elif ws > 1 and cfg["kind"] == "expr" and cfg["types"][0][0] < 100 and not args.rows:
        n_global, scaling = 1 << 30, "strong"
    else:
        n_global, scaling = (args.rows or cfg["rows"]) * ws, "weak"
    lo, hi = shard_range(n_global, ws, rank)
    rows = hi - lo
    gdev.build()
    wl = KINDS[cfg["kind"]](cfg, args, ctx, rows, n_global, lo)
    wl.setup()
    LA = wl.LA
    # one pass of the hot path = the rank's fused SUM kernel, then (N > 1) the
    # NCCL all-gather of the LA-limb partials and the exact combine kernel
    ss = ShardedSum(ctx, LA, wl.S, wl.kernel)
    partial = ss.partial
    # L2 flush buffer for working sets below L2 (cfg1: 16 MB)
    flush = None
    if getattr(wl, "bytes_per_row", 0) * rows < 256e6 and cfg["kind"] == "expr" and cfg["types"][0][0] < 100:
        flush = torch.empty(int(256e6) // 4, dtype=torch.int32, device="cuda")
        # then a 256 MB read: writes back the flush's dirty lines before the step starts, so the
        # timed kernel does not pay the flush's write-back (L2 left holding clean, unrelated lines)
        flush_rd = torch.zeros(int(256e6) // 4, dtype=torch.float32, device="cuda")
        flush_sum = torch.empty((), dtype=torch.float32, device="cuda")

    # Pipelined SUM launches (up_set_pipelined): consecutive steps
    # are queries over the same resident columns, so each step's kernel may
    # start streaming while the previous step's kernel finishes.  Not with the
    # L2 flush (the flush must complete before the step) nor for e2e (the
    # ingestion kernel right before the SUM writes its inputs).
    pipelined = flush is None and not args.no_pipelined
    ctx.set_pipelined(pipelined)

    def step():
        ss()

    for _ in range(max(3, args.warmup)):     # warm-up (includes the one-time specialisation / JIT)
        step()
    ctx.check()
    torch.cuda.synchronize()
    # W steps of a 60 us kernel are ~0.3 ms: keep warming (untimed) until ~0.4 s of
    # GPU work has run, so the timed steps see settled SM clocks
    t0 = time.perf_counter()
    for _ in range(3):
        step()
    torch.cuda.synchronize()
    per = max((time.perf_counter() - t0) / 3, 1e-6)
    warm_extra = int(min(20000, 0.4 / per))
    if ws > 1:      # the same count on every rank (each step has a collective)
        t = torch.tensor([warm_extra], dtype=torch.int64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        warm_extra = int(t.item())
    for i in range(warm_extra):
        step()
        if i % 64 == 63:
            torch.cuda.synchronize()
    torch.cuda.synchronize()

    # ---- timed region: K steps between a barrier + sync on both sides; CUDA
    # events on the launching stream.  Without an L2 flush: ONE event pair
    # around the K steps (events between steps would serialise them); with the
    # flush (cfg1 at 1M rows): an event pair around each step, the flush outside.
    K = args.steps

    def body():
        wl.kernel(partial)
        if ws > 1:     # the exchange step of ShardedSum.__call__
            dist.all_gather_into_tensor(ss.gathered, partial)
            ctx.sum_combine(ss.gathered, LA, out=ss.total)

    def ev():
        return torch.cuda.Event(enable_timing=True)

    l0 = ctx.launches
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        if flush is None:
            e0, e1 = ev(), ev()
            e0.record(stream)
            for i in range(K):
                body()
            e1.record(stream)
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1)
        else:
            sev = [(ev(), ev()) for _ in range(K)]
            for i in range(K):
                flush.zero_()            # evict the inputs from L2 (outside the step's events)
                torch.sum(flush_rd, dim=0, out=flush_sum)
                sev[i][0].record(stream)
                body()
                sev[i][1].record(stream)
            torch.cuda.synchronize()
            ms = sum(a.elapsed_time(b) for a, b in sev)
    if ws > 1:
        dist.barrier()
    launches = ctx.launches - l0
    if ws > 1:
        t = torch.tensor([ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    ms_per_step = ms / K
    value = n_global / (ms_per_step / 1e3)
    # the dominant kernel's average launch duration: when a step IS one launch
    # (N = 1, one fused kernel), the timed region's events give it directly
    # (ms / K); otherwise a second K-step pass with events around the kernel
    if ws == 1 and launches == K:
        kernel_ms, kernel_src = ms_per_step, "timed region: step = one launch (events around the K steps) / K"
    else:
        kev = [(ev(), ev()) for _ in range(K)]
        torch.cuda.synchronize()
        for i in range(K):
            if flush is not None:
                flush.zero_()
                torch.sum(flush_rd, dim=0, out=flush_sum)
            kev[i][0].record(stream)
            wl.kernel(partial)
            kev[i][1].record(stream)
        torch.cuda.synchronize()
        kernel_ms = sum(a.elapsed_time(b) for a, b in kev) / K
        kernel_src = "second K-step pass, events around the kernel launch"
    # the same K steps without programmatic dependent launch (reported beside the
    # pipelined value: what each step costs when launches are fully serialised)
    ms_unpiped = None
    if pipelined:
        ctx.set_pipelined(False)
        if ws > 1:
            dist.barrier()
        torch.cuda.synchronize()
        u0, u1 = ev(), ev()
        u0.record(stream)
        for i in range(K):
            body()
        u1.record(stream)
        torch.cuda.synchronize()
        ms_unpiped = u0.elapsed_time(u1) / K
        if ws > 1:
            t = torch.tensor([ms_unpiped], dtype=torch.float64, device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms_unpiped = float(t.item())
        ctx.set_pipelined(True)
    ctx.check()
    result = ss.result()
    peaks = _peaks()
    roofline = wl.roofline(kernel_ms, peaks)
    roofline["kernel_ms_source"] = kernel_src
    # traffic = dram__bytes_read + dram__bytes_write of the dominant kernel per
    # launch, from one `ncu --set full` capture of THIS workload (same config,
    # precision and rows per GPU), summarised by tools/ncu_summary.py
    tkey = traffic_key(cfg, rows, args.layout)
    tp = os.path.join(ROOT, "profiles", "traffic", f"{tkey}.json")
    roofline["traffic"] = None
    roofline["traffic_key"] = tkey
    if os.path.exists(tp):
        try:
            t = json.load(open(tp))
            roofline["traffic"] = t.get("dram_bytes_per_launch")
            roofline["traffic_source"] = t.get("source")
        except Exception:
            pass

    # ---- e2e through the C ABI from pinned host buffers (ingestion writes the
    # columns the SUM reads next: not pipelined)
    ctx.set_pipelined(False)
    host = wl.e2e_host_buffers()
    torch.cuda.synchronize()
    res_host = torch.empty(LA, dtype=torch.int32, pin_memory=True)

    ss_e2e = ShardedSum(ctx, LA, wl.S, wl.e2e_kernel)

    def e2e_step():
        wl.e2e_ingest(host)
        res_host.copy_(ss_e2e(), non_blocking=True)

    for _ in range(2):
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
    e2e_global = sum(min(E2E_MAX_ROWS, b - a) for a, b in (shard_range(n_global, ws, r) for r in range(ws)))
    if wl.e2e_rows == rows:
        assert up.format_decimal(res_host.tolist(), wl.S) == result, "e2e result differs from the resident run"
    h2d = sum(hb.numel() for hb in host)
    e2e = {"value": e2e_global / (ems / K2 / 1e3), "unit": "tuples/s", "h2d_bytes_per_step": h2d,
           "d2h_bytes_per_step": LA * 4, "ms_per_step": ems / K2,
           # the host link is the e2e roofline: the rows' bytes over the step time,
           # beside a plain pinned host->device copy of the same size measured here
           "h2d_gbs": round(h2d / (ems / K2 / 1e3) / 1e9, 2), "h2d_copy_gbs": _h2d_copy_gbs(h2d)}
    if wl.e2e_rows < rows:
        e2e["rows"] = f"first {wl.e2e_rows} rows of each rank's shard ({e2e_global} in total)"

    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        cpu, oracle_full = cpu_baseline(wl)
        if oracle_full is not None:
            assert oracle_full == result, f"bench SUM {result} != oracle SUM {oracle_full}"
            cpu["parity"] = "bench result == oracle SUM over every row"

    if rank == 0:
        desc = {"workload": cfg["name"], "rows_per_gpu": rows, "global_rows": n_global,
                "parallelism": f"rows sharded x{ws}, NCCL all-gather of partials + exact combine" if ws > 1
                else "1 GPU",
                "l2": ("flushed before every step (256 MB write, then a 256 MB read that writes the dirty lines back)" if flush is not None
                       else "inputs larger than L2 or compute-bound (no flush)")}
        desc.update(wl.workload_desc())
        if cfg["kind"] == "expr":
            desc["layout"] = args.layout
        desc["pipelined"] = pipelined
        if ms_unpiped is not None:
            desc["not_pipelined"] = {"ms_per_step": ms_unpiped, "value": n_global / (ms_unpiped / 1e3)}
        line = {
            "metric": METRIC, "value": value, "unit": "tuples/s", "n_gpus": ws, "steps": K,
            "warmup": args.warmup, "warmup_extra_untimed": warm_extra, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": scaling,
            "vs_baseline": None, "dtype": "u32", "data": "synthetic", "config": desc,
            "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches,
            "clocks": clk.summary(), "result": result, "jit_ms": round(ctx.jit_ms, 1),
        }
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
