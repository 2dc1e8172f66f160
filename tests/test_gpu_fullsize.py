"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (same generators, same kernels, same grid sizing).

Expected SUMs come from tests/golden/fullsize_sums.json, written by
tools/make_golden.py from gen/'s host generators and the ORACLE only (hours
of CPU work, done once on the build host; no value in it comes from libup).
Here the same columns are generated on the device (gen/'s device twin,
bit-identical to the host generator: test_gpu_parity.py::
test_device_generator_matches_host_twin) and summed through the C ABI.
cfg2 at 10M rows is also re-checked against the oracle live.  Column outputs
(modexp, sin_P) are checked on sampled rows against Python pow / the oracle."""
import json
import os

import numpy as np
import pytest

import oracle
from gen import device as gdev
from gen import synth
from tests import gpu_util as G

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

CORES = max(1, len(os.sched_getaffinity(0)))
GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "fullsize_sums.json")))


def _dev_cols(n, types, config, lead=()):
    cols = []
    for k, (p, s) in enumerate(types):
        mag, neg = gdev.uniform_decimal(n, p, config, k + 1, nonzero_lead=(k in lead))
        cols.append(G.ctx().column_from_device_bin(p, s, mag, neg))
        del mag, neg
    G.ctx().check()
    return cols


@pytest.mark.parametrize("name", ["cfg3_p200", "cfg3_p500", "cfg3_p1000"])
def test_full_size_cfg3_quads_vs_golden(name):
    """cfg3 as the bench runs it -- limb-quad columns, the tensor-core
    contraction fed straight from TMA (148 CTAs, several accumulation windows
    each) plus the top-limb division -- against the oracle's full SUM"""
    import torch
    g = _gold(name)
    w = g["workload"]
    types = [tuple(t) for t in w["types"]]
    lead = tuple(w.get("lead", ()))
    c = G.ctx()
    cols = []
    for k, (p, s) in enumerate(types):
        mag, neg = gdev.uniform_decimal(w["rows"], p, w["config"], k + 1, nonzero_lead=(k in lead))
        cols.append(c.column_from_device_bin(p, s, mag, neg, layout="quads"))
        del mag, neg
    c.check()
    got, P, S = G.gpu_sum_string(w["expr"], cols)
    assert (P, S) == (g["p"], g["s"])
    assert got == g["sum"]
    del cols
    torch.cuda.empty_cache()


def _gold(name):
    if name not in GOLD:   # oracle runs of ~0.5 h each are written off the GPU box (tools/make_golden.py)
        pytest.skip(f"golden entry {name} not computed yet: run tools/make_golden.py --only {name}")
    return GOLD[name]


@pytest.mark.parametrize("name", ["cfg2_10M", "cfg3_p200", "cfg3_p500", "cfg3_p1000", "cfg1_2p30", "cfg2_2p30"])
def test_full_size_expr_sum_vs_golden(name):
    import torch
    g = _gold(name)
    w = g["workload"]
    types = [tuple(t) for t in w["types"]]
    cols = _dev_cols(w["rows"], types, w["config"], tuple(w.get("lead", ())))
    got, P, S = G.gpu_sum_string(w["expr"], cols)
    assert (P, S) == (g["p"], g["s"])
    assert got == g["sum"]
    del cols
    torch.cuda.empty_cache()


def test_full_size_cfg2_live_oracle():
    """cfg2 (the headline) against the oracle computed here, not only the file."""
    types = [(35, 5), (32, 2)]
    n = 10_000_000
    host = []
    cols = []
    for k, (p, s) in enumerate(types):
        mag, neg = gdev.uniform_decimal(n, p, 2, k + 1)
        cols.append(G.ctx().column_from_device_bin(p, s, mag, neg))
        host.append((mag.cpu().numpy().view(np.uint32), neg.cpu().numpy()))
    got, P, S = G.gpu_sum_string("c1+c2", cols)
    want, oP, oS = oracle.eval_sum("c1+c2", [oracle.Column(p, s, m, g) for (m, g), (p, s) in zip(host, types)],
                                   threads=CORES)
    assert (P, S) == (oP, oS) and got == want == _gold("cfg2_10M")["sum"]


@pytest.mark.parametrize("name", ["cfg4_1024_e65537", "cfg4_1024_e3", "cfg4_2048_e65537"])
def test_full_size_modexp_sum_vs_golden(name):
    from paper_conf_icde_lixylz24_b200 import up
    g = _gold(name)
    w = g["workload"]
    N, _, _ = synth.rsa_modulus(w["bits"])
    n = w["rows"]
    mag, neg = gdev.uniform_range(synth.SEED, synth.stream_id(4, 0), n, 0, N - 1, signed=False)
    c = G.ctx()
    col = c.column_from_device_bin(len(str(N)), 0, mag, neg)
    total = c.modexp_sum(col, w["e"], N)
    c.check()
    assert up.result_to_string(total, 0) == g["sum"]
    if name == "cfg4_1024_e65537":
        # sampled rows of the full-size column output vs Python pow
        import torch
        out = c.modexp(col, w["e"], N)
        c.check()
        idx = np.random.default_rng(1).choice(n, 512, replace=False)
        rows = out.data[:, torch.as_tensor(idx, device="cuda")].cpu().numpy().view(np.uint32).T
        mh = mag.cpu().numpy().view(np.uint32)
        for r, i in zip(rows, idx):
            assert synth.words_to_int(r) == pow(synth.words_to_int(mh[i]), w["e"], N)


@pytest.mark.parametrize("name", ["cfg5_P500", "cfg5_P1000", "cfg5_P5000", "cfg5_P20000_100k"])
def test_full_size_sin_sum_vs_golden(name):
    from paper_conf_icde_lixylz24_b200 import up
    g = _gold(name)
    w = g["workload"]
    mag, neg = synth.normal_decimal(w["rows"], w["mu"], 0.01, 8, config=5, column=0)
    c = G.ctx()
    col = c.column_from_host_bin(9, 8, mag, neg)
    total = c.sin_taylor_sum(col, w["P"])
    c.check()
    assert up.result_to_string(total, w["P"]) == g["sum"]
    if name == "cfg5_P1000":
        import torch
        out = c.sin_taylor(col, w["P"])
        c.check()
        idx = np.random.default_rng(2).choice(w["rows"], 64, replace=False)
        got_rows = out.data[:, torch.as_tensor(idx, device="cuda")].cpu().numpy().view(np.uint32).T
        want = oracle.sin_rows(oracle.Column(9, 8, mag[idx], neg[idx]), w["P"])
        for gr, wr in zip(got_rows, want):
            assert G.limbs_int(gr.tolist()) == int(wr.replace(".", ""))
