"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (same kernels, same grid sizing): full-column SUMs where the oracle can
afford every row (cfg2 10M, cfg3 12.5M), sampled rows + the shard-combine
invariant where it cannot (cfg4 10M RSA, cfg5 1M sines).

Full-size inputs come from gen/'s device twin (bit-identical to the host
generator, tests/test_gpu_parity.py::test_device_generator_matches_host_twin)
and are copied to the host for the oracle; they never pass through libup."""
import os

import numpy as np
import pytest

import oracle
from gen import device as gdev
from gen import synth
from tests import gpu_util as G

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

CORES = max(1, len(os.sched_getaffinity(0)))


def _dev_cols(n, types, config, lead=()):
    cols, host = [], []
    for k, (p, s) in enumerate(types):
        mag, neg = gdev.uniform_decimal(n, p, config, k + 1, nonzero_lead=(k in lead))
        cols.append(G.ctx().column_from_device_bin(p, s, mag, neg))
        host.append((mag.cpu().numpy().view(np.uint32), neg.cpu().numpy()))
    G.ctx().check()
    return cols, host


@pytest.mark.parametrize("cfg", [(2, "c1+c2", [(35, 5), (32, 2)], 10_000_000, ()),
                                 (3, "c1*c2 - c3/c4", [(200, 50)] * 4, 12_500_000, (3,))])
def test_full_size_sum(cfg):
    config, expr, types, n, lead = cfg
    cols, host = _dev_cols(n, types, config, lead)
    got, P, S = G.gpu_sum_string(expr, cols)
    want, oP, oS = oracle.eval_sum(expr, [oracle.Column(p, s, m, g) for (m, g), (p, s) in zip(host, types)],
                                   threads=CORES)
    assert (P, S) == (oP, oS)
    assert got == want


def test_full_size_modexp_sampled_and_shard_invariant():
    from paper_conf_icde_lixylz24_b200 import up
    import torch
    N, _, _ = synth.rsa_modulus(1024)
    n = 10_000_000
    d = len(str(N))
    mag, neg = gdev.uniform_range(synth.SEED, synth.stream_id(4, 0), n, 0, N - 1, signed=False)
    c = G.ctx()
    col = c.column_from_device_bin(d, 0, mag, neg)
    total = c.modexp_sum(col, 65537, N)
    # shard invariant: SUM(all) == combine(SUM(first half), SUM(second half))
    h = n // 2
    halves = [c.column_from_device_bin(d, 0, mag[:h], neg[:h]), c.column_from_device_bin(d, 0, mag[h:], neg[h:])]
    parts = torch.cat([c.modexp_sum(x, 65537, N, n_global=n) for x in halves])
    comb = c.sum_combine(parts, total.numel())
    c.check()
    assert torch.equal(comb, total)
    # sampled rows of the full-size column output
    out = c.modexp(col, 65537, N)
    c.check()
    idx = np.random.default_rng(1).choice(n, 512, replace=False)
    rows = out.data[:, torch.as_tensor(idx, device="cuda")].cpu().numpy().view(np.uint32).T
    mh = mag.cpu().numpy().view(np.uint32)
    for r, i in zip(rows, idx):
        m = synth.words_to_int(mh[i])
        assert synth.words_to_int(r) == pow(m, 65537, N)


def test_full_size_sin_sampled_and_shard_invariant():
    from paper_conf_icde_lixylz24_b200 import up
    import torch
    n, P = 1_000_000, 1000
    mag, neg = synth.normal_decimal(n, 0.78, 0.01, 8, config=5, column=0)
    c = G.ctx()
    col = c.column_from_host_bin(9, 8, mag, neg)
    total = c.sin_taylor_sum(col, P)
    h = n // 2
    halves = [c.column_from_host_bin(9, 8, mag[:h], neg[:h]), c.column_from_host_bin(9, 8, mag[h:], neg[h:])]
    parts = torch.cat([c.sin_taylor_sum(x, P, n_global=n) for x in halves])
    assert torch.equal(c.sum_combine(parts, total.numel()), total)
    out = c.sin_taylor(col, P)
    c.check()
    idx = np.random.default_rng(2).choice(n, 64, replace=False)
    got_rows = out.data[:, torch.as_tensor(idx, device="cuda")].cpu().numpy().view(np.uint32).T
    sample = oracle.Column(9, 8, mag[idx], neg[idx])
    want = oracle.sin_rows(sample, P)
    for g, w in zip(got_rows, want):
        assert up.format_decimal(g.tolist(), P) == w
