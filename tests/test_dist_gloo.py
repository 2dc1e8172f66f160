"""Multi-rank host logic on CPU (gloo, world_size 2): row sharding, global-N
typing shared by all ranks, the all-gather of LA-limb two's-complement
partials, and the exact-combine invariant (sum of shard sums = whole SUM).
The GPU combine kernel itself is covered by tests/test_gpu_parity.py."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icde_lixylz24_b200.dist import shard_range


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_shard_range_partitions_rows():
    for n in (0, 1, 7, 10_000_000, 2 ** 30):
        for w in (1, 2, 3, 4, 8):
            parts = [shard_range(n, w, r) for r in range(w)]
            assert parts[0][0] == 0 and parts[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(parts, parts[1:]))
            sizes = [hi - lo for lo, hi in parts]
            assert max(sizes) - min(sizes) <= 1
    with pytest.raises(ValueError):
        shard_range(10, 2, 2)


def _to_limbs(v, la):
    u = v & ((1 << (32 * la)) - 1)
    return [((u >> (32 * j)) & 0xFFFFFFFF) - (1 << 32 if (u >> (32 * j)) & 0x80000000 else 0) for j in range(la)]


def _from_limbs(ls):
    v = 0
    for j, x in enumerate(ls):
        v |= (int(x) & 0xFFFFFFFF) << (32 * j)
    la = len(ls)
    return v - (1 << (32 * la)) if v >> (32 * la - 1) else v


def _worker(rank, world, port, n, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from gen import synth
    from paper_conf_icde_lixylz24_b200 import up
    types = [(35, 5), (32, 2)]
    lo, hi = shard_range(n, world, rank)
    # each rank generates its own shard, keyed by the global row index
    host = [synth.uniform_decimal(hi - lo, p, 2, k + 1, row0=lo) for k, (p, s) in enumerate(types)]
    ocols = [oracle.Column(p, s, m, g) for (m, g), (p, s) in zip(host, types)]
    part, P, S = oracle.eval_sum("c1+c2", ocols, n_global=n)
    la = up.limbs(P)
    assert P == up.sum_precision(36, n)
    mant = int(part.replace(".", ""))
    t = torch.tensor(_to_limbs(mant, la), dtype=torch.int32)
    out = torch.empty(la * world, dtype=torch.int32)
    dist.all_gather_into_tensor(out, t)
    total = sum(_from_limbs(out[r * la:(r + 1) * la].tolist()) for r in range(world))
    # every rank holds the same exact total
    tt = torch.tensor(_to_limbs(total, la), dtype=torch.int32)
    ref = tt.clone()
    dist.broadcast(ref, 0)
    assert torch.equal(ref, tt)
    if rank == 0:
        whole_host = [synth.uniform_decimal(n, p, 2, k + 1) for k, (p, s) in enumerate(types)]
        whole, wP, wS = oracle.eval_sum("c1+c2", [oracle.Column(p, s, m, g) for (m, g), (p, s) in
                                                  zip(whole_host, types)])
        q.put((whole, up.format_decimal([x & 0xFFFFFFFF for x in tt.tolist()], S)))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("n", [1, 2001])
def test_gloo_two_rank_sharded_sum(n):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, n, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(180)
        assert p.exitcode == 0
    whole, got = q.get(timeout=10)
    assert got == whole


class _OracleCtx:
    """Test double for libup's ctx on a GPU-less host: shard SUMs by the
    oracle, the combine by Python ints.  It lets the gloo test drive the
    product's ShardedSum plumbing (global-N typing, host staging, all-gather
    order, empty shards) without a GPU; the real ctx runs the same class in
    tests/test_gpu_dist.py."""

    def sum_type(self, expr, cols, n_global):
        import oracle
        from paper_conf_icde_lixylz24_b200 import up
        p, s = oracle.expr_type(expr, cols)
        P, S = oracle.sum_type(p, s, n_global)
        return P, S, up.limbs(P)

    def sum_expr(self, expr, cols, n_global, out):
        import oracle
        v, P, S = oracle.eval_sum(expr, cols, n_global=n_global)
        out.copy_(torch.tensor(_to_limbs(int(v.replace(".", "")), out.numel()), dtype=torch.int32))
        return out

    def sum_combine(self, gathered, la, out):
        tot = sum(_from_limbs(gathered[r * la:(r + 1) * la].tolist()) for r in range(gathered.numel() // la))
        out.copy_(torch.tensor(_to_limbs(tot, la), dtype=torch.int32))
        return out


def _sharded_worker(rank, world, port, n, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from gen import synth
    from paper_conf_icde_lixylz24_b200.dist import ShardedSum
    types = [(35, 5), (32, 2)]
    lo, hi = shard_range(n, world, rank)
    host = [synth.uniform_decimal(hi - lo, p, 2, k + 1, row0=lo) for k, (p, s) in enumerate(types)]
    cols = [oracle.Column(p, s, m, g) for (m, g), (p, s) in zip(host, types)]
    ss = ShardedSum.expr(_OracleCtx(), "c1+c2", cols, n, device=torch.device("cpu"))
    assert ss.stage_host and ss.world == world
    ss()
    from paper_conf_icde_lixylz24_b200 import up
    got = up.format_decimal([x & 0xFFFFFFFF for x in ss.result_tensor().tolist()], ss.S)
    allg = [None] * world
    dist.all_gather_object(allg, got)
    assert len(set(allg)) == 1            # every rank holds the same exact total
    if rank == 0:
        whole_host = [synth.uniform_decimal(n, p, 2, k + 1) for k, (p, s) in enumerate(types)]
        whole, _, _ = oracle.eval_sum("c1+c2", [oracle.Column(p, s, m, g) for (m, g), (p, s) in
                                                zip(whole_host, types)])
        q.put((whole, got))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,n", [(2, 1), (2, 2001), (3, 2)])
def test_gloo_sharded_sum_plumbing(world, n):
    """The product's ShardedSum over gloo (world 2 and 3) with a test-double
    ctx: includes empty shards (n_global < world)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_sharded_worker, args=(r, world, port, n, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(180)
        assert p.exitcode == 0
    whole, got = q.get(timeout=10)
    assert got == whole
