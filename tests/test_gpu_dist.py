"""Multi-rank product path on ONE GPU (rows a13 / e): two processes share
cuda:0 over a gloo process group (partials staged through host memory) and
run the product's ShardedSum end to end -- each rank generates its shard keyed
by the GLOBAL row index on the device, types with the global N, runs its fused
libup SUM kernel, all-gathers the LA-limb partials and runs libup's exact
combine kernel.  Every rank's result must equal the oracle's SUM over the
whole column.  With NCCL on N GPUs (bench.py --gpus N) the same class gathers
device to device; only the transport differs."""
import os
import socket

import pytest

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, kind, n, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    from gen import device as gdev
    from gen import synth
    from paper_conf_icde_lixylz24_b200 import up
    from paper_conf_icde_lixylz24_b200.dist import ShardedSum, shard_range
    ctx = up.Context(0)
    lo, hi = shard_range(n, world, rank)
    if kind == "expr":
        types = [(35, 5), (32, 2)]
        cols = []
        for k, (p, s) in enumerate(types):
            mag, neg = gdev.uniform_decimal(hi - lo, p, 2, k + 1, row0=lo)
            cols.append(ctx.column_from_device_bin(p, s, mag, neg))
        ss = ShardedSum.expr(ctx, "c1+c2", cols, n)
    elif kind == "cfg3q":
        # cfg3's SUM(c1*c2 - c3/c4) over limb quads: every rank runs the split
        # (tensor-core contraction + top-limb division) on its shard
        types = [(200, 50)] * 4
        cols = []
        for k, (p, s) in enumerate(types):
            mag, neg = gdev.uniform_decimal(hi - lo, p, 3, k + 1, row0=lo, nonzero_lead=(k == 3))
            cols.append(ctx.column_from_device_bin(p, s, mag, neg, layout="quads"))
        ss = ShardedSum.expr(ctx, "c1*c2 - c3/c4", cols, n)
    elif kind == "modexp":
        N, _, _ = synth.rsa_modulus(256)
        mag, neg = gdev.uniform_range(synth.SEED, synth.stream_id(4, 0), hi - lo, 0, N - 1, signed=False, row0=lo)
        ss = ShardedSum.modexp(ctx, ctx.column_from_device_bin(len(str(N)), 0, mag, neg), 65537, N, n)
    elif kind == "group":
        import numpy as np
        from paper_conf_icde_lixylz24_b200.dist import ShardedGroupAggregate
        types = [(12, 2), (12, 2), (3, 2)]
        cols = [ctx.column_from_host_bin(p, s, *synth.uniform_decimal(hi - lo, p, 8, k + 1, row0=lo))
                for k, (p, s) in enumerate(types)]
        gid = torch.as_tensor(_group_ids(n)[lo:hi].copy(), device="cuda")
        sga = ShardedGroupAggregate(ctx, GROUP_AGGS, cols, gid, 5, n)
        out, counts, layout = sga()
        ctx.check()
        res, cnt = up.group_results(out, counts, layout, 5)
        allg = [None] * world
        dist.all_gather_object(allg, (res, cnt))
        assert all(a == allg[0] for a in allg)
        if rank == 0:
            q.put((res, cnt))
        dist.barrier()
        dist.destroy_process_group()
        return
    else:
        mag, neg = synth.normal_decimal(hi - lo, 0.78, 0.01, 8, config=5, column=0, row0=lo)
        ss = ShardedSum.sin(ctx, ctx.column_from_host_bin(9, 8, mag, neg), 300, n)
    assert ss.stage_host and ss.world == world
    ss()
    ctx.check()
    got = ss.result()
    allg = [None] * world
    dist.all_gather_object(allg, got)
    assert len(set(allg)) == 1
    if rank == 0:
        q.put(got)
    dist.barrier()
    dist.destroy_process_group()


GROUP_AGGS = [("SUM", "c1"), ("AVG", "c2*(1-c3)"), ("MIN", "c1-c2"), ("MAX", "c2"), ("AVG", "c3")]


def _group_ids(n):
    import numpy as np
    g = np.random.default_rng(23).integers(0, 5, n).astype(np.int32)
    g[np.random.default_rng(24).random(n) < 0.1] = -1
    return g


def _oracle_whole(kind, n):
    import oracle
    from gen import synth
    if kind == "group":
        types = [(12, 2), (12, 2), (3, 2)]
        host = [synth.uniform_decimal(n, p, 8, k + 1) for k, (p, s) in enumerate(types)]
        res, cnt, _ = oracle.group_aggregate(GROUP_AGGS, [oracle.Column(p, s, m, g) for (m, g), (p, s) in zip(host, types)],
                                             _group_ids(n), 5, n)
        return (res, cnt)
    if kind == "expr":
        types = [(35, 5), (32, 2)]
        host = [synth.uniform_decimal(n, p, 2, k + 1) for k, (p, s) in enumerate(types)]
        return oracle.eval_sum("c1+c2", [oracle.Column(p, s, m, g) for (m, g), (p, s) in zip(host, types)],
                               threads=4)[0]
    if kind == "cfg3q":
        types = [(200, 50)] * 4
        host = [synth.uniform_decimal(n, p, 3, k + 1, nonzero_lead=(k == 3)) for k, (p, s) in enumerate(types)]
        return oracle.eval_sum("c1*c2 - c3/c4", [oracle.Column(p, s, m, g) for (m, g), (p, s) in zip(host, types)],
                               threads=4)[0]
    if kind == "modexp":
        N, _, _ = synth.rsa_modulus(256)
        m, g = synth.rsa_messages(n, N)
        return oracle.modexp_sum(oracle.Column(len(str(N)), 0, m, g), 65537, N, threads=4)
    m, g = synth.normal_decimal(n, 0.78, 0.01, 8, config=5, column=0)
    return oracle.sin_sum(oracle.Column(9, 8, m, g), 300, threads=4)


@pytest.mark.parametrize("kind,n,world", [("expr", 1, 2), ("expr", 100_003, 2), ("modexp", 3001, 2),
                                          ("sin", 2049, 2), ("expr", 50_000, 3), ("group", 30_001, 2),
                                          ("group", 7, 3), ("cfg3q", 4001, 2)])
def test_sharded_sum_two_processes_one_gpu(kind, n, world):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, kind, n, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(300)
        assert p.exitcode == 0
    assert q.get(timeout=10) == _oracle_whole(kind, n)
