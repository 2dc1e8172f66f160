"""Row-sharded SUM across GPUs (rows a13 / e): one process per GPU,
torch.distributed (NCCL over NVLink/NVSwitch) for the plumbing.

Rows are independent (the same expression is evaluated for every tuple,
P:L310-316) and the SUM is exact, so the only exchange is one all-gather of
the per-rank partials (LA int32 limbs each), followed by libup's exact
combine kernel on every rank (identical result everywhere).  Typing uses the
GLOBAL row count, so all ranks share LA.

With NCCL the partials are gathered device to device on the current stream.
With gloo (CPU process groups: tests, or several ranks sharing one GPU) the
partials are staged through host memory; the combine still runs on the GPU.
"""
from __future__ import annotations

from typing import Callable, Sequence, Tuple


def shard_range(n_global: int, world: int, rank: int) -> Tuple[int, int]:
    """Contiguous row block [lo, hi) of rank `rank` (sizes differ by <= 1)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad world/rank")
    lo = n_global * rank // world
    hi = n_global * (rank + 1) // world
    return lo, hi


class ShardedSum:
    """A row-sharded SELECT SUM: `local(out)` writes this rank's LA-limb
    partial into `out` (one fused libup kernel), then one all-gather of the
    partials and libup's exact combine kernel -- all on the current stream.

    Build with `ShardedSum.expr / .modexp / .sin` (SUM(expr), SUM(x^e mod N),
    SUM(sin_P(x))) or directly with any `local` writing LA limbs."""

    def __init__(self, ctx, LA: int, S: int, local: Callable, group=None, device=None, stage_host=None):
        import torch
        import torch.distributed as dist
        self.ctx, self.LA, self.S, self.local, self.group = ctx, LA, S, local, group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        if stage_host is None:
            stage_host = dist.is_initialized() and dist.get_backend(group) == "gloo"
        self.stage_host = stage_host
        dev = device if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.partial = torch.zeros(LA, dtype=torch.int32, device=dev)
        self.gathered = torch.empty(LA * self.world, dtype=torch.int32, device=dev)
        self.total = torch.empty(LA, dtype=torch.int32, device=dev)
        if stage_host:
            self.h_partial = torch.empty(LA, dtype=torch.int32)
            self.h_gathered = torch.empty(LA * self.world, dtype=torch.int32)

    # ------------------------------------------------------------------ builders
    @classmethod
    def expr(cls, ctx, expr: str, cols: Sequence, n_global: int, **kw):
        P, S, LA = ctx.sum_type(expr, list(cols), n_global)
        cols = list(cols)
        return cls(ctx, LA, S, lambda out: ctx.sum_expr(expr, cols, n_global, out=out), **kw)

    @classmethod
    def modexp(cls, ctx, base, exponent: int, modulus: int, n_global: int, **kw):
        _, LA = ctx.modexp_sum_type(modulus, n_global)
        return cls(ctx, LA, 0, lambda out: ctx.modexp_sum(base, exponent, modulus, n_global, out=out), **kw)

    @classmethod
    def sin(cls, ctx, x, P: int, n_global: int, **kw):
        from . import up
        LA = up.limbs(up.sum_precision(P + 1, n_global))
        return cls(ctx, LA, P, lambda out: ctx.sin_taylor_sum(x, P, n_global, out=out), **kw)

    # ------------------------------------------------------------------ step
    def __call__(self):
        import torch.distributed as dist
        self.local(self.partial)
        if self.world == 1:
            return self.partial
        if self.stage_host:
            self.h_partial.copy_(self.partial)
            dist.all_gather_into_tensor(self.h_gathered, self.h_partial, group=self.group)
            self.gathered.copy_(self.h_gathered)
        else:
            dist.all_gather_into_tensor(self.gathered, self.partial, group=self.group)
        self.ctx.sum_combine(self.gathered, self.LA, out=self.total)
        return self.total

    def result_tensor(self):
        return self.total if self.world > 1 else self.partial

    def result(self) -> str:
        from . import up
        return up.result_to_string(self.result_tensor(), self.S)


class ShardedGroupAggregate:
    """SELECT agg(expr), ... GROUP BY g over a row-sharded table (NEXT-4 across
    ranks): each rank runs the one-launch grouped aggregation over its rows
    with AVG computed as SUM (typing with the global row count), one
    all-gather of the packed partials and one of the group counts, then
    libup's up_group_combine kernel (exact SUM, MIN / MAX over non-empty
    ranks, AVG from the combined SUM and COUNT) -- identical on every rank."""

    def __init__(self, ctx, aggs, cols, group, n_groups: int, n_global: int, group_pg=None, stage_host=None):
        import torch
        import torch.distributed as dist
        self.ctx, self.aggs, self.cols, self.group = ctx, list(aggs), list(cols), group
        self.n_groups, self.n_global, self.pg = n_groups, n_global, group_pg
        self.world = dist.get_world_size(group_pg) if dist.is_initialized() else 1
        if stage_host is None:
            stage_host = dist.is_initialized() and dist.get_backend(group_pg) == "gloo"
        self.stage_host = stage_host

    def __call__(self):
        import torch
        import torch.distributed as dist
        out, counts, layout = self.ctx.group_aggregate(self.aggs, self.cols, self.group, self.n_groups,
                                                       self.n_global, partial=self.world > 1)
        if self.world == 1:
            return out, counts, layout
        W = self.world
        if self.stage_host:
            ho, hc = out.cpu(), counts.cpu()
            go = torch.empty(W * ho.numel(), dtype=ho.dtype)
            gc = torch.empty(W * hc.numel(), dtype=hc.dtype)
            dist.all_gather_into_tensor(go, ho, group=self.pg)
            dist.all_gather_into_tensor(gc, hc, group=self.pg)
            go, gc = go.to(out.device), gc.to(out.device)
        else:
            go = torch.empty(W * out.numel(), dtype=out.dtype, device=out.device)
            gc = torch.empty(W * counts.numel(), dtype=counts.dtype, device=counts.device)
            dist.all_gather_into_tensor(go, out, group=self.pg)
            dist.all_gather_into_tensor(gc, counts, group=self.pg)
        return self.ctx.group_combine(self.aggs, self.cols, go, gc, W, self.n_groups, self.n_global)
