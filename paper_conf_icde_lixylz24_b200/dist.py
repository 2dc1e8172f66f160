"""Row-sharded SUM across GPUs (rows a13 / e): one process per GPU,
torch.distributed (NCCL over NVLink/NVSwitch) for the plumbing.

Rows are independent (the same expression is evaluated for every tuple,
P:L310-316) and the SUM is exact, so the only exchange is one all-gather of
the per-rank partials (LA int32 limbs each), followed by libup's exact
combine kernel on every rank (identical result everywhere).  Typing uses the
GLOBAL row count, so all ranks share LA.
"""
from __future__ import annotations

from typing import Sequence, Tuple


def shard_range(n_global: int, world: int, rank: int) -> Tuple[int, int]:
    """Contiguous row block [lo, hi) of rank `rank` (sizes differ by <= 1)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad world/rank")
    lo = n_global * rank // world
    hi = n_global * (rank + 1) // world
    return lo, hi


class ShardedSum:
    """SELECT SUM(expr) over a row-sharded table: local fused kernel, NCCL
    all-gather of the partials, exact combine -- all on `stream`."""

    def __init__(self, ctx, expr: str, cols: Sequence, n_global: int, group=None):
        import torch
        import torch.distributed as dist
        self.ctx, self.expr, self.cols, self.n_global, self.group = ctx, expr, list(cols), n_global, group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.P, self.S, self.LA = ctx.sum_type(expr, self.cols, n_global)
        dev = self.cols[0].data.device
        self.partial = torch.empty(self.LA, dtype=torch.int32, device=dev)
        self.gathered = torch.empty(self.LA * self.world, dtype=torch.int32, device=dev)
        self.total = torch.empty(self.LA, dtype=torch.int32, device=dev)

    def __call__(self):
        import torch.distributed as dist
        self.ctx.sum_expr(self.expr, self.cols, self.n_global, out=self.partial)
        if self.world == 1:
            return self.partial
        dist.all_gather_into_tensor(self.gathered, self.partial, group=self.group)
        self.ctx.sum_combine(self.gathered, self.LA, out=self.total)
        return self.total

    def result(self) -> str:
        from . import up
        return up.result_to_string(self.total if self.world > 1 else self.partial, self.S)
