"""Multi-GPU plumbing for the migration path (S§8(e)): one process per GPU, torch process
groups ONLY to exchange the 512-byte pool handles and to run barriers / the max-over-ranks
timing reduction.  No collective touches KV bytes: those move by peer stores inside the
copy kernel (wind_kv_migrate / wind_kv_migrate_batch on an imported pool).

Sharding.  Prefill->decode hand-offs are independent units (each request's
KV goes from one prefill instance to one decode instance), so N ranks form N // 2 pairs
2k -> 2k+1 (every pairing is equivalent through NVSwitch); an odd last rank has no
partner and runs an intra-device migration.  All-to-all rebalancing (A8) is one exchange
step planned identically on every rank (rebalance.py).
"""
from __future__ import annotations

from typing import Optional, Sequence


def pair_role(rank: int, world: int) -> tuple[str, Optional[int]]:
    """('push', partner) for the prefill (source) rank of a pair, ('decode', partner) for
    the destination rank, ('solo', None) for a rank without a partner."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    if rank % 2 == 0 and rank + 1 < world:
        return "push", rank + 1
    if rank % 2 == 1:
        return "decode", rank - 1
    return "solo", None


def movers(world: int) -> int:
    """Ranks that issue a migration per step (pairs + an unpaired last rank)."""
    return world // 2 + world % 2


def exchange_handles(handle: Optional[bytes], group=None) -> list:
    """all_gather_object of this rank's exported pool handle (or None)."""
    import torch.distributed as dist
    out: list = [None] * dist.get_world_size(group)
    dist.all_gather_object(out, handle, group=group)
    return out


def max_over_ranks(values: Sequence[float], group=None) -> list[float]:
    """Element-wise max of per-rank floats (device times are maxed, never wall clock)."""
    import torch
    import torch.distributed as dist
    t = torch.tensor(list(values), dtype=torch.float64)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return [float(x) for x in t]
