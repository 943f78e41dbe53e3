"""All-to-all KV rebalancing across GPUs (S§8(a) A8; not in the paper — nearest are
Dynamic Rescheduling's decode->prefill moves of long-context requests, and
"load balancing across instances" as future work).

Host-side, deterministic, identical on every rank: given where each request's blocks live
and where each request should go (``plan_rebalance`` — longest-first greedy, P:227/P:233 —
or a uniform hash shuffle), assign destination slots lowest-free-first (R10) among the
slots that were free BEFORE the exchange (slots freed by outgoing requests are not reused
in the same step, so no write can land in a block another GPU is still reading), and emit
per (source GPU, destination GPU) block tables.  Each source GPU then pushes to all its
peers in ONE wind_kv_migrate_batch launch over the imported peer pools.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from . import MAX_BATCH, Pool, migrate_batch
from . import plan_rebalance as _plan_rebalance


@dataclass
class ExchangePlan:
    n_gpus: int
    dest_gpu: np.ndarray                      # final GPU per request
    moves: dict = field(default_factory=dict)  # (src_gpu, dst_gpu) -> (src_bt, dst_bt) int32
    new_tables: list = field(default_factory=list)  # per request: slots in its final pool
    blocks_moved: int = 0

    def items_for(self, gpu: int) -> list[tuple[int, np.ndarray, np.ndarray]]:
        """Outgoing (dst_gpu, src_bt, dst_bt) of `gpu`, ascending dst_gpu."""
        return [(d, s_bt, d_bt) for (s, d), (s_bt, d_bt) in sorted(self.moves.items())
                if s == gpu and s_bt.size]

    def incoming(self, gpu: int) -> int:
        return sum(int(s_bt.size) for (s, d), (s_bt, _) in self.moves.items() if d == gpu)


def plan_exchange(n_gpus: int, req_gpu, req_tables, free_masks, dest_gpu) -> ExchangePlan:
    """req_gpu[r]: current GPU; req_tables[r]: its slots there; free_masks[g]: bool array of
    GPU g's free slots before the exchange; dest_gpu[r]: target GPU."""
    req_gpu = np.asarray(req_gpu, np.int32)
    dest_gpu = np.asarray(dest_gpu, np.int32)
    free = [np.asarray(m, bool).copy() for m in free_masks]
    cursor = [0] * n_gpus
    acc: dict = {}
    new_tables = []
    moved = 0
    for r in range(req_gpu.size):
        s, d = int(req_gpu[r]), int(dest_gpu[r])
        tbl = np.asarray(req_tables[r], np.int32)
        if s == d or tbl.size == 0:
            new_tables.append(tbl.copy())
            continue
        # lowest free slots of GPU d at or after the cursor (slots before it are taken)
        cand = np.flatnonzero(free[d][cursor[d]:]) + cursor[d]
        if cand.size < tbl.size:
            raise ValueError(f"GPU {d} has {cand.size} free slots, request {r} needs {tbl.size}")
        slots = cand[:tbl.size].astype(np.int32)
        free[d][slots] = False
        cursor[d] = int(slots[-1]) + 1
        a = acc.setdefault((s, d), ([], []))
        a[0].append(tbl)
        a[1].append(slots)
        new_tables.append(slots)
        moved += int(tbl.size)
    moves = {k: (np.concatenate(v[0]).astype(np.int32), np.concatenate(v[1]).astype(np.int32))
             for k, v in acc.items()}
    return ExchangePlan(n_gpus, dest_gpu, moves, new_tables, moved)


def plan_rebalance_exchange(n_gpus: int, req_gpu, req_tables, free_masks) -> ExchangePlan:
    """The realistic plan: wind_kv_plan_rebalance chooses destinations, then slots."""
    blocks = np.array([len(t) for t in req_tables], np.int32)
    dest, _ = _plan_rebalance(n_gpus, req_gpu, blocks)
    return plan_exchange(n_gpus, req_gpu, req_tables, free_masks, dest)


def execute(plan: ExchangePlan, gpu: int, local: Pool, peers: dict, tables_on_device,
            layer_lo: int, layer_hi: int, stream=None) -> int:
    """Issue this GPU's outgoing pushes: one migrate_batch launch per <= 16 destinations.
    `peers[d]` is the (imported) pool of GPU d; `tables_on_device(np_array)` moves a table
    to device memory of this GPU (the caller keeps it alive until the op completes).
    Returns the number of blocks pushed."""
    items = plan.items_for(gpu)
    sent = 0
    for k in range(0, len(items), MAX_BATCH):
        chunk = items[k:k + MAX_BATCH]
        batch = [(peers[d], tables_on_device(s_bt), tables_on_device(d_bt)) for d, s_bt, d_bt in chunk]
        migrate_batch(local, batch, layer_lo, layer_hi, stream=stream)
        sent += sum(int(s.size) for _, s, _ in chunk)
    return sent
