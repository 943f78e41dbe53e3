"""N > 1 host logic on CPU with gloo process groups (world size 2 and 4): pairing, pool
handle exchange, max-over-ranks timing, and the all-to-all rebalancing plan (A8) that
every rank must derive identically.  The KV bytes of the exchange are simulated with the
CPU oracle to check that every request's logical KV survives the plan (S§8(c) P7)."""
import hashlib
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import oracle as O
from paper_conf_isca_fenghzly025_b200 import parallel, rebalance
from windgen import blocks_for_tokens, lengths_longtail, skewed_placement, hash_shuffle_dest


def free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def synthetic_cluster(G: int, R: int = 120, seed: int = 5):
    """Requests placed on G GPU pools (skewed, C5-like), slots shuffled inside each pool."""
    rng = np.random.default_rng(seed)
    blocks = np.minimum(blocks_for_tokens(lengths_longtail(R, seed), 16), 40).astype(np.int32)
    gpu = skewed_placement(R, G, seed)
    nb = [int(blocks[gpu == g].sum() * 2.5) + 64 for g in range(G)]
    nb = [max(nb)] * G  # equal pool sizes, as on identical GPUs
    tables, free = [], []
    perms = [rng.permutation(n) for n in nb]
    pos = [0] * G
    for r in range(R):
        g = int(gpu[r])
        tables.append(perms[g][pos[g]:pos[g] + blocks[r]].astype(np.int32))
        pos[g] += int(blocks[r])
    for g in range(G):
        m = np.ones(nb[g], bool)
        m[perms[g][:pos[g]]] = False
        free.append(m)
    return gpu, tables, free, nb, blocks


def plan_digest(plan) -> str:
    h = hashlib.sha256()
    for k in sorted(plan.moves):
        h.update(repr(k).encode())
        for a in plan.moves[k]:
            h.update(a.tobytes())
    return h.hexdigest()


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        role, partner = parallel.pair_role(rank, world)
        mine = bytes([rank + 1]) * 512 if role == "decode" else None
        handles = parallel.exchange_handles(mine)
        got = handles[partner] if role == "push" else None
        mx = parallel.max_over_ranks([float(rank), 10.0 - rank])
        gpu, tables, free, nb, blocks = synthetic_cluster(world)
        plan = rebalance.plan_rebalance_exchange(world, gpu, tables, free)
        shuffle = rebalance.plan_exchange(world, gpu, tables, free, hash_shuffle_dest(len(tables), world, 9))
        items = [(d, s.tolist(), t.tolist()) for d, s, t in plan.items_for(rank)]
        out = [None] * world
        dist.all_gather_object(out, (role, partner, got, mx, plan_digest(plan), plan_digest(shuffle), items))
        if rank == 0:
            q.put(out)
        dist.barrier()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3, 4])
def test_gloo_ranks_agree(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = q.get(timeout=180)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    roles = [o[0] for o in out]
    for r, (role, partner, got, mx, dig, dig2, items) in enumerate(out):
        assert mx == [float(world - 1), 10.0]
        if role == "push":
            assert out[partner][0] == "decode" and got == bytes([partner + 1]) * 512
        if role == "decode":
            assert out[partner][0] == "push"
    assert roles.count("solo") == world % 2
    assert parallel.movers(world) == roles.count("push") + roles.count("solo")
    # every rank derived the same plans
    assert len({o[4] for o in out}) == 1 and len({o[5] for o in out}) == 1
    # destinations of all ranks' outgoing items are disjoint and were free before
    gpu, tables, free, nb, blocks = synthetic_cluster(world)
    seen = [set() for _ in range(world)]
    for r, o in enumerate(out):
        for d, s_bt, d_bt in o[6]:
            assert len(s_bt) == len(d_bt) and d != r
            for b in d_bt:
                assert free[d][b] and b not in seen[d]
                seen[d].add(b)


@pytest.mark.parametrize("world", [2, 4, 8])
@pytest.mark.parametrize("kind", ["rebalance", "shuffle"])
def test_exchange_preserves_every_request(world, kind):
    """Apply the plan with the CPU oracle on host 'GPU pools': each request reads the same
    KV through its new table on its new GPU (P7), and loads are conserved."""
    gpu, tables, free, nb, blocks = synthetic_cluster(world, R=90, seed=world)
    if kind == "rebalance":
        plan = rebalance.plan_rebalance_exchange(world, gpu, tables, free)
    else:
        plan = rebalance.plan_exchange(world, gpu, tables, free, hash_shuffle_dest(90, world, 3))
    g = [O.Geom(0, 2, 2, 16, 16, 1, n) for n in nb]
    rng = np.random.default_rng(0)
    pools = [rng.integers(0, 256, gg.pool_bytes, dtype=np.uint8) for gg in g]
    before = [p.copy() for p in pools]
    for (s, d), (s_bt, d_bt) in sorted(plan.moves.items()):
        assert O.migrate(before[s], g[s], s_bt, pools[d], g[d], d_bt, 0, 2) == O.OK
    for r in range(len(tables)):
        s, d = int(gpu[r]), int(plan.dest_gpu[r])
        a = before[s].reshape(2, 2, nb[s], -1)[:, :, tables[r]]
        b = pools[d].reshape(2, 2, nb[d], -1)[:, :, plan.new_tables[r]]
        np.testing.assert_array_equal(a, b)
    load0 = np.bincount(gpu, weights=blocks, minlength=world)
    load1 = np.bincount(plan.dest_gpu, weights=blocks, minlength=world)
    assert load0.sum() == load1.sum()
    if kind == "rebalance":
        assert load1.max() <= load0.max()
