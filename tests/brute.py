"""Element-wise brute force for tiny pools — independent of the
oracle's C arithmetic.

The layout reading R2 is expressed here ONLY through numpy's
own multi-dimensional indexing of a [L][2][NB][H][bs][d][e_b] byte array, never through
an offset formula, and the table preconditions are checked by their literal O(n^2)
definitions.  A plausible slip in the oracle (a transposed kv/layer index, a missing
first_layer shift, an off-by-one in the layer range, a dropped snapshot) changes some
byte these loops compute differently.
"""
from __future__ import annotations

import numpy as np

OK, INVALID_ARG, GEOMETRY, LAYER_RANGE, BLOCK_RANGE, DUP_DST, ALIAS = 0, -1, -2, -3, -4, -5, -6


def as7d(pool: np.ndarray, g) -> np.ndarray:
    return pool.reshape(g.n_layers, 2, g.n_blocks, g.n_kv_heads, g.block_size, g.head_dim,
                        g.elem_bytes)


def expected_status(gs, src_bt, gd, dst_bt, lo, hi, same_pool) -> int:
    n = len(src_bt)
    if n < 0:
        return INVALID_ARG
    if (gs.n_kv_heads, gs.head_dim, gs.block_size, gs.elem_bytes) != \
       (gd.n_kv_heads, gd.head_dim, gd.block_size, gd.elem_bytes):
        return GEOMETRY
    if lo > hi:
        return LAYER_RANGE
    if lo < hi:
        for g in (gs, gd):
            if not (g.first_layer <= lo and hi <= g.first_layer + g.n_layers):
                return LAYER_RANGE
    for i in range(n):
        if not (0 <= src_bt[i] < gs.n_blocks and 0 <= dst_bt[i] < gd.n_blocks):
            return BLOCK_RANGE
    for i in range(n):
        for j in range(n):
            if i != j and dst_bt[i] == dst_bt[j]:
                return DUP_DST
    if same_pool:
        for i in range(n):
            for j in range(n):
                if i != j and dst_bt[i] == src_bt[j]:
                    return ALIAS
    return OK


def brute_migrate(src: np.ndarray, gs, src_bt, dst: np.ndarray, gd, dst_bt, lo, hi,
                  same_pool: bool) -> tuple[int, np.ndarray]:
    """Returns (status, new destination pool) computed element by element."""
    st = expected_status(gs, src_bt, gd, dst_bt, lo, hi, same_pool)
    out = dst.copy()
    if st != OK:
        return st, out
    S = as7d(src.copy(), gs)  # copy = the "src_before" snapshot
    D = as7d(out, gd)
    for i in range(len(src_bt)):
        for l in range(lo, hi):
            ls, ld = l - gs.first_layer, l - gd.first_layer
            for kv in range(2):
                for h in range(gs.n_kv_heads):
                    for t in range(gs.block_size):
                        for j in range(gs.head_dim):
                            for byte in range(gs.elem_bytes):
                                D[ld, kv, dst_bt[i], h, t, j, byte] = \
                                    S[ls, kv, src_bt[i], h, t, j, byte]
    return st, out
