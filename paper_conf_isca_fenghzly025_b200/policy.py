"""NEXT-4: the Dynamic Rescheduling trigger and victim policy on top of the migration path
(§3.2.1-3.3), host-side.

* Trigger ("when the KV blocks of decoding instances are nearly exhausted";
  reading R8): reschedule when the free blocks of the decode pool drop below 5 % of the
  pool, or below the blocks one decode step will allocate.
* Victims ("rescheduling long-context requests to free up more KV cache", P:233
  "WindServe tends to migrate longer sequences"; reading R7): longest first, ties to the
  lowest request id, until the freed blocks cover the deficit.
* Profiler Eq. 2: T_decode = a_d * sum(L) + c_d, fitted by least squares on
  measured decode steps ("parameters are obtained by profiling ... before runtime").
* Stall-free threshold (reading R6): the final pause should cost about one decode
  step, theta = floor(T_decode(sum L) * BW / (2 * L * C)) blocks, at least 1.
"""
from __future__ import annotations

import math

import numpy as np


def should_reschedule(free_blocks: int, n_blocks: int, new_blocks_per_step: int,
                      frac: float = 0.05) -> bool:
    """R8: free < frac * NB, or free < the blocks the next decode step needs."""
    return free_blocks < frac * n_blocks or free_blocks < new_blocks_per_step


def pick_victims(req_blocks, need: int) -> list[int]:
    """R7: request ids, longest first (lowest id on ties), until sum >= need."""
    b = np.asarray(req_blocks, dtype=np.int64)
    order = sorted(range(b.size), key=lambda r: (-int(b[r]), r))
    out, got = [], 0
    for r in order:
        if got >= need:
            break
        if b[r] <= 0:
            continue
        out.append(r)
        got += int(b[r])
    return out


def fit_decode_profile(sum_L, t_ms) -> tuple[float, float, float]:
    """Eq. 2 by least squares: returns (a_d [ms/token], c_d [ms], R^2)."""
    x = np.asarray(sum_L, dtype=np.float64)
    y = np.asarray(t_ms, dtype=np.float64)
    A = np.stack([x, np.ones_like(x)], axis=1)
    (a, c), *_ = np.linalg.lstsq(A, y, rcond=None)
    pred = A @ np.array([a, c])
    ss_res = float(((y - pred) ** 2).sum())
    ss_tot = float(((y - y.mean()) ** 2).sum()) or 1.0
    return float(a), float(c), 1.0 - ss_res / ss_tot


def predict_decode_ms(a_d: float, c_d: float, sum_L: float) -> float:
    return a_d * sum_L + c_d


def theta_from_profile(a_d: float, c_d: float, sum_L: float, bw_gbs: float, n_layers: int,
                       chunk_bytes: int) -> int:
    """R6 with Eq. 2: blocks movable during one predicted decode step, at least 1."""
    t = predict_decode_ms(a_d, c_d, sum_L)
    return max(1, int(math.floor(t * 1e-3 * bw_gbs * 1e9 / (2 * n_layers * chunk_bytes))))
