"""oracle — ORACLE (TEST INFRASTRUCTURE ONLY).

Thin ctypes wrapper over ``oracle/wind_oracle.c`` (plain C, built with gcc into
``oracle/libwind_oracle.so``).  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this package.
The product path (``paper_conf_isca_fenghzly025_b200``) never imports it and shares no
code with it.  See the header of wind_oracle.c for the paper passages each function
follows and for which functions are pinned by which tests.
"""
from __future__ import annotations

import ctypes as ct
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "wind_oracle.c")
_LIB = os.path.join(_HERE, "libwind_oracle.so")

OK, INVALID_ARG, GEOMETRY, LAYER_RANGE, BLOCK_RANGE, DUP_DST, ALIAS = 0, -1, -2, -3, -4, -5, -6
OOM, UNSUPPORTED = -9, -10


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (-O2, plain C11, pthreads)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-D_GNU_SOURCE", "-fPIC", "-shared",
                               "-Wall", "-Werror", "-o", tmp, _SRC, "-lpthread"])
        os.replace(tmp, _LIB)
    return _LIB


class _Geom(ct.Structure):
    _fields_ = [(n, ct.c_int32) for n in ("first_layer", "n_layers", "n_kv_heads", "head_dim",
                                         "block_size", "elem_bytes", "n_blocks")]


@dataclass(frozen=True)
class Geom:
    """O1: pool geometry (layer-major [L][2][NB][H][bs][d], reading R2)."""
    first_layer: int
    n_layers: int
    n_kv_heads: int
    head_dim: int
    block_size: int
    elem_bytes: int
    n_blocks: int

    def c(self) -> _Geom:
        return _Geom(self.first_layer, self.n_layers, self.n_kv_heads, self.head_dim,
                     self.block_size, self.elem_bytes, self.n_blocks)

    @property
    def chunk_bytes(self) -> int:
        return int(_lib().or_chunk_bytes(ct.byref(self.c())))

    @property
    def pool_bytes(self) -> int:
        return int(_lib().or_pool_bytes(ct.byref(self.c())))


_L = None


def _lib():
    global _L
    if _L is None:
        lib = ct.CDLL(build())
        P, I32, I64 = ct.c_void_p, ct.c_int32, ct.c_int64
        G = ct.POINTER(_Geom)
        sig = {
            "or_chunk_bytes": (I64, [G]),
            "or_pool_bytes": (I64, [G]),
            "or_chunk_offset": (I64, [G, I32, I32, I32]),
            "or_elem_offset": (I64, [G, I32, I32, I32, I32, I32, I32]),
            "or_geom_check": (ct.c_int, [G]),
            "or_check_op": (ct.c_int, [G, G, I32, I32, I32]),
            "or_validate_tables": (ct.c_int, [G, P, G, P, I32, ct.c_int]),
            "or_migrate": (ct.c_int, [P, G, P, P, G, P, I32, I32, I32]),
            "or_swap_out": (ct.c_int, [P, G, P, P, G, P, I32]),
            "or_swap_in": (ct.c_int, [P, G, P, P, G, P, I32]),
            "or_compact": (ct.c_int, [P, G, P, P, I32]),
            "or_expected_origin": (ct.c_int, [G, P, G, P, I32, I32, I32, P, P]),
            "or_plan_compact": (ct.c_int, [P, I32, P, P, P]),
            "or_plan_rebalance": (ct.c_int, [I32, I32, P, P, P, P]),
            "or_migrate_mt": (ct.c_int, [P, G, P, P, G, P, I32, I32, I32, I32]),
            "or_hw_threads": (I32, []),
            "or_stall_free_plan": (ct.c_int, [I32, I32, I32, P, I32, P, P, P, P]),
            "or_check_op_heads": (ct.c_int, [G, G, I32, I32, I32, I32, I32, I32]),
            "or_migrate_heads": (ct.c_int, [P, G, P, P, G, P, I32, I32, I32, I32, I32, I32]),
        }
        for name, (res, args) in sig.items():
            f = getattr(lib, name)
            f.restype, f.argtypes = res, args
        _L = lib
    return _L


def _p(a: np.ndarray | None):
    return None if a is None else a.ctypes.data_as(ct.c_void_p)


def _i32(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.int32))


def chunk_offset(g: Geom, layer: int, kv: int, block: int) -> int:
    return int(_lib().or_chunk_offset(ct.byref(g.c()), layer, kv, block))


def elem_offset(g: Geom, layer, kv, block, h, t, j) -> int:
    return int(_lib().or_elem_offset(ct.byref(g.c()), layer, kv, block, h, t, j))


def geom_check(g: Geom) -> int:
    return int(_lib().or_geom_check(ct.byref(g.c())))


def check_op(gs: Geom, gd: Geom, n: int, lo: int, hi: int) -> int:
    return int(_lib().or_check_op(ct.byref(gs.c()), ct.byref(gd.c()), n, lo, hi))


def validate(gs: Geom, src_bt, gd: Geom, dst_bt, same_pool: bool) -> int:
    s, d = _i32(src_bt), _i32(dst_bt)
    assert s.size == d.size
    return int(_lib().or_validate_tables(ct.byref(gs.c()), _p(s), ct.byref(gd.c()), _p(d),
                                         s.size, int(same_pool)))


def migrate(src: np.ndarray, gs: Geom, src_bt, dst: np.ndarray, gd: Geom, dst_bt,
            lo: int, hi: int) -> int:
    """O3, in place on ``dst`` (uint8, contiguous).  ``src is dst`` selects the same-pool
    (snapshot) semantics."""
    s, d = _i32(src_bt), _i32(dst_bt)
    assert s.size == d.size and src.dtype == np.uint8 and dst.dtype == np.uint8
    assert src.flags.c_contiguous and dst.flags.c_contiguous
    assert src.size == gs.pool_bytes and dst.size == gd.pool_bytes
    return int(_lib().or_migrate(_p(src), ct.byref(gs.c()), _p(s), _p(dst), ct.byref(gd.c()),
                                 _p(d), s.size, lo, hi))


def check_op_heads(gs: Geom, gd: Geom, n, lo, hi, sh0, dh0, nh) -> int:
    return int(_lib().or_check_op_heads(ct.byref(gs.c()), ct.byref(gd.c()), n, lo, hi, sh0, dh0, nh))


def migrate_heads(src: np.ndarray, gs: Geom, src_bt, dst: np.ndarray, gd: Geom, dst_bt,
                  lo: int, hi: int, src_head_lo: int, dst_head_lo: int, n_heads: int) -> int:
    """NEXT-3 head-range migrate (TP reshard); `src is dst` = same pool."""
    s, d = _i32(src_bt), _i32(dst_bt)
    assert src.size == gs.pool_bytes and dst.size == gd.pool_bytes
    return int(_lib().or_migrate_heads(_p(src), ct.byref(gs.c()), _p(s), _p(dst), ct.byref(gd.c()),
                                       _p(d), s.size, lo, hi, src_head_lo, dst_head_lo, n_heads))


def swap_out(dev: np.ndarray, gdev: Geom, dev_bt, host: np.ndarray, ghost: Geom, host_bt) -> int:
    s, d = _i32(dev_bt), _i32(host_bt)
    return int(_lib().or_swap_out(_p(dev), ct.byref(gdev.c()), _p(s), _p(host),
                                  ct.byref(ghost.c()), _p(d), s.size))


def swap_in(host: np.ndarray, ghost: Geom, host_bt, dev: np.ndarray, gdev: Geom, dev_bt) -> int:
    s, d = _i32(host_bt), _i32(dev_bt)
    return int(_lib().or_swap_in(_p(host), ct.byref(ghost.c()), _p(s), _p(dev),
                                 ct.byref(gdev.c()), _p(d), s.size))


def compact(pool: np.ndarray, g: Geom, src_bt, dst_bt) -> int:
    s, d = _i32(src_bt), _i32(dst_bt)
    return int(_lib().or_compact(_p(pool), ct.byref(g.c()), _p(s), _p(d), s.size))


def expected_origin(gs: Geom, src_bt, gd: Geom, dst_bt, lo: int, hi: int):
    """P2: (from_src uint8[L_d*2*NB_d], offset int64[...]) for every destination chunk."""
    s, d = _i32(src_bt), _i32(dst_bt)
    m = gd.n_layers * 2 * gd.n_blocks
    fs = np.zeros(m, dtype=np.uint8)
    off = np.zeros(m, dtype=np.int64)
    rc = int(_lib().or_expected_origin(ct.byref(gs.c()), _p(s), ct.byref(gd.c()), _p(d),
                                       s.size, lo, hi, _p(fs), _p(off)))
    if rc != OK:
        raise ValueError(f"expected_origin rc={rc}")
    return fs, off


def plan_compact(live) -> tuple[np.ndarray, np.ndarray]:
    lv = np.ascontiguousarray(np.asarray(live, dtype=np.uint8))
    src = np.zeros(lv.size, dtype=np.int32)
    dst = np.zeros(lv.size, dtype=np.int32)
    nm = np.zeros(1, dtype=np.int32)
    rc = int(_lib().or_plan_compact(_p(lv), lv.size, _p(src), _p(dst), _p(nm)))
    if rc != OK:
        raise ValueError(f"plan_compact rc={rc}")
    return src[:nm[0]].copy(), dst[:nm[0]].copy()


def plan_rebalance(n_gpus: int, req_gpu, req_blocks) -> tuple[np.ndarray, int]:
    g, b = _i32(req_gpu), _i32(req_blocks)
    out = np.zeros(g.size, dtype=np.int32)
    nm = np.zeros(1, dtype=np.int32)
    rc = int(_lib().or_plan_rebalance(n_gpus, g.size, _p(g), _p(b), _p(out), _p(nm)))
    if rc != OK:
        raise ValueError(f"plan_rebalance rc={rc}")
    return out, int(nm[0])


def migrate_mt(src: np.ndarray, gs: Geom, src_bt, dst: np.ndarray, gd: Geom, dst_bt,
               lo: int, hi: int, n_threads: int) -> int:
    s, d = _i32(src_bt), _i32(dst_bt)
    return int(_lib().or_migrate_mt(_p(src), ct.byref(gs.c()), _p(s), _p(dst),
                                    ct.byref(gd.c()), _p(d), s.size, lo, hi, n_threads))


def stall_free_plan(T0: int, bs: int, theta: int, appends) -> tuple[list, int]:
    """O8: [(begin_block, end_block), ...] (the last = pause stage) and the pause token
    count, for per-stage append counts `appends` (len = max_stages)."""
    a = _i32(appends)
    m = a.size
    b = np.zeros(m + 1, np.int32)
    e = np.zeros(m + 1, np.int32)
    ns = np.zeros(1, np.int32)
    ft = np.zeros(1, np.int32)
    rc = int(_lib().or_stall_free_plan(T0, bs, theta, _p(a), m, _p(b), _p(e), _p(ns), _p(ft)))
    if rc != OK:
        raise ValueError(f"stall_free_plan rc={rc}")
    return [(int(b[k]), int(e[k])) for k in range(ns[0])], int(ft[0])


def hw_threads() -> int:
    return int(_lib().or_hw_threads())
