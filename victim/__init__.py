"""victim — BENCH HARNESS ONLY, not part of the product library:
  * paged decode attention over a wind_kv pool: the co-running "decode stream" of the
    interference measurement (S§8(d)); validated against torch attention in
    tests/test_gpu_victim.py;
  * a copy-engine comparator (one cudaMemcpyAsync per chunk) for the same paged gather
    (S§7 step 4)."""
from __future__ import annotations

import ctypes as ct
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "decode_attn.cu")
LIB = os.path.join(HERE, "libwind_victim.so")
CE_SRC = os.path.join(HERE, "ce_gather.cu")
CE_LIB = os.path.join(HERE, "libwind_ce.so")
_L = None
_CE = None


def _nvcc(src: str, out: str) -> None:
    tmp = out + f".tmp{os.getpid()}"
    subprocess.check_call([os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc"), "-gencode",
                           "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-shared",
                           "-Xcompiler", "-fPIC", "-o", tmp, src])
    os.replace(tmp, out)


def build(force: bool = False) -> str:
    for src, out in ((SRC, LIB), (CE_SRC, CE_LIB)):
        if force or not os.path.exists(out) or os.path.getmtime(out) < os.path.getmtime(src):
            _nvcc(src, out)
    return LIB


def _lib():
    global _L
    if _L is None:
        if not os.path.exists(LIB):
            raise ImportError(f"{LIB} missing: run __graft_entry__.build()")
        L = ct.CDLL(LIB)
        f = L.victim_decode_attention
        f.argtypes = [ct.c_void_p] * 5 + [ct.c_int] * 7 + [ct.c_void_p, ct.c_void_p, ct.c_void_p]
        f.restype = ct.c_int
        _L = L
    return _L


def _ce():
    global _CE
    if _CE is None:
        if not os.path.exists(CE_LIB):
            raise ImportError(f"{CE_LIB} missing: run __graft_entry__.build()")
        L = ct.CDLL(CE_LIB)
        for name in ("ce_gather_loop",):
            f = getattr(L, name)
            f.argtypes = [ct.c_void_p, ct.c_int64, ct.c_void_p, ct.c_int64, ct.c_int64, ct.c_void_p,
                          ct.c_void_p, ct.c_int32, ct.c_int32, ct.c_void_p]
            f.restype = ct.c_int
        _CE = L
    return _CE


def scratch_floats(batch: int, hq: int, max_blocks: int, blocks_per_split: int) -> int:
    splits = -(-max_blocks // blocks_per_split)
    return batch * hq * splits * (128 + 2)


def decode_attention(q, k_plane_ptr: int, v_plane_ptr: int, bt, ctx, hkv: int, bs: int,
                     scratch, out, blocks_per_split: int = 32, stream: int = 0) -> None:
    """q: [B, Hq, 128] fp16 cuda; bt: [B, max_blocks] int32; ctx: [B] int32;
    scratch: fp32 >= scratch_floats(); out: [B, Hq, 128] fp32."""
    B, hq, d = q.shape
    rc = _lib().victim_decode_attention(q.data_ptr(), k_plane_ptr, v_plane_ptr, bt.data_ptr(),
                                        ctx.data_ptr(), B, bt.shape[1], hq, hkv, d, bs,
                                        blocks_per_split, scratch.data_ptr(), out.data_ptr(),
                                        stream or None)
    if rc != 0:
        raise RuntimeError(f"victim_decode_attention failed ({rc})")


def ce_gather(kind: str, src_plane0: int, s_stride: int, dst_plane0: int, d_stride: int, chunk: int,
              src_bt: np.ndarray, dst_bt: np.ndarray, planes: int, stream: int) -> None:
    """Copy-engine gather: kind 'loop' (one cudaMemcpyAsync per chunk), the only kind.
    Tables are host int32 arrays."""
    if kind != "loop":
        raise ValueError(f"unknown copy-engine comparator {kind!r}")
    s = np.ascontiguousarray(src_bt, np.int32)
    d = np.ascontiguousarray(dst_bt, np.int32)
    f = _ce().ce_gather_loop
    rc = f(src_plane0, s_stride, dst_plane0, d_stride, chunk, s.ctypes.data, d.ctypes.data, s.size,
           planes, stream or None)
    if rc != 0:
        raise RuntimeError(f"ce_gather_{kind} failed (cudaError {rc})")
