"""victim — BENCH HARNESS ONLY: paged decode attention over a wind_kv pool, the
co-running "decode stream" of the interference measurement (S§8(d)).  Not part of the
product library; validated against torch SDPA in tests/test_gpu_victim.py."""
from __future__ import annotations

import ctypes as ct
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "decode_attn.cu")
LIB = os.path.join(HERE, "libwind_victim.so")
_L = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call([os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc"), "-gencode",
                               "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-shared",
                               "-Xcompiler", "-fPIC", "-o", tmp, SRC])
        os.replace(tmp, LIB)
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
