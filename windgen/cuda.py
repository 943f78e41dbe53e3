"""ctypes binding of windgen/csrc/windgen_fill.cu (libwindgen_cuda.so): the O9 content
generator on the device (fill) and a chunk checker against it.  Test / bench input
infrastructure; never used by the product library."""
from __future__ import annotations

import ctypes as ct
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "csrc", "windgen_fill.cu")
LIB = os.path.join(HERE, "libwindgen_cuda.so")
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
        L.windgen_fill.argtypes = [ct.c_void_p, ct.c_uint64, ct.c_uint64, ct.c_uint64, ct.c_uint64,
                                   ct.c_void_p]
        L.windgen_fill.restype = ct.c_int
        L.windgen_check_chunks.argtypes = [ct.c_void_p, ct.c_uint64, ct.c_void_p, ct.c_void_p,
                                           ct.c_void_p, ct.c_int64, ct.c_void_p, ct.c_void_p]
        L.windgen_check_chunks.restype = ct.c_int
        _L = L
    return _L


def fill(ptr: int, nbytes: int, byte_offset: int, seed: int, tag: int, stream: int = 0) -> None:
    """Fill device bytes [ptr, ptr+nbytes) with pattern bytes [byte_offset, +nbytes) of
    pool (seed, tag)."""
    rc = _lib().windgen_fill(ptr, nbytes, byte_offset, seed, tag, stream or None)
    if rc != 0:
        raise RuntimeError(f"windgen_fill failed: cudaError {rc}")


def check_chunks(base: int, chunk_bytes: int, dst_off, exp_off, keys, device: int = 0,
                 stream: int = 0) -> tuple[int, int]:
    """Compare chunks at base+dst_off[c] with the pattern of keys[c] at exp_off[c].
    Returns (mismatching chunk count, lowest mismatching index or -1).  Synchronises."""
    import torch
    dev = torch.device("cuda", device)
    d = torch.as_tensor(np.asarray(dst_off, np.int64), device=dev)
    e = torch.as_tensor(np.asarray(exp_off, np.int64), device=dev)
    k = torch.as_tensor(np.asarray(keys, np.uint64).view(np.int64), device=dev)
    out = torch.tensor([0, -1], dtype=torch.int64, device=dev)
    rc = _lib().windgen_check_chunks(base, chunk_bytes, d.data_ptr(), e.data_ptr(), k.data_ptr(),
                                     d.numel(), out.data_ptr(), stream or None)
    if rc != 0:
        raise RuntimeError(f"windgen_check_chunks failed: cudaError {rc}")
    torch.cuda.synchronize(dev)
    cnt, first = out.tolist()
    return int(cnt), (int(first) if cnt else -1)
