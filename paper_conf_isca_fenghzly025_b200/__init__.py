"""paper_conf_isca_fenghzly025_b200 — B200-native paged KV-cache migration (WindServe,
ISCA '25: stall-free rescheduling and KV swap).

A thin ctypes binding over the C ABI in ``include/wind_kv.h`` (``libwind_kv.so``, built
in-tree for sm_100a).  Argument marshalling only: every step of the path runs in the
library's CUDA kernels.  PyTorch is used for device memory views and streams.  There is
no CPU fallback: if the shared library is missing this module raises on first use.

Names follow the ABI: ``migrate``, ``swap_out``, ``swap_in``, ``compact``,
``migrate_batch``, ``layer_ticket``, ``layer_wait``, ``validate``, ``plan_compact``,
``plan_rebalance``.
"""
from __future__ import annotations

import ctypes as ct
import os
from typing import Optional, Sequence

import numpy as np

__all__ = [
    "WindKVError", "Pool", "lib", "migrate", "migrate_batch", "migrate_heads", "swap_out", "swap_in", "compact",
    "layer_wait", "route", "migrate_stepped", "step_signal", "validate", "plan_compact", "plan_rebalance", "check_device_error",
    "set_tuning", "get_tuning", "launch_count", "STATUS", "PATH_INTRA", "PATH_PEER", "PATH_HOST",
    "KERNEL_AUTO", "KERNEL_TMA", "KERNEL_SIMT", "EXPORTED_SYMBOLS", "Partition",
]

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libwind_kv.so")

STATUS = {
    0: "WIND_OK", -1: "WIND_ERR_INVALID_ARG", -2: "WIND_ERR_GEOMETRY", -3: "WIND_ERR_LAYER_RANGE",
    -4: "WIND_ERR_BLOCK_RANGE", -5: "WIND_ERR_DUP_DST", -6: "WIND_ERR_ALIAS", -7: "WIND_ERR_NO_PEER",
    -8: "WIND_ERR_CUDA", -9: "WIND_ERR_OOM", -10: "WIND_ERR_UNSUPPORTED", -11: "WIND_ERR_DEVICE_CHECK",
}
OK = 0
LOC_DEVICE, LOC_HOST = 0, 1
POOL_DEBUG = 0x1
POOL_NO_STAGING = 0x2
PATH_INTRA, PATH_PEER, PATH_HOST = 0, 1, 2
KERNEL_AUTO, KERNEL_TMA, KERNEL_SIMT, KERNEL_COPY_ENGINE, KERNEL_STAGED = 0, 1, 2, 3, 4
IPC_HANDLE_BYTES = 512
MAX_BATCH = 16

# every function include/wind_kv.h declares (checked by tests/test_abi.py)
EXPORTED_SYMBOLS = [
    "wind_kv_pool_create", "wind_kv_pool_destroy", "wind_kv_pool_info", "wind_kv_pool_flags",
    "wind_kv_pool_export", "wind_kv_pool_import", "wind_kv_migrate", "wind_kv_swap_out",
    "wind_kv_swap_in", "wind_kv_compact", "wind_kv_migrate_batch", "wind_kv_migrate_heads",
    "wind_kv_layer_ticket",
    "wind_kv_layer_wait", "wind_kv_layer_count", "wind_kv_read_flags", "wind_kv_validate", "wind_kv_plan_compact",
    "wind_kv_plan_rebalance", "wind_kv_check_device_error", "wind_kv_set_tuning",
    "wind_kv_get_tuning", "wind_kv_migrate_ex", "wind_kv_launch_count", "wind_kv_status_string",
    "wind_kv_last_error",
    "wind_kv_version", "wind_kv_partition_sms", "wind_kv_partition_destroy", "wind_kv_route",
    "wind_kv_migrate_stepped", "wind_kv_step_signal",
]


class WindKVError(RuntimeError):
    def __init__(self, status: int, detail: str = ""):
        self.status = status
        self.name = STATUS.get(status, f"status {status}")
        super().__init__(f"{self.name}: {detail}" if detail else self.name)


class PoolDesc(ct.Structure):
    _fields_ = [("first_layer", ct.c_int32), ("n_layers", ct.c_int32), ("n_kv_heads", ct.c_int32),
                ("head_dim", ct.c_int32), ("block_size", ct.c_int32), ("elem_bytes", ct.c_int32),
                ("n_blocks", ct.c_int32), ("loc", ct.c_int32), ("device", ct.c_int32),
                ("flags", ct.c_uint32)]


class IpcHandle(ct.Structure):
    _fields_ = [("bytes", ct.c_ubyte * IPC_HANDLE_BYTES)]


class MigrateItem(ct.Structure):
    _fields_ = [("dst", ct.c_void_p), ("src_bt", ct.c_void_p), ("dst_bt", ct.c_void_p),
                ("n_blocks", ct.c_int32)]


class Tuning(ct.Structure):
    _fields_ = [("kernel", ct.c_int32), ("ctas_per_sm", ct.c_int32), ("stage_bytes", ct.c_int32),
                ("stages", ct.c_int32), ("max_ctas", ct.c_int32), ("evict_first", ct.c_int32),
                ("store_lag", ct.c_int32), ("rate_mbps", ct.c_int32)]


class SmPartition(ct.Structure):
    _fields_ = [("migration_stream", ct.c_void_p), ("compute_stream", ct.c_void_p),
                ("sms_migration", ct.c_int32), ("sms_compute", ct.c_int32),
                ("_internal", ct.c_void_p * 2)]


_LIB: Optional[ct.CDLL] = None


def lib() -> ct.CDLL:
    """Loads libwind_kv.so (fails loudly if it was not built: there is no fallback)."""
    global _LIB
    if _LIB is not None:
        return _LIB
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() (no CPU fallback)")
    L = ct.CDLL(LIB_PATH)
    P, I32, U32 = ct.c_void_p, ct.c_int32, ct.c_uint32
    sig = {
        "wind_kv_pool_create": [ct.POINTER(PoolDesc), P, ct.POINTER(P)],
        "wind_kv_pool_destroy": [P],
        "wind_kv_pool_info": [P, ct.POINTER(P), ct.POINTER(ct.c_size_t), ct.POINTER(PoolDesc)],
        "wind_kv_pool_flags": [P, ct.POINTER(P)],
        "wind_kv_pool_export": [P, ct.POINTER(IpcHandle)],
        "wind_kv_pool_import": [ct.POINTER(IpcHandle), I32, ct.POINTER(P)],
        "wind_kv_migrate": [P, P, P, P, I32, I32, I32, P],
        "wind_kv_swap_out": [P, P, P, P, I32, P],
        "wind_kv_swap_in": [P, P, P, P, I32, P],
        "wind_kv_compact": [P, P, P, I32, P],
        "wind_kv_migrate_batch": [P, ct.POINTER(MigrateItem), I32, I32, I32, P],
        "wind_kv_migrate_heads": [P, P, P, P, I32, I32, I32, I32, I32, I32, P],
        "wind_kv_layer_ticket": [P, ct.POINTER(U32)],
        "wind_kv_layer_wait": [P, I32, U32, P],
        "wind_kv_layer_count": [P, I32, ct.POINTER(U32)],
        "wind_kv_read_flags": [P, P, P],
        "wind_kv_validate": [P, P, P, P, I32, I32, I32],
        "wind_kv_plan_compact": [P, I32, P, P, P],
        "wind_kv_plan_rebalance": [I32, I32, P, P, P, P],
        "wind_kv_check_device_error": [P],
        "wind_kv_set_tuning": [I32, ct.POINTER(Tuning)],
        "wind_kv_get_tuning": [I32, ct.POINTER(Tuning)],
        "wind_kv_migrate_ex": [P, P, P, P, I32, I32, I32, ct.POINTER(Tuning), P],
        "wind_kv_partition_sms": [I32, I32, ct.POINTER(SmPartition)],
        "wind_kv_partition_destroy": [ct.POINTER(SmPartition)],
        "wind_kv_route": [P, P, ct.POINTER(I32), ct.POINTER(I32), ct.POINTER(I32)],
        "wind_kv_migrate_stepped": [P, P, P, P, I32, I32, I32, P, U32, ct.c_uint64, P],
        "wind_kv_step_signal": [P, P],
    }
    for name, args in sig.items():
        f = getattr(L, name)
        f.argtypes, f.restype = args, ct.c_int32
    L.wind_kv_launch_count.argtypes, L.wind_kv_launch_count.restype = [], ct.c_uint64
    for name in ("wind_kv_status_string",):
        getattr(L, name).argtypes, getattr(L, name).restype = [ct.c_int32], ct.c_char_p
    for name in ("wind_kv_last_error", "wind_kv_version"):
        getattr(L, name).argtypes, getattr(L, name).restype = [], ct.c_char_p
    _LIB = L
    return L


def _check(st: int) -> None:
    if st != OK:
        raise WindKVError(st, lib().wind_kv_last_error().decode(errors="replace"))


def last_error() -> str:
    return lib().wind_kv_last_error().decode(errors="replace")


# -------------------------------------------------------------------- marshalling

def _ptr(x) -> Optional[int]:
    """Device-accessible address of a table / buffer argument (torch tensor, numpy array
    in mapped memory is not supported: pass the mapped pointer as an int)."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        import torch
        if x.dtype != torch.int32:
            raise TypeError(f"block tables must be int32 tensors, got {x.dtype}")
        if not x.is_contiguous():
            raise ValueError("tables must be contiguous")
        if not x.is_cuda and x.numel() > 0 and not x.is_pinned():
            # the kernels read tables on the device: pageable host memory is not accessible
            raise ValueError("block tables must be device tensors or pinned host tensors")
        return x.data_ptr()
    raise TypeError(f"cannot pass {type(x).__name__} as a device pointer")


def _len(x) -> int:
    return int(x.numel()) if hasattr(x, "numel") else len(x)


def _stream(stream, device: int) -> Optional[int]:
    if stream is None:
        import torch
        return torch.cuda.current_stream(device).cuda_stream or None
    if isinstance(stream, int):
        return stream or None
    return stream.cuda_stream or None


class _CudaArray:
    """__cuda_array_interface__ wrapper so torch can view library-owned device memory."""

    def __init__(self, ptr: int, nbytes: int, owner=None):
        self._owner = owner  # the Pool: kept alive as long as a tensor view exists
        self.__cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1",
                                         "data": (ptr, False), "version": 3}


class Pool:
    """A KV block pool (include/wind_kv.h wind_kv_pool_*)."""

    def __init__(self, n_layers: int, n_kv_heads: int, head_dim: int, block_size: int,
                 elem_bytes: int, n_blocks: int, *, loc: str = "device", device: int = 0,
                 first_layer: int = 0, debug: bool = False, external_base: Optional[int] = None,
                 staging: bool = True, _handle: Optional[int] = None):
        if _handle is None:
            d = PoolDesc(first_layer, n_layers, n_kv_heads, head_dim, block_size, elem_bytes,
                         n_blocks, LOC_HOST if loc == "host" else LOC_DEVICE, device,
                         (POOL_DEBUG if debug else 0) | (0 if staging else POOL_NO_STAGING))
            h = ct.c_void_p()
            _check(lib().wind_kv_pool_create(ct.byref(d), external_base, ct.byref(h)))
            _handle = h.value
        self._h = _handle
        base, nbytes, desc = ct.c_void_p(), ct.c_size_t(), PoolDesc()
        _check(lib().wind_kv_pool_info(self._h, ct.byref(base), ct.byref(nbytes), ct.byref(desc)))
        self.base, self.nbytes, self.desc = int(base.value or 0), int(nbytes.value), desc
        f = ct.c_void_p()
        _check(lib().wind_kv_pool_flags(self._h, ct.byref(f)))
        self.flags_ptr = int(f.value or 0)

    # geometry
    @property
    def handle(self) -> int:
        if not self._h:
            raise ValueError("pool destroyed")
        return self._h

    @property
    def is_host(self) -> bool:
        return self.desc.loc == LOC_HOST

    @property
    def device(self) -> int:
        return self.desc.device

    @property
    def chunk_bytes(self) -> int:
        d = self.desc
        return d.n_kv_heads * d.block_size * d.head_dim * d.elem_bytes

    @property
    def layers(self) -> tuple[int, int]:
        return self.desc.first_layer, self.desc.first_layer + self.desc.n_layers

    def tensor(self):
        """A torch uint8 view of the whole pool (device pools: on the pool's device; host
        pools: a CPU tensor over the mapped pinned memory)."""
        import torch
        if self.is_host:
            arr = np.ctypeslib.as_array((ct.c_ubyte * self.nbytes).from_address(self.base))
            return torch.from_numpy(arr)
        with torch.cuda.device(self.device):
            return torch.as_tensor(_CudaArray(self.base, self.nbytes, self), device=f"cuda:{self.device}")

    def flags_tensor(self, device: Optional[int] = None):
        """A torch int32 view of layer_done[n_layers] (device-accessible flags)."""
        import torch
        dev = self.device if device is None else device
        with torch.cuda.device(dev):
            t = torch.as_tensor(_CudaArray(self.flags_ptr, 4 * self.desc.n_layers, self),
                                device=f"cuda:{dev}")
        return t.view(torch.int32)

    # flags
    def layer_ticket(self) -> int:
        t = ct.c_uint32()
        _check(lib().wind_kv_layer_ticket(self.handle, ct.byref(t)))
        return int(t.value)

    def read_flags(self, out, stream=None) -> None:
        """wind_kv_read_flags: async copy of layer_done[n_layers] into `out` (a pinned host
        or device int32/uint32 tensor, or an address) on `stream`."""
        ptr = out if isinstance(out, int) else out.data_ptr()
        _check(lib().wind_kv_read_flags(self.handle, ptr, _stream(stream, self.device)))

    def layer_count(self, layer: int) -> int:
        v = ct.c_uint32()
        _check(lib().wind_kv_layer_count(self.handle, layer, ct.byref(v)))
        return int(v.value)

    # IPC
    def export(self) -> bytes:
        h = IpcHandle()
        _check(lib().wind_kv_pool_export(self.handle, ct.byref(h)))
        return bytes(h.bytes)

    @classmethod
    def import_(cls, handle: bytes, local_device: int) -> "Pool":
        if len(handle) != IPC_HANDLE_BYTES:
            raise ValueError("bad IPC handle size")
        h = IpcHandle()
        ct.memmove(h.bytes, handle, IPC_HANDLE_BYTES)
        out = ct.c_void_p()
        _check(lib().wind_kv_pool_import(ct.byref(h), local_device, ct.byref(out)))
        return cls(0, 0, 0, 0, 0, 0, _handle=out.value)

    def destroy(self) -> None:
        if getattr(self, "_h", None):
            lib().wind_kv_pool_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass


# ------------------------------------------------------------------------- ops

def _exec_device(src: Pool, dst: Pool) -> int:
    return src.device if not src.is_host else dst.device


def migrate(src: Pool, src_bt, dst: Pool, dst_bt, n: Optional[int] = None,
            layer_lo: Optional[int] = None, layer_hi: Optional[int] = None, stream=None) -> None:
    """wind_kv_migrate: dst[l][kv][dst_bt[i]] := src[l][kv][src_bt[i]] for l in [lo, hi)."""
    n = _len(src_bt) if n is None else n
    lo = max(src.layers[0], dst.layers[0]) if layer_lo is None else layer_lo
    hi = min(src.layers[1], dst.layers[1]) if layer_hi is None else layer_hi
    _check(lib().wind_kv_migrate(src.handle, _ptr(src_bt), dst.handle, _ptr(dst_bt), n, lo, hi,
                                 _stream(stream, _exec_device(src, dst))))


def tuning(kernel: int = KERNEL_TMA, ctas_per_sm: int = 1, stage_bytes: int = 49152, stages: int = 4,
           max_ctas: int = 0, evict_first: bool = False, store_lag: int = 2, rate_mbps: int = 0) -> Tuning:
    """A complete per-op tuning (every field explicit) for migrate_ex."""
    return Tuning(kernel, ctas_per_sm, stage_bytes, stages, max_ctas, int(evict_first), store_lag, rate_mbps)


def migrate_ex(src: Pool, src_bt, dst: Pool, dst_bt, tuning_override: Optional[Tuning],
               n: Optional[int] = None, layer_lo: Optional[int] = None, layer_hi: Optional[int] = None,
               stream=None) -> None:
    """wind_kv_migrate_ex: migrate with a per-op tuning (None = the path's current one)."""
    n = _len(src_bt) if n is None else n
    lo = max(src.layers[0], dst.layers[0]) if layer_lo is None else layer_lo
    hi = min(src.layers[1], dst.layers[1]) if layer_hi is None else layer_hi
    tp = ct.byref(tuning_override) if tuning_override is not None else None
    _check(lib().wind_kv_migrate_ex(src.handle, _ptr(src_bt), dst.handle, _ptr(dst_bt), n, lo, hi, tp,
                                    _stream(stream, _exec_device(src, dst))))


def migrate_heads(src: Pool, src_bt, dst: Pool, dst_bt, src_head_lo: int, dst_head_lo: int,
                  n_heads: int, n: Optional[int] = None, layer_lo: Optional[int] = None,
                  layer_hi: Optional[int] = None, stream=None) -> None:
    """wind_kv_migrate_heads: heads [src_head_lo, +n_heads) of each source block into heads
    [dst_head_lo, +n_heads) of the destination block (TP reshard, NEXT-3)."""
    n = _len(src_bt) if n is None else n
    lo = max(src.layers[0], dst.layers[0]) if layer_lo is None else layer_lo
    hi = min(src.layers[1], dst.layers[1]) if layer_hi is None else layer_hi
    _check(lib().wind_kv_migrate_heads(src.handle, _ptr(src_bt), dst.handle, _ptr(dst_bt), n, lo, hi,
                                       src_head_lo, dst_head_lo, n_heads,
                                       _stream(stream, _exec_device(src, dst))))


def migrate_batch(src: Pool, items: Sequence[tuple], layer_lo: int, layer_hi: int,
                  stream=None) -> None:
    """wind_kv_migrate_batch: items = [(dst_pool, src_bt, dst_bt[, n]), ...] in one launch
    (n is required when the tables are passed as raw addresses)."""
    arr = (MigrateItem * len(items))()
    for k, item in enumerate(items):
        dst, sbt, dbt = item[:3]
        n = item[3] if len(item) > 3 else _len(sbt)
        arr[k] = MigrateItem(dst.handle, _ptr(sbt), _ptr(dbt), n)
    dev = src.device if not src.is_host else items[0][0].device
    _check(lib().wind_kv_migrate_batch(src.handle, arr, len(items), layer_lo, layer_hi,
                                       _stream(stream, dev)))


def swap_out(dev: Pool, dev_bt, host: Pool, host_bt, n: Optional[int] = None, stream=None) -> None:
    n = _len(dev_bt) if n is None else n
    _check(lib().wind_kv_swap_out(dev.handle, _ptr(dev_bt), host.handle, _ptr(host_bt), n,
                                  _stream(stream, dev.device)))


def swap_in(host: Pool, host_bt, dev: Pool, dev_bt, n: Optional[int] = None, stream=None) -> None:
    n = _len(dev_bt) if n is None else n
    _check(lib().wind_kv_swap_in(host.handle, _ptr(host_bt), dev.handle, _ptr(dev_bt), n,
                                 _stream(stream, dev.device)))


def compact(pool: Pool, src_bt, dst_bt, n: Optional[int] = None, stream=None) -> None:
    n = _len(src_bt) if n is None else n
    _check(lib().wind_kv_compact(pool.handle, _ptr(src_bt), _ptr(dst_bt), n,
                                 _stream(stream, pool.device)))


def migrate_stepped(src: Pool, src_bt, dst: Pool, dst_bt, step_counter, first_step: int,
                    bytes_per_step: int, n: Optional[int] = None, layer_lo: Optional[int] = None,
                    layer_hi: Optional[int] = None, stream=None) -> None:
    """wind_kv_migrate_stepped: the migrate cut into ~bytes_per_step slices, slice k released
    when the int32/uint32 device tensor (or address) `step_counter` reaches first_step + k."""
    n = _len(src_bt) if n is None else n
    lo = max(src.layers[0], dst.layers[0]) if layer_lo is None else layer_lo
    hi = min(src.layers[1], dst.layers[1]) if layer_hi is None else layer_hi
    cp = step_counter if isinstance(step_counter, int) else step_counter.data_ptr()
    _check(lib().wind_kv_migrate_stepped(src.handle, _ptr(src_bt), dst.handle, _ptr(dst_bt), n, lo, hi, cp,
                                         first_step, bytes_per_step, _stream(stream, _exec_device(src, dst))))


def step_signal(step_counter, stream=None) -> None:
    """wind_kv_step_signal: +1 on the step counter, in stream order (a decode step starts)."""
    cp = step_counter if isinstance(step_counter, int) else step_counter.data_ptr()
    dev = 0 if isinstance(step_counter, int) else step_counter.device.index
    _check(lib().wind_kv_step_signal(cp, _stream(stream, dev)))


def route(src: Pool, dst: Pool) -> tuple[int, int, bool]:
    """wind_kv_route: (executing device, path PATH_INTRA / PATH_PEER / PATH_HOST, system-scope
    flag publication) of an op from src to dst."""
    e, p, s = ct.c_int32(), ct.c_int32(), ct.c_int32()
    _check(lib().wind_kv_route(src.handle, dst.handle, ct.byref(e), ct.byref(p), ct.byref(s)))
    return int(e.value), int(p.value), bool(s.value)


def layer_wait(dst: Pool, layer: int, ticket: int, stream=None) -> None:
    _check(lib().wind_kv_layer_wait(dst.handle, layer, ticket, _stream(stream, dst.device)))


def validate(src: Pool, src_bt, dst: Pool, dst_bt, layer_lo: int, layer_hi: int) -> int:
    """wind_kv_validate on HOST tables; returns the status code (does not raise)."""
    s = np.ascontiguousarray(np.asarray(src_bt, dtype=np.int32))
    d = np.ascontiguousarray(np.asarray(dst_bt, dtype=np.int32))
    if s.size != d.size:
        raise ValueError("table lengths differ")
    return int(lib().wind_kv_validate(src.handle, s.ctypes.data, dst.handle, d.ctypes.data,
                                      s.size, layer_lo, layer_hi))


def plan_compact(live) -> tuple[np.ndarray, np.ndarray]:
    lv = np.ascontiguousarray(np.asarray(live, dtype=np.uint8))
    s = np.zeros(max(1, lv.size), np.int32)
    d = np.zeros(max(1, lv.size), np.int32)
    n = ct.c_int32()
    _check(lib().wind_kv_plan_compact(lv.ctypes.data, lv.size, s.ctypes.data, d.ctypes.data,
                                      ct.byref(n)))
    return s[:n.value].copy(), d[:n.value].copy()


def plan_rebalance(n_gpus: int, req_gpu, req_blocks) -> tuple[np.ndarray, int]:
    g = np.ascontiguousarray(np.asarray(req_gpu, dtype=np.int32))
    b = np.ascontiguousarray(np.asarray(req_blocks, dtype=np.int32))
    out = np.zeros(max(1, g.size), np.int32)
    n = ct.c_int32()
    _check(lib().wind_kv_plan_rebalance(n_gpus, g.size, g.ctypes.data, b.ctypes.data,
                                        out.ctypes.data, ct.byref(n)))
    return out[:g.size].copy(), int(n.value)


def check_device_error(pool: Pool) -> None:
    _check(lib().wind_kv_check_device_error(pool.handle))


def set_tuning(path: int, kernel: int = KERNEL_AUTO, ctas_per_sm: int = 0, stage_bytes: int = 0,
               stages: int = 0, max_ctas: int = 0, evict_first: bool = False,
               store_lag: int = 0, rate_mbps: int = 0) -> None:
    t = Tuning(kernel, ctas_per_sm, stage_bytes, stages, max_ctas, int(evict_first), store_lag,
               rate_mbps)
    _check(lib().wind_kv_set_tuning(path, ct.byref(t)))


def get_tuning(path: int) -> dict:
    t = Tuning()
    _check(lib().wind_kv_get_tuning(path, ct.byref(t)))
    return {k: getattr(t, k) for k, _ in Tuning._fields_}


class Partition:
    """wind_kv_partition_sms: two green contexts with disjoint SM sets on `device` — a
    migration partition of >= `min_sms` SMs and a compute partition with the rest — and a
    torch stream in each (`.migration`, `.compute`).  Call destroy() when both are idle."""

    def __init__(self, device: int, min_sms: int):
        import torch
        self._p = SmPartition()
        _check(lib().wind_kv_partition_sms(device, min_sms, ct.byref(self._p)))
        self.sms_migration, self.sms_compute = self._p.sms_migration, self._p.sms_compute
        self.migration = torch.cuda.ExternalStream(self._p.migration_stream, device=f"cuda:{device}")
        self.compute = torch.cuda.ExternalStream(self._p.compute_stream, device=f"cuda:{device}")

    def destroy(self) -> None:
        if self._p.migration_stream:
            _check(lib().wind_kv_partition_destroy(ct.byref(self._p)))


def launch_count() -> int:
    return int(lib().wind_kv_launch_count())


def version() -> str:
    return lib().wind_kv_version().decode()
