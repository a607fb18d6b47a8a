"""Thin ctypes binding of include/accmg.h (argument marshalling only).

Every function here forwards to the same-named C entry point of libaccmg.so (built in-tree by
__graft_entry__.build() / `make accmg`); every step of the loop runs in the library's CUDA
kernels. Importing this module fails loudly if the library is missing — there is no fallback.
"""
from __future__ import annotations

import ctypes
import os
import re

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# ACCMG_LIBRARY: another in-tree build of the same library (same-box A/B measurements only)
LIB_PATH = os.environ.get("ACCMG_LIBRARY") or os.path.join(_HERE, "libaccmg.so")
HEADER = os.path.join(os.path.dirname(_HERE), "include", "accmg.h")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with __graft_entry__.build() or `make accmg`")
_lib = ctypes.CDLL(LIB_PATH)

# ---- constants (mirrors of include/accmg.h) --------------------------------------------------
OK, EINVAL, ECUDA, ENCCL, ENOMEM, ESTATE, EUNSUPPORTED, ECONFLICT, EDATA = 0, -1, -2, -3, -4, -5, -6, -7, -8
XCHG_AUTO, XCHG_NCCL_ALL, XCHG_NCCL = 0, 1, 2
DIRTY_RUNS, DIRTY_CHUNKS = 0, 1
HALO_AUTO, HALO_PULL = 0, 1
MC_OFF, MC_AUTO, MC_VMM = 0, 1, 2
R, W, RW, REDUCE_SUM = 1, 2, 3, 4
BODY_JACOBI2D_5PT, BODY_GEMM_BF16_F32, BODY_KMEANS_ASSIGN, BODY_KMEANS_UPDATE = 1, 2, 3, 4
KMEANS_EXACT, KMEANS_WINDOWS = -1, 9  # accmg_args_kmeans.shift for arbitrary finite points; windows
BODY_SCATTER = 5
BODY_JACOBI3D_7PT = 6
BODY_JACOBI2D_DEEP = 7
BODY_TEST_SPARSE_WRITE = 100
BODY_TEST_MASKED_WRITE = 101


class accmg_config(ctypes.Structure):
    _fields_ = [("num_partitions", ctypes.c_int32), ("world_size", ctypes.c_int32), ("rank", ctypes.c_int32),
                ("device", ctypes.c_int32), ("dirty_chunk_bytes", ctypes.c_int64),
                ("exchange_mode", ctypes.c_int32), ("debug_checks", ctypes.c_int32), ("profile", ctypes.c_int32),
                ("dirty_protocol", ctypes.c_int32), ("halo_mode", ctypes.c_int32), ("multicast", ctypes.c_int32),
                ("nccl_unique_id", ctypes.c_uint8 * 128)]


class accmg_bounds(ctypes.Structure):
    _fields_ = [("ndim", ctypes.c_int32), ("pad", ctypes.c_int32), ("lo", ctypes.c_int64 * 3),
                ("hi", ctypes.c_int64 * 3)]


class accmg_access(ctypes.Structure):
    _fields_ = [("region", ctypes.c_void_p), ("mode", ctypes.c_int32), ("declared", ctypes.c_int32),
                ("stride", ctypes.c_int64), ("left", ctypes.c_int64), ("right", ctypes.c_int64)]


class accmg_args_jacobi2d(ctypes.Structure):
    _fields_ = [("rows", ctypes.c_int64), ("cols", ctypes.c_int64)]


class accmg_args_gemm(ctypes.Structure):
    _fields_ = [("M", ctypes.c_int64), ("N", ctypes.c_int64), ("K", ctypes.c_int64)]


class accmg_args_kmeans(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("d", ctypes.c_int32), ("k", ctypes.c_int32), ("shift", ctypes.c_int32),
                ("pad", ctypes.c_int32)]


class accmg_args_sparse(ctypes.Structure):
    _fields_ = [("rows", ctypes.c_int64), ("cols", ctypes.c_int64), ("period", ctypes.c_int64)]


class accmg_args_masked(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64)]


class accmg_args_jacobi3d(ctypes.Structure):
    _fields_ = [("n0", ctypes.c_int64), ("n1", ctypes.c_int64), ("n2", ctypes.c_int64)]


class accmg_args_jacobi2d_deep(ctypes.Structure):
    _fields_ = [("rows", ctypes.c_int64), ("cols", ctypes.c_int64), ("h", ctypes.c_int64)]


class accmg_args_scatter(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("m", ctypes.c_int64)]


_STAT_FIELDS = ["loops", "bytes_interpartition", "bytes_declared", "bytes_undeclared_payload",
                "bytes_undeclared_headers", "bytes_reduce", "bytes_paper_protocol", "bytes_remote", "bytes_h2d",
                "bytes_d2h", "body_launches", "kernel_launches", "device_bytes_user", "device_bytes_system"]


class accmg_stats(ctypes.Structure):
    _fields_ = [(f, ctypes.c_int64) for f in _STAT_FIELDS] + [
        ("ms_body", ctypes.c_double), ("ms_compact", ctypes.c_double), ("ms_exchange", ctypes.c_double),
        ("write_misses", ctypes.c_int64), ("bytes_write_miss", ctypes.c_int64),
        ("bytes_link", ctypes.c_int64), ("bytes_link_remote", ctypes.c_int64),
        ("bytes_multicast", ctypes.c_int64), ("multicast_regions", ctypes.c_int64)]


_vp, _i32, _i64, _sz = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_size_t
_p64 = ctypes.POINTER(ctypes.c_int64)
_SIGS = {
    "accmg_nccl_unique_id": [_vp],
    "accmg_unique_id": [_vp],
    "accmg_init": [ctypes.POINTER(accmg_config)],
    "accmg_finalize": [],
    "accmg_region_create": [_vp, _sz, _i64, ctypes.POINTER(_vp)],
    "accmg_region_destroy": [_vp],
    "accmg_loop_launch": [ctypes.POINTER(accmg_bounds), _i32, ctypes.POINTER(accmg_access), _i32, _vp, _sz],
    "accmg_sync_to_host": [_vp],
    "accmg_sync_to_host_owned": [_vp],
    "accmg_barrier": [],
    "accmg_get_stats": [ctypes.POINTER(accmg_stats)],
    "accmg_reset_stats": [],
    "accmg_set_profile": [_i32],
    "accmg_multicast_probe": [_i32, ctypes.c_char_p, _i32],
    "accmg_chunk": [_i64, _i64, _i32, _i32, _p64, _p64],
    "accmg_debug_dirty_bitmap": [_vp, _i32, _vp, _i64],
    "accmg_debug_chunk_bits": [_vp, _i32, _vp, _i64],
    "accmg_debug_packed": [_vp, _i32, _vp, _i64, _p64],
    "accmg_debug_replica": [_vp, _i32, _vp],
    "accmg_debug_valid": [_vp, _i32, _vp, _i64, _p64],
}
for _name, _args in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.argtypes = _args
    _f.restype = ctypes.c_int
_lib.accmg_last_error.argtypes = []
_lib.accmg_last_error.restype = ctypes.c_char_p
_lib.accmg_stream.argtypes = []
_lib.accmg_stream.restype = ctypes.c_void_p


def header_symbols() -> list[str]:
    """Entry points declared in include/accmg.h (for the export check)."""
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"^\s*(?:int|const char\*|void\*)\s+(accmg_\w+)\s*\(", txt, re.M)))


class AccmgError(RuntimeError):
    def __init__(self, code: int, fn: str):
        self.code = code
        super().__init__(f"{fn} failed with {code}: {accmg_last_error()}")


def _check(rc: int, fn: str) -> None:
    if rc != 0:
        raise AccmgError(rc, fn)


def _addr(a) -> int:
    if isinstance(a, np.ndarray):
        if not a.flags.c_contiguous:
            raise ValueError("host array must be C-contiguous")
        return a.ctypes.data
    return a.data_ptr()  # CPU torch tensor (e.g. pinned)


class Region:
    """Handle of a registered host array (keeps the host array alive, as the ABI borrows it)."""

    def __init__(self, handle: int, host, elem_size: int, extent: int):
        self.handle, self.host, self.elem_size, self.extent = handle, host, elem_size, extent

    @property
    def _as_parameter_(self):
        return ctypes.c_void_p(self.handle)


# ---- entry points (same names as the C ABI) ----------------------------------------------------
def accmg_nccl_unique_id() -> bytes:
    buf = (ctypes.c_uint8 * 128)()
    _check(_lib.accmg_nccl_unique_id(buf), "accmg_nccl_unique_id")
    return bytes(buf)


def accmg_unique_id() -> bytes:
    buf = (ctypes.c_uint8 * 128)()
    _check(_lib.accmg_unique_id(buf), "accmg_unique_id")
    return bytes(buf)


def accmg_init(num_partitions: int = 1, world_size: int = 1, rank: int = 0, device: int = 0,
               dirty_chunk_bytes: int = 0, exchange_mode: int = XCHG_AUTO, debug_checks: int = 0,
               profile: int = 0, nccl_unique_id: bytes | None = None, dirty_protocol: int = DIRTY_RUNS,
               halo_mode: int = HALO_AUTO, multicast: int = MC_OFF) -> None:
    c = accmg_config(num_partitions, world_size, rank, device, dirty_chunk_bytes, exchange_mode, debug_checks,
                     profile, dirty_protocol, halo_mode, multicast)
    if nccl_unique_id is not None:
        ctypes.memmove(c.nccl_unique_id, nccl_unique_id, 128)
    _check(_lib.accmg_init(ctypes.byref(c)), "accmg_init")


def accmg_multicast_probe(num_devices: int) -> tuple[bool, str]:
    """(True, "") if an NVLS multicast object over num_devices GPUs can be created, else (False, why)."""
    buf = ctypes.create_string_buffer(512)
    rc = _lib.accmg_multicast_probe(num_devices, buf, 512)
    if rc < 0:
        raise AccmgError(rc, "accmg_multicast_probe")
    return rc == 1, buf.value.decode()


def accmg_finalize() -> None:
    _check(_lib.accmg_finalize(), "accmg_finalize")


def accmg_region_create(host_array, elem_size: int | None = None, extent: int | None = None) -> Region:
    if elem_size is None:
        elem_size = host_array.itemsize if isinstance(host_array, np.ndarray) else host_array.element_size()
    if extent is None:
        extent = host_array.size if isinstance(host_array, np.ndarray) else host_array.numel()
    out = ctypes.c_void_p()
    _check(_lib.accmg_region_create(_addr(host_array), elem_size, extent, ctypes.byref(out)), "accmg_region_create")
    return Region(out.value, host_array, elem_size, extent)


def accmg_region_destroy(r: Region) -> None:
    _check(_lib.accmg_region_destroy(r), "accmg_region_destroy")


def bounds(lo, hi) -> accmg_bounds:
    b = accmg_bounds()
    b.ndim = len(lo)
    for i, (l, h) in enumerate(zip(lo, hi)):
        b.lo[i], b.hi[i] = l, h
    return b


def access(region: Region, mode: int, declared: bool = False, stride: int = 0, left: int = 0,
           right: int = 0) -> accmg_access:
    return accmg_access(region.handle, mode, int(declared), stride, left, right)


def accmg_loop_launch(b: accmg_bounds, body_id: int, descs, args) -> None:
    arr = (accmg_access * len(descs))(*descs)
    _check(_lib.accmg_loop_launch(ctypes.byref(b), body_id, arr, len(descs), ctypes.byref(args),
                                  ctypes.sizeof(args)), "accmg_loop_launch")


def accmg_sync_to_host(r: Region) -> None:
    _check(_lib.accmg_sync_to_host(r), "accmg_sync_to_host")


def accmg_sync_to_host_owned(r: Region) -> None:
    _check(_lib.accmg_sync_to_host_owned(r), "accmg_sync_to_host_owned")


def accmg_barrier() -> None:
    _check(_lib.accmg_barrier(), "accmg_barrier")


def accmg_get_stats() -> dict:
    s = accmg_stats()
    _check(_lib.accmg_get_stats(ctypes.byref(s)), "accmg_get_stats")
    return {f: getattr(s, f) for f, _ in accmg_stats._fields_}


def accmg_reset_stats() -> None:
    _check(_lib.accmg_reset_stats(), "accmg_reset_stats")


def accmg_set_profile(on: bool) -> None:
    _check(_lib.accmg_set_profile(1 if on else 0), "accmg_set_profile")


def accmg_last_error() -> str:
    return _lib.accmg_last_error().decode()


def accmg_stream() -> int | None:
    return _lib.accmg_stream()


def accmg_chunk(lo: int, hi: int, num_partitions: int, partition: int) -> tuple[int, int]:
    a, b = ctypes.c_int64(), ctypes.c_int64()
    _check(_lib.accmg_chunk(lo, hi, num_partitions, partition, ctypes.byref(a), ctypes.byref(b)), "accmg_chunk")
    return a.value, b.value


def accmg_debug_dirty_bitmap(r: Region, partition: int) -> np.ndarray:
    out = np.empty((r.extent + 31) // 32, dtype=np.uint32)
    _check(_lib.accmg_debug_dirty_bitmap(r, partition, out.ctypes.data, out.size), "accmg_debug_dirty_bitmap")
    return out


def accmg_debug_chunk_bits(r: Region, partition: int, chunk_elems: int) -> np.ndarray:
    nch = (r.extent + chunk_elems - 1) // chunk_elems
    out = np.empty((nch + 31) // 32, dtype=np.uint32)
    _check(_lib.accmg_debug_chunk_bits(r, partition, out.ctypes.data, out.size), "accmg_debug_chunk_bits")
    return out


def accmg_debug_packed(r: Region, partition: int) -> np.ndarray:
    used = ctypes.c_int64()
    _check(_lib.accmg_debug_packed(r, partition, None, 0, ctypes.byref(used)), "accmg_debug_packed")
    out = np.empty(used.value, dtype=np.uint8)
    _check(_lib.accmg_debug_packed(r, partition, out.ctypes.data, out.size, ctypes.byref(used)), "accmg_debug_packed")
    return out


def accmg_debug_replica(r: Region, partition: int, dtype) -> np.ndarray:
    out = np.empty(r.extent, dtype=dtype)
    assert out.itemsize == r.elem_size
    _check(_lib.accmg_debug_replica(r, partition, out.ctypes.data), "accmg_debug_replica")
    return out


def accmg_debug_valid(r: Region, partition: int) -> list[tuple[int, int]]:
    n = ctypes.c_int64()
    _check(_lib.accmg_debug_valid(r, partition, None, 0, ctypes.byref(n)), "accmg_debug_valid")
    out = np.empty(2 * max(n.value, 1), dtype=np.int64)
    _check(_lib.accmg_debug_valid(r, partition, out.ctypes.data, n.value, ctypes.byref(n)), "accmg_debug_valid")
    return [(int(out[2 * i]), int(out[2 * i + 1])) for i in range(n.value)]
