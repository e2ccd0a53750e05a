"""Thin ctypes binding of include/sesa.h (argument marshalling only; every step runs in libsesa.so's kernels).

The C names are kept: ``sesa_trace_create``, ``sesa_race_check``, ``sesa_races_get``, ``sesa_expand`` ...
``Trace`` wraps a handle for convenience; torch is used only for device memory and streams.  There is no CPU
fallback: if ``libsesa.so`` is missing or no CUDA device is present, calls raise.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libsesa.so")

SESA_OK, SESA_EINVAL, SESA_ERANGE, SESA_ENOMEM, SESA_ECUDA, SESA_ENCCL, SESA_ESTATE, SESA_ETRUNC = range(8)
SESA_SPACE_SHARED, SESA_SPACE_GLOBAL = 0, 1
SESA_READ, SESA_WRITE, SESA_ATOMIC = 0, 1, 2
SESA_RACE_RW, SESA_RACE_WW, SESA_RACE_WW_BENIGN = 1, 2, 3
SESA_FLAG_REPORT_BENIGN = 1

# numpy views of the ABI structs (declared here from include/sesa.h)
ACCESS_DTYPE = np.dtype(
    [("addr", "<u8"), ("value_hash", "<u8"), ("block", "<u4"), ("thread", "<u4"), ("interval", "<u4"),
     ("size", "<u2"), ("space", "u1"), ("rw", "u1")], align=True)
RACE_DTYPE = np.dtype(
    [("addr", "<u8"), ("first", "<u8"), ("second", "<u8"), ("block", "<u4"), ("interval", "<u4"),
     ("space", "u1"), ("kind", "u1"), ("reserved", "u1", (2,)), ("epoch", "<u4")], align=True)
FLOW_DTYPE = np.dtype(
    [("base", "<u8"), ("bstride", "<i8"), ("tstride", "<i8"), ("istride", "<i8"), ("value_seed", "<u8"),
     ("block_lo", "<u4"), ("block_hi", "<u4"), ("nthreads", "<u4"), ("interval", "<u4"),
     ("pmask", "<u4"), ("pval", "<u4"), ("pmod", "<u4"), ("prem", "<u4"), ("plo", "<u4"), ("phi", "<u4"),
     ("fkind", "<u4"), ("fc", "<u4"), ("fm", "<u4"), ("count", "<u4"),
     ("size", "<u2"), ("space", "u1"), ("rw", "u1"), ("flags", "<u4")], align=True)


REGION_DTYPE = np.dtype([("base", "<u8"), ("size", "<u8"), ("space", "<u4"), ("reserved", "<u4")], align=True)


class sesa_oob_report(ctypes.Structure):
    _fields_ = [("n_oob", ctypes.c_uint64), ("first_index", ctypes.c_uint64), ("first", ctypes.c_uint8 * 32)]


class sesa_config(ctypes.Structure):
    _fields_ = [("warp_size", ctypes.c_uint32), ("lockstep", ctypes.c_uint32), ("granularity", ctypes.c_uint32),
                ("flags", ctypes.c_uint32)]


class sesa_kernel_stat(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char * 32), ("launches", ctypes.c_uint32), ("ms", ctypes.c_float),
                ("bytes", ctypes.c_double)]


class sesa_flow_check_info(ctypes.Structure):
    _fields_ = [("n_flows", ctypes.c_uint64), ("n_flows_checked", ctypes.c_uint64), ("n_records", ctypes.c_uint64),
                ("n_records_checked", ctypes.c_uint64)]


class sesa_check_info(ctypes.Structure):
    _fields_ = [("n_records", ctypes.c_uint64), ("n_entries", ctypes.c_uint64), ("n_races", ctypes.c_uint64),
                ("n_multi", ctypes.c_uint64), ("sort_bits", ctypes.c_uint32), ("pos_bits", ctypes.c_uint32), ("digit_bits", ctypes.c_uint32),
                ("sort_passes", ctypes.c_uint32), ("sorted_input", ctypes.c_uint32), ("launches", ctypes.c_uint32),
                ("crossing_tiles", ctypes.c_uint32), ("n_stats", ctypes.c_uint32),
                ("fused_first_pass", ctypes.c_uint32), ("bucket_path", ctypes.c_uint32),
                ("wbit_filter", ctypes.c_uint32)]


# every symbol include/sesa.h declares (tests assert the library exports all of them)
EXPORTS = ["sesa_trace_create", "sesa_trace_create_dist", "sesa_nccl_unique_id", "sesa_race_check",
           "sesa_race_check_host", "sesa_races_get", "sesa_races_device", "sesa_expand", "sesa_trace_set_profiling",
           "sesa_trace_info", "sesa_trace_kernel_stats", "sesa_trace_destroy", "sesa_status_str", "sesa_last_error",
           "sesa_abi_version", "sesa_race_check_loopback", "sesa_trace_set_regions", "sesa_oob_get",
           "sesa_race_check_launches", "sesa_race_check_warp", "sesa_race_check_flows", "sesa_flow_check_get"]

_lib = None


def load() -> ctypes.CDLL:
    """Load libsesa.so (raises if it has not been built: there is no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} missing: build it with `python -m paper_conf_sc_lilg14_b200.build`")
    lib = ctypes.CDLL(LIB_PATH)
    P, U64, U32, I = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
    PP = ctypes.POINTER(ctypes.c_void_p)
    lib.sesa_trace_create.argtypes = [ctypes.POINTER(sesa_config), PP]
    lib.sesa_trace_create_dist.argtypes = [ctypes.POINTER(sesa_config), I, I, P, PP]
    lib.sesa_nccl_unique_id.argtypes = [P]
    lib.sesa_race_check.argtypes = [P, P, U64, U64, P]
    lib.sesa_race_check_host.argtypes = [P, P, U64, U64, P]
    lib.sesa_race_check_launches.argtypes = [P, P, U64, P, U32, U64, P]
    lib.sesa_race_check_warp.argtypes = [P, P, P, U64, U64, P]
    lib.sesa_race_check_flows.argtypes = [P, P, U64, P]
    lib.sesa_flow_check_get.argtypes = [P, ctypes.POINTER(sesa_flow_check_info)]
    lib.sesa_race_check_loopback.argtypes = [ctypes.POINTER(sesa_config), P, P, I, U64, P, PP]
    lib.sesa_races_get.argtypes = [P, P, U64, ctypes.POINTER(U64)]
    lib.sesa_races_device.argtypes = [P, PP, ctypes.POINTER(U64)]
    lib.sesa_expand.argtypes = [P, P, U64, P, U64, ctypes.POINTER(U64), P]
    lib.sesa_trace_set_profiling.argtypes = [P, I]
    lib.sesa_trace_info.argtypes = [P, ctypes.POINTER(sesa_check_info)]
    lib.sesa_trace_kernel_stats.argtypes = [P, ctypes.POINTER(sesa_kernel_stat), U32, ctypes.POINTER(U32)]
    lib.sesa_trace_destroy.argtypes = [P]
    lib.sesa_trace_destroy.restype = None
    lib.sesa_status_str.argtypes = [I]
    lib.sesa_status_str.restype = ctypes.c_char_p
    lib.sesa_last_error.argtypes = [P]
    lib.sesa_last_error.restype = ctypes.c_char_p
    lib.sesa_abi_version.restype = I
    for name in EXPORTS:
        if name not in ("sesa_trace_destroy", "sesa_status_str", "sesa_last_error", "sesa_abi_version"):
            getattr(lib, name).restype = I
    _lib = lib
    return lib


class SesaError(RuntimeError):
    def __init__(self, status: int, detail: str):
        super().__init__(f"{load().sesa_status_str(status).decode()}: {detail}")
        self.status = status
        self.detail = detail


def _stream_ptr(stream):
    if stream is None:
        import torch
        return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return ctypes.c_void_p(stream)
    return ctypes.c_void_p(stream.cuda_stream)


class Trace:
    """One sesa_trace handle (single GPU, or one rank of a distributed check)."""

    def __init__(self, warp_size: int = 32, lockstep: int = 0, granularity: int = 4, *, dist=None,
                 benign: bool = False):
        lib = load()
        # flags bit 0 = SESA_FLAG_REPORT_BENIGN: also report benign W/W locations as kind 3
        self.cfg = sesa_config(warp_size, lockstep, granularity, 1 if benign else 0)
        h = ctypes.c_void_p()
        if dist is None:
            st = lib.sesa_trace_create(ctypes.byref(self.cfg), ctypes.byref(h))
        else:
            rank, world, uid = dist
            buf = (ctypes.c_uint8 * 128).from_buffer_copy(bytes(uid))
            st = lib.sesa_trace_create_dist(ctypes.byref(self.cfg), rank, world, buf, ctypes.byref(h))
        if st != SESA_OK:
            raise SesaError(st, "sesa_trace_create")
        self.h = h
        self.lib = lib

    def close(self):
        if getattr(self, "h", None):
            self.lib.sesa_trace_destroy(self.h)
            self.h = None

    __del__ = close

    def _raise(self, st, what):
        raise SesaError(st, f"{what}: {self.lib.sesa_last_error(self.h).decode()}")

    def check(self, d_records, n: int | None = None, index_base: int = 0, stream=None) -> int:
        """Race-check device records (a torch uint8/any tensor or raw pointer); returns the race count."""
        ptr, count = _dev_ptr(d_records, n)
        st = self.lib.sesa_race_check(self.h, ctypes.c_void_p(ptr), count, index_base, _stream_ptr(stream))
        if st != SESA_OK:
            self._raise(st, "sesa_race_check")
        return self.n_races()

    def check_launches(self, d_records, n: int, launch_offsets, index_base: int = 0, stream=None) -> int:
        """Multi-launch trace: records [launch_offsets[e], launch_offsets[e+1]) came from kernel launch e."""
        ptr, count = _dev_ptr(d_records, n)
        offs = np.ascontiguousarray(np.asarray(launch_offsets, dtype=np.uint64))
        st = self.lib.sesa_race_check_launches(self.h, ctypes.c_void_p(ptr), count, ctypes.c_void_p(offs.ctypes.data),
                                               len(offs) - 1, index_base, _stream_ptr(stream))
        if st != SESA_OK:
            self._raise(st, "sesa_race_check_launches")
        return self.n_races()

    def check_warp(self, d_records, d_ext, n: int, index_base: int = 0, stream=None) -> int:
        """Precise warp model (NEXT-3): d_ext = device array of n {pc, div} u32 pairs."""
        ptr, count = _dev_ptr(d_records, n)
        eptr = d_ext if isinstance(d_ext, int) else d_ext.data_ptr()
        st = self.lib.sesa_race_check_warp(self.h, ctypes.c_void_p(ptr), ctypes.c_void_p(eptr), count, index_base,
                                           _stream_ptr(stream))
        if st != SESA_OK:
            self._raise(st, "sesa_race_check_warp")
        return self.n_races()

    def check_flows(self, d_flows, n_flows: int, stream=None) -> int:
        """Descriptor-level check (NEXT-2): the race list of the expansion of n_flows device descriptors."""
        ptr = d_flows if isinstance(d_flows, int) else d_flows.data_ptr()
        st = self.lib.sesa_race_check_flows(self.h, ctypes.c_void_p(ptr), n_flows, _stream_ptr(stream))
        if st != SESA_OK:
            self._raise(st, "sesa_race_check_flows")
        return self.n_races()

    def flow_info(self) -> dict:
        i = sesa_flow_check_info()
        self.lib.sesa_flow_check_get(self.h, ctypes.byref(i))
        return {k: getattr(i, k) for k, _ in sesa_flow_check_info._fields_}

    def check_host(self, h_records: np.ndarray, index_base: int = 0, stream=None) -> int:
        a = np.ascontiguousarray(h_records)
        assert a.dtype.itemsize == 32
        st = self.lib.sesa_race_check_host(self.h, ctypes.c_void_p(a.ctypes.data if len(a) else 0), len(a),
                                           index_base, _stream_ptr(stream))
        if st != SESA_OK:
            self._raise(st, "sesa_race_check_host")
        return self.n_races()

    def check_host_ptr(self, ptr: int, n: int, index_base: int = 0, stream=None) -> int:
        st = self.lib.sesa_race_check_host(self.h, ctypes.c_void_p(ptr), n, index_base, _stream_ptr(stream))
        if st != SESA_OK:
            self._raise(st, "sesa_race_check_host")
        return self.n_races()

    def n_races(self) -> int:
        n = ctypes.c_uint64()
        st = self.lib.sesa_races_get(self.h, None, 0, ctypes.byref(n))
        if st != SESA_OK:
            self._raise(st, "sesa_races_get")
        return n.value

    def races(self) -> np.ndarray:
        n = self.n_races()
        out = np.zeros(n, RACE_DTYPE)
        got = ctypes.c_uint64()
        st = self.lib.sesa_races_get(self.h, ctypes.c_void_p(out.ctypes.data if n else 0), n, ctypes.byref(got))
        if st != SESA_OK:
            self._raise(st, "sesa_races_get")
        return out

    def races_device(self):
        p = ctypes.c_void_p()
        n = ctypes.c_uint64()
        st = self.lib.sesa_races_device(self.h, ctypes.byref(p), ctypes.byref(n))
        if st != SESA_OK:
            self._raise(st, "sesa_races_device")
        return p.value, n.value

    def expand(self, d_flows, n_flows: int, d_out=None, cap: int = 0, stream=None) -> int:
        fptr, _ = _dev_ptr(d_flows, n_flows)
        optr = 0 if d_out is None else _dev_ptr(d_out, cap)[0]
        n = ctypes.c_uint64()
        st = self.lib.sesa_expand(self.h, ctypes.c_void_p(fptr), n_flows, ctypes.c_void_p(optr), cap,
                                  ctypes.byref(n), _stream_ptr(stream))
        if st not in (SESA_OK, SESA_ETRUNC) or (st == SESA_ETRUNC and d_out is not None):
            self._raise(st, "sesa_expand")
        return n.value

    def set_regions(self, regions: np.ndarray):
        """Register memory regions (REGION_DTYPE array: base, size, space) for the out-of-bound check."""
        a = np.ascontiguousarray(regions, dtype=REGION_DTYPE)
        st = self.lib.sesa_trace_set_regions(self.h, ctypes.c_void_p(a.ctypes.data if len(a) else 0),
                                             ctypes.c_uint32(len(a)))
        if st != SESA_OK:
            self._raise(st, "sesa_trace_set_regions")

    def oob(self) -> dict:
        """The last check's OOB report: n_oob, first_index (2**64-1 if none), first (record, ACCESS_DTYPE)."""
        r = sesa_oob_report()
        st = self.lib.sesa_oob_get(self.h, ctypes.byref(r))
        if st != SESA_OK:
            self._raise(st, "sesa_oob_get")
        return dict(n_oob=r.n_oob, first_index=r.first_index,
                    first=np.frombuffer(bytes(r.first), ACCESS_DTYPE)[0])

    def set_profiling(self, on: bool = True):
        self.lib.sesa_trace_set_profiling(self.h, 1 if on else 0)

    def info(self) -> dict:
        i = sesa_check_info()
        self.lib.sesa_trace_info(self.h, ctypes.byref(i))
        return {k: getattr(i, k) for k, _ in sesa_check_info._fields_}

    def kernel_stats(self) -> list[dict]:
        n = ctypes.c_uint32()
        self.lib.sesa_trace_kernel_stats(self.h, None, 0, ctypes.byref(n))
        arr = (sesa_kernel_stat * max(n.value, 1))()
        self.lib.sesa_trace_kernel_stats(self.h, arr, n.value, ctypes.byref(n))
        return [dict(name=arr[i].name.decode(), launches=arr[i].launches, ms=arr[i].ms, bytes=arr[i].bytes)
                for i in range(n.value)]


def _dev_ptr(x, n):
    """(pointer, element count) of a torch tensor of records (dtype uint8 with 32*n bytes, or int64 [n, 4]) or
    of an int pointer with an explicit n."""
    if isinstance(x, int):
        assert n is not None
        return x, n
    nbytes = x.numel() * x.element_size()
    return x.data_ptr(), (n if n is not None else nbytes // 32)


def check_loopback(d_records, offs, warp_size=32, lockstep=0, granularity=4, index_base=0, stream=None,
                   benign=False):
    """Distributed check with len(offs)-1 virtual ranks on this GPU; returns the merged race array."""
    lib = load()
    cfg = sesa_config(warp_size, lockstep, granularity, SESA_FLAG_REPORT_BENIGN if benign else 0)
    o = (ctypes.c_uint64 * len(offs))(*offs)
    h = ctypes.c_void_p()
    ptr, _ = _dev_ptr(d_records, offs[-1])
    st = lib.sesa_race_check_loopback(ctypes.byref(cfg), ctypes.c_void_p(ptr), o, len(offs) - 1, index_base,
                                      _stream_ptr(stream), ctypes.byref(h))
    try:
        if st != SESA_OK:
            raise SesaError(st, lib.sesa_last_error(h).decode() if h.value else "sesa_race_check_loopback")
        n = ctypes.c_uint64()
        lib.sesa_races_get(h, None, 0, ctypes.byref(n))
        out = np.zeros(n.value, RACE_DTYPE)
        if n.value:
            lib.sesa_races_get(h, ctypes.c_void_p(out.ctypes.data), n.value, ctypes.byref(n))
        return out
    finally:
        if h.value:
            lib.sesa_trace_destroy(h)


def nccl_unique_id() -> bytes:
    buf = (ctypes.c_uint8 * 128)()
    st = load().sesa_nccl_unique_id(buf)
    if st != SESA_OK:
        raise SesaError(st, "sesa_nccl_unique_id")
    return bytes(buf)


def to_device(records: np.ndarray, device="cuda"):
    """Copy a record array (32-byte items) to a torch uint8 device tensor."""
    import torch
    a = np.ascontiguousarray(records)
    return torch.from_numpy(a.view(np.uint8).reshape(-1)).to(device)
