"""CPU oracle loader — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline / ``--impl reference`` legs may
import this module.  It compiles and loads ``oracle/sesa_oracle.c`` (plain C, written from the paper — see its
header for the rule-by-rule citations) with ctypes.  It shares no code with the CUDA path
(``paper_conf_sc_lilg14_b200``): the numpy layouts below are declared here independently and a test asserts
they match the C structs' sizes.

Functions
  check(records, index_base=0, warp_size=32, lockstep=0, granularity=4, method="grouped", threads=None) -> races
      method = "brute" | "grouped" | "partitioned" (T threads, locations split by hash; same bytes as "grouped")
  pair_kind(rec_a, rec_b, warp_size, lockstep) -> 0 | 1 (RW) | 2 (WW)
  benign_pair(rec_a, rec_b) -> 0 | 1   (benign W/W pair: kind 3 with check(..., benign=True), NEXT-4)
  validate(records) -> None or lowest bad index
  expand(flows) -> records  (canonical schedule order)
  oob(records, regions, index_base=0) -> (count, first_index or None)   out-of-bound check (NEXT-1)
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import time

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "sesa_oracle.c")
_SO = os.path.join(_HERE, "_build", "libsesa_oracle.so")

REC_DTYPE = np.dtype(
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

EXT_DTYPE = np.dtype([("pc", "<u4"), ("div", "<u4")])  # precise warp model extension (NEXT-3)

_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle (gcc -O2).  Building the checker is not using it (it is only called by tests)."""
    os.makedirs(os.path.dirname(_SO), exist_ok=True)
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-fPIC", "-shared", "-pthread", "-Wall", "-o", tmp, _SRC])
        os.replace(tmp, _SO)
    return _SO


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        P, U64, U32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32
        for name in ("oracle_check_brute", "oracle_check_grouped"):
            f = getattr(lib, name)
            f.argtypes = [P, U64, U64, U32, U32, U32, U32, P, U64, ctypes.POINTER(U64)]
            f.restype = ctypes.c_int
        lib.oracle_check_partitioned.argtypes = [P, U64, U64, U32, U32, U32, U32, U32, P, U64, ctypes.POINTER(U64)]
        lib.oracle_check_partitioned.restype = ctypes.c_int
        for name in ("oracle_check_brute_ep", "oracle_check_grouped_ep"):
            f = getattr(lib, name)
            f.argtypes = [P, P, U64, U64, U32, U32, U32, U32, P, U64, ctypes.POINTER(U64)]
            f.restype = ctypes.c_int
        lib.oracle_check_partitioned_ep.argtypes = [P, P, U64, U64, U32, U32, U32, U32, U32, P, U64,
                                                    ctypes.POINTER(U64)]
        lib.oracle_check_partitioned_ep.restype = ctypes.c_int
        for name in ("oracle_check_warp_brute", "oracle_check_warp_grouped"):
            f = getattr(lib, name)
            f.argtypes = [P, P, U64, U64, U32, U32, U32, P, U64, ctypes.POINTER(U64)]
            f.restype = ctypes.c_int
        lib.oracle_pair_kind_warp.argtypes = [P, P, P, P, U32, U32]
        lib.oracle_pair_kind_warp.restype = ctypes.c_int
        lib.oracle_pair_kind.argtypes = [P, P, U32, U32]
        lib.oracle_pair_kind.restype = ctypes.c_int
        lib.oracle_benign_pair.argtypes = [P, P]
        lib.oracle_benign_pair.restype = ctypes.c_int
        lib.oracle_validate.argtypes = [P, U64, ctypes.POINTER(U64)]
        lib.oracle_validate.restype = ctypes.c_int
        lib.oracle_expand.argtypes = [P, U64, P, U64]
        lib.oracle_expand.restype = U64
        for name in ("oracle_sizeof_rec", "oracle_sizeof_race", "oracle_sizeof_flow"):
            getattr(lib, name).restype = U64
        assert lib.oracle_sizeof_rec() == REC_DTYPE.itemsize == 32
        assert lib.oracle_sizeof_race() == RACE_DTYPE.itemsize == 40
        assert lib.oracle_sizeof_flow() == FLOW_DTYPE.itemsize == 104
        _lib = lib
    return _lib


class OracleError(RuntimeError):
    def __init__(self, code: int, detail: int):
        super().__init__(f"oracle error {code} (detail {detail})")
        self.code, self.detail = code, detail


def _as_recs(records) -> np.ndarray:
    r = np.ascontiguousarray(records)
    if r.dtype != REC_DTYPE:
        r = r.view(REC_DTYPE) if r.dtype.itemsize == 32 or r.dtype == np.uint8 else r.astype(REC_DTYPE)
    return r


def nthreads() -> int:
    """Host threads the partitioned checker uses by default (the cores this process may run on)."""
    try:
        return max(1, len(os.sched_getaffinity(0)))
    except AttributeError:  # pragma: no cover
        return max(1, os.cpu_count() or 1)


def check(records, index_base: int = 0, warp_size: int = 32, lockstep: int = 0, granularity: int = 4,
          method: str = "grouped", benign: bool = False, threads: int | None = None, launches=None) -> np.ndarray:
    """Canonical race list (sorted by (epoch, space, block, interval, addr, kind)) of ``records``; with ``benign``
    also one kind-3 record per location holding a benign W/W pair (config flags bit 0, oracle_benign_pair).
    method: "brute" (all pairs), "grouped" (1 thread), "partitioned" (``threads`` threads, default nthreads()).
    launches: multi-launch trace (NEXT-4): offsets [0, o1, ..., n] — records [o_e, o_{e+1}) ran in kernel launch
    e; accesses of different launches are ordered and never race (the race's `epoch` field names its launch)."""
    lib = _load()
    r = _as_recs(records)
    T = nthreads() if threads is None else int(threads)
    ep = None
    if launches is not None:
        offs = np.asarray(launches, dtype=np.int64)
        assert offs[0] == 0 and offs[-1] == len(r) and (np.diff(offs) >= 0).all()
        ep = np.repeat(np.arange(len(offs) - 1, dtype=np.uint32), np.diff(offs))
    cap = 1024
    while True:
        out = np.zeros(cap, RACE_DTYPE)
        nout = ctypes.c_uint64(0)
        rp = r.ctypes.data if len(r) else None
        args = (len(r), index_base, warp_size, lockstep, granularity, 1 if benign else 0)
        if ep is not None:
            epp = ep.ctypes.data if len(ep) else None
            if method == "partitioned":
                rc = lib.oracle_check_partitioned_ep(rp, epp, *args, T, out.ctypes.data, cap, ctypes.byref(nout))
            else:
                fn = lib.oracle_check_brute_ep if method == "brute" else lib.oracle_check_grouped_ep
                rc = fn(rp, epp, *args, out.ctypes.data, cap, ctypes.byref(nout))
        elif method == "partitioned":
            rc = lib.oracle_check_partitioned(rp, *args, T, out.ctypes.data, cap, ctypes.byref(nout))
        else:
            fn = lib.oracle_check_brute if method == "brute" else lib.oracle_check_grouped
            rc = fn(rp, *args, out.ctypes.data, cap, ctypes.byref(nout))
        if rc == 7:
            cap = int(nout.value)
            continue
        if rc != 0:
            raise OracleError(rc, int(nout.value))
        return out[: nout.value].copy()


def check_warp(records, ext, index_base: int = 0, warp_size: int = 32, lockstep: int = 1, granularity: int = 4,
               method: str = "grouped") -> np.ndarray:
    """Precise warp model (NEXT-3, oracle_pair_kind_warp): ``ext`` holds one {pc, div} per record."""
    lib = _load()
    r = _as_recs(records)
    e = np.ascontiguousarray(np.asarray(ext).view(EXT_DTYPE) if np.asarray(ext).dtype != EXT_DTYPE else ext)
    assert len(e) == len(r)
    fn = lib.oracle_check_warp_brute if method == "brute" else lib.oracle_check_warp_grouped
    cap = 1024
    while True:
        out = np.zeros(cap, RACE_DTYPE)
        nout = ctypes.c_uint64(0)
        rc = fn(r.ctypes.data if len(r) else None, e.ctypes.data if len(e) else None, len(r), index_base, warp_size,
                lockstep, granularity, out.ctypes.data, cap, ctypes.byref(nout))
        if rc == 7:
            cap = int(nout.value)
            continue
        if rc != 0:
            raise OracleError(rc, int(nout.value))
        return out[: nout.value].copy()


def timed_check(records, **kw):
    t0 = time.perf_counter()
    races = check(records, **kw)
    return races, time.perf_counter() - t0


def pair_kind(a, b, warp_size: int = 32, lockstep: int = 0) -> int:
    lib = _load()
    ra = _as_recs(np.asarray(a).reshape(1))
    rb = _as_recs(np.asarray(b).reshape(1))
    return int(lib.oracle_pair_kind(ra.ctypes.data, rb.ctypes.data, warp_size, lockstep))


def benign_pair(a, b) -> int:
    lib = _load()
    ra = _as_recs(np.asarray(a).reshape(1))
    rb = _as_recs(np.asarray(b).reshape(1))
    return int(lib.oracle_benign_pair(ra.ctypes.data, rb.ctypes.data))


def validate(records):
    lib = _load()
    r = _as_recs(records)
    bad = ctypes.c_uint64(0)
    if lib.oracle_validate(r.ctypes.data if len(r) else None, len(r), ctypes.byref(bad)):
        return int(bad.value)
    return None


def expand(flows) -> np.ndarray:
    lib = _load()
    f = np.ascontiguousarray(flows)
    if f.dtype != FLOW_DTYPE:
        f = f.view(FLOW_DTYPE)
    n = lib.oracle_expand(f.ctypes.data if len(f) else None, len(f), None, 0)
    if n == 2**64 - 1:
        raise OracleError(1, 0)
    out = np.zeros(n, REC_DTYPE)
    lib.oracle_expand(f.ctypes.data if len(f) else None, len(f), out.ctypes.data if n else None, n)
    return out


def race_tuples(races: np.ndarray):
    """Races as plain tuples (for readable comparisons in tests)."""
    return [(int(x["space"]), int(x["block"]), int(x["interval"]), int(x["addr"]), int(x["kind"]),
             int(x["first"]), int(x["second"])) for x in races]


def oob(records: np.ndarray, regions: np.ndarray, index_base: int = 0):
    """Out-of-bound records, by the definition in include/sesa.h (sesa_region; Table IV "OOB" P:467, Fig. 9
    P:569-571): a valid record of a space with registered regions is OOB iff NO region of its space contains all
    its bytes (base <= addr and addr + size <= base + size).  Spaces without regions are not checked.  Plain
    definition: every record against every region of its space (no search structure).  Returns
    (count, lowest index_base-adjusted OOB index or None)."""
    r = np.asarray(records)
    addr = r["addr"].astype(np.uint64)
    end = addr + r["size"].astype(np.uint64)  # one past the last byte (records do not wrap: validated)
    bad = np.zeros(len(r), bool)
    for sp in (0, 1):
        regs = regions[regions["space"] == sp]
        if len(regs) == 0:
            continue
        sel = r["space"] == sp
        inside = np.zeros(len(r), bool)
        for g in regs:  # each region in turn: the definition, record by record
            b, e = np.uint64(g["base"]), np.uint64(g["base"]) + np.uint64(g["size"])
            inside |= sel & (addr >= b) & (end <= e)
        bad |= sel & ~inside
    idx = np.nonzero(bad)[0]
    return int(len(idx)), (int(idx[0]) + index_base if len(idx) else None)

