"""BASELINE configs C3-C5: host generation (numpy, for the oracle) and device generation (torch, for the bench).

Recipes (formulas in csrc/gen_common.h):
  C3  Parboil-histo-shaped: 1024 x 512 threads, 96 grid-stride pixels each: R img[p]; 1/64 guarded R bins[b];
      ATOMIC bins[b], b ~ Zipf(s=1) over 4096 bins.  ~101.4 M records.  ws 32, lockstep 0.
  C4  Lonestar-bfs-shaped: 2^24 nodes (32768 x 512), power-law degrees (alpha 2.1, 4..1024, mean 16.8), R-MAT
      destinations, 45% frontier / 5% visited / 50% unvisited.  ~410 M records.  ws 32, lockstep 1.
  C5  scaling sweep: 1e9 records, unique words via a Feistel permutation, R/W/A 70/25/5, 1e5 injected races.
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass

import numpy as np

from . import SEED_BASE
from .build import DEV_SO, HOST_SO, build
from .layout import REC_DTYPE


class C5Cfg(ctypes.Structure):
    _fields_ = [("seed", ctypes.c_uint64), ("n", ctypes.c_uint64), ("base", ctypes.c_uint64)]


class C3Cfg(ctypes.Structure):
    _fields_ = [("seed", ctypes.c_uint64), ("blocks", ctypes.c_uint32), ("threads", ctypes.c_uint32),
                ("ppt", ctypes.c_uint32), ("nbins", ctypes.c_uint32), ("img_base", ctypes.c_uint64),
                ("bins_base", ctypes.c_uint64)]


class C4Cfg(ctypes.Structure):
    _fields_ = [("seed", ctypes.c_uint64), ("log2n", ctypes.c_uint32), ("dmin", ctypes.c_uint32),
                ("ndeg", ctypes.c_uint32), ("pad", ctypes.c_uint32), ("dist_base", ctypes.c_uint64),
                ("row_base", ctypes.c_uint64), ("col_base", ctypes.c_uint64), ("changed_base", ctypes.c_uint64)]


class RndCfg(ctypes.Structure):
    _fields_ = [("seed", ctypes.c_uint64), ("n", ctypes.c_uint64), ("blocks", ctypes.c_uint32),
                ("threads", ctypes.c_uint32), ("intervals", ctypes.c_uint32), ("words", ctypes.c_uint32),
                ("shared_pm", ctypes.c_uint32), ("atomic_pm", ctypes.c_uint32), ("write_pm", ctypes.c_uint32),
                ("values", ctypes.c_uint32), ("nsizes", ctypes.c_uint32), ("sorted", ctypes.c_uint32),
                ("unaligned", ctypes.c_uint32), ("pad", ctypes.c_uint32), ("sizes", ctypes.c_uint16 * 4),
                ("gbase", ctypes.c_uint64)]


_host = _dev = None


def _hostlib():
    global _host
    if _host is None:
        build()
        _host = ctypes.CDLL(HOST_SO)
        P, U64 = ctypes.c_void_p, ctypes.c_uint64
        _host.gen_c5_host.argtypes = [P, U64, U64, P]
        _host.gen_c3_count_host.argtypes = [P]
        _host.gen_c3_count_host.restype = U64
        _host.gen_c3_host.argtypes = [P, P, P]
        _host.gen_c4_layout_host.argtypes = [P, P, P, P]
        _host.gen_c4_layout_host.restype = U64
        _host.gen_c4_host.argtypes = [P, P, P, P, P]
        _host.gen_random_host.argtypes = [P, U64, U64, P]
        assert _host.gen_sizeof_rndcfg() == ctypes.sizeof(RndCfg)
        assert _host.gen_sizeof_c3cfg() == ctypes.sizeof(C3Cfg)
        assert _host.gen_sizeof_c4cfg() == ctypes.sizeof(C4Cfg)
        assert _host.gen_sizeof_c5cfg() == ctypes.sizeof(C5Cfg)
    return _host


def _devlib():
    global _dev
    if _dev is None:
        build()
        _dev = ctypes.CDLL(DEV_SO)
        P, U64 = ctypes.c_void_p, ctypes.c_uint64
        _dev.gen_c5_dev.argtypes = [P, U64, U64, P, P]
        _dev.gen_c3_count_dev.argtypes = [P, P, P]
        _dev.gen_c3_write_dev.argtypes = [P, P, P, P, P]
        _dev.gen_c4_degree_dev.argtypes = [P, P, P, P]
        _dev.gen_c4_count_dev.argtypes = [P, P, P, P, P]
        _dev.gen_c4_write_dev.argtypes = [P, P, P, P, P, P]
    return _dev


def _cdf_u64(p: np.ndarray) -> np.ndarray:
    c = np.cumsum(p / p.sum())
    out = np.minimum(np.floor(c * 2.0**64), 2.0**64 - 1).astype(np.float64)
    cdf = np.array([int(x) if x < 2.0**64 else 2**64 - 1 for x in out], dtype=object)
    cdf = np.array([min(int(x), 2**64 - 1) for x in cdf], dtype=np.uint64)
    cdf[-1] = np.uint64(2**64 - 1)
    return cdf


def zipf_cdf(nbins: int = 4096, s: float = 1.0) -> np.ndarray:
    return _cdf_u64(1.0 / np.arange(1, nbins + 1, dtype=np.float64) ** s)


def degree_cdf(dmin: int = 4, dmax: int = 1024, alpha: float = 2.1) -> np.ndarray:
    return _cdf_u64(np.arange(dmin, dmax + 1, dtype=np.float64) ** -alpha)


# ---------------------------------------------------------------------------------------------------------- C5
C5_BASE = 0x7F6000000000


def c5_cfg(n: int = 10**9) -> C5Cfg:
    return C5Cfg(SEED_BASE + 5, n, C5_BASE)


def c5_host(n: int = 10**9, lo: int = 0, hi: int | None = None) -> np.ndarray:
    hi = n if hi is None else hi
    out = np.zeros(hi - lo, REC_DTYPE)
    c = c5_cfg(n)
    _hostlib().gen_c5_host(ctypes.byref(c), lo, hi, out.ctypes.data if hi > lo else None)
    return out


def c5_device(n: int = 10**9, out=None, stream=None):
    import torch
    if out is None:
        out = torch.empty(n * 32, dtype=torch.uint8, device="cuda")
    c = c5_cfg(n)
    s = torch.cuda.current_stream().cuda_stream if stream is None else stream
    rc = _devlib().gen_c5_dev(ctypes.byref(c), 0, n, ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(s))
    assert rc == 0, rc
    return out


def c5_truth(n: int = 10**9, index_base: int = 0) -> np.ndarray:
    """Expected races of C5 by construction: one per stratum at the victim's word, witness (victim, partner)."""
    from .layout import RACE_DTYPE
    K = max(1, n // 10000)
    S = n // K
    half = S // 2
    from . import mix
    seed = SEED_BASE + 5
    ks = np.arange(K, dtype=np.uint64)
    v = np.array([k * S + mix(seed ^ 0x1A1A ^ k) % half for k in range(K)], dtype=np.uint64)
    p = v + np.uint64(half)
    recv = np.concatenate([c5_host(n, int(i), int(i) + 1) for i in v]) if K <= 2000 else _c5_pick(n, v)
    recp = np.concatenate([c5_host(n, int(i), int(i) + 1) for i in p]) if K <= 2000 else _c5_pick(n, p)
    races = np.zeros(K, RACE_DTYPE)
    races["addr"] = recv["addr"]
    races["first"] = v + np.uint64(index_base)
    races["second"] = p + np.uint64(index_base)
    races["block"] = 0xFFFFFFFF
    races["interval"] = 0xFFFFFFFF
    races["space"] = 1
    races["kind"] = np.where((recv["rw"] == 0) | (recp["rw"] == 0), 1, 2)
    del ks
    return races[np.argsort(races["addr"], kind="stable")]


def _c5_pick(n, idx):
    out = np.zeros(len(idx), REC_DTYPE)
    c = c5_cfg(n)
    lib = _hostlib()
    tmp = np.zeros(1, REC_DTYPE)
    for j, i in enumerate(idx):
        lib.gen_c5_host(ctypes.byref(c), int(i), int(i) + 1, tmp.ctypes.data)
        out[j] = tmp[0]
    return out


# ---------------------------------------------------------------------------------------------------------- C3
C3_IMG = 0x7F5000000000


@dataclass
class C3:
    blocks: int = 1024
    threads: int = 512
    ppt: int = 96
    nbins: int = 4096

    def cfg(self) -> C3Cfg:
        npix = self.blocks * self.threads * self.ppt
        bins = C3_IMG + 4 * npix + 4096
        return C3Cfg(SEED_BASE + 3, self.blocks, self.threads, self.ppt, self.nbins, C3_IMG, bins)

    def cdf(self) -> np.ndarray:
        return zipf_cdf(self.nbins)

    def host(self) -> np.ndarray:
        lib = _hostlib()
        c = self.cfg()
        n = lib.gen_c3_count_host(ctypes.byref(c))
        out = np.zeros(n, REC_DTYPE)
        cdf = self.cdf()
        lib.gen_c3_host(ctypes.byref(c), cdf.ctypes.data, out.ctypes.data)
        return out

    def device(self):
        import torch
        lib = _devlib()
        c = self.cfg()
        T = self.blocks * self.threads
        s = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
        cnt = torch.empty(T, dtype=torch.int32, device="cuda")
        assert lib.gen_c3_count_dev(ctypes.byref(c), ctypes.c_void_p(cnt.data_ptr()), s) == 0
        off = torch.cumsum(cnt.to(torch.int64), 0) - cnt.to(torch.int64)
        n = int(off[-1].item() + cnt[-1].item())
        out = torch.empty(n * 32, dtype=torch.uint8, device="cuda")
        cdf = torch.from_numpy(self.cdf().view(np.int64)).cuda()
        assert lib.gen_c3_write_dev(ctypes.byref(c), ctypes.c_void_p(cdf.data_ptr()), ctypes.c_void_p(off.data_ptr()),
                                    ctypes.c_void_p(out.data_ptr()), s) == 0
        return out, n


# ---------------------------------------------------------------------------------------------------------- C4
C4_DIST = 0x7F4000000000


@dataclass
class C4:
    log2n: int = 24
    dmin: int = 4
    dmax: int = 1024

    def cfg(self) -> C4Cfg:
        N = 1 << self.log2n
        dist = C4_DIST
        row = dist + 4 * N + 4096
        col = row + 4 * (N + 1) + 4096
        changed = dist - 64
        return C4Cfg(SEED_BASE + 4, self.log2n, self.dmin, self.dmax - self.dmin + 1, 0, dist, row, col, changed)

    def cdf(self) -> np.ndarray:
        return degree_cdf(self.dmin, self.dmax)

    def host(self) -> np.ndarray:
        lib = _hostlib()
        c = self.cfg()
        N = 1 << self.log2n
        rows = np.zeros(N + 1, np.uint64)
        counts = np.zeros(N, np.uint64)
        cdf = self.cdf()
        n = lib.gen_c4_layout_host(ctypes.byref(c), cdf.ctypes.data, rows.ctypes.data, counts.ctypes.data)
        out = np.zeros(n, REC_DTYPE)
        lib.gen_c4_host(ctypes.byref(c), cdf.ctypes.data, rows.ctypes.data, counts.ctypes.data, out.ctypes.data)
        return out

    def device(self):
        import torch
        lib = _devlib()
        c = self.cfg()
        N = 1 << self.log2n
        s = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
        cdf = torch.from_numpy(self.cdf().view(np.int64)).cuda()
        deg = torch.empty(N, dtype=torch.int32, device="cuda")
        assert lib.gen_c4_degree_dev(ctypes.byref(c), ctypes.c_void_p(cdf.data_ptr()),
                                     ctypes.c_void_p(deg.data_ptr()), s) == 0
        rows = torch.cumsum(deg.to(torch.int64), 0) - deg.to(torch.int64)
        cnt = torch.empty(N, dtype=torch.int32, device="cuda")
        assert lib.gen_c4_count_dev(ctypes.byref(c), ctypes.c_void_p(cdf.data_ptr()),
                                    ctypes.c_void_p(rows.data_ptr()), ctypes.c_void_p(cnt.data_ptr()), s) == 0
        off = torch.cumsum(cnt.to(torch.int64), 0) - cnt.to(torch.int64)
        n = int(off[-1].item() + cnt[-1].item())
        out = torch.empty(n * 32, dtype=torch.uint8, device="cuda")
        assert lib.gen_c4_write_dev(ctypes.byref(c), ctypes.c_void_p(cdf.data_ptr()),
                                    ctypes.c_void_p(rows.data_ptr()), ctypes.c_void_p(off.data_ptr()),
                                    ctypes.c_void_p(out.data_ptr()), s) == 0
        return out, n


# ---------------------------------------------------------------------------------------------------- random
def rnd_cfg(n: int, seed: int, *, blocks: int = 3, threads: int = 70, intervals: int = 3, words: int = 24,
            shared_frac: float = 0.5, sizes=(1, 2, 4, 8), atomic_frac: float = 0.15, write_frac: float = 0.35,
            values: int = 3, sort: bool = True, unaligned: bool = True) -> RndCfg:
    sz = (ctypes.c_uint16 * 4)(*(list(sizes) + [1] * (4 - len(sizes))))
    return RndCfg(SEED_BASE + 0x100 + seed, n, blocks, threads, intervals, words, int(round(shared_frac * 1000)),
                  int(round(atomic_frac * 1000)), int(round(write_frac * 1000)), values, len(sizes), int(sort),
                  int(unaligned), 0, sz, 0x10000000000)


def rnd_host(n: int, seed: int, **kw) -> np.ndarray:
    """Counter-based random trace (gen_common.h rnd_record): a C twin of sesagen.random_trace for large sweeps."""
    c = rnd_cfg(n, seed, **kw)
    out = np.zeros(n, REC_DTYPE)
    if n:
        _hostlib().gen_random_host(ctypes.byref(c), 0, n, out.ctypes.data)
    return out
