"""oracle — TEST INFRASTRUCTURE ONLY.

ctypes wrapper around oracle/oracle.c, the plain CPU oracle of the HB+-tree
(§4.1, §5.2-5.3, §5.6).  Only tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / --impl reference legs may import this package; the
product package paper_conf_sigmod_shahvaranij16_b200 never does.

Keys and values cross this wrapper as uint64 numpy arrays (u32 keys are
zero-extended); `width` (4 or 8) selects the key width's MAX = 2^(8*width)-1.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_HDR = os.path.join(_HERE, "oracle.h")
_LIB = os.path.join(_HERE, "liboracle.so")

END = 0x7FFFFFFFFFFFFFFF
FOUND = 0x8000000000000000
MAXLEV = 64


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain C11 + OpenMP)."""
    stale = (not os.path.exists(_LIB)) or max(os.path.getmtime(_SRC), os.path.getmtime(_HDR)) > os.path.getmtime(_LIB)
    if force or stale:
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-std=c11", "-O2", "-fPIC", "-shared", "-fopenmp",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


class _ITree(C.Structure):
    _fields_ = [("kmax", C.c_uint64), ("F", C.c_uint32), ("P", C.c_uint32), ("n", C.c_uint64),
                ("H", C.c_uint32), ("L0", C.c_uint64),
                ("nodes", C.c_uint64 * MAXLEV), ("offset", C.c_uint64 * (MAXLEV + 1)),
                ("inner", C.POINTER(C.c_uint64)), ("lkeys", C.POINTER(C.c_uint64)),
                ("lvals", C.POINTER(C.c_uint64))]


class _RTree(C.Structure):
    _fields_ = [("kmax", C.c_uint64), ("F", C.c_uint32), ("P", C.c_uint32), ("kpl", C.c_uint32),
                ("NI", C.c_uint32), ("B", C.c_uint32), ("b", C.c_uint32), ("n", C.c_uint64),
                ("pool", C.c_uint64), ("cap", C.c_uint64),
                ("lkeys", C.POINTER(C.c_uint64)), ("lvals", C.POINTER(C.c_uint64)),
                ("lcount", C.POINTER(C.c_uint32)), ("lsep", C.POINTER(C.c_uint64)),
                ("lidx", C.POINTER(C.c_uint64)), ("nchain", C.c_uint64),
                ("chain", C.POINTER(C.c_uint64)), ("U", C.c_uint32),
                ("unodes", C.c_uint64 * MAXLEV), ("uoff", C.c_uint64 * (MAXLEV + 1)),
                ("ukeys", C.POINTER(C.c_uint64)), ("uidx", C.POINTER(C.c_uint64)),
                ("urefs", C.POINTER(C.c_uint32))]


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        u64p = C.POINTER(C.c_uint64)
        L.orc_dedupe.restype = C.c_uint64
        L.orc_dedupe.argtypes = [u64p, u64p, C.c_uint64, u64p, u64p]
        L.orc_itree_build.restype = C.POINTER(_ITree)
        L.orc_itree_build.argtypes = [u64p, u64p, C.c_uint64, C.c_uint32, C.c_uint32]
        L.orc_itree_free.argtypes = [C.POINTER(_ITree)]
        L.orc_itree_search.argtypes = [C.POINTER(_ITree), u64p, C.c_uint64, u64p, u64p, C.c_int]
        L.orc_itree_update.restype = C.POINTER(_ITree)
        L.orc_itree_update.argtypes = [C.POINTER(_ITree), u64p, u64p, C.POINTER(C.c_uint8), C.c_uint64]
        L.orc_rtree_build.restype = C.POINTER(_RTree)
        L.orc_rtree_build.argtypes = [u64p, u64p, C.c_uint64, C.c_uint32, C.c_uint32]
        L.orc_rtree_free.argtypes = [C.POINTER(_RTree)]
        L.orc_rtree_search.argtypes = [C.POINTER(_RTree), u64p, C.c_uint64, u64p, u64p, C.c_int]
        L.orc_rtree_update.restype = C.c_int
        L.orc_rtree_update.argtypes = [C.POINTER(_RTree), u64p, u64p, C.POINTER(C.c_uint8), C.c_uint64]
        L.orc_lower_bound.argtypes = [u64p, u64p, C.c_uint64, u64p, C.c_uint64, u64p, u64p, C.c_int]
        u32p = C.POINTER(C.c_uint32)
        L.orc_itree_range.argtypes = [C.POINTER(_ITree), u64p, u64p, C.c_uint64, C.c_uint32, u64p, u64p, u32p]
        L.orc_rtree_range.argtypes = [C.POINTER(_RTree), u64p, u64p, C.c_uint64, C.c_uint32, u64p, u64p, u32p]
        _lib = L
    return _lib


def _p64(a):
    return a.ctypes.data_as(C.POINTER(C.c_uint64))


def _as_u64(a):
    return np.ascontiguousarray(np.asarray(a).astype(np.uint64, copy=False))


def _copy(ptr, count, dtype=np.uint64):
    if count == 0:
        return np.zeros(0, dtype=dtype)
    return np.ctypeslib.as_array(ptr, shape=(count,)).astype(dtype, copy=True)


def default_threads() -> int:
    return os.cpu_count() or 1


def dedupe(keys, vals):
    """Stable sort by unsigned key; duplicates collapse to the last occurrence."""
    k, v = _as_u64(keys), _as_u64(vals)
    ok = np.empty(len(k), np.uint64)
    ov = np.empty(len(k), np.uint64)
    m = lib().orc_dedupe(_p64(k), _p64(v), len(k), _p64(ok), _p64(ov))
    return ok[:m].copy(), ov[:m].copy()


def lower_bound(Kd, Vd, q, nthreads: int = 1):
    Kd, Vd, q = _as_u64(Kd), _as_u64(Vd), _as_u64(q)
    pf = np.empty(len(q), np.uint64)
    vals = np.empty(len(q), np.uint64)
    lib().orc_lower_bound(_p64(Kd), _p64(Vd), len(Kd), _p64(q), len(q), _p64(pf), _p64(vals), nthreads)
    return pf, vals


def _range(fn, ptr, lo, hi, k):
    lo, hi = _as_u64(lo), _as_u64(hi)
    m = len(lo)
    ok = np.empty(m * k, np.uint64)
    ov = np.empty(m * k, np.uint64)
    oc = np.empty(m, np.uint32)
    fn(ptr, _p64(lo), _p64(hi), m, k, _p64(ok), _p64(ov), oc.ctypes.data_as(C.POINTER(C.c_uint32)))
    return ok.reshape(m, k), ov.reshape(m, k), oc


class ITree:
    """Implicit tree: build from sorted distinct (Kd, Vd)."""

    def __init__(self, Kd, Vd, fanout: int, width: int, _ptr=None):
        self.width = width
        if _ptr is None:
            Kd, Vd = _as_u64(Kd), _as_u64(Vd)
            _ptr = lib().orc_itree_build(_p64(Kd), _p64(Vd), len(Kd), fanout, width)
        self._p = _ptr

    @classmethod
    def from_pairs(cls, keys, vals, fanout, width):
        Kd, Vd = dedupe(keys, vals)
        return cls(Kd, Vd, fanout, width)

    def __del__(self):
        if getattr(self, "_p", None) is not None and _lib is not None:
            _lib.orc_itree_free(self._p)
            self._p = None

    @property
    def s(self):
        return self._p.contents

    def search(self, q, nthreads: int = 1):
        q = _as_u64(q)
        pf = np.empty(len(q), np.uint64)
        vals = np.empty(len(q), np.uint64)
        lib().orc_itree_search(self._p, _p64(q), len(q), _p64(pf), _p64(vals), nthreads)
        return pf, vals

    def range(self, lo, hi, k):
        """Up to k pairs with lo <= key <= hi per query."""
        return _range(lib().orc_itree_range, self._p, lo, hi, k)

    def update(self, keys, vals, ops):
        k, v = _as_u64(keys), _as_u64(vals)
        o = np.ascontiguousarray(np.asarray(ops, dtype=np.uint8))
        p = lib().orc_itree_update(self._p, _p64(k), _p64(v), o.ctypes.data_as(C.POINTER(C.c_uint8)), len(k))
        return ITree(None, None, self.s.F, self.width, _ptr=p)

    def arrays(self):
        s = self.s
        H = s.H
        total = s.offset[H]
        return dict(F=s.F, P=s.P, n=s.n, H=H, L0=s.L0, kmax=s.kmax,
                    nodes=[s.nodes[d] for d in range(H)],
                    offset=[s.offset[d] for d in range(H + 1)],
                    inner=_copy(s.inner, total * s.F).reshape(total, s.F),
                    lkeys=_copy(s.lkeys, s.L0 * s.P).reshape(s.L0, s.P),
                    lvals=_copy(s.lvals, s.L0 * s.P).reshape(s.L0, s.P))


class RTree:
    """Regular tree, generalised to fanout F."""

    def __init__(self, Kd, Vd, fanout: int, width: int):
        self.width = width
        Kd, Vd = _as_u64(Kd), _as_u64(Vd)
        self._p = lib().orc_rtree_build(_p64(Kd), _p64(Vd), len(Kd), fanout, width)

    @classmethod
    def from_pairs(cls, keys, vals, fanout, width):
        Kd, Vd = dedupe(keys, vals)
        return cls(Kd, Vd, fanout, width)

    def __del__(self):
        if getattr(self, "_p", None) is not None and _lib is not None:
            _lib.orc_rtree_free(self._p)
            self._p = None

    @property
    def s(self):
        return self._p.contents

    def search(self, q, nthreads: int = 1):
        q = _as_u64(q)
        pf = np.empty(len(q), np.uint64)
        vals = np.empty(len(q), np.uint64)
        lib().orc_rtree_search(self._p, _p64(q), len(q), _p64(pf), _p64(vals), nthreads)
        return pf, vals

    def range(self, lo, hi, k):
        """Up to k pairs with lo <= key <= hi per query, through the chain."""
        return _range(lib().orc_rtree_range, self._p, lo, hi, k)

    def update(self, keys, vals, ops):
        k, v = _as_u64(keys), _as_u64(vals)
        o = np.ascontiguousarray(np.asarray(ops, dtype=np.uint8))
        rc = lib().orc_rtree_update(self._p, _p64(k), _p64(v), o.ctypes.data_as(C.POINTER(C.c_uint8)), len(k))
        if rc != 0:
            raise RuntimeError("oracle regular update: non-monotone routing")

    def arrays(self):
        s = self.s
        F, P, NI, pool, U = s.F, s.P, s.NI, s.pool, s.U
        total = s.uoff[U]
        return dict(F=F, P=P, NI=NI, kpl=s.kpl, B=s.B, b=s.b, n=s.n, kmax=s.kmax, pool=pool, U=U,
                    unodes=[s.unodes[u] for u in range(U)], uoff=[s.uoff[u] for u in range(U + 1)],
                    lkeys=_copy(s.lkeys, pool * F * P).reshape(pool, F * P),
                    lvals=_copy(s.lvals, pool * F * P).reshape(pool, F * P),
                    lcount=_copy(s.lcount, pool, np.uint32),
                    lsep=_copy(s.lsep, pool * F).reshape(pool, F),
                    lidx=_copy(s.lidx, pool * NI).reshape(pool, NI),
                    chain=_copy(s.chain, s.nchain),
                    ukeys=_copy(s.ukeys, total * F).reshape(total, F),
                    uidx=_copy(s.uidx, total * NI).reshape(total, NI),
                    urefs=_copy(s.urefs, total * F, np.uint32).reshape(total, F))
