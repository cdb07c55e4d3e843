"""paper_conf_sigmod_shahvaranij16_b200 — B200-native HB+-tree lookups.

A thin ctypes binding of libhbt.so (include/hbt.h).  It only marshals
arguments: every step of build, search and update runs in the library's CUDA
kernels.  PyTorch provides device memory and streams.  There is no CPU
fallback: importing this package without the built library raises, and every
call on a machine without a CUDA device fails with HBTError.

    import torch, paper_conf_sigmod_shahvaranij16_b200 as hbt
    t = hbt.Tree(keys_u64_cuda, values_u64_cuda, fanout=16, layout="implicit")
    pos_found, values = t.search(queries_u64_cuda)

The result of a lookup (PAPER.md:190 node search): with Kd the
sorted distinct keys (last duplicate wins) and r = lower_bound(Kd, q),
found = r < n' and Kd[r] == q; pos = r for the implicit tree, the physical slot
(v*F + j)*P + s for the regular tree, or END; pos_found = pos | found << 63.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# HBT_LIB_ALT (A/B experiments only): another in-tree build of the same library
LIB_PATH = os.path.join(_HERE, os.environ.get("HBT_LIB_ALT", "libhbt.so"))

OK, EINVAL, ENOMEM, ECUDA, ENCCL, EUNSUPPORTED = 0, -1, -2, -3, -4, -5
IMPLICIT, REGULAR, KEY32, KEY64 = 0x0, 0x1, 0x00, 0x10
POS_END = 0x7FFFFFFFFFFFFFFF
FOUND_BIT = 0x8000000000000000
MAX_LEVELS = 32
SEG_INNER, SEG_LEAF, SEG_COUNT, SEG_LAST_KEYS, SEG_LAST_IDX = 0, 1, 2, 3, 4
SEG_UPPER_KEYS, SEG_UPPER_IDX, SEG_UPPER_REFS, SEG_CHAIN, SEG_INNER_IDX = 5, 6, 7, 8, 9
UPSERT, DELETE = 0, 1

EXPORTED = ["hbt_bulk_build", "hbt_search", "hbt_search_host", "hbt_bulk_update", "hbt_destroy",
            "hbt_info", "hbt_export", "hbt_set_param", "hbt_last_error", "hbt_version",
            "hbt_range", "hbt_comm_unique_id", "hbt_comm_init", "hbt_comm_init_host", "hbt_comm_destroy", "hbt_bulk_build_sharded",
            "hbt_search_sharded", "hbt_shard_local_init", "hbt_search_sharded_local", "hbt_last_phases",
            "hbt_set_leaf_placement", "hbt_get_leaf_placement", "hbt_versioned_create", "hbt_versioned_search",
            "hbt_versioned_update", "hbt_versioned_current", "hbt_versioned_destroy", "hbt_comm_shard_table"]


class HBTError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"hbt error {code}: {msg}")
        self.code = code


class _Out(C.Structure):
    _fields_ = [("pos_found", C.c_void_p), ("values", C.c_void_p)]


class _Batch(C.Structure):
    _fields_ = [("keys", C.c_void_p), ("values", C.c_void_p), ("ops", C.c_void_p), ("count", C.c_uint64)]


class _Phases(C.Structure):
    _fields_ = [("phases", C.c_uint32), ("launches", C.c_uint32), ("ms", C.c_float * 8)]


class _Info(C.Structure):
    _fields_ = [("layout", C.c_uint32), ("width", C.c_uint32), ("fanout", C.c_uint32),
                ("pairs_per_line", C.c_uint32), ("n_distinct", C.c_uint64), ("height", C.c_uint32),
                ("smem_levels", C.c_uint32), ("level_nodes", C.c_uint64 * MAX_LEVELS),
                ("leaf_lines", C.c_uint64), ("chain_len", C.c_uint64), ("inner_bytes", C.c_uint64),
                ("leaf_bytes", C.c_uint64)]


ALLGATHER_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_void_p, C.c_uint64, C.c_void_p)


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `make` or __graft_entry__.build() "
                          "(there is no CPU fallback)")
    L = C.CDLL(LIB_PATH)
    vp, u64, u32 = C.c_void_p, C.c_uint64, C.c_uint32
    L.hbt_bulk_build.argtypes = [vp, vp, u64, u32, u32, vp, C.POINTER(vp)]
    L.hbt_search.argtypes = [vp, vp, u64, _Out, vp]
    L.hbt_search_host.argtypes = [vp, vp, u64, vp, vp, vp]
    L.hbt_bulk_update.argtypes = [vp, C.POINTER(_Batch), vp]
    L.hbt_destroy.argtypes = [vp]
    L.hbt_info.argtypes = [vp, C.POINTER(_Info)]
    L.hbt_export.argtypes = [vp, u32, vp, u64, C.POINTER(u64)]
    L.hbt_set_param.argtypes = [vp, C.c_char_p, C.c_int64]
    L.hbt_range.argtypes = [vp, vp, vp, u64, u32, vp, vp, vp, vp]
    L.hbt_comm_unique_id.argtypes = [vp]
    L.hbt_comm_init.argtypes = [C.c_int, C.c_int, vp, C.POINTER(vp)]
    L.hbt_comm_init_host.argtypes = [C.c_int, C.c_int, ALLGATHER_FN, vp, C.POINTER(vp)]
    L.hbt_comm_destroy.argtypes = [vp]
    L.hbt_bulk_build_sharded.argtypes = [vp, vp, vp, u64, u32, u32, vp, C.POINTER(vp)]
    L.hbt_search_sharded.argtypes = [vp, vp, u64, _Out, vp]
    L.hbt_shard_local_init.argtypes = [C.POINTER(vp), C.c_int]
    L.hbt_search_sharded_local.argtypes = [C.POINTER(vp), C.c_int, C.POINTER(vp), C.POINTER(u64),
                                           C.POINTER(_Out), vp]
    L.hbt_last_phases.argtypes = [vp, vp]
    L.hbt_set_leaf_placement.argtypes = [vp, u32]
    L.hbt_get_leaf_placement.argtypes = [vp, C.POINTER(u32)]
    L.hbt_versioned_create.argtypes = [vp, C.POINTER(vp)]
    L.hbt_versioned_search.argtypes = [vp, vp, u64, _Out, vp, C.POINTER(u64)]
    L.hbt_versioned_update.argtypes = [vp, C.POINTER(_Batch), vp, C.POINTER(u64)]
    L.hbt_versioned_current.argtypes = [vp, C.POINTER(vp), C.POINTER(u64)]
    L.hbt_versioned_destroy.argtypes = [vp]
    L.hbt_comm_shard_table.argtypes = [vp, u64, u64, u64, vp, vp, vp]
    L.hbt_last_error.restype = C.c_char_p
    L.hbt_version.restype = C.c_char_p
    for f in ["hbt_bulk_build", "hbt_search", "hbt_search_host", "hbt_bulk_update", "hbt_destroy",
              "hbt_info", "hbt_export", "hbt_set_param", "hbt_range", "hbt_comm_unique_id", "hbt_comm_init",
              "hbt_comm_init_host",
              "hbt_comm_destroy", "hbt_bulk_build_sharded", "hbt_search_sharded", "hbt_shard_local_init",
              "hbt_search_sharded_local", "hbt_last_phases", "hbt_set_leaf_placement",
              "hbt_get_leaf_placement", "hbt_versioned_create", "hbt_versioned_search", "hbt_versioned_update",
              "hbt_versioned_current", "hbt_versioned_destroy", "hbt_comm_shard_table"]:
        getattr(L, f).restype = C.c_int
    return L


lib = _load()


def _check(rc):
    if rc != OK:
        raise HBTError(rc, lib.hbt_last_error().decode(errors="replace"))


def version() -> str:
    return lib.hbt_version().decode()


def _stream_ptr(stream):
    import torch
    if stream is None:  # torch's current stream on the current device (raw handle, no Stream object)
        return C.c_void_p(torch._C._cuda_getCurrentRawStream(torch._C._cuda_getDevice()))
    return C.c_void_p(stream.cuda_stream)


def _width(t) -> int:
    w = t.element_size()
    if w not in (4, 8):
        raise ValueError("keys/values must be 32- or 64-bit integer tensors")
    return w


def _dtype(width):
    import torch
    return torch.int32 if width == 4 else torch.int64


class Tree:
    """A device-resident HB+-tree (implicit or regular layout)."""

    @classmethod
    def _adopt(cls, handle, width, fanout, layout):
        import torch
        t = cls.__new__(cls)
        t._h, t.width, t.fanout, t.layout, t._torch = handle, width, fanout, layout, torch
        return t

    def __init__(self, keys, values, fanout: int = 16, layout: str = "implicit", stream=None):
        import torch
        if keys.numel() and not (keys.is_cuda and values.is_cuda):
            raise ValueError("keys/values must be CUDA tensors")
        if keys.numel() != values.numel() or keys.element_size() != values.element_size():
            raise ValueError("keys and values must have equal length and width")
        self.width = _width(keys)
        self.fanout = fanout
        self.layout = layout
        word = (REGULAR if layout == "regular" else IMPLICIT) | (KEY64 if self.width == 8 else KEY32)
        keys = keys.contiguous()
        values = values.contiguous()
        h = C.c_void_p()
        _check(lib.hbt_bulk_build(C.c_void_p(keys.data_ptr() if keys.numel() else 0),
                                  C.c_void_p(values.data_ptr() if values.numel() else 0),
                                  keys.numel(), fanout, word, _stream_ptr(stream), C.byref(h)))
        self._h = h
        self._torch = torch

    # -- lifetime
    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            lib.hbt_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @property
    def handle(self):
        return self._h

    # -- lookups
    def search(self, queries, out_pos=None, out_vals=None, stream=None):
        torch = self._torch
        if queries.element_size() != self.width:
            raise ValueError("query width differs from the tree's key width")
        queries = queries.contiguous()
        m = queries.numel()
        if out_pos is None:
            out_pos = torch.empty(m, dtype=torch.int64, device=queries.device)
        if out_vals is None:
            out_vals = torch.empty(m, dtype=_dtype(self.width), device=queries.device)
        if m:
            _check(lib.hbt_search(self._h, C.c_void_p(queries.data_ptr()), m,
                                  _Out(out_pos.data_ptr(), out_vals.data_ptr()), _stream_ptr(stream)))
        return out_pos, out_vals

    # -- placement of the L-segment (hbt_set_leaf_placement)
    def set_leaf_placement(self, where: str):
        """'device' (HBM) or 'host' (pinned host memory read by zero-copy loads)."""
        _check(lib.hbt_set_leaf_placement(self._h, {"device": 0, "host": 1}[where]))

    @property
    def leaf_placement(self) -> str:
        w = C.c_uint32()
        _check(lib.hbt_get_leaf_placement(self._h, C.byref(w)))
        return "host" if w.value else "device"

    def search_host(self, queries, out_pos, out_vals, stream=None):
        """End-to-end lookups from/to HOST buffers (numpy arrays or pinned CPU tensors)."""
        def ptr(a):
            return a.ctypes.data if isinstance(a, np.ndarray) else a.data_ptr()
        m = len(queries)
        _check(lib.hbt_search_host(self._h, C.c_void_p(ptr(queries)), m, C.c_void_p(ptr(out_pos)),
                                   C.c_void_p(ptr(out_vals)), _stream_ptr(stream)))
        return out_pos, out_vals

    def range(self, lo, hi, k: int, stream=None):
        """Up to k pairs with lo <= key <= hi per query.
        Returns (keys [m, k], values [m, k], count [m] int32)."""
        torch = self._torch
        lo, hi = lo.contiguous(), hi.contiguous()
        m = lo.numel()
        dt = _dtype(self.width)
        ok = torch.empty((m, k), dtype=dt, device=lo.device)
        ov = torch.empty((m, k), dtype=dt, device=lo.device)
        oc = torch.empty(m, dtype=torch.int32, device=lo.device)
        if m:
            _check(lib.hbt_range(self._h, C.c_void_p(lo.data_ptr()), C.c_void_p(hi.data_ptr()), m, k,
                                 C.c_void_p(ok.data_ptr()), C.c_void_p(ov.data_ptr()), C.c_void_p(oc.data_ptr()),
                                 _stream_ptr(stream)))
        return ok, ov, oc

    # -- updates
    def update(self, keys, values, ops, stream=None):
        keys, values, ops = keys.contiguous(), values.contiguous(), ops.contiguous()
        b = _Batch(keys.data_ptr() if keys.numel() else 0, values.data_ptr() if values.numel() else 0,
                   ops.data_ptr() if ops.numel() else 0, keys.numel())
        _check(lib.hbt_bulk_update(self._h, C.byref(b), _stream_ptr(stream)))

    # -- introspection
    def info(self) -> dict:
        i = _Info()
        _check(lib.hbt_info(self._h, C.byref(i)))
        d = {f: getattr(i, f) for f, _ in _Info._fields_ if f != "level_nodes"}
        nl = i.height if i.layout == IMPLICIT else max(i.height - 1, 0)
        d["level_nodes"] = [i.level_nodes[k] for k in range(nl)]
        return d

    def export(self, segment: int) -> np.ndarray:
        """Raw bytes of one device segment (uint8 numpy array)."""
        need = C.c_uint64(0)
        rc = lib.hbt_export(self._h, segment, C.c_void_p(1), 0, C.byref(need))
        if rc != OK and need.value == 0:
            _check(rc)
        buf = np.empty(max(need.value, 1), np.uint8)
        _check(lib.hbt_export(self._h, segment, C.c_void_p(buf.ctypes.data), buf.nbytes, C.byref(need)))
        return buf[: need.value]

    def set_param(self, name: str, value: int):
        _check(lib.hbt_set_param(self._h, name.encode(), int(value)))

    PHASES = ("count", "scan", "scatter", "search", "gather")

    def last_phases(self) -> dict:
        """Device ms of each phase of the last bucketed search (needs set_param("phase_timing", 1))."""
        p = _Phases()
        _check(lib.hbt_last_phases(self._h, C.byref(p)))
        d = {self.PHASES[i]: float(p.ms[i]) for i in range(p.phases)}
        d["launches"] = int(p.launches)
        return d

    def set_search_config(self, ctas_per_sm: int = 0, smem_mode=None):
        """Launch-shape knobs of the search (results never depend on them)."""
        self.set_param("ctas_per_sm", ctas_per_sm)
        if smem_mode is not None:
            self.set_param("smem_mode", smem_mode)


class VersionedTree:
    """Searches concurrent with bulk updates (hbt_versioned_*): every search reads the
    version current at its call; update() derives and publishes the next version
    while searches on other streams keep reading the previous one."""

    def __init__(self, tree: Tree):
        h = C.c_void_p()
        _check(lib.hbt_versioned_create(tree._h, C.byref(h)))
        tree._h = C.c_void_p()  # owned by the versioned handle now
        self._h, self.width, self._torch = h, tree.width, tree._torch

    def search(self, queries, out_pos=None, out_vals=None, stream=None):
        """Returns (pos_found, values, version)."""
        torch = self._torch
        queries = queries.contiguous()
        m = queries.numel()
        if out_pos is None:
            out_pos = torch.empty(m, dtype=torch.int64, device=queries.device)
        if out_vals is None:
            out_vals = torch.empty(m, dtype=_dtype(self.width), device=queries.device)
        ver = C.c_uint64(0)
        if m:
            _check(lib.hbt_versioned_search(self._h, C.c_void_p(queries.data_ptr()), m,
                                            _Out(out_pos.data_ptr(), out_vals.data_ptr()), _stream_ptr(stream),
                                            C.byref(ver)))
        return out_pos, out_vals, ver.value

    def update(self, keys, values, ops, stream=None) -> int:
        keys, values, ops = keys.contiguous(), values.contiguous(), ops.contiguous()
        b = _Batch(keys.data_ptr() if keys.numel() else 0, values.data_ptr() if values.numel() else 0,
                   ops.data_ptr() if ops.numel() else 0, keys.numel())
        ver = C.c_uint64(0)
        _check(lib.hbt_versioned_update(self._h, C.byref(b), _stream_ptr(stream), C.byref(ver)))
        return ver.value

    @property
    def version(self) -> int:
        t, ver = C.c_void_p(), C.c_uint64(0)
        _check(lib.hbt_versioned_current(self._h, C.byref(t), C.byref(ver)))
        return ver.value

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            lib.hbt_versioned_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ---------------------------------------------------------------- sharding


def unique_id() -> bytes:
    """ncclGetUniqueId (call on one rank and broadcast the 128 bytes)."""
    buf = C.create_string_buffer(128)
    _check(lib.hbt_comm_unique_id(buf))
    return buf.raw


def shard_plan(n_total: int, world: int, rank: int):
    """Contiguous key-index range [lo, hi) of shard `rank` when n_total generated
    keys (stratified, i.e. sorted by index, c4) are split over `world` ranks."""
    return rank * n_total // world, (rank + 1) * n_total // world


def broadcast_unique_id(group=None) -> bytes:
    """Rank 0 creates the NCCL id; every rank receives it (torch.distributed,
    any backend)."""
    import torch.distributed as dist
    obj = [unique_id() if dist.get_rank(group) == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]


class Comm:
    """An NCCL communicator owned by libhbt (one process per GPU)."""

    def __init__(self, nranks: int, rank: int, uid: bytes):
        h = C.c_void_p()
        _check(lib.hbt_comm_init(nranks, rank, C.c_char_p(uid), C.byref(h)))
        self._h, self.nranks, self.rank = h, nranks, rank

    @classmethod
    def from_torch(cls, group=None):
        import torch.distributed as dist
        uid = broadcast_unique_id(group)
        return cls(dist.get_world_size(group), dist.get_rank(group), uid)

    @classmethod
    def from_torch_host(cls, group=None):
        """A communicator without NCCL: the library's small host-side exchanges go
        through torch.distributed (any backend, e.g. gloo) all-gathers; the data
        path is the fused peer-memory exchange.  Allows several ranks per GPU."""
        import torch
        import torch.distributed as dist
        world, rank = dist.get_world_size(group), dist.get_rank(group)

        def allgather(send, recv, nbytes, ctx):
            try:
                mine = torch.frombuffer(bytearray(C.string_at(send, nbytes)), dtype=torch.uint8)
                out = [torch.empty(nbytes, dtype=torch.uint8) for _ in range(world)]
                dist.all_gather(out, mine, group=group)
                C.memmove(recv, torch.cat(out).numpy().tobytes(), nbytes * world)
                return 0
            except Exception:
                return 1

        self = cls.__new__(cls)
        self._fn = ALLGATHER_FN(allgather)  # keep the callback alive
        h = C.c_void_p()
        _check(lib.hbt_comm_init_host(world, rank, self._fn, None, C.byref(h)))
        self._h, self.nranks, self.rank = h, world, rank
        return self

    @classmethod
    def single(cls):
        """A one-rank communicator without NCCL (the host all-gather is a copy)."""
        self = cls.__new__(cls)

        def allgather(send, recv, nbytes, ctx):
            C.memmove(recv, send, nbytes)
            return 0

        self._fn = ALLGATHER_FN(allgather)
        h = C.c_void_p()
        _check(lib.hbt_comm_init_host(1, 0, self._fn, None, C.byref(h)))
        self._h, self.nranks, self.rank = h, 1, 0
        return self

    def shard_table(self, n_local: int, kmin: int, kmax: int):
        """Collective, host only: (counts, bases, maxima) of every rank's shard (uint64
        numpy arrays), the routing table of the key-range-sharded search."""
        arr = [np.zeros(self.nranks, np.uint64) for _ in range(3)]
        _check(lib.hbt_comm_shard_table(self._h, int(n_local), int(kmin), int(kmax),
                                        *[C.c_void_p(a.ctypes.data) for a in arr]))
        return tuple(arr)

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            lib.hbt_comm_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class ShardedTree(Tree):
    """This rank's shard of a key-range-sharded implicit tree (collective calls)."""

    def __init__(self, comm: Comm, keys, values, fanout: int = 16, stream=None):
        import torch
        self.width = _width(keys)
        self.fanout, self.layout, self._torch, self.comm = fanout, "implicit", torch, comm
        word = IMPLICIT | (KEY64 if self.width == 8 else KEY32)
        keys, values = keys.contiguous(), values.contiguous()
        h = C.c_void_p()
        _check(lib.hbt_bulk_build_sharded(comm._h, C.c_void_p(keys.data_ptr() if keys.numel() else 0),
                                          C.c_void_p(values.data_ptr() if values.numel() else 0), keys.numel(),
                                          fanout, word, _stream_ptr(stream), C.byref(h)))
        self._h = h

    def update(self, keys, values, ops, stream=None):
        raise HBTError(EUNSUPPORTED, "bulk update of a key-range shard is not supported "
                                     "(rebuild the sharded tree)")

    def search(self, queries, out_pos=None, out_vals=None, stream=None):
        torch = self._torch
        queries = queries.contiguous()
        m = queries.numel()
        if out_pos is None:
            out_pos = torch.empty(m, dtype=torch.int64, device="cuda")
        if out_vals is None:
            out_vals = torch.empty(m, dtype=_dtype(self.width), device="cuda")
        _check(lib.hbt_search_sharded(self._h, C.c_void_p(queries.data_ptr() if m else 0), m,
                                      _Out(out_pos.data_ptr() if m else 0, out_vals.data_ptr() if m else 0),
                                      _stream_ptr(stream)))
        return out_pos, out_vals


class LocalShardGroup:
    """G implicit trees on ONE device used as a key-range shard group: the same
    route / search / unpermute kernels as ShardedTree, the exchange being
    device-to-device copies."""

    def __init__(self, trees):
        self.trees = list(trees)
        G = len(self.trees)
        self._arr = (C.c_void_p * G)(*[t.handle.value for t in self.trees])
        _check(lib.hbt_shard_local_init(self._arr, G))

    def search(self, queries, stream=None):
        torch = self.trees[0]._torch
        G = len(self.trees)
        qs = [q.contiguous() for q in queries]
        outs = [(torch.empty(q.numel(), dtype=torch.int64, device="cuda"),
                 torch.empty(q.numel(), dtype=_dtype(self.trees[0].width), device="cuda")) for q in qs]
        qa = (C.c_void_p * G)(*[q.data_ptr() if q.numel() else 0 for q in qs])
        ma = (C.c_uint64 * G)(*[q.numel() for q in qs])
        oa = (_Out * G)(*[_Out(p.data_ptr() if p.numel() else 0, v.data_ptr() if v.numel() else 0) for p, v in outs])
        _check(lib.hbt_search_sharded_local(self._arr, G, qa, ma, oa, _stream_ptr(stream)))
        return outs


def unpack(pos_found, values, width: int):
    """Split device results into numpy (pos, found, value) with unsigned views."""
    pf = pos_found.cpu().numpy().view(np.uint64)
    vals = values.cpu().numpy().view(np.uint32 if width == 4 else np.uint64)
    return pf, vals
