"""Host-side logic of key-range sharding on CPU, world_size 2 over gloo.

The CUDA kernels of the sharded search are tested on a GPU (virtual shards on
one device, tests/test_gpu_sharded.py).  Here, without a GPU, two processes run
the same PROTOCOL with torch.distributed (gloo) and the oracle standing in for
each shard's local search, and compare with the unsharded oracle:
  owner(q) = #(shard_max < q) over the non-empty shards (clamped to the last),
  all-to-all of counts, queries and results, global pos = shard base + rank,
  unpermute to the original order — including an empty shard and keys beyond
  every shard (they must come back END from the last non-empty shard).
Also: the NCCL unique id broadcast (package helper) reaches every rank intact,
and shard_plan covers [0, n) without gaps.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
import oracle


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _a2a(x, send_counts, recv_counts):
    out = torch.empty(sum(recv_counts), dtype=x.dtype)
    dist.all_to_all_single(out, x, recv_counts, send_counts)
    return out


def _worker(rank, world, port, case, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_sigmod_shahvaranij16_b200 as hbt
        uid = hbt.broadcast_unique_id()
        ids = [None] * world
        dist.all_gather_object(ids, uid)
        assert all(i == ids[0] for i in ids) and len(uid) == 128

        n = 20000
        allk = gen.stratified_keys(n, gen.stream_seed(4, gen.STREAM_K))
        allv = gen.values(n, 8, gen.stream_seed(4, gen.STREAM_V))
        lo, hi = hbt.shard_plan(n, world, rank)
        if case == "empty_first" and rank == 0:
            lo, hi = 0, 0
        if case == "empty_first" and rank == 1:
            lo = 0
        k, v = allk[lo:hi], allv[lo:hi]
        shard = oracle.ITree.from_pairs(k, v, 16, 8)
        meta = torch.tensor(np.array([len(k), k.min() if len(k) else 0, k.max() if len(k) else 0],
                                     dtype=np.uint64).view(np.int64))
        allmeta = [torch.empty(3, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(allmeta, meta)
        cnt = [int(m[0]) for m in allmeta]
        mx = [int(np.int64(m[2]).astype(np.uint64)) for m in allmeta]
        base = np.cumsum([0] + cnt)[:-1]
        table = [(mx[g], g) for g in range(world) if cnt[g]]

        rng = np.random.default_rng(rank)
        qs = np.concatenate([allk[rng.integers(0, n, 3000)],                       # hits anywhere
                             rng.integers(0, 2**64 - 1, 2000, dtype=np.uint64, endpoint=True),  # misses
                             np.array([0, 2**64 - 1, allk[0], allk[-1], allk[-1] + 1], np.uint64)])
        # route
        owner = np.array([table[min(sum(1 for m_, _ in table if m_ < int(x)), len(table) - 1)][1] for x in qs])
        order = np.argsort(owner, kind="stable")
        send_counts = [int((owner == g).sum()) for g in range(world)]
        rc = torch.empty(world, dtype=torch.int64)
        dist.all_to_all_single(rc, torch.tensor(send_counts, dtype=torch.int64))
        recv_counts = rc.tolist()
        rq = _a2a(torch.from_numpy(qs[order].view(np.int64)), send_counts, recv_counts).numpy().view(np.uint64)
        # local search + global position
        pf, vals = shard.search(rq)
        pos = pf & np.uint64(oracle.END)
        pf = np.where(pos != np.uint64(oracle.END), pf + np.uint64(base[rank]), pf)
        back_pf = _a2a(torch.from_numpy(pf.view(np.int64)), recv_counts, send_counts).numpy().view(np.uint64)
        back_v = _a2a(torch.from_numpy(vals.view(np.int64)), recv_counts, send_counts).numpy().view(np.uint64)
        out_pf = np.empty_like(back_pf)
        out_v = np.empty_like(back_v)
        out_pf[order] = back_pf
        out_v[order] = back_v
        # unsharded oracle
        full = oracle.ITree.from_pairs(allk, allv, 16, 8)
        epf, ev = full.search(qs)
        ok = bool(np.array_equal(out_pf, epf) and np.array_equal(out_v, ev))
        q.put((rank, ok, int((out_pf != epf).sum())))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("case", ["even", "empty_first"])
def test_sharded_protocol_two_ranks_gloo(case):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, case, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(ok for _, ok, _ in res), res


def test_shard_plan_covers_range():
    import paper_conf_sigmod_shahvaranij16_b200 as hbt
    for n, w in [(10, 3), (1 << 31, 8), (7, 8), (0, 2)]:
        spans = [hbt.shard_plan(n, w, r) for r in range(w)]
        assert spans[0][0] == 0 and spans[-1][1] == n
        assert all(spans[i][1] == spans[i + 1][0] for i in range(w - 1))


def _host_comm_worker(rank, world, port, q):
    import ctypes as C
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_sigmod_shahvaranij16_b200 as hbt
        comm = hbt.Comm.from_torch_host()
        # drive the callback the library calls, through its C function pointer
        send = (C.c_uint64 * 3)(100 + rank, 2**64 - 1 - rank, 7)
        recv = (C.c_uint64 * (3 * world))()
        rc = comm._fn(C.cast(send, C.c_void_p), C.cast(recv, C.c_void_p), C.sizeof(send), None)
        want = [x for r in range(world) for x in (100 + r, 2**64 - 1 - r, 7)]
        ok = rc == 0 and list(recv) == want and comm.nranks == world and comm.rank == rank
        comm.close()
        q.put((rank, ok))
    finally:
        dist.destroy_process_group()


def test_host_allgather_communicator_two_ranks_gloo():
    """hbt_comm_init_host + the torch.distributed all-gather callback that carries
    the sharded calls' host-side exchanges when NCCL is not used (exchange = 0)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_host_comm_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(ok for _, ok in res), res


def _shard_table_worker(rank, world, port, case, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_sigmod_shahvaranij16_b200 as hbt
        comm = hbt.Comm.from_torch_host()
        n = 3000
        allk = gen.stratified_keys(n, 11)
        lo, hi = hbt.shard_plan(n, world, rank)
        if case == "empty_middle" and rank == 1:
            lo = hi = 0
        if case == "overlap" and rank == 1:
            lo -= 5  # shares five keys with rank 0's range
        if case == "out_of_order":  # rank 0 holds the upper range
            lo, hi = hbt.shard_plan(n, world, world - 1 - rank)
        k = allk[lo:hi]
        try:
            counts, bases, maxima = comm.shard_table(len(k), int(k.min()) if len(k) else 0,
                                                     int(k.max()) if len(k) else 0)
            got = ("ok", counts.tolist(), bases.tolist(), maxima.tolist())
        except hbt.HBTError as e:
            got = ("err", e.code)
        comm.close()
        q.put((rank, got))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("case", ["even3", "empty_middle", "overlap", "out_of_order"])
def test_library_shard_table_gloo(case):
    """The library's own multi-process host path (hbt_comm_shard_table: all-gather of
    every rank's (n', min, max) through the host-callback communicator over gloo, key-order
    validation, bases and maxima of the routing table), no GPU needed."""
    world = 3 if case in ("even3", "empty_middle") else 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_shard_table_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    import paper_conf_sigmod_shahvaranij16_b200 as hbt
    if case in ("overlap", "out_of_order"):
        assert all(r == ("err", hbt.EINVAL) for r in res.values()), res
        return
    allk = gen.stratified_keys(3000, 11)
    spans = [hbt.shard_plan(3000, world, r) for r in range(world)]
    if case == "empty_middle":
        spans[1] = (0, 0)
    counts = [hi - lo for lo, hi in spans]
    bases = list(np.cumsum([0] + counts)[:-1])
    maxima = [int(allk[hi - 1]) if hi > lo else 0 for lo, hi in spans]
    for r in range(world):
        assert res[r] == ("ok", counts, bases, maxima), (r, res[r])
