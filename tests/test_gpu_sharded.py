"""GPU parity of the key-range-sharded search.

* Virtual shard groups on one B200 (hbt_search_sharded_local): G shards built
  from key-ordered disjoint ranges, empty shards included; every shard's query
  batch (hits anywhere, misses, edges, keys beyond every shard) must equal the
  UNSHARDED oracle bit for bit (global pos = rank).
* The NCCL path (hbt_comm_init + hbt_bulk_build_sharded + hbt_search_sharded)
  with one rank on one GPU.
"""
import numpy as np
import pytest
import torch

import gen
import oracle
from gpu_util import from_dev, to_dev

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def hbt():
    import paper_conf_sigmod_shahvaranij16_b200 as m
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    return m


def split_points(n, G, empty):
    cuts = [g * n // G for g in range(G + 1)]
    spans = [(cuts[g], cuts[g + 1]) for g in range(G)]
    for g in empty:  # make shard g empty, give its keys to a neighbour
        lo, hi = spans[g]
        spans[g] = (lo, lo)
        if g + 1 < G:
            spans[g + 1] = (lo, spans[g + 1][1])
        else:
            spans[g - 1] = (spans[g - 1][0], hi)
    return spans


def queries(allk, rng, m):
    n = len(allk)
    return np.concatenate([allk[rng.integers(0, n, m // 2)],
                           rng.integers(0, 2**64 - 1, m // 2, dtype=np.uint64, endpoint=True),
                           np.array([0, 2**64 - 1, allk[0], allk[-1], allk[-1] + 1, allk[0] - 1], np.uint64)])


@pytest.mark.parametrize("bucket", [0, 1])
@pytest.mark.parametrize("exchange", [0, 1])
@pytest.mark.parametrize("G,empty", [(1, []), (2, []), (3, [1]), (5, [0, 4]), (8, []), (8, [2, 3])])
def test_virtual_shards_match_unsharded_oracle(hbt, G, empty, exchange, bucket):
    """bucket = 1: the owner side searches its received queries through the bucketed
    path (item directory, global positions = shard base + local rank)."""
    n = 200000
    allk = gen.stratified_keys(n, gen.stream_seed(4, gen.STREAM_K))
    allv = gen.values(n, 8, gen.stream_seed(4, gen.STREAM_V))
    full = oracle.ITree.from_pairs(allk, allv, 16, 8)
    spans = split_points(n, G, empty)
    trees = []
    for lo, hi in spans:
        k, v = allk[lo:hi], allv[lo:hi]
        perm = np.random.default_rng(lo).permutation(len(k))  # unsorted within the shard is fine
        trees.append(hbt.Tree(to_dev(k[perm], 8), to_dev(v[perm], 8), fanout=16))
        trees[-1].set_param("exchange", exchange)
        if bucket:
            trees[-1].set_param("bucket", 1)
            trees[-1].set_param("bucket_slice", 4096)
    grp = hbt.LocalShardGroup(trees)
    rng = np.random.default_rng(G)
    for rep in range(2):  # second batch: larger, forces the windows to grow
        qs = [queries(allk, rng, (4000 + 1000 * g) * (1 + 3 * rep)) for g in range(G)]
        outs = grp.search([to_dev(q, 8) for q in qs])
        torch.cuda.synchronize()
        for q, (pf, v) in zip(qs, outs):
            epf, ev = full.search(q)
            assert np.array_equal(pf.cpu().numpy().view(np.uint64), epf)
            assert np.array_equal(from_dev(v, 8), ev)


def test_virtual_shards_reject_overlap(hbt):
    k = np.arange(1, 1001, dtype=np.uint64)
    a = hbt.Tree(to_dev(k[:600], 8), to_dev(k[:600], 8), fanout=8)
    b = hbt.Tree(to_dev(k[500:], 8), to_dev(k[500:], 8), fanout=8)
    with pytest.raises(hbt.HBTError):
        hbt.LocalShardGroup([a, b])


@pytest.mark.parametrize("exchange,g1_direct", [(0, 0), (0, 1), (1, 1)])
def test_nccl_path_one_rank(hbt, exchange, g1_direct):
    """One rank over the real communicator: exchange 0 = fused peer-memory path
    (IPC window export/all-gather, device barriers; g1_direct = 1 searches the single
    shard in place), 1 = NCCL send/recv."""
    uid = hbt.unique_id()
    comm = hbt.Comm(1, 0, uid)
    n = 100000
    allk = gen.stratified_keys(n, 7)
    allv = gen.values(n, 8, 9)
    t = hbt.ShardedTree(comm, to_dev(allk, 8), to_dev(allv, 8), fanout=16)
    t.set_param("exchange", exchange)
    t.set_param("g1_direct", g1_direct)
    o = oracle.ITree.from_pairs(allk, allv, 16, 8)
    for rep in range(3):
        q = queries(allk, np.random.default_rng(rep), 20000 * (1 + rep))
        pf, v = t.search(to_dev(q, 8))
        torch.cuda.synchronize()
        epf, ev = o.search(q)
        assert np.array_equal(pf.cpu().numpy().view(np.uint64), epf)
        assert np.array_equal(from_dev(v, 8), ev)
    t.close()
    comm.close()


@pytest.mark.parametrize("bucket,chunks,cnode", [(0, 1, 0), (1, 1, 0), (0, 2, 0), (1, 3, 0), (1, 4, 0), (1, 1, 1),
                                                (1, 2, 1)])
def test_fused_exchange_two_processes_one_gpu(bucket, chunks, cnode):
    """Two ranks (processes) on one GPU through the host-callback communicator:
    CUDA IPC windows, device flag barriers, count rows published by peer stores and
    queries put into the owner's window (exchange = 0); bucket = 1: the owner's
    bucketed gather stores results straight into the requester's window; chunks > 1:
    the batch is exchanged in chunks, the owner searching chunk c on a second stream
    while chunk c+1 is put; cnode = 1: a 2^21-key tree whose owner searches read the compact
    last-inner-level nodes.  Seven
    batches of growing and shrinking size per rank, each rank's results vs the
    unsharded oracle (tools/two_rank_one_gpu.py)."""
    import os
    import socket
    import subprocess
    import sys
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nproc-per-node", "2",
                        "--master-addr", "127.0.0.1", "--master-port", str(port),
                        os.path.join(root, "tools", "two_rank_one_gpu.py"), "0", str(bucket), str(chunks),
                        str(cnode)],
                       capture_output=True, text=True, timeout=600, cwd=root)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
    assert r.stdout.count("ok=True") == 2, r.stdout[-2000:]
