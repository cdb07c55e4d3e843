"""Two processes on ONE GPU running the sharded search through the real
communicator: exercises CUDA IPC window export/import, the device-side flag
barriers and the peer-store exchange (exchange=0) or NCCL send/recv (1), and
checks every rank's results against the unsharded oracle.  Launch with
torchrun --nproc-per-node 2 (gloo for the host-side plumbing)."""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gen  # noqa: E402
import oracle  # noqa: E402  (test tool: checks the results)
import paper_conf_sigmod_shahvaranij16_b200 as hbt  # noqa: E402


def main():
    exchange = int(sys.argv[1]) if len(sys.argv) > 1 else 0
    bucket = int(sys.argv[2]) if len(sys.argv) > 2 else 2  # 1: owner search bucketed (fused remote gather)
    chunks = int(sys.argv[3]) if len(sys.argv) > 3 else 2  # exchange chunks (put of c+1 overlaps search of c)
    # 1: a larger tree with one bucket per shard, so the owner's item directory sits on the last
    # inner level and the search reads its compact nodes (item_cnode forced)
    cnode = int(sys.argv[4]) if len(sys.argv) > 4 else 0
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    torch.cuda.set_device(0)
    comm = hbt.Comm.from_torch_host() if exchange == 0 else hbt.Comm.from_torch()
    n = 1 << 21 if cnode else 200000
    allk = gen.stratified_keys(n, 7)
    allv = gen.values(n, 8, 9)
    lo, hi = hbt.shard_plan(n, world, rank)
    k = torch.from_numpy(allk[lo:hi].view(np.int64)).cuda()
    v = torch.from_numpy(allv[lo:hi].view(np.int64)).cuda()
    t = hbt.ShardedTree(comm, k, v, fanout=16)
    t.set_param("exchange", exchange)
    t.set_param("bucket", bucket)
    if exchange == 0:
        t.set_param("exchange_chunks", chunks)
    if bucket == 1:
        t.set_param("bucket_slice", 1 << 30 if cnode else 4096)
    if cnode:
        t.set_param("l2_levels_bytes", 4096)
        t.set_param("item_cnode", 2)
    full = oracle.ITree.from_pairs(allk, allv, 16, 8)
    ok = True
    # batch sizes grow (window regrowth, a collective re-export) and shrink; several
    # batches in a row exercise the device-side count publication (matrix parity)
    for rep, mq in enumerate([30000, 90000, 20000, 250000, 10000, 400000, 5000]):
        rng = np.random.default_rng(100 * rank + rep)
        q = np.concatenate([allk[rng.integers(0, n, mq * (rank + 1))],
                            rng.integers(0, 2**64 - 1, 5000, dtype=np.uint64, endpoint=True)])
        pf, vals = t.search(torch.from_numpy(q.view(np.int64)).cuda())
        torch.cuda.synchronize()
        epf, ev = full.search(q)
        ok &= np.array_equal(pf.cpu().numpy().view(np.uint64), epf)
        ok &= np.array_equal(vals.cpu().numpy().view(np.uint64), ev)
    print(f"rank {rank} exchange {exchange} ok={ok}", flush=True)
    t.close()
    comm.close()
    dist.destroy_process_group()
    sys.exit(0 if ok else 1)


if __name__ == "__main__":
    main()
