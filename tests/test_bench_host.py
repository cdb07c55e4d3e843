"""Host-side logic of bench.py (no GPU): the workload description both arms print, the
--gpus re-launch under torch.distributed.run, and the c4 oracle sample behind
cpu_baseline / --impl reference (its answers against the stratified closed form)."""
import sys
import types

import numpy as np

import bench
import gen
import oracle


def _args(**kw):
    a = dict(gpus=1, steps=3, warmup=3, impl="hbt", config="c4", queries=None, range_k=0, exchange=None)
    a.update(kw)
    return types.SimpleNamespace(**a)


def test_config_is_the_same_for_both_arms_and_names_the_workload():
    for world in (1, 2, 8):
        a = bench.bench_config(_args(), world)
        b = bench.bench_config(_args(impl="reference"), world)
        assert a == b
        assert a["workload"].startswith("c4")
        assert a["n_keys"] == 1 << 31 and a["queries_total"] == 1 << 28
        assert a["queries_per_rank"] == (1 << 28) // world
        assert ("sharded" in a["parallelism"]) == (world > 1)
    c2 = bench.bench_config(_args(config="c2"), 4)
    assert c2["queries_total"] == 4 * (1 << 24) and "replicated" in c2["parallelism"]


def test_gpus_flag_relaunches_under_torchrun(monkeypatch):
    calls = []
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    monkeypatch.setattr(bench.subprocess, "call", lambda cmd: calls.append(cmd) or 0)
    monkeypatch.setattr(sys, "argv", ["bench.py", "--gpus", "4", "--steps", "2"])
    assert bench.maybe_spawn(_args(gpus=4)) == 0
    cmd = calls[0]
    assert cmd[1:3] == ["-m", "torch.distributed.run"]
    assert "--nproc-per-node=4" in cmd and "--master-addr=127.0.0.1" in cmd
    assert cmd[-3:] == ["--gpus", "4", "--steps", "2"][-3:]
    # inside torchrun, one GPU, or the reference arm: no re-launch
    monkeypatch.setenv("WORLD_SIZE", "4")
    assert bench.maybe_spawn(_args(gpus=4)) is None
    monkeypatch.delenv("WORLD_SIZE")
    assert bench.maybe_spawn(_args(gpus=1)) is None
    assert bench.maybe_spawn(_args(gpus=4, impl="reference")) is None


def test_c4_oracle_sample_matches_the_stratified_closed_form(monkeypatch):
    monkeypatch.setattr(bench, "C4_SLICE", 1 << 14)
    c, k, v, q = bench.c4_oracle_sample(5000)
    assert np.all(np.diff(k.astype(np.uint64)) > 0)  # a sorted contiguous slice of the c4 keys
    sk = gen.stream_seed(4, gen.STREAM_K)
    sv = gen.stream_seed(4, gen.STREAM_V)
    t = oracle.ITree.from_pairs(k, v, c["fanout"], 8)
    pf, val = t.search(q)
    i = q >> np.uint64(33)                    # closed form: every query is a hit on K_i
    assert np.array_equal(pf, i | np.uint64(1 << 63))
    assert np.array_equal(val, gen.mix64(i ^ np.uint64(sv)))
    assert np.array_equal(k[i.astype(np.int64)], q)
    assert sk != sv


def test_c5_splits_its_batch_over_the_replicas():
    """BASELINE configs[4] 'query-batch split at 8 GPUs': c5's 2^26 queries are divided
    among the ranks (strong scaling); c1-c3 keep a full batch per rank (weak)."""
    for world in (1, 2, 8):
        c5 = bench.bench_config(_args(config="c5"), world)
        assert c5["queries_total"] == 1 << 26 and c5["queries_per_rank"] == (1 << 26) // world
        c3 = bench.bench_config(_args(config="c3"), world)
        assert c3["queries_total"] == world * (1 << 26) and c3["queries_per_rank"] == 1 << 26


def test_roofline_model_bytes_of_the_c4_item_search():
    """tools/roofline.py's bucketed model as bench.py calls it (the line's algorithmic bytes,
    DESIGN.md §6): query 8 + record 16 + distinct leaf lines touched by 2^28 uniform queries
    (64 B each) + one pass over the directory keys at leaf-line granularity (8 B per line):
    90.4 B/q for the c4 geometry."""
    from tools import roofline
    info = {"width": 8, "fanout": 16, "layout": 0, "n_distinct": 1 << 31, "height": 8, "smem_levels": 4,
            "level_nodes": [1, 2, 32, 512, 8192, 131072, 2097152, 33554432], "leaf_lines": 1 << 29}
    m = 1 << 28
    b = roofline.model_bucketed(info, m)["hbm_bytes_per_query"]
    lines = (1 << 29) * (1 - np.exp(-m / (1 << 29))) * 64 / m
    assert abs(b - (24 + lines + (1 << 29) * 8 / m)) < 1e-6, b
    assert abs(b - 90.36) < 0.01
