"""Pins for the regular-tree oracle (oracle/oracle.c) — CPU only.

Fixed by things other than the oracle:
* found / value: numpy.searchsorted + a Python dict (the textbook map), also
  after batches of UPSERT/DELETE (reading R12);
* pos: key_at(pos) == the lower-bound successor read back from the oracle's
  leaf arrays, END iff no successor, all keys at distinct slots;
* the leaf partition: closed form Kd[floor(v n/nb) .. floor((v+1) n/nb)) with
  nb = ceil(n / floor(3B/4)) (reading R11);
* hand-worked golden tree + split in tests/golden/regular_u64_F4_n30.json
  (PAPER.md:134-138);
* structural invariants (sorted chain, counts <= B, separators = max key).
"""
import json
import os

import numpy as np
import pytest

import oracle
from test_oracle_implicit import END, expected, gen_keys, kmax, query_set

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def key_at(a, pos):
    F, P = a["F"], a["P"]
    v, rem = divmod(pos, F * P)
    return int(a["lkeys"][v][rem])


def check_positions(t, d, q, width):
    """pos points at the successor slot; END iff no successor; slots distinct."""
    a = t.arrays()
    pf, val = t.search(q)
    keys_ = np.array(sorted(d), dtype=np.uint64)
    for qq, p in zip(q.tolist(), pf.tolist()):
        r = int(np.searchsorted(keys_, np.uint64(qq), side="left"))
        pos = p & END
        if r == len(keys_):
            assert pos == END, (qq, p)
        else:
            assert pos != END, qq
            assert key_at(a, pos) == int(keys_[r]), (qq, pos)
    pf_all, _ = t.search(keys_)
    slots = (pf_all & np.uint64(END)).tolist()
    assert len(set(slots)) == len(slots)


def check_invariants(t, width):
    a = t.arrays()
    F, P, B, mx = a["F"], a["P"], a["B"], kmax(width)
    chain = a["chain"].tolist()
    prev_max = None
    for v in chain:
        c = int(a["lcount"][v])
        assert c <= B
        ks = a["lkeys"][v]
        assert (ks[c:] == mx).all() and (a["lvals"][v][c:] == 0).all()
        assert all(ks[i] < ks[i + 1] for i in range(c - 1))
        if c and prev_max is not None:
            assert int(ks[0]) > prev_max
        if c:
            prev_max = int(ks[c - 1])
        lines = max(1, -(-c // P))
        sep = a["lsep"][v]
        for j in range(F):
            if j < lines - 1:
                assert int(sep[j]) == int(ks[j * P + P - 1])
            else:
                assert int(sep[j]) == mx
    assert sum(int(a["lcount"][v]) for v in chain) == a["n"]
    # upper levels: sizes ceil(./F) up to one root
    c = len(chain)
    sizes = []
    while c > 1:
        c = -(-c // F)
        sizes.append(c)
    assert a["unodes"] == sizes


@pytest.mark.parametrize("width", [4, 8])
@pytest.mark.parametrize("F", [4, 8, 16, 32])
def test_regular_search_matches_lower_bound(width, F):
    P = 64 // (2 * width)
    rng = np.random.default_rng(77 * F + width)
    for n in [0, 1, 2, P, F * P, F * P + 1, 3 * F * P, 2000]:
        k, v = gen_keys(n, width, rng, dup=True, with_max=(n % 2 == 0))
        t = oracle.RTree.from_pairs(k, v, F, width)
        q = query_set(k, width, rng)
        pf, val = t.search(q)
        epf, evl = expected(k, v, q, width)
        assert np.array_equal(pf >> np.uint64(63), epf >> np.uint64(63)), (n, F)
        assert np.array_equal(val, evl), (n, F)
        d = dict(zip(k.tolist(), v.tolist()))
        check_positions(t, d, q, width)
        check_invariants(t, width)


@pytest.mark.parametrize("width,F", [(8, 32), (4, 32), (8, 8)])
def test_regular_build_partition_closed_form(width, F):
    rng = np.random.default_rng(5)
    k, v = gen_keys(5000, width, rng)
    Kd, Vd = oracle.dedupe(k, v)
    t = oracle.RTree(Kd, Vd, F, width)
    a = t.arrays()
    P = 64 // (2 * width)
    B = F * P
    b = (3 * B) // 4
    n = len(Kd)
    nb = -(-n // b)
    assert a["pool"] == nb and a["chain"].tolist() == list(range(nb))
    for vv in range(nb):
        lo, hi = vv * n // nb, (vv + 1) * n // nb
        assert a["lcount"][vv] == hi - lo
        assert a["lkeys"][vv][: hi - lo].tolist() == Kd[lo:hi].tolist()
        assert a["lvals"][vv][: hi - lo].tolist() == Vd[lo:hi].tolist()


def test_regular_golden():
    g = json.load(open(os.path.join(GOLDEN, "regular_u64_F4_n30.json")))
    t = oracle.RTree.from_pairs(np.array(g["keys"], np.uint64), np.array(g["values"], np.uint64),
                                g["fanout"], g["width"])

    def check(spec, qs):
        a = t.arrays()
        assert a["pool"] == spec["pool"]
        assert a["lcount"].tolist() == spec["lcount"]
        assert a["chain"].tolist() == spec["chain"]
        assert a["ukeys"].tolist() == spec["ukeys"]
        assert a["urefs"].tolist() == spec["urefs"]
        if "lsep" in spec:
            assert a["lsep"].tolist() == spec["lsep"]
        q = np.array([x["q"] for x in qs], np.uint64)
        pf, val = t.search(q)
        for x, p, vv in zip(qs, pf.tolist(), val.tolist()):
            want = END if x["pos"] == "END" else x["pos"]
            assert (p & END) == want, x
            assert bool(p >> 63) == x["found"], x
            assert vv == x["value"], x

    check(g, g["queries"])
    u = g["update"]
    t.update(np.array(u["keys"], np.uint64), np.array(u["values"], np.uint64), np.array(u["ops"], np.uint8))
    check(u, u["queries"])


@pytest.mark.parametrize("width", [4, 8])
@pytest.mark.parametrize("F", [4, 8])
def test_regular_update_vs_dict(width, F):
    """Random UPSERT/DELETE batches on tiny fanouts force splits, removals and
    the empty tree (reading R11/R12)."""
    rng = np.random.default_rng(1234 + F + width)
    mx = kmax(width)
    for trial in range(12):
        n = int(rng.integers(0, 400))
        k, v = gen_keys(n, width, rng, dup=True)
        t = oracle.RTree.from_pairs(k, v, F, width)
        d = dict(zip(k.tolist(), v.tolist()))
        for batch in range(4):
            nops = int(rng.integers(0, 300))
            live = np.array(list(d) or [0], np.uint64)
            pick = live[rng.integers(0, len(live), nops)]
            fresh = rng.integers(0, mx, nops, dtype=np.uint64, endpoint=True)
            ok = np.where(rng.random(nops) < 0.5, pick, fresh).astype(np.uint64)
            ov = rng.integers(0, mx, nops, dtype=np.uint64, endpoint=True)
            p_del = [0.2, 0.5, 0.95, 1.0][batch]
            op = (rng.random(nops) < p_del).astype(np.uint8)
            if batch == 3:  # delete everything that is left
                ok = np.array(list(d), np.uint64)
                ov = np.zeros(len(ok), np.uint64)
                op = np.ones(len(ok), np.uint8)
            t.update(ok, ov, op)
            for a_, b_, o_ in zip(ok.tolist(), ov.tolist(), op.tolist()):
                if o_ == 0:
                    d[a_] = b_
                else:
                    d.pop(a_, None)
            q = query_set(np.array(list(d) or [0], np.uint64), width, rng, 100)
            pf, val = t.search(q)
            keys_ = np.array(list(d.keys()), np.uint64)
            vals_ = np.array(list(d.values()), np.uint64)
            epf, evl = expected(keys_, vals_, q, width)
            assert np.array_equal(pf >> np.uint64(63), epf >> np.uint64(63))
            assert np.array_equal(val, evl)
            check_positions(t, d, q, width)
            check_invariants(t, width)
            if batch == 3:
                a = t.arrays()
                assert a["n"] == 0 and a["pool"] == 1 and a["chain"].tolist() == [0]


def test_regular_split_appends_pool_indices_in_key_order():
    """Two leaves overflow in one batch: new indices are appended in key order."""
    width, F = 8, 4
    keys_ = np.arange(2, 62, 2, dtype=np.uint64)       # golden tree: 3 leaves of 10
    t = oracle.RTree(keys_, keys_, F, width)
    ins = np.array([1, 3, 5, 7, 9, 11, 13, 43, 45, 47, 49, 51, 53, 55], np.uint64)
    t.update(ins, ins, np.zeros(len(ins), np.uint8))
    a = t.arrays()
    # leaf 0 (2..20 + 7) and leaf 2 (42..60 + 7) split; leaf 0's right part gets 3, leaf 2's gets 4
    assert a["chain"].tolist() == [0, 3, 1, 2, 4]
    assert a["pool"] == 5
    assert a["lcount"].tolist() == [8, 10, 8, 9, 9]


@pytest.mark.parametrize("layout", ["implicit", "regular"])
@pytest.mark.parametrize("width", [4, 8])
def test_range_scan_matches_sorted_slices(layout, width):
    """Range scan = the first up-to-k sorted keys in [lo, hi]: pinned by
    numpy.searchsorted + slicing of the sorted key array (and a dict for values),
    also after updates that split / remove leaves (regular: chain traversal)."""
    rng = np.random.default_rng(width + (layout == "regular"))
    mx = kmax(width)
    k, v = gen_keys(3000, width, rng, dup=True)
    T = oracle.ITree if layout == "implicit" else oracle.RTree
    t = T.from_pairs(k, v, 4, width)
    d = dict(zip(k.tolist(), v.tolist()))
    if layout == "regular":  # make the chain non-trivial: splits and removals
        ins = rng.integers(0, mx, 2000, dtype=np.uint64, endpoint=True)
        dels = k[:1000]
        ok = np.concatenate([ins, dels])
        ov = rng.integers(0, mx, len(ok), dtype=np.uint64, endpoint=True)
        op = np.concatenate([np.zeros(len(ins), np.uint8), np.ones(len(dels), np.uint8)])
        t.update(ok, ov, op)
        for a_, b_, o_ in zip(ok.tolist(), ov.tolist(), op.tolist()):
            if o_ == 0:
                d[a_] = b_
            else:
                d.pop(a_, None)
    Kd = np.array(sorted(d), np.uint64)
    lo = query_set(Kd[:200], width, rng, 300)
    span = rng.integers(0, mx // 200, len(lo), dtype=np.uint64)
    hi = np.minimum(lo.astype(object) + span.astype(object), mx).astype(np.uint64)
    hi[:10] = mx
    for kk in (1, 5, 32):
        ok_, ov_, oc = t.range(lo, hi, kk)
        for x in range(len(lo)):
            a = int(np.searchsorted(Kd, lo[x], side="left"))
            b = int(np.searchsorted(Kd, hi[x], side="right"))
            want = Kd[a:min(b, a + kk)]
            assert oc[x] == len(want), (x, kk)
            assert ok_[x, : len(want)].tolist() == want.tolist()
            assert ov_[x, : len(want)].tolist() == [d[int(z)] for z in want.tolist()]
            assert (ok_[x, len(want):] == mx).all() and (ov_[x, len(want):] == 0).all()
