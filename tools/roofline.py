"""Roofline model for batched B+-tree lookups, used by bench.py.

Algorithmic bytes per query (what the method must move):
  I/O      2S + 8          (query in; value + pos|found out)
  per inner level: implicit nodes wider than 32 B = index sector + one key
                   sector (64 B; the paper's index line), else F*S;
                            regular index sector 32 + key line 64 + ref sector 32
                            (last level: 32 + 64)
  leaf     key sector 32 + value sector 32 (the value sector only when found)
Only bytes that miss the L2 count toward HBM.  The cache model is an ideal
static cache: the L2 capacity holds the byte ranges with the highest access
probability per byte (levels top-down for uniform queries; the Zipf pmf can
be supplied per leaf line).  Levels pinned in shared memory cost nothing.
"""
from __future__ import annotations

import numpy as np


def _sect(b):
    return ((b + 31) // 32) * 32


def implicit_tiers(info, hit_rate=1.0, smem_levels=None):
    """(total_bytes, bytes_per_query) tiers of the implicit tree below the
    shared-memory levels, for uniform queries (every node of a level equally
    likely).  A node wider than one 32 B sector is read as its index sector plus
    ONE key sector (the search kernel's access pattern); narrower nodes whole."""
    S, F = info["width"], info["fanout"]
    SL = info["smem_levels"] if smem_levels is None else smem_levels
    node = F * S
    tiers = []
    for d, nodes in enumerate(info["level_nodes"]):
        if d < SL:
            continue
        if node > 32:
            idx_stride = max(16, (node // 32) * S)
            tiers.append((nodes * idx_stride, 32.0))   # index sector
            tiers.append((nodes * node, 32.0))         # one key sector
        else:
            tiers.append((nodes * _sect(node), float(_sect(node))))
    L0 = info["leaf_lines"]
    tiers.append((L0 * 32, 32.0))             # key half of the leaf line
    tiers.append((L0 * 32, 32.0 * hit_rate))  # value half (needed when found)
    return tiers


def regular_tiers(info, hit_rate=1.0, smem_levels=None):
    S, F = info["width"], info["fanout"]
    kpl = 64 // S
    SL = info["smem_levels"] if smem_levels is None else smem_levels
    per_upper = (32 if F > kpl else 0) + min(64, F * S) + 32
    per_last = (32 if F > kpl else 0) + min(64, F * S)
    levels = list(reversed(info["level_nodes"]))  # root first
    tiers = []
    node_bytes = (32 if F > kpl else 0) + F * S + 4 * F
    for d, nodes in enumerate(levels):
        if d < SL:
            continue
        tiers.append((nodes * node_bytes, per_upper))
    pool = info["leaf_lines"]
    tiers.append((pool * ((32 if F > kpl else 0) + F * S), per_last))
    tiers.append((pool * F * 32, 32.0))
    tiers.append((pool * F * 32, 32.0 * hit_rate))
    return tiers


def static_cache_bytes(tiers, capacity):
    """Per-query bytes that miss an ideal static cache of `capacity` bytes."""
    miss = 0.0
    left = float(capacity)
    for total, per_q in sorted(tiers, key=lambda t: -(t[1] / max(t[0], 1))):
        cached = min(1.0, left / total) if total > 0 else 1.0
        left = max(0.0, left - total)
        miss += per_q * (1.0 - cached)
    return miss


def model(info, l2_bytes, hit_rate=1.0):
    S = info["width"]
    io = 2 * S + 8
    tiers = implicit_tiers(info, hit_rate) if info["layout"] == 0 else regular_tiers(info, hit_rate)
    hbm = io + static_cache_bytes(tiers, l2_bytes)
    l2 = io + sum(t[1] for t in tiers)
    return {"hbm_bytes_per_query": hbm, "l2_bytes_per_query": l2, "io_bytes_per_query": io}


def _touched(units, m):
    """Expected distinct units touched by m uniform accesses over `units` units."""
    if units <= 0:
        return 0.0
    return units * (1.0 - np.exp(-float(m) / units))


def model_bucketed(info, m, level=None):
    """Algorithmic bytes per query of the BUCKETED tree search kernel (csrc/bucketed.cu,
    item directory): the query in (S), the 16 B result record out, and the tree lines
    below the shared-memory directory, each fetched from HBM once per pass when the
    queries of a bucket share it (uniform queries: distinct lines touched = U (1 - e^(-m/U))).
    regular: one 64 B key line of a last-level node + one 64 B leaf line per query;
    implicit: the levels from `level` down (index sector + key sector, or the whole
    node when wider than the L2 budget) + the 64 B leaf line.  The staged directory
    maxima (S per unit) are read once per pass."""
    S, F, n = info["width"], info["fanout"], info["n_distinct"]
    P = 64 // (2 * S)
    io = S + 16
    if info["layout"] == 1:  # regular
        kpl = 64 // S
        ni = F // kpl if F > kpl else 1
        key_lines = max(1.0, n / (kpl * P))
        leaf_lines = max(1.0, n / P)
        dram = (_touched(key_lines, m) * 64 + _touched(leaf_lines, m) * 64
                + info["chain_len"] * (ni * S + 4)) / m
        l2 = 64 + 64
    else:
        L0 = info["leaf_lines"]
        lv = info["height"] if level is None else level
        nodes = info["level_nodes"]
        dram = _touched(L0, m) * 64 / m
        l2 = 64
        for d in range(lv, info["height"]):
            node_b = F * S
            dram += _touched(nodes[d], m) * node_b / m
            l2 += 64 if node_b > 32 else _sect(node_b)
        units = L0 if lv >= info["height"] else nodes[lv]
        dram += units * S / m
    return {"hbm_bytes_per_query": io + dram, "l2_bytes_per_query": io + l2, "io_bytes_per_query": io}


def l2_granularity(info, hit_rate=1.0, bucketed=False, level=None):
    """The L2 model bytes per query split by access granularity (bytes per request):
    {32: random 32 B sectors, 64: random 64 B lines and the coalesced query / result
    streams}.  bench.py divides each class by the in-run probe of that granularity, so
    the L2 roof of a mixed pattern is sum(bytes_c / BW_c), not bytes / BW_32."""
    S, F = info["width"], info["fanout"]
    io = 2 * S + 8 if not bucketed else S + 16
    out = {32: 0.0, 64: float(io)}
    if info["layout"] == 1:  # regular
        kpl = 64 // S
        if bucketed:
            out[64] += 64 + 64  # key line + leaf line (256-bit lane loads: one 64 B request each)
            return out
        levels = len(info["level_nodes"]) - (info["smem_levels"] or 0)
        idx = 32 if F > kpl else 0
        out[32] += max(0, levels) * (idx + 32) + idx
        out[64] += max(0, levels) * min(64, F * S) + min(64, F * S) + 32 + 32 * hit_rate
        return out
    node = F * S
    lv = info["smem_levels"] if level is None else level
    for d in range(lv, info["height"]):
        if node > 32:
            out[32] += 64  # index sector + one key sector
        else:
            out[32] += _sect(node)
    out[64] += 32 + 32 * hit_rate  # the leaf line as one request (key + value sectors)
    return out
