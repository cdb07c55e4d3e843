"""Build one config's tree once and time the search under several hbt_set_param
settings (device time per batch with CUDA events; phase times of bucketed searches).

  python tools/param_sweep.py --config c4 --set item_rounds=1,item_l2_hint=0 --set item_rounds=16
Each --set is a comma-separated list of NAME=VALUE applied in order (knobs keep
their values across sets: name every knob a set depends on).  Prints one JSON line
per set; same_result_hash checks every set returns the first set's outputs."""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_sigmod_shahvaranij16_b200 as hbt  # noqa: E402
from gen.device import GenLib  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c4")
    ap.add_argument("--set", action="append", default=[])
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--m", type=int, default=0)
    ap.add_argument("--sorted", action="store_true", help="sort the batch first (locality experiments)")
    a = ap.parse_args()
    c = gen.CONFIGS[a.config]
    g = GenLib()
    sk, sv, sq = (gen.stream_seed(c["cfg"], s) for s in (gen.STREAM_K, gen.STREAM_V, gen.STREAM_Q))
    n, w, m = c["n"], c["width"], a.m or c["m"]
    if a.config == "c4":
        keys, vals = g.stratified_keys(n, sk), g.mix_stream(n, w, sv)
        q = g.stratified_queries(m, n, sq, sk)
    elif c["queries"] == "zipf":
        keys, vals = g.mix_stream(n, w, sk), g.mix_stream(n, w, sv)
        hk = gen.keys(n, w, sk)
        q = torch.from_numpy(hk[gen.zipf_ranks(m, n, c["theta"], sq) - 1].view("int64")).cuda()
    else:
        keys, vals = g.mix_stream(n, w, sk), g.mix_stream(n, w, sv)
        q = g.uniform_queries(m, n, w, sq, sk)
    if a.sorted:
        q = (q.view(torch.int64) ^ (1 << 63)).sort().values.__xor__(1 << 63).view(q.dtype)  # unsigned order
    tree = hbt.Tree(keys, vals, fanout=c["fanout"], layout=c["layout"])
    del keys, vals
    torch.cuda.empty_cache()
    pf = torch.empty(m, dtype=torch.int64, device="cuda")
    vv = torch.empty(m, dtype=q.dtype, device="cuda")
    ref = None
    for s in (a.set or [""]):
        kv = [x.split("=") for x in s.split(",") if x]
        for k, v in kv:
            tree.set_param(k, int(v, 0))
        for _ in range(3):
            tree.search(q, pf, vv)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(a.steps):
            tree.search(q, pf, vv)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / a.steps
        ph = None
        try:
            tree.set_param("phase_timing", 1)
            tree.search(q, pf, vv)
            ph = tree.last_phases()
            tree.set_param("phase_timing", 0)
        except hbt.HBTError:
            pass
        h = int(pf.sum().item()) ^ int(vv.sum().item())
        same = ref is None or h == ref
        ref = h if ref is None else ref
        print(json.dumps({"config": a.config, "set": s, "ms": round(ms, 4), "gqps": round(m / ms / 1e6, 2),
                          "phases": ph, "same_result_hash": same}), flush=True)


if __name__ == "__main__":
    main()
