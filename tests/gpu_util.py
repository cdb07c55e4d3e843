"""Helpers shared by the -m gpu parity tests (test code only)."""
import os

import numpy as np
import torch

import gen
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
END = oracle.END


def np_dtype(width):
    return np.uint32 if width == 4 else np.uint64


def to_dev(a, width):
    a = np.ascontiguousarray(np.asarray(a).astype(np_dtype(width)))
    sgn = a.view(np.int32 if width == 4 else np.int64)
    return torch.from_numpy(sgn.copy()).cuda()


def from_dev(t, width):
    return t.cpu().numpy().view(np_dtype(width)).astype(np.uint64)


def gpu_build(hbt, keys, vals, F, width, layout="implicit"):
    return hbt.Tree(to_dev(keys, width), to_dev(vals, width), fanout=F, layout=layout)


def gpu_search(tree, q, width):
    pf, v = tree.search(to_dev(q, width))
    torch.cuda.synchronize()
    return pf.cpu().numpy().view(np.uint64), from_dev(v, width)


def expected_implicit_bytes(o_tree, width):
    a = o_tree.arrays()
    dt = np_dtype(width)
    inner = a["inner"].astype(dt).tobytes()
    leaf = np.concatenate([a["lkeys"], a["lvals"]], axis=1).astype(dt).tobytes()
    return inner, leaf


from gen.device import GenLib  # noqa: E402,F401
