"""Random-read bandwidth over a large buffer vs cudaLimitMaxL2FetchGranularity."""
import ctypes as C
import json
import os

import torch  # noqa: F401

L = C.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "libhbtprobe.so"))
L.probe_random_read_gbs.restype = C.c_double
L.probe_random_read_gbs.argtypes = [C.c_uint64, C.c_int, C.c_int]
out = {"default_granularity": L.probe_get_l2_fetch()}
for g in [0, 32, 64, 128]:
    rc = L.probe_set_l2_fetch(g)
    out[f"g{g}"] = {"rc": rc, "now": L.probe_get_l2_fetch(),
                    **{f"{mb}MB_{ch}B": round(L.probe_random_read_gbs(mb << 20, ch, 2), 1)
                       for mb in (1024, 96) for ch in (32, 64)}}
print(json.dumps(out))
