"""Random-read bandwidth vs buffer size (where the L2 stops holding the working set)."""
import ctypes as C
import json
import os
import sys

import torch  # noqa: F401  (initialises CUDA)

L = C.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "libhbtprobe.so"))
L.probe_random_read_gbs.restype = C.c_double
L.probe_random_read_gbs.argtypes = [C.c_uint64, C.c_int, C.c_int]
out = {}
for mb in [8, 16, 32, 48, 64, 80, 96, 112, 128, 160, 256, 1024]:
    out[mb] = {ch: round(L.probe_random_read_gbs(mb << 20, ch, 2), 1) for ch in (32, 64)}
print(json.dumps(out))
