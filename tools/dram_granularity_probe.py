"""Random-read DRAM probe: all-SM random reads of 32/64/128/256 B aligned chunks over a
1 GB and a 4 GB buffer (far beyond the L2): useful GB/s per chunk size.  If the useful
rate doubles from 64 B to 128 B chunks, a random read costs a ~128 B transfer."""
import ctypes as C
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
L = C.CDLL(os.path.join(ROOT, "tools", "libhbtprobe.so"))
L.probe_random_read_gbs.restype = C.c_double
L.probe_random_read_gbs.argtypes = [C.c_uint64, C.c_int, C.c_int]
out = {}
for nb in (1 << 30, 4 << 30):
    for chunk in (32, 64, 128, 256):
        out[f"{nb >> 20}MB_{chunk}B"] = round(L.probe_random_read_gbs(nb, chunk, 3), 1)
print(json.dumps(out))
