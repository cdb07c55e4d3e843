"""Does splitting the SMs into two halves that each read only half of a random
working set restore L2 capacity (cross-die duplication test)?  map: 0 none,
1 smid < nsm/2, 2 smid & 1, 3 (smid>>1)&1, 4 (smid>>2)&1, 5 (smid>>3)&1,
6 the measured die of each SM (tools/sm_die_map.py)."""
import ctypes as C
import json
import os
import subprocess
import sys

import torch  # noqa: F401

HERE = os.path.dirname(os.path.abspath(__file__))
L = C.CDLL(os.path.join(HERE, "libhbtprobe.so"))
L.probe_random_read_aff_gbs.restype = C.c_double
L.probe_random_read_aff_gbs.argtypes = [C.c_uint64, C.c_int, C.c_int, C.c_int, C.c_void_p]
subprocess.run([sys.executable, os.path.join(HERE, "sm_die_map.py")], check=True)
d = json.load(open("gpurun_out/sm_die_map.json"))
die = (C.c_uint8 * 256)()
for s, g in zip(d["smid"], d["die"]):
    die[s] = g
out = {}
for mb in [32, 64, 96, 128, 160, 256]:
    out[mb] = {m: round(L.probe_random_read_aff_gbs(mb << 20, 32, m, 2, C.cast(die, C.c_void_p)), 1) for m in (0, 5, 6)}
    print(mb, out[mb], flush=True)
print(json.dumps(out))
