"""Random 32 B reads where each SM group (die, tools/sm_die_map.py) reads only
256 B chunks homed on its own die (mode 1) / the other die (2) / anywhere (0)."""
import ctypes as C
import json
import os
import subprocess
import sys

import torch  # noqa: F401

HERE = os.path.dirname(os.path.abspath(__file__))
L = C.CDLL(os.path.join(HERE, "libhbtprobe.so"))
L.probe_affinity_read_gbs.restype = C.c_double
L.probe_affinity_read_gbs.argtypes = [C.c_uint64, C.c_int, C.c_void_p, C.c_uint32, C.POINTER(C.c_double)]
subprocess.run([sys.executable, os.path.join(HERE, "sm_die_map.py")], check=True)
d = json.load(open("gpurun_out/sm_die_map.json"))
die = (C.c_uint8 * 256)()
for s, g in zip(d["smid"], d["die"]):
    die[s] = g
out = {}
for mb in [32, 64, 80, 96, 112, 128, 160]:
    r = {}
    for mode in (0, 1, 2):
        f = C.c_double()
        r[mode] = round(L.probe_affinity_read_gbs(mb << 20, mode, C.cast(die, C.c_void_p), 290, C.byref(f)), 1)
    r["frac_home0"] = round(f.value, 3)
    out[mb] = r
    print(mb, r, flush=True)
json.dump(out, open("gpurun_out/l2_home_affinity.json", "w"))
