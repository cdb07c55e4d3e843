"""Home-die interleave of device memory: per-SM latency to addresses 64 B apart;
cluster SMs (die) and addresses (home) jointly; print the run lengths."""
import ctypes as C
import json
import os

import numpy as np
import torch  # noqa: F401

L = C.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "libhbtprobe.so"))
n = torch.cuda.get_device_properties(0).multi_processor_count
for stride, na in [(64, 4096), (4096, 2048)]:
    lat = (C.c_uint16 * (na * n))()
    sm = (C.c_uint32 * n)()
    print("rc", L.probe_addr_latency(lat, sm, n, stride, na))
    lat = np.array(lat, dtype=np.float64).reshape(n, na)
    z = lat - lat.mean(axis=0)
    u, s, vt = np.linalg.svd(z, full_matrices=False)
    die = (u[:, 0] > 0).astype(int)
    home = (vt[0] > 0).astype(int)
    print("stride", stride, "sv", np.round(s[:3], 1), "SMs per group", np.bincount(die), "addr per group", np.bincount(home))
    runs = np.diff(np.flatnonzero(np.diff(np.r_[-1, home, -1]) != 0))
    print("run lengths (addresses):", np.bincount(runs)[:40].tolist())
    print("home pattern first 256:", "".join(map(str, home[:256])))
    # how clean: mean latency near vs far
    near = np.where(die[:, None] == home[None, :], lat, np.nan)
    print("median lat group-match / mismatch", np.nanmedian(near), np.nanmedian(np.where(die[:, None] != home[None, :], lat, np.nan)))
