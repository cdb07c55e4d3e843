"""Discover which SMs share a die: per-SM latency to 64 L2-resident lines;
SMs on the same die see the same near/far pattern."""
import ctypes as C
import json
import os

import numpy as np
import torch  # noqa: F401

L = C.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "libhbtprobe.so"))
n = torch.cuda.get_device_properties(0).multi_processor_count
lat = (C.c_uint32 * (64 * n))()
sm = (C.c_uint32 * n)()
print("rc", L.probe_sm_latency(lat, sm, n))
lat = np.array(lat, dtype=np.float64).reshape(n, 64)
sm = np.array(sm)
print("distinct sms", len(set(sm.tolist())))
print("latency range", lat.min(), np.median(lat), lat.max())
z = lat - lat.mean(axis=0)
u, s, vt = np.linalg.svd(z, full_matrices=False)
score = u[:, 0]
grp = (score > 0).astype(int)
order = np.argsort(sm)
print("singular values", np.round(s[:4], 1))
print("die by smid:", "".join(str(grp[i]) for i in order))
print("per-address near/far (group0 mean, group1 mean):")
print(np.round(lat[grp == 0].mean(0)[:16]), np.round(lat[grp == 1].mean(0)[:16]))
json.dump({"smid": sm[order].tolist(), "die": grp[order].tolist()}, open("gpurun_out/sm_die_map.json", "w"))
