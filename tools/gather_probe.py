"""Random 64 B line gather probe (tools/probe.cu probe_gather64): G lines/s from an
8 GB DRAM-resident buffer vs lines in flight per SM, for lane-pair 256-bit loads (mode 0,
the item search's leaf read) and per-lane cp.async.bulk copies into shared memory
(mode 1).  One JSON line per setting."""
import ctypes
import json
import os

lib = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "libhbtprobe.so"))
lib.probe_gather64.restype = ctypes.c_double
lib.probe_gather64.argtypes = [ctypes.c_uint64, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int]
B = 8 << 30
for mode, u, th, cps in [(0, 1, 1024, 1), (0, 2, 1024, 1), (0, 4, 1024, 1), (0, 8, 1024, 1),
                         (0, 1, 1024, 2), (0, 2, 1024, 2), (0, 4, 1024, 2), (0, 2, 512, 4),
                         (1, 1, 1024, 1), (1, 2, 1024, 1), (1, 1, 512, 2), (1, 2, 512, 2), (1, 4, 256, 2),
                         (1, 8, 128, 2), (1, 4, 512, 1), (1, 8, 256, 1)]:
    r = lib.probe_gather64(B, mode, u, th, cps, 3)
    inflight = th * cps * u // (2 if mode == 0 else 1)
    print(json.dumps({"mode": ["ldg256_pair", "tma_bulk64"][mode], "u": u, "threads": th, "ctas_per_sm": cps,
                      "lines_in_flight_per_sm": inflight, "glines_per_s": round(r, 2)}), flush=True)
# windowed: all SMs draw random lines from one sliding window (DRAM-row / L2 locality)
lib.probe_gather64_window.restype = ctypes.c_double
lib.probe_gather64_window.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int]
for wmb in (0, 2048, 512, 128, 64, 32, 16, 8, 2):
    r = lib.probe_gather64_window(B, wmb << 20, 3)
    print(json.dumps({"mode": "ldg256_pair_window", "window_mb": wmb or "whole 8 GB", "lines_in_flight_per_sm": 1024,
                      "glines_per_s": round(r, 2)}), flush=True)
