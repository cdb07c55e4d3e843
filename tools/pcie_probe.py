"""Host link probe: pinned H2D / D2H copy rates alone and concurrently (two streams),
the ceiling of the e2e number (hbt_search_host moves 8 B in and 16 B out per u64 query)."""
import json
import time

import torch

N = 1 << 30
h_in = torch.empty(2 * N, dtype=torch.uint8, pin_memory=True)
h_out = torch.empty(4 * N, dtype=torch.uint8, pin_memory=True)
d_in = torch.empty(2 * N, dtype=torch.uint8, device="cuda")
d_out = torch.empty(4 * N, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def timed(fn, reps=3):
    best = 1e9
    for _ in range(reps + 1):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        fn()
        torch.cuda.synchronize()
        best = min(best, time.perf_counter() - t0)
    return best


def h2d():
    with torch.cuda.stream(s1):
        d_in.copy_(h_in, non_blocking=True)


def d2h():
    with torch.cuda.stream(s2):
        h_out.copy_(d_out, non_blocking=True)


def both():
    h2d()
    d2h()


t1, t2, t3 = timed(h2d), timed(d2h), timed(both)
print(json.dumps({"h2d_gbs": round(2 * N / t1 / 1e9, 1), "d2h_gbs": round(4 * N / t2 / 1e9, 1),
                  "concurrent_s": round(t3, 4), "concurrent_h2d_2GiB_d2h_4GiB_gbs_total": round(6 * N / t3 / 1e9, 1),
                  "c4_e2e_ceiling_gqps": round((1 << 28) / t3 / 1e9, 3)}))
