"""ctypes binding of gen/libhbtgen.so, the device twin of gen/'s integer
streams (no method arithmetic).  Needs torch with CUDA."""
import ctypes as C
import os

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


class GenLib:
    """ctypes view of gen/libhbtgen.so (device twin of gen/)."""

    def __init__(self):
        L = C.CDLL(os.path.join(ROOT, "gen", "libhbtgen.so"))
        vp, u64, u32 = C.c_void_p, C.c_uint64, C.c_uint32
        L.hbtgen_mix_stream.argtypes = [vp, u64, u64, u32, u64, vp]
        L.hbtgen_uniform_queries.argtypes = [vp, u64, u64, u64, u32, u64, u64, vp]
        L.hbtgen_stratified_keys.argtypes = [vp, u64, u64, u64, vp]
        L.hbtgen_stratified_queries.argtypes = [vp, u64, u64, u64, u64, u64, vp]
        self.L = L

    @staticmethod
    def _s():
        return C.c_void_p(torch.cuda.current_stream().cuda_stream)

    def mix_stream(self, n, width, seed, start=0):
        out = torch.empty(n, dtype=torch.int32 if width == 4 else torch.int64, device="cuda")
        assert self.L.hbtgen_mix_stream(out.data_ptr(), start, n, width, seed, self._s()) == 0
        return out

    def uniform_queries(self, m, rng, width, seed_q, seed_k, start=0):
        out = torch.empty(m, dtype=torch.int32 if width == 4 else torch.int64, device="cuda")
        assert self.L.hbtgen_uniform_queries(out.data_ptr(), start, m, rng, width, seed_q, seed_k, self._s()) == 0
        return out

    def stratified_keys(self, n, seed, start=0):
        out = torch.empty(n, dtype=torch.int64, device="cuda")
        assert self.L.hbtgen_stratified_keys(out.data_ptr(), start, n, seed, self._s()) == 0
        return out

    def stratified_queries(self, m, rng, seed_q, seed_k, start=0):
        out = torch.empty(m, dtype=torch.int64, device="cuda")
        assert self.L.hbtgen_stratified_queries(out.data_ptr(), start, m, rng, seed_q, seed_k, self._s()) == 0
        return out
