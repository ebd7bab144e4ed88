"""Helpers shared by the GPU tests (buffers, oracle comparison).  Test
infrastructure: may import both the oracle and the product binding."""
import numpy as np

import oracle
from ddt_inputs import random_bytes, SENTINEL


def cuda_bytes(arr: np.ndarray):
    import torch
    return torch.from_numpy(np.ascontiguousarray(arr).view(np.uint8).reshape(-1).copy()).cuda()


def host(t) -> np.ndarray:
    return t.cpu().numpy()


class Case:
    """A (spec, count) request with device/host source & destination buffers laid
    out so the footprint (with negative lb) fits, plus a byte misalignment."""

    def __init__(self, ddt, spec, count=1, misalign=0, seed=1, pk_misalign=0):
        self.spec, self.count = spec, count
        self.o = oracle.Type(spec)
        self.t = ddt.Type.from_spec(spec)
        lo, hi = self.o.footprint(count)
        self.margin = 64
        self.off = self.margin - lo + misalign          # MPI buffer address inside the allocation
        self.nbytes = (hi - lo) + 2 * self.margin + 16
        self.src = random_bytes(self.nbytes, seed)
        self.psize = count * self.o.size
        self.pk_off = pk_misalign
        self.packed_src = random_bytes(self.psize + 32, seed + 7)

    # GPU
    def gpu_pack(self, q):
        import torch
        s = cuda_bytes(self.src)
        d = torch.full((self.psize + 32,), SENTINEL, dtype=torch.uint8, device="cuda")
        uid = q.pack(self.t, (s, self.off), self.count, (d, self.pk_off))
        return uid, s, d

    def gpu_unpack(self, q):
        import torch
        s = cuda_bytes(self.packed_src)
        d = torch.full((self.nbytes,), SENTINEL, dtype=torch.uint8, device="cuda")
        uid = q.unpack(self.t, (s, self.pk_off), self.count, (d, self.off))
        return uid, s, d

    # oracle
    def expect_pack(self):
        out = np.full(self.psize + 32, SENTINEL, np.uint8)
        out[self.pk_off:self.pk_off + self.psize] = oracle.pack(self.o, self.src, self.count, self.off)
        return out

    def expect_unpack(self):
        out = np.full(self.nbytes, SENTINEL, np.uint8)
        oracle.unpack(self.o, self.packed_src[self.pk_off:self.pk_off + self.psize], out, self.count, self.off)
        return out


def assert_bytes_equal(got: np.ndarray, exp: np.ndarray, what=""):
    if not np.array_equal(got, exp):
        bad = np.nonzero(got != exp)[0]
        raise AssertionError(f"{what}: {bad.size} bytes differ; first at {bad[:8].tolist()} "
                             f"got {got[bad[:8]].tolist()} expected {exp[bad[:8]].tolist()}")


def occupier():
    """ctypes handle of tests/c/occupy.cu (built here with nvcc for sm_100a on
    first use; test support, not part of the library)."""
    import ctypes
    import os
    import subprocess
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    src = os.path.join(root, "tests", "c", "occupy.cu")
    out = os.path.join(root, "build", "occupy.so")
    if not os.path.exists(out) or os.path.getmtime(out) < os.path.getmtime(src):
        os.makedirs(os.path.dirname(out), exist_ok=True)
        tmp = out + f".tmp{os.getpid()}"
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O2",
                               "-shared", "-Xcompiler", "-fPIC", "-o", tmp, src])
        os.replace(tmp, out)
    L = ctypes.CDLL(out)
    L.occupy_launch.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                                ctypes.c_longlong]
    L.occupy_launch.restype = ctypes.c_int
    return L
