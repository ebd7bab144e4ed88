"""L2 fetch-granularity probe (diagnostic): does cudaLimitMaxL2FetchGranularity
change the DRAM over-fetch of the sparse configs[2] layout (10^5 x 12-B blocks)
or the COMB x-face cells?  Times a 32-request configs[2] pack plan (L2 flushed
before each launch) and the configs[3] x-face class at each granularity."""
import ctypes
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import config3_spec  # noqa: E402

RT = ctypes.CDLL(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib",
                              "libcudart.so.12"))
LIMIT = 0x05  # cudaLimitMaxL2FetchGranularity


def get_limit():
    v = ctypes.c_size_t()
    RT.cudaDeviceGetLimit(ctypes.byref(v), LIMIT)
    return v.value


def main():
    torch.cuda.set_device(0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    out = []
    for shuffled in (False, True):
        spec, fp = config3_spec(shuffled=shuffled)
        t = ddt.Type.from_spec(spec)
        B = 32
        src = torch.empty((B, fp), dtype=torch.uint8, device="cuda")
        src.random_(0, 256)
        dst = torch.empty((B, t.size), dtype=torch.uint8, device="cuda")
        q = ddt.Queue()
        for b in range(B):
            q.pack(t, src[b], 1, dst[b])
        plan = ddt.Plan(q)
        s = torch.cuda.current_stream()
        for g in (0, 32, 64, 128, 32, 0):
            RT.cudaDeviceSetLimit(LIMIT, ctypes.c_size_t(g))
            got = get_limit()
            ts = []
            for _ in range(15):
                flush.fill_(1)
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(s)
                plan.launch()
                b.record(s)
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(b) * 1e3)
            us = statistics.median(ts)
            r = {"layout": "configs[2]" + (" shuffled" if shuffled else ""), "set": g, "limit": got,
                 "us": round(us, 2), "alg_GBs": round(2 * B * t.size / us / 1e3, 1)}
            print(json.dumps(r), flush=True)
            out.append(r)
        plan.destroy()
        q.destroy()


if __name__ == "__main__":
    main()
