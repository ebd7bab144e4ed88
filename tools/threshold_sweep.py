"""Fig 8 analog on B200 (§IV-C): 32 back-to-back pack
requests of a specfem3D_cm-style sparse layout (struct of 3 indexed float
components) through one queue with the auto-flush threshold T; the time from
the first enqueue until every request is complete (host enqueue + launches +
kernels), for T from 16 KB to "everything in one batch".  The paper's rule --
fuse until the fused kernel runs longer than a launch -- is checked against
the measured per-batch kernel times.  There is no network here, so only the
under-fusion side of the paper's curve can appear (over-fusion costs overlap
with communication).  Prints one JSON document."""
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import config3_cm_spec  # noqa: E402


def main():
    torch.cuda.set_device(0)
    res = {"workload": "32 x specfem3D_cm-style struct-on-indexed pack requests", "cells": []}
    for npts in (1365, 5461, 21845):   # ~16 KB, 64 KB, 256 KB packed per message
        spec, nb = config3_cm_spec(nblocks=npts, npoints=1 << 16)
        t = ddt.Type.from_spec(spec)
        n = 32
        src = torch.randint(0, 255, (n, nb), dtype=torch.uint8, device="cuda")
        dst = torch.empty((n, t.size), dtype=torch.uint8, device="cuda")
        sp = [src[i].data_ptr() for i in range(n)]
        dp = [dst[i].data_ptr() for i in range(n)]
        total = n * t.size
        for T in (16 << 10, 64 << 10, 256 << 10, 512 << 10, 1 << 20, 4 << 20, 0):
            q = ddt.Queue()
            q.set_flush_threshold(T)
            times = []
            for rep in range(25):
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                for i in range(n):
                    q.pack(t, sp[i], 1, dp[i])
                q.wait()
                times.append((time.perf_counter() - t0) * 1e6)
            st = q.stats()
            res["cells"].append({"msg_bytes": t.size, "threshold": T if T else "all", "us": round(statistics.median(times[5:]), 2),
                                 "launches_per_round": round(st["launches"] / 25, 2), "total_bytes": total})
            q.destroy()
    print(json.dumps(res))


if __name__ == "__main__":
    main()
