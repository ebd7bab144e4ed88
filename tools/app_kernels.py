"""Application-kernel layouts of the paper's Fig 12 on
one B200: per layout, a batch of B pack requests + B unpack requests (each its
own source / packed / destination buffer), frozen into two persistent plans
(one fused launch each), timed with CUDA events after an L2 read sweep, median
of `reps`.  Algorithmic bytes = 2 S per request (pack) + 2 S (unpack).

  specfem3D_oc : indexed 3-float blocks at 10^5 sorted random points (configs[2])
  specfem3D_cm : struct-on-indexed, 3 float components (x, y, z arrays)
  MILC         : hvector-of-vector face of an L^4 su3 lattice (L = 32)
  NAS_MG       : the x, y and z vector faces of a 258^3 grid of doubles (3 requests per batch entry)

usage: python tools/app_kernels.py [B] [reps]   -> one JSON line per layout (diagnostic)"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import config3_spec, config3_cm_spec, milc_spec, nas_mg_specs  # noqa: E402


def layouts():
    oc, fp_oc = config3_spec()
    cm, fp_cm = config3_cm_spec()
    mi, fp_mi = milc_spec(32)
    nas, fp_nas = nas_mg_specs(258, 258, 258)
    return [("specfem3D_oc", [oc], fp_oc), ("specfem3D_cm", [cm], fp_cm), ("MILC", [mi], fp_mi),
            ("NAS_MG", [nas["x"], nas["y"], nas["z"]], fp_nas)]


def main():
    B = int(sys.argv[1]) if len(sys.argv) > 1 else 16
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 20
    torch.cuda.set_device(0)
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for name, specs, fp in layouts():
        types = [ddt.Type.from_spec(sp) for sp in specs]
        q = ddt.Queue()
        srcs = [torch.empty(fp, dtype=torch.uint8, device="cuda").random_(0, 256) for _ in range(B)]
        dsts = [torch.empty(fp, dtype=torch.uint8, device="cuda") for _ in range(B)]
        pks = [[torch.empty(t.size, dtype=torch.uint8, device="cuda") for t in types] for _ in range(B)]
        for b in range(B):
            for t, pk in zip(types, pks[b]):
                q.pack(t, srcs[b], 1, pk)
        pack = ddt.Plan(q)
        for b in range(B):
            for t, pk in zip(types, pks[b]):
                q.unpack(t, pk, 1, dsts[b])
        unpack = ddt.Plan(q)
        S = B * sum(t.size for t in types)
        res = {"pack": [], "unpack": []}
        for _ in range(3):
            pack.launch()
            unpack.launch()
        for _ in range(reps):
            for arm, plan in (("pack", pack), ("unpack", unpack)):
                flush.max()
                a, b_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(s)
                plan.launch()
                b_.record(s)
                torch.cuda.synchronize()
                res[arm].append(a.elapsed_time(b_) * 1e3)
        out = {"layout": name, "B": B, "requests_per_launch": B * len(types), "packed_bytes_per_launch": S}
        for arm, v in res.items():
            us = statistics.median(v)
            out[arm] = {"us": round(us, 2), "alg_GBs": round(2 * S / us / 1e3, 1)}
        print(json.dumps(out), flush=True)
        pack.destroy()
        unpack.destroy()
        q.destroy()
        del srcs, dsts, pks
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
