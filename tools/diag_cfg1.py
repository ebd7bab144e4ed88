"""Per-CTA timeline of the configs[1] step in the bench harness (diagnostic).

Needs a library built with -DDDT_DIAG_TRACE=1 (tools/build_alt.sh diag
-DDDT_DIAG_TRACE=1), loaded through DDT_LIBDDT.  Builds bench.py's configs[1]
workload (R = 96 replicas, P2P plan at P = 1), captures K steps in one graph,
replays it after the L2 read sweep, and reads back one {start, after the PDL
wait, end} globaltimer record per CTA of every launch.  Per launch (ordered by
completion): how early its CTAs start relative to the predecessor's end, when
they pass griddepcontrol.wait, when the last one ends.

  DDT_LIBDDT=build/alt/libddt_diag.so python tools/diag_cfg1.py [K]
"""
import ctypes
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import FACE_DIRS  # noqa: E402

REC = np.dtype([("t0", "<u8"), ("t1", "<u8"), ("t2", "<u8"), ("cta", "<u4"), ("tag", "<u4")])


def main():
    K = int(sys.argv[1]) if len(sys.argv) > 1 else 500
    torch.cuda.set_device(0)
    torch.cuda.set_stream(torch.cuda.Stream())  # as bench.py: the queue binds the current stream
    lib = ddt.lib()
    fn = lib.ddt_diag_trace
    fn.argtypes = [ctypes.c_void_p, ctypes.c_int32]
    fn.restype = ctypes.c_int32
    c = ddt.Comm.single(0)
    wl = bench.HaloWorkload(ddt, torch, 0, 1, (128, 128, 128), FACE_DIRS, 1, os.environ.get("MODE", "p2p"), c, 2,
                            replicas=96, graph=False)
    flush = torch.empty(bench.L2_FLUSH_BYTES, dtype=torch.uint8, device="cuda")
    for _ in range(50):
        wl.step()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=torch.cuda.current_stream()):
        for _ in range(K):
            wl.step()
    g.replay()
    torch.cuda.synchronize()
    fn(None, 0)  # reset
    bench.l2_evict(torch, flush)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    g.replay()
    b.record()
    torch.cuda.synchronize()
    us = a.elapsed_time(b) * 1e3 / K
    buf = np.zeros(1 << 20, REC)
    n = fn(buf.ctypes.data, len(buf))
    r = buf[:n]
    # launches: records of one tag, split where consecutive starts are > 20 us apart
    launches = []
    for tag in np.unique(r["tag"]):
        x = np.sort(r[r["tag"] == tag], order="t0")
        cut = np.where(np.diff(x["t0"].astype(np.int64)) > 20000)[0] + 1
        for part in np.split(x, cut):
            launches.append(part)
    launches.sort(key=lambda p: int(p["t2"].max()))
    rows = []
    for i in range(1, len(launches)):
        p, q = launches[i - 1], launches[i]
        e = int(p["t2"].max())
        rows.append({
            "step_ns": int(q["t2"].max()) - e,
            "start_first": int(q["t0"].min()) - e, "start_last": int(q["t0"].max()) - e,
            "wait_first": (int(q["t1"].min()) - e) if q["t1"].min() else None,
            "wait_last": (int(q["t1"].max()) - e) if q["t1"].min() else None,
            "end_first": int(q["t2"].min()) - e,
            "ctas": len(q)})
    mid = rows[len(rows) // 4: 3 * len(rows) // 4]

    def med(k):
        v = [x[k] for x in mid if x[k] is not None]
        return statistics.median(v) if v else None
    # per CTA index (the batch's items in order): median time from passing the wait to the CTA's end
    mids = launches[len(launches) // 4: 3 * len(launches) // 4]
    by_cta = {}
    for q in mids:
        if not q["t1"].min():
            continue
        for rec in q:
            by_cta.setdefault(int(rec["cta"]), []).append(int(rec["t2"]) - int(rec["t1"]))
    cta_ns = {c: statistics.median(v) for c, v in sorted(by_cta.items())}
    buckets = {}
    for c, v in cta_ns.items():
        buckets.setdefault(c // 20 * 20, []).append(v)
    out_b = {f"{b}-{b + 19}": round(statistics.median(v)) for b, v in buckets.items()}
    out = {"lib": os.environ.get("DDT_LIBDDT", ""), "K": K, "us_per_step_events": round(us, 3), "records": int(n),
           "wait_to_end_ns_by_cta": out_b,
           "launches": len(launches), "median_over_middle_half_ns": {k: med(k) for k in rows[0]},
           "sample": rows[len(rows) // 2: len(rows) // 2 + 5]}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
