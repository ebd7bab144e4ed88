"""Measurement sweep over BASELINE.json configs 1, 3 and 5 on one B200 (the
bench line carries configs[1]; this tool produces the per-config tables in
profiles/).  Device times from CUDA events on the queue's stream; L2 evicted
(256 MiB read sweep) before every timed repetition unless the working set exceeds
L2 by itself.  Prints one JSON document.

configs[0]  vector(16,4,64) of double: pack+unpack per iteration (2 flushes or
            one 2-request plan), us/iter, launches/iter.
configs[2]  hindexed 10^5 x 3 floats (sorted and shuffled), batch B in {1,16,32}:
            pack GB/s algorithmic (2S per request) and vs the 32-B-sector floor.
configs[4]  dense vector (256 B blocks, 50% density), S = 64 B .. 64 MiB,
            B in {1,4,16,64,256,1024} with B*S <= 4 GiB (subset by --quick):
            arms fused (one flush), fused-plan (persistent table, 1 launch),
            per-request (B flushes, 1 sync: Alg 2 shape), per-request+sync
            (B flushes each synchronised: Alg 1 / GPU-Sync shape).
"""
import argparse
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import (config1_spec, config3_spec, config3_cm_spec, config5_spec, CONFIG5_SIZES,  # noqa: E402
                        CONFIG5_BATCHES)

FLUSH = None


def flush_l2():
    FLUSH.max()  # read sweep: evicts L2 without leaving dirty lines to write back in the timed region


def timed(fn, reps, flush=True, setup=None):
    s = torch.cuda.current_stream()
    out = []
    for i in range(reps + 3):
        if setup:
            setup()
        if flush:
            flush_l2()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        fn()
        b.record(s)
        torch.cuda.synchronize()
        if i >= 3:
            out.append(a.elapsed_time(b) * 1e3)
    return statistics.median(out)


def cfg1(reps):
    t = ddt.Type.from_spec(config1_spec())
    src = torch.randint(0, 255, (8192,), dtype=torch.uint8, device="cuda")
    pk = torch.empty(512, dtype=torch.uint8, device="cuda")
    dst = torch.empty(8192, dtype=torch.uint8, device="cuda")
    q = ddt.Queue()

    def two_flushes():
        q.pack(t, src, 1, pk)
        q.flush()
        q.unpack(t, pk, 1, dst)
        q.flush()

    l0 = q.stats()["launches"]
    us = timed(two_flushes, reps)
    launches = (q.stats()["launches"] - l0) / (reps + 3)
    # persistent plans (one per direction)
    q.pack(t, src, 1, pk)
    p1 = ddt.Plan(q)
    q.unpack(t, pk, 1, dst)
    p2 = ddt.Plan(q)

    def plans():
        p1.launch()
        p2.launch()

    us_plan = timed(plans, reps)
    # the iteration as a solver would replay it: K iterations (2 dependent
    # launches each) captured once into a CUDA graph, device time per iteration
    K = 200
    st = torch.cuda.Stream()
    qg = ddt.Queue(stream=st)  # plans launch on their queue's stream: the capturing one
    qg.pack(t, src, 1, pk)
    g1 = ddt.Plan(qg)
    qg.unpack(t, pk, 1, dst)
    g2 = ddt.Plan(qg)
    torch.cuda.synchronize()
    with torch.cuda.stream(st):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            for _ in range(K):
                g1.launch()
                g2.launch()
        g.replay()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        g.replay()
        b.record(st)
        torch.cuda.synchronize()
    us_graph = a.elapsed_time(b) * 1e3 / K
    return {"workload": "configs[0]", "us_per_iter_flush": round(us, 2), "launches_per_iter": launches,
            "us_per_iter_plan": round(us_plan, 2), "us_per_iter_graph": round(us_graph, 3), "graph_note": "K=200 iterations captured once, L2-hot (1 KB footprint)",
            "bytes_per_iter": 4 * 512}


def cfg3(reps):
    res = []
    for variant in ("sorted", "shuffled", "cm_struct"):
        if variant == "cm_struct":
            spec, nb = config3_cm_spec()
            t = ddt.Type.from_spec(spec)
            idx = np.array(spec[3][0][2], dtype=np.int64)
            offs = np.concatenate([4 * idx + k * 4 * (1 << 20) for k in range(3)])
            seglen = 4
        else:
            spec, nb = config3_spec(shuffled=(variant == "shuffled"))
            t = ddt.Type.from_spec(spec)
            offs = np.array(spec[2], dtype=np.int64)
            seglen = 12
        sectors = len(np.unique(np.concatenate([offs // 32, (offs + seglen - 1) // 32])))
        for B in (1, 16, 32):
            src = torch.randint(0, 255, (B, nb), dtype=torch.uint8, device="cuda")
            dst = torch.empty((B, t.size), dtype=torch.uint8, device="cuda")
            q = ddt.Queue()
            for b in range(B):
                q.pack(t, src[b], 1, dst[b])
            plan = ddt.Plan(q)
            us = timed(plan.launch, reps)
            alg = 2 * t.size * B
            floor = (sectors * 32 + t.size) * B
            res.append({"variant": variant, "B": B, "us": round(us, 2), "alg_gbs": round(alg / us / 1e3, 1),
                        "sector_floor_gbs_equiv": round(floor / us / 1e3, 1), "payload_bytes": t.size * B,
                        "sector_read_bytes": sectors * 32 * B})
            plan.destroy()
            q.destroy()
    return {"workload": "configs[2]", "cells": res}


def cfg5(reps, quick):
    cells = []
    sizes = CONFIG5_SIZES if not quick else [64, 4096, 65536, 1 << 20, 16 << 20, 64 << 20]
    batches = CONFIG5_BATCHES if not quick else [1, 16, 256]
    for S in sizes:
        spec, fp = config5_spec(S)
        t = ddt.Type.from_spec(spec)
        for B in batches:
            if B * S > (1 << 30) or B * (fp + S) > (3 << 30):
                continue
            src = torch.empty((B, fp), dtype=torch.uint8, device="cuda")
            src.random_(0, 256)
            dst = torch.empty((B, S), dtype=torch.uint8, device="cuda")
            q = ddt.Queue()
            big = B * (fp + S) > (512 << 20)
            r = max(3, reps // (4 if big else 1))

            # the fused arm enqueues the batch through ddt_enqueue_many (one call
            # across the ABI; a Python loop of single enqueues would time ctypes)
            tys = np.full(B, t.handle.value, dtype=np.uint64)
            sp = np.asarray([src[b].data_ptr() for b in range(B)], dtype=np.uint64)
            dp = np.asarray([dst[b].data_ptr() for b in range(B)], dtype=np.uint64)
            cn = np.ones(B, dtype=np.int64)

            def fused():
                q.enqueue_many_raw(0, tys, sp, cn, dp)
                q.flush()

            def per_request():
                for b in range(B):
                    q.pack(t, src[b], 1, dst[b])
                    q.flush()

            def per_request_sync():
                for b in range(B):
                    q.pack(t, src[b], 1, dst[b])
                    q.flush()
                    torch.cuda.current_stream().synchronize()

            cell = {"S": S, "B": B}
            cell["fused_us"] = round(timed(fused, r, flush=not big), 2)
            for b in range(B):
                q.pack(t, src[b], 1, dst[b])
            plan = ddt.Plan(q)
            cell["plan_us"] = round(timed(plan.launch, r, flush=not big), 2)
            plan.destroy()
            if B <= 256:
                cell["per_request_us"] = round(timed(per_request, r, flush=not big), 2)
                cell["per_request_sync_us"] = round(timed(per_request_sync, max(3, r // 2), flush=not big), 2)
            alg = 2.0 * S * B
            cell["plan_gbs"] = round(alg / cell["plan_us"] / 1e3, 1)
            cells.append(cell)
            q.destroy()
            del src, dst
            torch.cuda.empty_cache()
    return {"workload": "configs[4]", "cells": cells}


def main():
    global FLUSH
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=30)
    ap.add_argument("--quick", action="store_true")
    args = ap.parse_args()
    torch.cuda.set_device(0)
    FLUSH = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    t0 = time.time()
    out = {"gpu": torch.cuda.get_device_name(0), "reps": args.reps}
    out["config1"] = cfg1(args.reps)
    out["config3"] = cfg3(args.reps)
    out["config5"] = cfg5(args.reps, args.quick)
    out["wall_s"] = round(time.time() - t0, 1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
