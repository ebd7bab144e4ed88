"""Dense-pack probe (configs[4] layout: 256-B blocks at 50% density): the fused
plan against library arms on the same buffers, interleaved round robin, median
of N rounds, device time from CUDA events.

arms:  plan        ddt_plan_launch (bench.py's pack_roofline arm)
       plan_ubK    same, items of K vectors per thread (DDT_UB=K at plan build)
       torch       torch strided copy (dst.view(B,n,256) <- src.view(B,n,512)[..., :256])
       memcpy2d    one cudaMemcpy2DAsync per request (B calls)
       copy        contiguous torch copy of the same S*B bytes (this box's copy rate)
usage: python tools/pack_probe.py [rounds]   -> one JSON document on stdout
"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import config5_spec  # noqa: E402


def main():
    rounds = int(sys.argv[1]) if len(sys.argv) > 1 else 9
    from cuda.bindings import runtime as rt
    torch.cuda.set_device(0)
    stream = torch.cuda.current_stream()
    out = []
    for S, B in [(1 << 20, 1024), (4 << 20, 256), (16 << 20, 64), (64 << 20, 16)]:
        spec, fp = config5_spec(S)
        assert fp <= (S // 256) * 512
        t = ddt.Type.from_spec(spec)
        src = torch.empty((B, (S // 256) * 512), dtype=torch.uint8, device="cuda")
        src.random_(0, 256)
        dst = torch.empty((B, S), dtype=torch.uint8, device="cuda")
        ref = src.view(B, S // 256, 512)[:, :, :256].reshape(B, S)
        csrc = torch.empty((B, S), dtype=torch.uint8, device="cuda")
        arms = {}
        q = ddt.Queue()
        plans = {}
        for ub in (None, 4, 2, 1):
            if ub:
                os.environ["DDT_UB"] = str(ub)
            ddt.reload_env()
            for b in range(B):
                q.pack(t, src[b], 1, dst[b])
            plans["plan" if ub is None else f"plan_ub{ub}"] = ddt.Plan(q)
            os.environ.pop("DDT_UB", None)
            ddt.reload_env()
        for k, p in plans.items():
            arms[k] = p.launch
        lib_arms = os.environ.get("PROBE_LIB_ARMS", "1") == "1"
        arms["torch"] = lambda: dst.view(B, S // 256, 256).copy_(src.view(B, S // 256, 512)[:, :, :256])
        h = stream.cuda_stream

        def m2d():
            for b in range(B):
                rt.cudaMemcpy2DAsync(dst[b].data_ptr(), 256, src[b].data_ptr(), 512, 256, S // 256,
                                     rt.cudaMemcpyKind.cudaMemcpyDeviceToDevice, h)
        arms["memcpy2d"] = m2d
        arms["copy"] = lambda: dst.copy_(csrc)
        if not lib_arms:
            for k in ("torch", "memcpy2d", "copy"):
                arms.pop(k)
        times = {k: [] for k in arms}
        for k, f in arms.items():  # warm-up + parity of every arm that writes dst
            dst.zero_()
            f()
            torch.cuda.synchronize()
            if k != "copy":
                assert torch.equal(dst, ref), f"{k} differs"
        for _ in range(rounds):
            for k, f in arms.items():
                a, b_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                f()
                b_.record(stream)
                torch.cuda.synchronize()
                times[k].append(a.elapsed_time(b_) * 1e3)
        cell = {"S": S, "B": B}
        for k, v in times.items():
            us = statistics.median(v)
            cell[k] = {"us": round(us, 2), "alg_gbs": round(2.0 * S * B / us / 1e3, 1)}
        out.append(cell)
        print(json.dumps(cell), file=sys.stderr, flush=True)
        for p in plans.values():
            p.destroy()
        q.destroy()
        del src, dst, csrc, ref
        torch.cuda.empty_cache()
    print(json.dumps({"probe": "pack_probe", "rounds": rounds, "cells": out}))


if __name__ == "__main__":
    main()
