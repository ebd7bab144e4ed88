"""COMB P = 1 breakdown / A-B probe (diagnostic, not a bench line).

Times the configs[3] 26-neighbour self exchange (512^3 x 4 vars, DirectIPC
plan) restricted to direction classes, back to back over 2 replicas (each step
touches > 2 x L2).  All variants are plans over the SAME arrays and are timed
interleaved (round r times every variant once, K steps each), and the median
over rounds is reported: the x-face cells (one 8-B access per 4112-B row) make
single runs vary by ~10 %, so only interleaved medians compare variants.

Library knobs (DDT_UB, DDT_NO_GROUP, DDT_ITEM_ORDER, DDT_NO_PHASE) are read
when a plan is built; PROBE_KNOBS='[{}, {"DDT_NO_PHASE": "1"}]' selects the
variants.

usage: python tools/comb_probe.py [classes...]   -> one JSON line per (class, knobs)
"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import halo_messages, ALL_DIRS  # noqa: E402

CLASSES = {
    "all": ALL_DIRS,
    "xface": [d for d in ALL_DIRS if d[2] != 0 and d[0] == 0 and d[1] == 0],
    "x_any": [d for d in ALL_DIRS if d[2] != 0],
    "dense": [d for d in ALL_DIRS if d[2] == 0],
    "zyface": [d for d in ALL_DIRS if d[2] == 0 and abs(d[0]) + abs(d[1]) == 1],
}


def build(arrays, dirs, knobs, nvars, local):
    for k, v in knobs.items():
        os.environ[k] = v
    ddt.reload_env()
    try:
        msgs = halo_messages(0, 1, local, dirs=dirs, nvars=nvars)
        cache = {}

        def T(spec):
            if repr(spec) not in cache:
                cache[repr(spec)] = ddt.Type.from_spec(spec)
            return cache[repr(spec)]

        q = ddt.Queue()
        plans = []
        for arrs in arrays:
            sends = [(m["peer"], m["tag"], T(m["send_spec"]), arrs[m["var"]], 1) for m in msgs]
            recvs = [(m["recv_peer"], m["recv_tag"], T(m["recv_spec"]), arrs[m["var"]], 1) for m in msgs]
            mode = os.environ.get("PROBE_MODE", "nccl")  # p2p + DDT_SELF_VIA_WINDOW=1: the exchange kernel
            plans.append(ddt.Halo(q, ddt.Comm.single(0), sends, recvs, mode=mode, graph=(mode == "nccl")))
        S = sum(T(m["send_spec"]).size for m in msgs)
        return q, plans, S, len(msgs)
    finally:
        for k in knobs:
            os.environ.pop(k, None)
        ddt.reload_env()


def time_steps(plans, K):
    s = torch.cuda.current_stream()
    for k in range(4):
        plans[k % len(plans)].exchange()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for k in range(K):
        plans[k % len(plans)].exchange()
    b.record(s)
    torch.cuda.synchronize()
    return a.elapsed_time(b) * 1e3 / K


def main():
    torch.cuda.set_device(0)
    local, nvars, R = (512, 512, 512), 4, 2
    rounds, K = int(os.environ.get("PROBE_ROUNDS", "7")), int(os.environ.get("PROBE_K", "30"))
    classes = sys.argv[1:] or list(CLASSES)
    knob_sets = [{}, {"DDT_NO_GROUP": "1"}, {"DDT_UB": "1"}, {"DDT_UB": "2"}, {"DDT_ITEM_ORDER": "blocked"}]
    if os.environ.get("PROBE_KNOBS"):
        knob_sets = json.loads(os.environ["PROBE_KNOBS"])
    shape = tuple(n + 2 for n in local)
    arrays = []
    for _ in range(R):
        arrs = [torch.empty(shape, dtype=torch.int64, device="cuda") for _ in range(nvars)]
        for a in arrs:
            a.random_()
        arrays.append(arrs)
    variants = []
    for c in classes:
        for kn in knob_sets:
            q, plans, S, n = build(arrays, CLASSES[c], kn, nvars, local)
            variants.append(dict(cls=c, knobs=kn, q=q, plans=plans, S=S, n=n, t=[]))
    for _ in range(rounds):
        for v in variants:
            v["t"].append(time_steps(v["plans"], K))
    for v in variants:
        us = statistics.median(v["t"])
        print(json.dumps({"class": v["cls"], "knobs": v["knobs"], "msgs": v["n"], "S_bytes": v["S"],
                          "us": round(us, 2), "min_us": round(min(v["t"]), 2), "max_us": round(max(v["t"]), 2),
                          "alg_GBs": round(2 * v["S"] / us / 1e3, 1)}), flush=True)


if __name__ == "__main__":
    main()
