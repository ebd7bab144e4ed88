"""Kernel launches per batch / per exchange, counted by CUPTI (torch.profiler)
-- the SURVEY §8(d) cross-check of the ncu launch lists (nsys is not in the
image).  For each workload: K iterations under the profiler, the number of
device kernels whose name starts with ddt_ divided by K, and every other
kernel seen inside the profiled region (there should be none).

usage: python tools/cupti_launches.py  -> one JSON document"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from torch.profiler import profile, ProfilerActivity  # noqa: E402

import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import halo_messages, FACE_DIRS, ALL_DIRS, config1_spec, config5_spec  # noqa: E402


def count(fn, K):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for _ in range(K):
            fn()
        torch.cuda.synchronize()
    names = {}
    for e in prof.events():
        if e.device_type.name == "CUDA" and not e.name.startswith(("Memcpy", "Memset", "cudaGraph")):
            names[e.name] = names.get(e.name, 0) + 1
    ours = sum(v for k, v in names.items() if "ddt_" in k)
    return {"iterations": K, "ddt_kernels_per_iter": ours / K,
            "other_kernels": {k: v for k, v in names.items() if "ddt_" not in k}}


def halo(local, dirs, nvars, mode):
    msgs = halo_messages(0, 1, local, dirs=dirs, nvars=nvars)
    arrs = [torch.zeros(tuple(n + 2 for n in local), dtype=torch.int64, device="cuda") for _ in range(nvars)]
    cache = {}

    def T(spec):
        if repr(spec) not in cache:
            cache[repr(spec)] = ddt.Type.from_spec(spec)
        return cache[repr(spec)]
    q = ddt.Queue()
    sends = [(m["peer"], m["tag"], T(m["send_spec"]), arrs[m["var"]], 1) for m in msgs]
    recvs = [(m["recv_peer"], m["recv_tag"], T(m["recv_spec"]), arrs[m["var"]], 1) for m in msgs]
    return q, ddt.Halo(q, ddt.Comm.single(0), sends, recvs, mode=mode, graph=False), len(msgs)


def main():
    torch.cuda.set_device(0)
    out = {}
    for name, local, dirs, nvars in [("configs[1] 128^3 faces", (128, 128, 128), FACE_DIRS, 1),
                                     ("configs[3] COMB 512^3 x 4 vars", (512, 512, 512), ALL_DIRS, 4)]:
        for mode in ("nccl", "p2p"):
            q, h, n = halo(local, dirs, nvars, mode)
            r = count(h.exchange, 20)
            r["messages_per_iter"] = 2 * n
            out[f"{name} exchange ({mode} plan, P=1)"] = r
            h.destroy()
            q.destroy()
            torch.cuda.empty_cache()
    # configs[0]: pack flush + unpack flush
    t = ddt.Type.from_spec(config1_spec())
    src = torch.zeros(8192, dtype=torch.uint8, device="cuda")
    pk = torch.zeros(512, dtype=torch.uint8, device="cuda")
    q = ddt.Queue()

    def c0():
        q.pack(t, src, 1, pk)
        q.flush()
        q.unpack(t, pk, 1, src)
        q.flush()
    out["configs[0] pack flush + unpack flush"] = count(c0, 50)
    # configs[4]: a fused batch of B requests = one launch
    S, B = 1 << 16, 256
    spec, fp = config5_spec(S)
    t5 = ddt.Type.from_spec(spec)
    s5 = torch.zeros((B, fp), dtype=torch.uint8, device="cuda")
    d5 = torch.zeros((B, S), dtype=torch.uint8, device="cuda")

    def c4():
        q.enqueue_many("pack", t5, list(s5), 1, list(d5))
        q.flush()
    r = count(c4, 20)
    r["requests_per_iter"] = B
    out[f"configs[4] fused batch of {B} x {S} B packs"] = r
    q.destroy()
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
