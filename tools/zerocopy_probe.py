"""Zero-copy halo exchange on HOST arrays: the fused kernel gathers the send
faces from and scatters the ghost faces into pinned host memory (UVA) -- only
the halo bytes cross PCIe -- against the staged flow (copy whole arrays
host->device, exchange, copy back).  configs[1] (128^3, 6 faces, P = 1) and
configs[3] (512^3 x 4 vars, 26 directions, P = 1).  Checks both flows agree.
usage: python tools/zerocopy_probe.py  -> JSON lines"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402
from ddt_inputs import halo_messages, FACE_DIRS, ALL_DIRS  # noqa: E402


def plan(q, comm, arrs, msgs, cache):
    def T(spec):
        k = repr(spec)
        if k not in cache:
            cache[k] = ddt.Type.from_spec(spec)
        return cache[k]
    sends = [(m["peer"], m["tag"], T(m["send_spec"]), arrs[m["var"]], 1) for m in msgs]
    recvs = [(m["recv_peer"], m["recv_tag"], T(m["recv_spec"]), arrs[m["var"]], 1) for m in msgs]
    return ddt.Halo(q, comm, sends, recvs, mode="nccl", graph=False)


def timeit(fn, K, stream):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(stream)
    for _ in range(K):
        fn()
    b.record(stream)
    torch.cuda.synchronize()
    return a.elapsed_time(b) / K * 1e3


def main():
    torch.cuda.set_device(0)
    stream = torch.cuda.current_stream()
    comm = ddt.Comm.single(0)
    for name, local, dirs, nvars, K in [("configs[1]", (128, 128, 128), FACE_DIRS, 1, 50),
                                       ("configs[3]", (512, 512, 512), ALL_DIRS, 4, 10)]:
        shape = tuple(n + 2 for n in local)
        msgs = halo_messages(0, 1, local, dirs=dirs, nvars=nvars)
        g = torch.Generator().manual_seed(5)
        hosts = [torch.randint(-2**62, 2**62, shape, dtype=torch.int64, generator=g).pin_memory()
                 for _ in range(nvars)]
        devs = [h.cuda() for h in hosts]
        outs = [torch.empty_like(h).pin_memory() for h in hosts]
        q = ddt.Queue()
        cache = {}
        hz = plan(q, comm, hosts, msgs, cache)   # zero-copy: the plan points at host memory
        hd = plan(q, comm, devs, msgs, cache)    # staged: the plan points at device copies

        def staged():
            for h, d in zip(hosts, devs):
                d.copy_(h, non_blocking=True)
            hd.exchange()
            for o, d in zip(outs, devs):
                o.copy_(d, non_blocking=True)

        us_z = timeit(hz.exchange, K, stream)
        us_s = timeit(staged, K, stream)
        us_d = timeit(hd.exchange, K, stream)
        torch.cuda.synchronize()
        ok = all(torch.equal(h, o) for h, o in zip(hosts, outs))
        halo_bytes = sum(cache[repr(m["send_spec"])].size for m in msgs)
        print(json.dumps({"workload": name, "zero_copy_us": round(us_z, 2), "staged_us": round(us_s, 2),
                          "device_us": round(us_d, 2), "agree": ok, "halo_bytes_each_way": halo_bytes,
                          "array_bytes": sum(h.numel() * 8 for h in hosts),
                          "zero_copy_GBs_each_way": round(halo_bytes / us_z / 1e3, 2)}), flush=True)
        hz.destroy()
        hd.destroy()
        q.destroy()


if __name__ == "__main__":
    main()
