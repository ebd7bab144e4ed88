"""Vector-width probe (diagnostic, not a bench line): does the 8-B vector width
that 8-mod-16 rows force (halo faces: rows start at x = 1) cost bandwidth on
long dense rows?  Fused persistent-plan batches of 16 requests, each
hvector(8192 rows x 4096 B, stride 4112 B) = 32 MiB packed (1 GiB of
algorithmic bytes per launch, working set >> L2), in three shapes:
  pack16  : source 16-B aligned  -> w = 16
  pack8   : source at +8 B        -> w = 8
  direct8 : DirectIPC row gather -> row scatter, both at +8 B (the P = 1 face
            self message), w = 8; direct16: both aligned.
"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_cluster_chukzsp20_b200 as ddt  # noqa: E402

ROWS, ROWB, STRIDE, B = 8192, 4096, 4112, 16


def timed(plan, reps=15):
    s = torch.cuda.current_stream()
    for _ in range(3):
        plan.launch()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        plan.launch()
        b.record(s)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) * 1e3)
    return statistics.median(ts)


def main():
    torch.cuda.set_device(0)
    t = ddt.Type.hvector(ROWS, ROWB, STRIDE, ddt.Type.basic("byte")).commit()
    fp = ROWS * STRIDE + 64
    src = torch.empty((B, fp), dtype=torch.uint8, device="cuda")
    src.random_(0, 256)
    dst = torch.empty((B, fp), dtype=torch.uint8, device="cuda")
    pk = torch.empty((B, ROWS * ROWB + 64), dtype=torch.uint8, device="cuda")
    for name, off in [("pack16", 0), ("pack8", 8), ("direct16", 0), ("direct8", 8)]:
        q = ddt.Queue()
        for b in range(B):
            if name.startswith("pack"):
                q.pack(t, (src[b], off), 1, pk[b])
            else:
                q.direct(t, (src[b], off), 1, t, (dst[b], off), 1)
        plan = ddt.Plan(q)
        us = timed(plan)
        alg = 2.0 * B * ROWS * ROWB
        print(json.dumps({"variant": name, "us": round(us, 2), "alg_GBs": round(alg / us / 1e3, 1)}), flush=True)
        plan.destroy()
        q.destroy()


if __name__ == "__main__":
    main()
