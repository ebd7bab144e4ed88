"""Diagnostic: can two ranks on ONE GPU form an NCCL communicator (the
library's NCCL-mode data path at nranks > 1)?  Prints each rank's result."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
from mp_util import free_port, init  # noqa: E402


def worker(rank, world, port, q):
    try:
        init(rank, world, port)
        import torch
        torch.cuda.set_device(0)
        import paper_conf_cluster_chukzsp20_b200 as ddt
        c = ddt.Comm.from_torch(0, nccl=True)
        q.put((rank, "ok: NCCL communicator of 2 ranks on one GPU created"))
        c.close()
    except Exception as e:
        q.put((rank, f"{type(e).__name__}: {e}"))


if __name__ == "__main__":
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    ps = [ctx.Process(target=worker, args=(r, 2, port, q)) for r in range(2)]
    [p.start() for p in ps]
    for _ in range(2):
        print(q.get(timeout=120), flush=True)
    [p.join(30) for p in ps]
