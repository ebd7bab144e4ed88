"""Debug (scratch): the SM-occupancy exchange test with progress reporting."""
import ctypes, os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
os.environ["DDT_SELF_VIA_WINDOW"] = "1"; os.environ["DDT_NO_LL"] = "1"
import torch
import paper_conf_cluster_chukzsp20_b200 as ddt
from gpu_util import occupier
from test_gpu_exchange_protocols import Plan
from ddt_inputs import ALL_DIRS
occ = occupier()
nsm = torch.cuda.get_device_properties(0).multi_processor_count
local = tuple(int(x) for x in os.environ.get("LOCAL", "64,128,128").split(","))
p = Plan(ddt, local, ALL_DIRS, 2, "p2p")
p.h.set_timeout(2.0)
rd = p.h.trace(200000)
p.fill(0); p.h.exchange(); p.check("warm")
print("warm trace records", len(rd()), flush=True)
rd = p.h.trace(200000)
p.fill(1); torch.cuda.synchronize()
stop = torch.zeros(1, dtype=torch.int32).pin_memory()
s_occ = torch.cuda.Stream()
ctas = 2 * nsm - int(os.environ.get("FREE", "1"))
started = torch.zeros(ctas, dtype=torch.int32).pin_memory()
occ.occupy_launch(ctypes.c_void_p(s_occ.cuda_stream), ctas, 1024, ctypes.c_void_p(stop.data_ptr()),
                  ctypes.c_void_p(started.data_ptr()), int(30e9))
t0 = time.time()
while int(started.sum()) < ctas and time.time() - t0 < 10:
    time.sleep(0.001)
print("occupier resident", int(started.sum()), flush=True)
p.h.exchange()
ds = torch.cuda.current_stream()
trace_buf = p.h._trace_buf
for i in range(8):
    time.sleep(1.0)
    # trace counter lives in the control block; read records already written via a copy on another stream
    s2 = torch.cuda.Stream()
    with torch.cuda.stream(s2):
        host = trace_buf[: 48 * 200000].to("cpu", non_blocking=False)
    import numpy as np
    rec = host.numpy().view(np.uint64).reshape(-1, 6)
    n = int((rec[:, 5] > 0).sum())
    print(f"t={i+1}s done_items={n} finished={ds.query()}", flush=True)
    if ds.query():
        break
stop[0] = 1
torch.cuda.synchronize()
print("after stop: records", len(rd()), flush=True)
