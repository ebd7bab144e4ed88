"""PCIe probe (diagnostic): how fast can the x-face cells of a 130^3 double
array in pinned HOST memory move to / from the device?
  zero-copy kernel : the library's DirectIPC of the two x faces on host arrays
  dma2d            : cudaMemcpy2DAsync of 16-B row ends (x = 0..1 or 128..129),
                     pitch 1040 B, one row per (z, y) of the interior (3-D copy
                     with 16-B width), host -> device and device -> host
  dma_dense        : one contiguous 128 KiB copy each way (the link's bulk rate)"""
import json
import os
import sys
import statistics

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from cuda.bindings import runtime as rt  # noqa: E402

torch.cuda.set_device(0)
s = torch.cuda.current_stream()
h = torch.zeros((130, 130, 130), dtype=torch.int64).pin_memory()
d = torch.zeros((130, 130, 130), dtype=torch.int64, device="cuda")
stage = torch.zeros((128 * 128, 2), dtype=torch.int64, device="cuda")


def timeit(fn, n=50):
    for _ in range(5):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(n):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        fn()
        b.record(s)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) * 1e3)
    return round(statistics.median(ts), 2)


def p3d(src_ptr, src_pitch, dst_ptr, dst_pitch, width, height, depth, kind, src_slice, dst_slice):
    prm = rt.cudaMemcpy3DParms()
    prm.srcPtr = rt.make_cudaPitchedPtr(src_ptr, src_pitch, width, src_slice // src_pitch)
    prm.dstPtr = rt.make_cudaPitchedPtr(dst_ptr, dst_pitch, width, dst_slice // dst_pitch)
    prm.extent = rt.make_cudaExtent(width, height, depth)
    prm.kind = kind
    return prm


row = 130 * 8
hp, dp = h.data_ptr(), d.data_ptr()
H2D, D2H = rt.cudaMemcpyKind.cudaMemcpyHostToDevice, rt.cudaMemcpyKind.cudaMemcpyDeviceToHost
# 16-B row ends of the interior rows: x = 0..1 at byte 0, 128..129 at byte 1024 of rows (z, y), z, y in 1..128
off = (1 * 130 + 1) * row
prm_in = p3d(hp + off, row, stage.data_ptr(), 16, 16, 128, 128, H2D, 130 * row, 128 * 16)
prm_out = p3d(stage.data_ptr(), 16, hp + off, row, 16, 128, 128, D2H, 128 * 16, 130 * row)
res = {}
res["dma3d_16B_rows_h2d_us"] = timeit(lambda: rt.cudaMemcpy3DAsync(prm_in, s.cuda_stream))
res["dma3d_16B_rows_d2h_us"] = timeit(lambda: rt.cudaMemcpy3DAsync(prm_out, s.cuda_stream))
dense_h = torch.zeros(128 * 1024, dtype=torch.uint8).pin_memory()
dense_d = torch.zeros(128 * 1024, dtype=torch.uint8, device="cuda")
res["dma_dense_128KiB_h2d_us"] = timeit(lambda: dense_d.copy_(dense_h, non_blocking=True))
res["dma_dense_128KiB_d2h_us"] = timeit(lambda: dense_h.copy_(dense_d, non_blocking=True))
res["rows"] = 128 * 128
print(json.dumps(res))
