"""Zero-copy requests on PINNED HOST buffers (include/ddt.h conventions: data
buffers may be page-locked host memory, which the fused kernel reads / writes
through unified addressing -- only the typemap's bytes cross PCIe).  Bit-exact
against the CPU oracle for pack (host source), unpack (host destination) and
DirectIPC (host -> host) in one fused batch each, and a halo exchange on host
arrays against numpy's periodic padding (the same pins as the device tests)."""
import numpy as np
import pytest

import oracle
from ddt_inputs import halo_messages, ghost_mask, FACE_DIRS, ALL_DIRS, random_bytes, SENTINEL, config1_spec, \
    config3_spec
from gpu_util import assert_bytes_equal

pytestmark = pytest.mark.gpu

SPECS = [
    config1_spec(),
    ("subarray", [10, 12, 14], [8, 10, 1], [1, 1, 12], "C", ("basic", "double")),
    ("subarray", [6, 7, 9], [4, 5, 7], [1, 1, 1], "F", ("basic", "float")),
    ("hvector", 5, 3, -40, ("basic", "int32")),
    ("indexed", [2, 0, 3, 1], [7, 1, 0, 12], ("basic", "double")),
    config3_spec(nblocks=2000, npoints=1 << 12)[0],
]


@pytest.fixture(scope="module")
def ddt():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_cluster_chukzsp20_b200.build import build
    build()
    import paper_conf_cluster_chukzsp20_b200 as m
    return m


def _pinned(arr):
    import torch
    return torch.from_numpy(np.ascontiguousarray(arr)).pin_memory()


@pytest.mark.parametrize("count", [1, 2])
def test_host_pack_unpack_direct(ddt, count):
    import torch
    q = ddt.Queue()
    cases = []
    for i, spec in enumerate(SPECS):
        o = oracle.Type(spec)
        t = ddt.Type.from_spec(spec)
        lo, hi = o.footprint(count)
        off = 64 - lo
        nb = hi - lo + 160
        src = random_bytes(nb, 300 + i)
        psrc = random_bytes(count * o.size + 16, 400 + i)
        cases.append(dict(o=o, t=t, off=off, nb=nb, src=src, psrc=psrc,
                          h_src=_pinned(src),
                          d_pk=torch.full((count * o.size + 16,), SENTINEL, dtype=torch.uint8, device="cuda"),
                          h_psrc=_pinned(psrc),
                          h_un=_pinned(np.full(nb, SENTINEL, np.uint8)),
                          h_dir=_pinned(np.full(nb, SENTINEL, np.uint8))))
    for c in cases:  # pack: host source -> device packed
        q.pack(c["t"], (c["h_src"], c["off"]), count, c["d_pk"])
    assert q.flush() == len(cases)
    for c in cases:  # unpack: host packed -> host destination; direct: host -> host
        q.unpack(c["t"], c["h_psrc"], count, (c["h_un"], c["off"]))
        q.direct(c["t"], (c["h_src"], c["off"]), count, c["t"], (c["h_dir"], c["off"]), count)
    assert q.flush() == 2 * len(cases)
    q.wait()
    for i, c in enumerate(cases):
        o, n = c["o"], count * c["o"].size
        exp_pk = np.full(n + 16, SENTINEL, np.uint8)
        exp_pk[:n] = oracle.pack(o, c["src"], count, c["off"])
        assert_bytes_equal(c["d_pk"].cpu().numpy(), exp_pk, f"host-source pack {i}")
        exp_un = np.full(c["nb"], SENTINEL, np.uint8)
        oracle.unpack(o, c["psrc"][:n], exp_un, count, c["off"])
        assert_bytes_equal(c["h_un"].numpy(), exp_un, f"host-destination unpack {i}")
        exp_dir = np.full(c["nb"], SENTINEL, np.uint8)
        oracle.unpack(o, exp_pk[:n], exp_dir, count, c["off"])
        assert_bytes_equal(c["h_dir"].numpy(), exp_dir, f"host->host direct {i}")
    q.destroy()


@pytest.mark.parametrize("local,dirs,nvars", [((9, 4, 3), FACE_DIRS, 1), ((5, 6, 7), ALL_DIRS, 2),
                                              ((32, 32, 32), FACE_DIRS, 1)])
def test_host_halo_exchange(ddt, local, dirs, nvars):
    import torch
    shape = tuple(n + 2 for n in local)
    arrs = []
    for v in range(nvars):
        a = np.full(shape, 0, np.int64)
        a.view(np.uint8)[...] = SENTINEL
        a[1:-1, 1:-1, 1:-1] = random_bytes(int(np.prod(local)) * 8, 50 + v).view(np.int64).reshape(local)
        arrs.append(_pinned(a))
    msgs = halo_messages(0, 1, local, dirs=dirs, nvars=nvars)
    cache = {}

    def T(spec):
        if repr(spec) not in cache:
            cache[repr(spec)] = ddt.Type.from_spec(spec)
        return cache[repr(spec)]
    q = ddt.Queue()
    sends = [(m["peer"], m["tag"], T(m["send_spec"]), arrs[m["var"]], 1) for m in msgs]
    recvs = [(m["recv_peer"], m["recv_tag"], T(m["recv_spec"]), arrs[m["var"]], 1) for m in msgs]
    h = ddt.Halo(q, ddt.Comm.single(torch.cuda.current_device()), sends, recvs, mode="nccl", graph=False)
    before = [a.numpy()[1:-1, 1:-1, 1:-1].copy() for a in arrs]
    h.exchange()
    torch.cuda.synchronize()
    gm = ghost_mask(local, dirs)
    for i, a in enumerate(arrs):
        x = a.numpy()
        assert np.array_equal(x[1:-1, 1:-1, 1:-1], before[i]), "interior modified"
        exp = np.pad(x[1:-1, 1:-1, 1:-1], 1, mode="wrap")
        assert np.array_equal(x[gm], exp[gm]), "ghosts differ from np.pad(wrap)"
        rest = ~gm
        rest[1:-1, 1:-1, 1:-1] = False
        assert np.all(x.view(np.uint8).reshape(x.shape + (8,))[rest] == SENTINEL)
    h.destroy()
    q.destroy()
