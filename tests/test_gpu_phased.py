"""GPU parity of phased 16-B units (batch.cpp phase_batch): closed-form rows
whose start is 8 mod 16 on both sides move as [8-B head][16-B body][8-B tail]
instead of 8-B vectors.  Every case is bit-exact against the CPU oracle with
0xA5 sentinels around every footprint, and asserts whether the phased path was
taken (queue stats) so the test exercises what it claims."""
import numpy as np
import pytest

import oracle
from ddt_inputs import SENTINEL, random_bytes
from gpu_util import Case, cuda_bytes, host, assert_bytes_equal

pytestmark = pytest.mark.gpu

DOUBLE = ("basic", "double")


@pytest.fixture(scope="module")
def ddt():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_cluster_chukzsp20_b200.build import build
    build()
    import paper_conf_cluster_chukzsp20_b200 as m
    return m


@pytest.fixture(scope="module")
def q(ddt):
    return ddt.Queue()


def _pack_unpack(ddt, q, c, expect_phased):
    import torch
    ph0 = q.stats()["phased"]
    _, _, dp = c.gpu_pack(q)
    _, _, du = c.gpu_unpack(q)
    assert q.flush() == 2
    q.wait()
    torch.cuda.synchronize()
    assert_bytes_equal(host(dp), c.expect_pack(), f"pack {c.spec}")
    assert_bytes_equal(host(du), c.expect_unpack(), f"unpack {c.spec}")
    got = q.stats()["phased"] - ph0
    assert got == (2 if expect_phased else 0), (c.spec, got)


# (row bytes L, stride bytes, src misalign, packed misalign, phased?)
#   start 8, L = 8 + 16m + 8 -> head + tail.  Head-only / tail-only rows (L = 8 mod 16) phase only
#   when both sides are strided (DirectIPC): a packed side would alternate phase row to row.
ROWS = [
    (4096, 4112, 8, 8, True),     # a 512-double halo row at x = 1 (configs[1] / COMB faces)
    (1024, 1040, 8, 8, True),     # configs[1] 128^3 face row
    (48, 64, 8, 8, True),         # head + 2 body + tail (smallest phased case)
    (56, 80, 8, 8, False),        # L = 8 mod 16: packed rows would alternate phase (direct-only case)
    (40, 48, 0, 0, False),        # likewise
    (24, 32, 8, 8, False),        # m = 1 < 2: stays 8-B vectors
    (4096, 4112, 8, 0, False),    # packed side at another phase: 8-B vectors
    (4096, 4104, 8, 8, False),    # stride 8 mod 16: the phase flips row to row
]


@pytest.mark.parametrize("L,stride,mis,pkm,phased", ROWS)
@pytest.mark.parametrize("count", [1, 3])
def test_rows(ddt, q, L, stride, mis, pkm, phased, count):
    nrows = 37
    spec = ("hvector", nrows, L // 8, stride, DOUBLE)
    if count > 1:   # instances 16-B apart in phase: extent = (nrows-1)*stride + L, resize to a multiple of 16
        ext = ((nrows - 1) * stride + L + 15) // 16 * 16 + 16
        spec = ("resized", spec, 0, ext)
    c = Case(ddt, spec, count, misalign=mis, seed=L + stride + count, pk_misalign=pkm)
    _pack_unpack(ddt, q, c, phased and (count == 1 or stride % 16 == 0))


@pytest.mark.parametrize("sub", [((130, 130, 130), (1, 128, 128), (1, 1, 1)),     # z-face: 128 x 128 rows of 1 KiB
                                 ((130, 130, 130), (128, 1, 128), (1, 128, 1)),   # y-face
                                 ((20, 30, 42), (5, 7, 40), (3, 4, 1))])
def test_subarray_faces(ddt, q, sub):
    sizes, subsizes, starts = sub
    spec = ("subarray", list(sizes), list(subsizes), list(starts), "C", DOUBLE)
    # Case puts the footprint's first byte (row 0 of the face, x = 1) at 64 + misalign
    c = Case(ddt, spec, 1, misalign=8, seed=7, pk_misalign=8)
    _pack_unpack(ddt, q, c, True)


def test_contiguous_both_at_8(ddt, q):
    c = Case(ddt, ("contiguous", 1001, DOUBLE), 1, misalign=8, seed=3, pk_misalign=8)
    _pack_unpack(ddt, q, c, True)


def _direct_case(ddt, q, sspec, dspec, smis, dmis, seed_):
    """DirectIPC src layout -> dst layout; returns (got, expected) host bytes."""
    import torch
    so, do = oracle.Type(sspec), oracle.Type(dspec)
    st, dt = ddt.Type.from_spec(sspec), ddt.Type.from_spec(dspec)
    slo, shi = so.footprint(1)
    dlo, dhi = do.footprint(1)
    sbuf = random_bytes(shi - slo + 128, seed_)
    soff = 32 - slo + smis
    doff = 32 - dlo + dmis
    dn = dhi - dlo + 128
    gs = cuda_bytes(sbuf)
    gd = torch.full((dn,), SENTINEL, dtype=torch.uint8, device="cuda")
    q.direct(st, (gs, soff), 1, dt, (gd, doff), 1)
    _keep.append(gs)  # the caller owns the source until the request completes
    return gd, (so, sbuf, soff), (do, dn, doff)


_keep = []


def test_direct_faces_and_mixed_batch(ddt, q):
    """P = 1 self messages of a 130^3 halo in ONE flush: four phased face rows
    (z / y faces, send layer -> ghost layer) plus two 8-B x-face cell messages
    that stay plain vectors -> the runtime-width phased variant."""
    import torch
    n = 130
    sizes = [n, n, n]

    def sub(subsizes, starts):
        return ("subarray", sizes, subsizes, starts, "C", DOUBLE)

    pairs = [(sub([1, 128, 128], [1, 1, 1]), sub([1, 128, 128], [129, 1, 1])),
             (sub([1, 128, 128], [128, 1, 1]), sub([1, 128, 128], [0, 1, 1])),
             (sub([128, 1, 128], [1, 1, 1]), sub([128, 1, 128], [1, 129, 1])),
             (sub([128, 1, 128], [1, 128, 1]), sub([128, 1, 128], [1, 0, 1])),
             (sub([128, 128, 1], [1, 1, 1]), sub([128, 128, 1], [1, 1, 129])),
             (sub([128, 128, 1], [1, 1, 128]), sub([128, 128, 1], [1, 1, 0]))]
    ph0 = q.stats()["phased"]
    # _direct_case puts each footprint's first byte (x = 1 for the faces) at 32 + misalign
    cases = [_direct_case(ddt, q, s, d, 8, 8, 40 + i) for i, (s, d) in enumerate(pairs)]
    assert q.flush() == len(pairs)
    q.wait()
    torch.cuda.synchronize()
    assert q.stats()["phased"] - ph0 == 4
    for gd, (so, sbuf, soff), (do, dn, doff) in cases:
        exp = np.full(dn, SENTINEL, np.uint8)
        oracle.unpack(do, oracle.pack(so, sbuf, 1, soff), exp, 1, doff)
        assert_bytes_equal(host(gd), exp, "direct")


def test_direct_different_strides_same_rows(ddt, q):
    """Both sides strided with equal row length but different strides / dims."""
    import torch
    sspec = ("hvector", 64, 64, 1040, DOUBLE)                    # 64 rows of 512 B
    dspec = ("subarray", [8, 9, 80], [8, 8, 64], [0, 1, 3], "C", DOUBLE)  # 64 rows of 512 B at x = 3
    ph0 = q.stats()["phased"]
    gd, (so, sbuf, soff), (do, dn, doff) = _direct_case(ddt, q, sspec, dspec, 8, 8, 5)
    q.flush()
    q.wait()
    torch.cuda.synchronize()
    assert q.stats()["phased"] - ph0 == 1
    exp = np.full(dn, SENTINEL, np.uint8)
    oracle.unpack(do, oracle.pack(so, sbuf, 1, soff), exp, 1, doff)
    assert_bytes_equal(host(gd), exp, "direct strided")


def test_no_phase_knob_same_bytes(ddt, monkeypatch):
    """DDT_NO_PHASE=1 (A/B knob) gives the same bytes through plain vectors."""
    import torch
    monkeypatch.setenv("DDT_NO_PHASE", "1")
    q2 = ddt.Queue()
    c = Case(ddt, ("hvector", 37, 512, 4112, DOUBLE), 1, misalign=8, seed=11, pk_misalign=8)
    _pack_unpack(ddt, q2, c, False)
    q2.destroy()


@pytest.mark.parametrize("L,sstride,dstride,mis,phased", [
    (56, 80, 96, 8, True),     # head + 3 body units, no tail
    (40, 48, 64, 0, True),     # 2 body units + tail
    (56, 80, 88, 8, False),    # destination stride 8 mod 16
])
def test_direct_head_or_tail_only(ddt, q, L, sstride, dstride, mis, phased):
    import torch
    sspec = ("hvector", 29, L // 8, sstride, DOUBLE)
    dspec = ("hvector", 29, L // 8, dstride, DOUBLE)
    ph0 = q.stats()["phased"]
    gd, (so, sbuf, soff), (do, dn, doff) = _direct_case(ddt, q, sspec, dspec, mis, mis, 9)
    q.flush()
    q.wait()
    torch.cuda.synchronize()
    assert q.stats()["phased"] - ph0 == (1 if phased else 0)
    exp = np.full(dn, SENTINEL, np.uint8)
    oracle.unpack(do, oracle.pack(so, sbuf, 1, soff), exp, 1, doff)
    assert_bytes_equal(host(gd), exp, "direct head/tail")


def test_narrow_list_batch_device_table(ddt):
    """40 sparse 4-B-vector list requests in one flush: the device-table form of
    the narrow-list variant (8 loads in flight per thread), pack then unpack."""
    import torch
    from ddt_inputs import config3_spec
    q2 = ddt.Queue()
    cases = [Case(ddt, config3_spec(nblocks=700, npoints=1 << 12, s=100 + i, shuffled=(i % 3 == 0))[0], 1 + i % 2,
                  misalign=4 * (i % 4), seed=i, pk_misalign=4 * (i % 2)) for i in range(40)]
    outs = [c.gpu_pack(q2) for c in cases]
    assert q2.flush() == 40
    ins = [c.gpu_unpack(q2) for c in cases]
    assert q2.flush() == 40
    q2.wait()
    torch.cuda.synchronize()
    for c, (_, _, dp), (_, _, du) in zip(cases, outs, ins):
        assert_bytes_equal(host(dp), c.expect_pack(), "narrow pack")
        assert_bytes_equal(host(du), c.expect_unpack(), "narrow unpack")
    assert q2.stats()["launches"] == 2
    q2.destroy()
