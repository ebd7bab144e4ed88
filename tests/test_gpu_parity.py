"""GPU parity: the CUDA path through the C ABI vs the CPU oracle, bit-exact
(zero tolerance: pure byte movement), with 0xA5 sentinels
outside every footprint.  Covers random nested types, misaligned pointers,
count > 1, the BASELINE.json configs 1, 3, 5 at full size, fused mixed
batches (one launch per flush), the request-list states and limits."""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st, HealthCheck

import oracle
from ddt_inputs import (random_bytes, SENTINEL, config1_spec, config3_spec, config5_spec, seed)
from gpu_util import Case, cuda_bytes, host, assert_bytes_equal

pytestmark = pytest.mark.gpu


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


def _run_case(ddt, q, c: Case):
    import torch
    launches0 = q.stats()["launches"]
    uid_p, _, dp = c.gpu_pack(q)
    uid_u, _, du = c.gpu_unpack(q)
    n = q.flush()
    assert n == 2
    q.wait()
    assert q.query(uid_p) == "completed" and q.query(uid_u) == "completed"
    torch.cuda.synchronize()
    assert_bytes_equal(host(dp), c.expect_pack(), f"pack {c.spec} count={c.count}")
    if not c.o.num_entries or not _overlaps(c):
        assert_bytes_equal(host(du), c.expect_unpack(), f"unpack {c.spec} count={c.count}")
    assert q.stats()["launches"] - launches0 == (1 if c.psize else 0)


def _overlaps(c):
    d, ln = c.o.typemap(c.count)
    b = np.concatenate([np.arange(a, a + n) for a, n in zip(d, ln)]) if len(d) else np.zeros(0)
    return len(np.unique(b)) != len(b)


# --------------------------------------------------------------- random types
from test_abi_cpu import spec_strategy  # noqa: E402


@settings(max_examples=250, deadline=None, suppress_health_check=list(HealthCheck))
@given(spec=spec_strategy(), count=st.integers(1, 3), mis=st.integers(0, 15), pkm=st.sampled_from([0, 0, 4, 8, 1]),
       s=st.integers(0, 1000))
def test_random_types_bit_exact(ddt, q, spec, count, mis, pkm, s):
    c = Case(ddt, spec, count, misalign=mis, seed=s, pk_misalign=pkm)
    if c.psize and _overlaps(c):
        # unpack into overlapping entries is rejected (R5); pack still parity-checked
        import torch
        uid, _, dp = c.gpu_pack(q)
        q.flush()
        q.wait()
        assert_bytes_equal(host(dp), c.expect_pack(), f"pack {spec}")
        from paper_conf_cluster_chukzsp20_b200 import DDTError
        with pytest.raises(DDTError):
            c.gpu_unpack(q)
        return
    _run_case(ddt, q, c)


# --------------------------------------------------------------- config 1
@pytest.mark.parametrize("count", [1, 2, 5])
@pytest.mark.parametrize("mis", [0, 8, 3])
def test_config1_vector(ddt, q, count, mis):
    _run_case(ddt, q, Case(ddt, config1_spec(), count, misalign=mis, seed=seed(1)))


def test_config1_golden_values(ddt, q):
    """Labelled source: the packed doubles are the golden byte offsets."""
    import torch
    t = ddt.Type.from_spec(config1_spec())
    lab = torch.arange(1000, dtype=torch.int64, device="cuda") * 8
    out = torch.zeros(64, dtype=torch.int64, device="cuda")
    q.pack(t, lab, 1, out)
    q.wait()
    exp = np.concatenate([np.arange(512 * i, 512 * i + 32, 8) for i in range(16)])
    assert host(out).tolist() == exp.tolist()


# --------------------------------------------------------------- config 3
@pytest.mark.parametrize("shuffled", [False, True])
def test_config3_sparse_hindexed_full(ddt, q, shuffled):
    """10^5 blocks of 3 floats over 2^20 points (12 MiB source), batch of 4
    requests with distinct sources, all in one launch."""
    import torch
    spec, nb = config3_spec(shuffled=shuffled)
    t = ddt.Type.from_spec(spec)
    o = oracle.Type(spec)
    assert t.layout_kind == "uniform_list"
    B = 4
    srcs = [random_bytes(nb, seed(3, v)) for v in range(B)]
    d_src = [cuda_bytes(s) for s in srcs]
    d_pk = [torch.full((t.size,), SENTINEL, dtype=torch.uint8, device="cuda") for _ in range(B)]
    d_un = [torch.full((nb,), SENTINEL, dtype=torch.uint8, device="cuda") for _ in range(B)]
    l0 = q.stats()["launches"]
    for v in range(B):
        q.pack(t, d_src[v], 1, d_pk[v])
    q.flush()
    for v in range(B):
        q.unpack(t, d_pk[v], 1, d_un[v])
    q.flush()
    q.wait()
    assert q.stats()["launches"] - l0 == 2
    for v in range(B):
        exp = oracle.pack(o, srcs[v])
        assert_bytes_equal(host(d_pk[v]), exp, "config3 pack")
        eu = np.full(nb, SENTINEL, np.uint8)
        oracle.unpack(o, exp, eu)
        assert_bytes_equal(host(d_un[v]), eu, "config3 unpack")


# --------------------------------------------------------------- config 5
@pytest.mark.parametrize("S,B", [(64, 1), (64, 64), (1024, 16), (16384, 4), (262144, 16), (4 << 20, 4),
                                 (64 << 20, 1)])
def test_config5_dense_vector_batches(ddt, q, S, B):
    """Message-size sweep cells: B requests of S bytes, fused pack then fused
    unpack; every request checked against the oracle."""
    import torch
    spec, fp = config5_spec(S)
    t = ddt.Type.from_spec(spec)
    o = oracle.Type(spec)
    srcs = [random_bytes(fp, seed(5, i)) for i in range(B)]
    d_src = [cuda_bytes(s) for s in srcs]
    d_pk = [torch.full((S,), SENTINEL, dtype=torch.uint8, device="cuda") for _ in range(B)]
    d_un = [torch.full((fp,), SENTINEL, dtype=torch.uint8, device="cuda") for _ in range(B)]
    for i in range(B):
        q.pack(t, d_src[i], 1, d_pk[i])
    assert q.flush() == B
    for i in range(B):
        q.unpack(t, d_pk[i], 1, d_un[i])
    assert q.flush() == B
    q.wait()
    for i in range(B):
        exp = oracle.pack(o, srcs[i])
        assert_bytes_equal(host(d_pk[i]), exp, f"config5 pack S={S}")
        eu = np.full(fp, SENTINEL, np.uint8)
        oracle.unpack(o, exp, eu)
        assert_bytes_equal(host(d_un[i]), eu, f"config5 unpack S={S}")


# --------------------------------------------------------------- batches / scheduler
def test_mixed_batch_one_launch_equals_sequential_oracle(ddt, q):
    """A fused batch of 96 mixed pack/unpack requests of different types is ONE
    launch and equals the oracle executing the requests one by one (R6)."""
    import torch
    rng = np.random.default_rng(7)
    specs = [config1_spec(), ("subarray", [9, 10, 11], [3, 4, 5], [1, 2, 3], "C", ("basic", "double")),
             ("subarray", [9, 10, 11], [9, 1, 11], [0, 4, 0], "F", ("basic", "float")),
             ("hindexed", [3, 1, 2], [100, 4, 37], ("basic", "byte")),
             ("indexed", [1, 2, 3], [0, 10, 20], ("basic", "int32")),
             ("vector", 5, 3, -4, ("basic", "int64"))]
    cases = [Case(ddt, specs[i % len(specs)], count=int(rng.integers(1, 4)), misalign=int(rng.integers(0, 16)),
                  seed=i) for i in range(96)]
    bufs = []
    l0 = q.stats()["launches"]
    for i, c in enumerate(cases):
        bufs.append(c.gpu_pack(q) if i % 2 == 0 else c.gpu_unpack(q))
    assert q.flush() == 96
    q.wait()
    assert q.stats()["launches"] - l0 == 1
    for i, (c, (_, _, d)) in enumerate(zip(cases, bufs)):
        exp = c.expect_pack() if i % 2 == 0 else c.expect_unpack()
        assert_bytes_equal(host(d), exp, f"batch item {i}")


def test_shared_buffer_batch_equals_oracle_run_batch(ddt, q):
    """One fused launch of 48 packs of mixed layouts into disjoint slices of ONE
    packed buffer, then one launch of 48 unpacks from ONE packed buffer into
    disjoint regions of ONE destination array: byte-equal to oracle.run_batch
    (the requests executed one by one on the host, R6)."""
    import torch
    specs = [config1_spec(), ("subarray", [9, 10, 11], [3, 4, 5], [1, 2, 3], "C", ("basic", "double")),
             ("hindexed", [3, 1, 2], [100, 4, 37], ("basic", "byte")),
             ("struct", [1, 2, 1], [0, 8, 24], [("basic", "byte"), ("basic", "double"), ("basic", "int32")]),
             ("vector", 5, 3, -4, ("basic", "int64"))]
    rng = np.random.default_rng(11)
    src = random_bytes(1 << 20, 12)
    ots = [oracle.Type(sp) for sp in specs]
    tts = [ddt.Type.from_spec(sp) for sp in specs]
    reqs, pk_off, src_offs = [], 16, []
    for i in range(48):
        k = i % len(specs)
        cnt = int(rng.integers(1, 4))
        lo, hi = ots[k].footprint(cnt)
        so = int(rng.integers(0, (1 << 20) - (hi - lo) - 64)) - lo
        reqs.append(dict(op="pack", type=ots[k], count=cnt, src=src, src_offset=so, dst=None, dst_offset=pk_off, k=k))
        pk_off += cnt * ots[k].size + int(rng.integers(0, 9))
    packed_h = np.full(pk_off + 64, SENTINEL, np.uint8)
    for r in reqs:
        r["dst"] = packed_h
    s_d = cuda_bytes(src)
    p_d = torch.full((pk_off + 64,), SENTINEL, dtype=torch.uint8, device="cuda")
    l0 = q.stats()["launches"]
    for r in reqs:
        q.pack(tts[r["k"]], (s_d, r["src_offset"]), r["count"], (p_d, r["dst_offset"]))
    assert q.flush() == 48
    oracle.run_batch([{k: v for k, v in r.items() if k != "k"} for r in reqs])
    q.wait()
    assert q.stats()["launches"] - l0 == 1
    assert_bytes_equal(host(p_d), packed_h, "shared packed buffer")
    # unpacks: instances placed back to back (disjoint footprints) in one array
    dst_h = np.full(1 << 21, SENTINEL, np.uint8)
    ureqs, pos = [], 128
    for r in reqs:
        t = r["type"]
        lo, hi = t.footprint(r["count"])
        ureqs.append(dict(op="unpack", type=t, count=r["count"], src=packed_h, src_offset=r["dst_offset"],
                          dst=dst_h, dst_offset=pos - lo, k=r["k"]))
        pos += (hi - lo) + 8
    d_d = torch.full((1 << 21,), SENTINEL, dtype=torch.uint8, device="cuda")
    for r in ureqs:
        q.unpack(tts[r["k"]], (p_d, r["src_offset"]), r["count"], (d_d, r["dst_offset"]))
    q.flush()
    oracle.run_batch([{k: v for k, v in r.items() if k != "k"} for r in ureqs])
    q.wait()
    assert_bytes_equal(host(d_d), dst_h, "shared destination array")


def test_queue_full_gives_negative_uid_then_recovers(ddt):
    import torch
    q4 = ddt.Queue(capacity=4)
    t = ddt.Type.from_spec(config1_spec())
    s = torch.zeros(8192, dtype=torch.uint8, device="cuda")
    d = torch.zeros(512 * 8, dtype=torch.uint8, device="cuda")
    uids = [q4.pack(t, s, 1, (d, 512 * i)) for i in range(4)]
    assert uids == [0, 1, 2, 3]
    assert q4.try_pack(t, s, 1, d) == -3  # DDT_ERR_QUEUE_FULL: the paper's negative UID
    assert q4.query(3) == "pending"
    q4.flush()
    q4.wait()
    assert all(q4.query(u) == "completed" for u in uids)
    assert q4.pack(t, s, 1, d) == 4
    q4.wait()
    q4.destroy()


def test_enqueue_many_equals_oracle_and_stops_at_full_ring(ddt):
    """ddt_enqueue_many: 40 mixed-type packs in one call, then 40 unpacks, two
    launches, bit-exact vs the oracle; on a ring of 24 the bulk call stops at
    the first DDT_ERR_QUEUE_FULL (returned for that request), the caller
    flushes and resubmits the rest."""
    import torch
    specs = [config1_spec(), ("subarray", [9, 10, 11], [3, 4, 5], [1, 2, 3], "C", ("basic", "double")),
             ("hindexed", [3, 1, 2], [100, 4, 37], ("basic", "byte")), ("vector", 5, 3, -4, ("basic", "int64"))]
    cases = [Case(ddt, specs[i % len(specs)], count=1 + i % 3, misalign=i % 16, seed=500 + i) for i in range(40)]
    srcs = [cuda_bytes(c.src) for c in cases]
    pks = [torch.full((c.psize + 32,), SENTINEL, dtype=torch.uint8, device="cuda") for c in cases]
    psrcs = [cuda_bytes(c.packed_src) for c in cases]
    uns = [torch.full((c.nbytes,), SENTINEL, dtype=torch.uint8, device="cuda") for c in cases]
    for cap in (0, 24):
        qq = ddt.Queue(capacity=cap)
        for p in pks:
            p.fill_(SENTINEL)
        for u in uns:
            u.fill_(SENTINEL)
        for op, ins, outs in (("pack", [(s, c.off) for s, c in zip(srcs, cases)], [(p, c.pk_off) for p, c in zip(pks, cases)]),
                              ("unpack", [(s, c.pk_off) for s, c in zip(psrcs, cases)], [(u, c.off) for u, c in zip(uns, cases)])):
            k0, partial = 0, 0
            while k0 < len(cases):
                k, uids = qq.try_enqueue_many(op, [c.t for c in cases[k0:]], ins[k0:],
                                              [c.count for c in cases[k0:]], outs[k0:])
                if k0 + k < len(cases):
                    assert cap and uids[k] == -3, (k, uids[k])  # DDT_ERR_QUEUE_FULL for request k
                    partial += 1
                k0 += k
                qq.wait()  # flush + completion frees the ring
            assert partial == (0 if not cap else (len(cases) - 1) // cap)
        for i, c in enumerate(cases):
            assert_bytes_equal(host(pks[i]), c.expect_pack(), f"enqueue_many pack {i} cap={cap}")
            assert_bytes_equal(host(uns[i]), c.expect_unpack(), f"enqueue_many unpack {i} cap={cap}")
        qq.destroy()


@pytest.mark.parametrize("mode", ["0", "1", "2"])
def test_grid_modes_bit_exact_and_reusable(ddt, mode, monkeypatch):
    """Every multi-wave work distribution (static order, dynamic item tickets,
    one CTA per item) gives the oracle's bytes, and the ticket
    counter is reset between launches: three flushes and three launches of a
    plan of the same 8 x 8 MiB batch (4096 items) all match."""
    import torch
    monkeypatch.setenv("DDT_GRID_MODE", mode)
    S, B = 8 << 20, 8
    spec, fp = config5_spec(S)
    o = oracle.Type(spec)
    t = ddt.Type.from_spec(spec)
    srcs = [random_bytes(fp, 900 + b) for b in range(B)]
    exp = [oracle.pack(o, x) for x in srcs]
    d_src = [cuda_bytes(x) for x in srcs]
    d_dst = [torch.empty(S, dtype=torch.uint8, device="cuda") for _ in range(B)]
    qq = ddt.Queue()

    def check(what):
        torch.cuda.synchronize()
        for b in range(B):
            assert_bytes_equal(host(d_dst[b]), exp[b], f"{what} mode={mode} request {b}")
            d_dst[b].fill_(SENTINEL)

    for it in range(3):
        qq.enqueue_many("pack", t, d_src, 1, d_dst)
        assert qq.flush() == B
        check(f"flush {it}")
    qq.enqueue_many("pack", t, d_src, 1, d_dst)
    plan = ddt.Plan(qq)
    for it in range(3):
        plan.launch()
        check(f"plan launch {it}")
    plan.destroy()
    qq.destroy()


@pytest.mark.parametrize("blk,base,count,shuffled", [(3, "float", 1, False), (3, "float", 2, True),
                                                     (2, "int32", 3, False), (4, "float", 1, True),
                                                     (1, "int32", 2, False), (3, "float", 1, "far")])
def test_segment_per_thread_variant(ddt, blk, base, count, shuffled):
    """Variant 10 (one whole <= 16-B segment per thread, uniform lists; DESIGN.md
    §7k) for pack and unpack in one batch each, several segment sizes, count > 1,
    shuffled block order and int64 offsets ("far": displacements beyond 2^31)."""
    import torch
    rng = np.random.default_rng(77 + blk)
    n = 3000
    npts = 1 << 15
    idx = np.sort(rng.choice(npts, n, replace=False))
    if shuffled is True:
        rng.shuffle(idx)
    disp = [int(i) * 4 * blk for i in idx]
    if shuffled == "far":
        disp = [d + (1 << 31) for d in disp]
    spec = ("hindexed", [blk] * n, disp, ("basic", base))
    cases = [Case(ddt, spec, count=count, misalign=4 * k, seed=700 + k) for k in range(3)]
    q = ddt.Queue()
    outs = [c.gpu_pack(q) for c in cases]
    q.flush()
    q.wait()
    for c, (_, _, d) in zip(cases, outs):
        assert_bytes_equal(host(d), c.expect_pack(), f"segment pack blk={blk}")
    outs = [c.gpu_unpack(q) for c in cases]
    q.flush()
    q.wait()
    for c, (_, _, d) in zip(cases, outs):
        assert_bytes_equal(host(d), c.expect_unpack(), f"segment unpack blk={blk}")
    q.destroy()


def test_pdl_launches_respect_stream_order(ddt):
    """Programmatic dependent launch keeps every stream
    dependency: 40 rounds of [torch kernel writes the source] -> [ddt pack
    flush] -> [ddt unpack flush of that packed buffer] -> [torch kernel reads
    the result], all on one stream with no host synchronisation, each round's
    bytes checked afterwards against the oracle (a PDL kernel that ran ahead of
    its predecessor would read the previous round's values)."""
    import torch
    spec = ("subarray", [20, 24, 28], [18, 22, 1], [1, 1, 26], "C", ("basic", "double"))
    o = oracle.Type(spec)
    t = ddt.Type.from_spec(spec)
    lo, hi = o.footprint(1)
    q = ddt.Queue()
    src = torch.empty(hi + 64, dtype=torch.uint8, device="cuda")
    pk = torch.empty(o.size, dtype=torch.uint8, device="cuda")
    out = torch.empty(hi + 64, dtype=torch.uint8, device="cuda")
    snaps = []
    for k in range(40):
        src.fill_((7 * k + 3) & 0xFF)                # torch kernel writes the source
        src[k: k + 8].fill_(k)                       # and a second, dependent one
        out.fill_(0xA5)
        q.pack(t, src, 1, pk)
        q.flush()                                    # reads src
        q.unpack(t, pk, 1, out)
        q.flush()                                    # reads pk written by the previous kernel
        snaps.append(out.clone())                    # torch kernel reads the result
    torch.cuda.synchronize()
    for k, got in enumerate(snaps):
        s_host = np.full(hi + 64, (7 * k + 3) & 0xFF, np.uint8)
        s_host[k: k + 8] = k
        exp = np.full(hi + 64, 0xA5, np.uint8)
        oracle.unpack(o, oracle.pack(o, s_host), exp)
        assert_bytes_equal(host(got), exp, f"round {k}")
    q.destroy()


def test_pdl_read_after_write_inside_a_captured_graph(ddt):
    """Inside ONE captured CUDA graph (programmatic edges between consecutive
    ddt kernels): 30 rounds of [pack A -> packed buffer] -> [unpack of that
    buffer into B] -> [pack of B's typemap -> a per-round buffer], each kernel
    reading what its immediate predecessor wrote (persistent plans launched
    during capture), so a load scheduled above griddepcontrol.wait would read
    the previous round's bytes; torch kernels rewrite the source between
    rounds.  Every round is checked vs the oracle."""
    import torch
    spec = ("vector", 64, 3, 7, ("basic", "double"))
    o = oracle.Type(spec)
    t = ddt.Type.from_spec(spec)
    lo, hi = o.footprint(1)
    R = 30
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        q = ddt.Queue()
        src = torch.empty(hi, dtype=torch.uint8, device="cuda")
        pk = torch.empty(o.size, dtype=torch.uint8, device="cuda")
        mid = torch.empty(hi, dtype=torch.uint8, device="cuda")
        pk2 = torch.empty((R, o.size), dtype=torch.uint8, device="cuda")
        q.pack(t, src, 1, pk)
        p_pack = ddt.Plan(q)
        q.unpack(t, pk, 1, mid)
        p_unpack = ddt.Plan(q)
        p_out = []
        for k in range(R):
            q.pack(t, mid, 1, pk2[k])
            p_out.append(ddt.Plan(q))
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for k in range(R):
                src.fill_((11 * k + 5) & 0xFF)
                src[k: k + 16].fill_(k)
                mid.fill_(0xA5)
                p_pack.launch()
                p_unpack.launch()
                p_out[k].launch()
        g.replay()
    torch.cuda.synchronize()
    got = pk2.cpu().numpy()
    for k in range(R):
        s_host = np.full(hi, (11 * k + 5) & 0xFF, np.uint8)
        s_host[k: k + 16] = k
        assert_bytes_equal(got[k], oracle.pack(o, s_host), f"round {k}")
    del g
    for p_ in [p_pack, p_unpack] + p_out:
        p_.destroy()
    q.destroy()


def test_ring_reclaim_with_many_inflight_batches(ddt):
    """A 64-slot ring driven by 300 one-request flushes with no host wait: the
    ring fills repeatedly and enqueue reclaims completed batches (newest-first
    query + binary search over the in-order batches); every uid ends COMPLETED
    and every packed result equals the oracle."""
    import torch
    qq = ddt.Queue(capacity=64)
    spec = config1_spec()
    o = oracle.Type(spec)
    t = ddt.Type.from_spec(spec)
    srcs = [random_bytes(8192, 1200 + i) for i in range(8)]
    d_src = [cuda_bytes(x) for x in srcs]
    outs = torch.full((300, o.size), SENTINEL, dtype=torch.uint8, device="cuda")
    uids = []
    for i in range(300):
        uids.append(qq.pack(t, d_src[i % 8], 1, outs[i]))
        assert qq.flush() == 1
    qq.wait()
    assert all(qq.query(u) == "completed" for u in uids)
    got = outs.cpu().numpy()
    for i in range(300):
        assert_bytes_equal(got[i], oracle.pack(o, srcs[i % 8]), f"request {i}")
    qq.destroy()


def test_zero_size_and_empty_requests(ddt, q):
    import torch
    t = ddt.Type.from_spec(("vector", 0, 3, 2, ("basic", "double")))
    s = torch.zeros(16, dtype=torch.uint8, device="cuda")
    uid = q.pack(t, s, 5, s)
    assert q.query(uid) == "completed"
    t1 = ddt.Type.from_spec(config1_spec())
    uid2 = q.pack(t1, s, 0, s)
    assert q.query(uid2) == "completed"
    l0 = q.stats()["launches"]
    q.flush()
    q.wait()
    assert q.stats()["launches"] == l0  # nothing to move -> no launch


def test_oversized_request_rejected(ddt, q):
    from paper_conf_cluster_chukzsp20_b200 import DDTError
    t = ddt.Type.from_spec(("contiguous", 1 << 33, ("basic", "byte")))
    with pytest.raises(DDTError) as e:
        q.pack(t, 1, 1, 3)  # odd pointers -> 1-byte vectors -> 2^33 vectors > 2^32
    assert e.value.code == -10


def test_failed_enqueue_publishes_nothing(ddt):
    """Enqueue builds the descriptors in place in the free Tail slot; a request
    that fails while being built must leave the ring untouched: the next uid is
    unchanged and the next request (same slot) packs bit-exactly."""
    q1 = ddt.Queue(capacity=2)
    c = Case(ddt, config1_spec(), 3, 8, 0)
    big = ddt.Type.from_spec(("contiguous", 1 << 33, ("basic", "byte")))
    u0, _, d0 = c.gpu_pack(q1)
    assert q1.try_pack(big, 1, 1, 3) == -10  # DDT_ERR_UNSUPPORTED while building the Tail slot
    u1, _, d1 = c.gpu_pack(q1)
    assert (u0, u1) == (0, 1)
    assert q1.flush() == 2
    q1.wait()
    for d in (d0, d1):
        assert_bytes_equal(host(d), c.expect_pack(), "pack after a failed enqueue")
    q1.destroy()


def test_nan_and_negative_zero_survive(ddt, q):
    import torch
    vals = np.array([np.nan, -0.0, np.inf, -np.inf, 5e-324, 1.0] * 40, dtype=np.float64)
    vals.view(np.uint64)[0] = 0x7FF0000000000123  # signalling-NaN payload
    t = ddt.Type.from_spec(("vector", 60, 2, 4, ("basic", "double")))
    s = cuda_bytes(vals)
    d = torch.zeros(t.size, dtype=torch.uint8, device="cuda")
    q.pack(t, s, 1, d)
    q.wait()
    exp = oracle.pack(oracle.Type(("vector", 60, 2, 4, ("basic", "double"))), vals.view(np.uint8))
    assert_bytes_equal(host(d), exp, "nan payloads")


# --------------------------------------------------------------- launch forms, DirectIPC, plans
@pytest.mark.parametrize("n", [1, 5, 8, 9, 20, 32, 33, 70])
def test_batch_forms_param_and_device_table(ddt, q, n):
    """Batches of <= 8 / <= 32 requests ride in the kernel parameters, larger
    ones in a device table: all three forms are bit-exact and one launch."""
    rng = np.random.default_rng(n)
    specs = [config1_spec(), ("subarray", [7, 8, 9], [2, 8, 3], [4, 0, 5], "C", ("basic", "float")),
             ("hindexed", [2, 5, 1], [3, 40, 17], ("basic", "byte"))]
    cases = [Case(ddt, specs[i % 3], count=int(rng.integers(1, 3)), misalign=int(rng.integers(0, 8)), seed=50 + i)
             for i in range(n)]
    outs = [c.gpu_pack(q) for c in cases]
    l0 = q.stats()["launches"]
    assert q.flush() == n
    q.wait()
    assert q.stats()["launches"] - l0 == 1
    for c, (_, _, d) in zip(cases, outs):
        assert_bytes_equal(host(d), c.expect_pack(), f"form n={n}")


@pytest.mark.parametrize("mis_s,mis_d", [(0, 0), (8, 0), (4, 12), (1, 3)])
def test_direct_enqueue_equals_unpack_of_pack(ddt, q, mis_s, mis_d):
    """DirectIPC: one gather->scatter pass == oracle unpack(pack(x))."""
    import torch
    pairs = [(("subarray", [10, 11, 12], [8, 9, 1], [1, 1, 10], "C", ("basic", "double")),
              ("subarray", [10, 11, 12], [8, 9, 1], [1, 1, 0], "C", ("basic", "double"))),
             (("vector", 72, 1, 3, ("basic", "double")), ("subarray", [12, 12], [8, 9], [2, 1], "F", ("basic", "double"))),
             (config3_spec(nblocks=500, npoints=4096)[0], ("vector", 500, 3, 5, ("basic", "float")))]
    for ss, ds in pairs:
        os_, od = oracle.Type(ss), oracle.Type(ds)
        assert os_.size == od.size
        ts, td = ddt.Type.from_spec(ss), ddt.Type.from_spec(ds)
        _, shi = os_.footprint()
        _, dhi = od.footprint()
        src = random_bytes(shi + 64, 9)
        s = cuda_bytes(src)
        d = torch.full((dhi + 64,), SENTINEL, dtype=torch.uint8, device="cuda")
        q.direct(ts, (s, mis_s), 1, td, (d, mis_d), 1)
        q.wait()
        exp = np.full(dhi + 64, SENTINEL, np.uint8)
        oracle.unpack(od, oracle.pack(os_, src, 1, mis_s), exp, 1, mis_d)
        assert_bytes_equal(host(d), exp, f"direct {ss[0]}->{ds[0]}")


def test_direct_size_mismatch_rejected(ddt, q):
    from paper_conf_cluster_chukzsp20_b200 import DDTError
    a = ddt.Type.from_spec(("vector", 4, 1, 2, ("basic", "double")))
    b = ddt.Type.from_spec(("vector", 3, 1, 2, ("basic", "double")))
    with pytest.raises(DDTError) as e:
        q.direct(a, 256, 1, b, 512, 1)
    assert e.value.code == -8


@pytest.mark.parametrize("n", [3, 40])
def test_plan_replay(ddt, q, n):
    """A persistent plan relaunches the same fused batch; results follow the
    current source contents each launch."""
    import torch
    spec, fp = config5_spec(4096)
    o = oracle.Type(spec)
    t = ddt.Type.from_spec(spec)
    src = torch.zeros((n, fp), dtype=torch.uint8, device="cuda")
    dst = torch.zeros((n, 4096), dtype=torch.uint8, device="cuda")
    for i in range(n):
        q.pack(t, src[i], 1, dst[i])
    plan = ddt.Plan(q)
    for it in range(3):
        hs = random_bytes(n * fp, 300 + it).reshape(n, fp)
        src.copy_(torch.from_numpy(hs))
        plan.launch()
        torch.cuda.synchronize()
        got = host(dst)
        for i in range(n):
            assert_bytes_equal(got[i], oracle.pack(o, hs[i]), f"plan it={it} req={i}")
    plan.destroy()


# --------------------------------------------------------------- scheduler triggers / response status
def test_auto_flush_threshold(ddt):
    """§IV-C trigger (2): the enqueue that makes the pending bytes reach the
    threshold launches the batch; the results are unchanged."""
    import torch
    q2 = ddt.Queue()
    spec, fp = config5_spec(65536)
    o = oracle.Type(spec)
    t = ddt.Type.from_spec(spec)
    hs = random_bytes(8 * fp, 77).reshape(8, fp)
    src = torch.from_numpy(hs).cuda()
    dst = torch.zeros((8, 65536), dtype=torch.uint8, device="cuda")
    q2.set_flush_threshold(3 * 65536)
    uids = [q2.pack(t, src[i], 1, dst[i]) for i in range(8)]
    st = q2.stats()
    assert st["flushes"] == 2 and st["launches"] == 2  # after requests 3 and 6
    assert q2.query(uids[7]) == "pending" and q2.query(uids[0]) in ("busy", "completed")
    q2.wait()
    assert q2.stats()["launches"] == 3
    got = host(dst)
    for i in range(8):
        assert_bytes_equal(got[i], oracle.pack(o, hs[i]), f"threshold req {i}")
    q2.destroy()


def test_gpu_written_response_status(ddt):
    """Scheduler (3) per request: a small request fused ahead of a
    1 GiB request reports COMPLETED while the batch is still running."""
    import torch
    q3 = ddt.Queue()
    q3.set_response_flags(True)
    small_spec, sfp = config5_spec(4096)
    big_spec, bfp = config5_spec(64 << 20)
    ts, tb = ddt.Type.from_spec(small_spec), ddt.Type.from_spec(big_spec)
    hs = random_bytes(sfp, 5)
    s_src = torch.from_numpy(hs).cuda()
    s_dst = torch.zeros(4096, dtype=torch.uint8, device="cuda")
    b_src = torch.zeros((16, bfp), dtype=torch.uint8, device="cuda")
    b_dst = torch.zeros((16, 64 << 20), dtype=torch.uint8, device="cuda")
    torch.cuda.synchronize()
    u_small = q3.pack(ts, s_src, 1, s_dst)
    u_big = [q3.pack(tb, b_src[i], 1, b_dst[i]) for i in range(16)]
    q3.flush()
    early = False
    stream = torch.cuda.current_stream()
    for _ in range(200000):
        if q3.query(u_small) == "completed":
            early = not stream.query()
            break
    q3.wait()
    assert all(q3.query(u) == "completed" for u in [u_small] + u_big)
    assert early, "the small request's response status did not arrive before its batch finished"
    assert_bytes_equal(host(s_dst), oracle.pack(oracle.Type(small_spec), hs), "response-flag batch")
    q3.destroy()


def test_config3_cm_struct_on_indexed_full(ddt, q):
    """specfem3D_cm-style struct of three indexed float components (10^5 points
    each over 2^20): pack and unpack bit-exact, one launch each."""
    import torch
    from ddt_inputs import config3_cm_spec
    spec, nb = config3_cm_spec()
    t = ddt.Type.from_spec(spec)
    o = oracle.Type(spec)
    src = random_bytes(nb, seed(3, 8))
    d_src = cuda_bytes(src)
    d_pk = torch.full((t.size,), SENTINEL, dtype=torch.uint8, device="cuda")
    d_un = torch.full((nb,), SENTINEL, dtype=torch.uint8, device="cuda")
    q.pack(t, d_src, 1, d_pk)
    q.flush()
    q.unpack(t, d_pk, 1, d_un)
    q.wait()
    exp = oracle.pack(o, src)
    assert_bytes_equal(host(d_pk), exp, "config3-cm pack")
    eu = np.full(nb, SENTINEL, np.uint8)
    oracle.unpack(o, exp, eu)
    assert_bytes_equal(host(d_un), eu, "config3-cm unpack")


@pytest.mark.parametrize("L", [6, 16])
def test_milc_nested_vector(ddt, q, L):
    """MILC-style hvector-of-vector face of an L^4 su3 lattice: pack + unpack bit-exact."""
    from ddt_inputs import milc_spec
    spec, fp = milc_spec(L)
    _run_case(ddt, q, Case(ddt, spec, 1, misalign=0, seed=L))
    _run_case(ddt, q, Case(ddt, spec, 2, misalign=8, seed=L + 1))


@pytest.mark.parametrize("face", ["x", "y", "z"])
@pytest.mark.parametrize("n", [(34, 34, 34), (66, 34, 18)])
def test_nas_mg_vector_faces(ddt, q, face, n):
    """NAS_MG-style vector faces (x: one element per row, y: one row per plane,
    z: a whole plane): pack + unpack bit-exact vs the oracle, one instance at an
    aligned base and two at a misaligned one."""
    from ddt_inputs import nas_mg_specs
    specs, _ = nas_mg_specs(*n)
    _run_case(ddt, q, Case(ddt, specs[face], 1, misalign=0, seed=sum(n)))
    _run_case(ddt, q, Case(ddt, specs[face], 2, misalign=8, seed=sum(n) + 1))


def _irregular_hindexed(nblocks, npoints, base, maxlen, seed_, ones=False):
    """hindexed with irregular block lengths (a GENERAL_LIST layout); ones=True:
    mostly 1-element blocks of bytes (windows overflow -> per-vector fallback)."""
    rng = np.random.default_rng(seed_)
    esz = {"float": 4, "double": 8, "byte": 1}[base]
    if ones:  # every other element at most: few merges, ~1 segment per byte packed
        idx = 2 * np.sort(rng.choice(npoints // 2 - maxlen, nblocks, replace=False))
    else:
        idx = np.sort(rng.choice(npoints - maxlen, nblocks, replace=False))
    lens = np.where(rng.random(nblocks) < 0.9, 1, 2) if ones else rng.integers(1, maxlen + 1, nblocks)
    gaps = np.diff(np.append(idx, npoints))
    lens = np.minimum(lens, gaps)
    return ("hindexed", [int(x) for x in lens], [int(x) * esz for x in idx], ("basic", base))


@pytest.mark.parametrize("spec,count,mis", [
    (_irregular_hindexed(5000, 1 << 16, "float", 5, 1), 1, 0),
    (_irregular_hindexed(5000, 1 << 16, "float", 5, 2), 2, 4),
    (("indexed", [1, 3, 2, 5], [0, 4, 9, 20], ("basic", "double")), 200, 8),
    (_irregular_hindexed(400000, 1 << 21, "byte", 2, 3, ones=True), 1, 1),
    (_irregular_hindexed(3000, 1 << 15, "double", 7, 4), 3, 0),
])
def test_general_list_windows(ddt, q, spec, count, mis):
    """GENERAL_LIST layouts: items whose segments fit a shared-memory window
    (staged through the skip table), items spanning instances and byte-granular
    windows that overflow (per-vector fallback) -- pack and unpack bit-exact."""
    t = ddt.Type.from_spec(spec)
    assert t.layout_kind == "general_list"
    _run_case(ddt, q, Case(ddt, spec, count, misalign=mis, seed=count + mis))


def test_general_list_direct_both_sides(ddt, q):
    """DirectIPC general -> general (the source side uses the window, the
    destination the per-vector lookup) == oracle unpack(pack(x))."""
    import torch
    ss = _irregular_hindexed(4000, 1 << 15, "float", 4, 5)
    ds = _irregular_hindexed(4000, 1 << 15, "float", 4, 5)
    os_, od = oracle.Type(ss), oracle.Type(ds)
    ts, td = ddt.Type.from_spec(ss), ddt.Type.from_spec(ds)
    _, shi = os_.footprint()
    _, dhi = od.footprint()
    src = random_bytes(shi + 64, 19)
    s = cuda_bytes(src)
    d = torch.full((dhi + 64,), SENTINEL, dtype=torch.uint8, device="cuda")
    q.direct(ts, s, 1, td, d, 1)
    q.wait()
    exp = np.full(dhi + 64, SENTINEL, np.uint8)
    oracle.unpack(od, oracle.pack(os_, src, 1, 0), exp, 1, 0)
    assert_bytes_equal(host(d), exp, "direct general->general")
