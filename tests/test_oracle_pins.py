"""Pins for the CPU oracle (oracle/ddt_oracle.c) against things other than itself.

Each test names what fixes the expected value (SURVEY §8(c) "Pins"):
  * numpy basic slicing / as_strided / concatenation   -- library routines
  * closed forms for size / lb / extent                 -- MPI-3.1 §4.1 formulas
  * self-describing buffers (each element holds its own byte offset)
  * invariants: round trip, count*size, sentinel outside the footprint
  * the config-1 golden file (hand-derived, cited in the file)
A plausible oracle bug (dropped term, wrong sign, transposed index, C/Fortran
mix-up, extent instead of true extent ...) fails at least one of these.
"""
import json
import os

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st, HealthCheck

import oracle
from ddt_inputs import random_bytes, SENTINEL, config1_spec, config3_spec, config5_spec

GOLD = os.path.join(os.path.dirname(__file__), "golden")
HSET = settings(max_examples=60, deadline=None, suppress_health_check=[HealthCheck.too_slow])


def _labels(nbytes_elems: int, elem=8):
    """Self-describing int64 buffer: element i holds its own byte offset i*8."""
    return (np.arange(nbytes_elems, dtype=np.int64) * elem)


def _spec_from_json(j):
    """JSON lists -> spec tuples (a spec is a list whose first item is its kind;
    a struct's oldtypes are a list of specs)."""
    def is_spec(x):
        return isinstance(x, list) and bool(x) and isinstance(x[0], str)
    if not is_spec(j):
        return j
    out = [j[0]]
    for x in j[1:]:
        if is_spec(x):
            out.append(_spec_from_json(x))
        elif isinstance(x, list) and x and all(is_spec(y) for y in x):
            out.append([_spec_from_json(y) for y in x])
        else:
            out.append(x)
    return tuple(out)


# ------------------------------------------------------------ golden config 1
def test_config1_golden():
    g = json.load(open(os.path.join(GOLD, "config1_vector.json")))
    spec = _spec_from_json(g["spec"])
    assert spec == config1_spec()
    t = oracle.Type(spec)
    assert t.size == g["size"]
    assert t.extent() == (g["lb"], g["extent"])
    assert t.true_extent() == (g["true_lb"], g["true_extent"])
    assert t.num_entries == g["num_entries"]
    # merge the oracle's entry list into contiguous segments (typemap order)
    d, ln = t.typemap()
    segs = []
    for a, b in zip(d.tolist(), ln.tolist()):
        if segs and segs[-1][0] + segs[-1][1] == a:
            segs[-1][1] += b
        else:
            segs.append([a, b])
    assert segs == g["segments_offset_len"]
    d2, _ = t.typemap(2)
    assert d2[64] == g["count2_second_instance_first_byte"]
    # pack of a labelled buffer = the golden byte offsets
    src = _labels(1000)
    out = oracle.pack(t, src).view(np.int64)
    expect = np.concatenate([np.arange(o, o + n, 8) for o, n in g["segments_offset_len"]])
    np.testing.assert_array_equal(out, expect)


# ------------------------------------------------------------ subarray vs numpy
@HSET
@given(st.data())
def test_subarray_matches_numpy_slicing(data):
    nd = data.draw(st.integers(1, 4))
    sizes = [data.draw(st.integers(1, 6)) for _ in range(nd)]
    subs = [data.draw(st.integers(1, s)) for s in sizes]
    starts = [data.draw(st.integers(0, s - b)) for s, b in zip(sizes, subs)]
    order = data.draw(st.sampled_from(["C", "F"]))
    base = data.draw(st.sampled_from(["double", "float", "byte", "int32"]))
    esz = oracle.BASIC_SIZES[base]
    n = int(np.prod(sizes))
    src = random_bytes(n * esz, 11)
    t = oracle.Type(("subarray", sizes, subs, starts, order, ("basic", base)))
    elems = src.view({1: np.uint8, 4: np.uint32, 8: np.uint64}[esz])
    a = elems.reshape(sizes, order=order)
    sl = tuple(slice(s, s + b) for s, b in zip(starts, subs))
    expect = a[sl].flatten(order=order)
    got = oracle.pack(t, src).view(expect.dtype)
    np.testing.assert_array_equal(got, expect)
    # subarray is resized: lb 0, extent = prod(sizes)*esz (MPI-3.1 §4.1.3)
    assert t.extent() == (0, n * esz)
    assert t.size == int(np.prod(subs)) * esz


def test_subarray_fortran_is_not_c():
    """C and Fortran orders must differ on a non-symmetric 2-D box."""
    sizes, subs, starts = [3, 4], [2, 3], [1, 0]
    src = _labels(12)
    c = oracle.pack(oracle.Type(("subarray", sizes, subs, starts, "C", ("basic", "double"))), src).view(np.int64)
    f = oracle.pack(oracle.Type(("subarray", sizes, subs, starts, "F", ("basic", "double"))), src).view(np.int64)
    # C: rows 1..2, cols 0..2 of a 3x4 row-major array
    np.testing.assert_array_equal(c // 8, [4, 5, 6, 8, 9, 10])
    # Fortran: dim0 fastest; element (i0,i1) at i0 + 3*i1, i0 in 1..2, i1 in 0..2
    np.testing.assert_array_equal(f // 8, [1, 2, 4, 5, 7, 8])


# ------------------------------------------------------------ vector / hvector
def _vector_closed_bounds(c, b, S, E, olb=0, oub=None):
    oub = E if oub is None else oub
    lb = min(0, (c - 1) * S) + min(0, (b - 1) * E) + olb
    ub = max(0, (c - 1) * S) + max(0, (b - 1) * E) + oub
    return lb, ub


@HSET
@given(c=st.integers(1, 6), b=st.integers(1, 5), stride=st.integers(-9, 9),
       base=st.sampled_from(["double", "float", "int64"]))
def test_vector_matches_as_strided(c, b, stride, base):
    esz = oracle.BASIC_SIZES[base]
    t = oracle.Type(("vector", c, b, stride, ("basic", base)))
    lb, ub = _vector_closed_bounds(c, b, stride * esz, esz)
    assert t.extent() == (lb, ub - lb)
    assert t.size == c * b * esz
    # buffer with room on both sides; the MPI buffer address sits at -lb
    nel = (ub - lb) // esz + 2
    src = random_bytes(nel * esz, 5)
    off = -lb
    got = oracle.pack(t, src, src_offset=off)
    el = np.dtype({4: np.uint32, 8: np.uint64}[esz])
    view = np.lib.stride_tricks.as_strided(src[off:].view(np.uint8), shape=(c, b, esz),
                                           strides=(stride * esz, esz, 1))
    np.testing.assert_array_equal(got, view.reshape(-1))
    assert got.view(el).size == c * b


@HSET
@given(c=st.integers(1, 5), b=st.integers(1, 4), S=st.integers(-40, 40))
def test_hvector_matches_as_strided(c, b, S):
    esz = 4
    t = oracle.Type(("hvector", c, b, S, ("basic", "float")))
    lb, ub = _vector_closed_bounds(c, b, S, esz)
    assert t.extent() == (lb, ub - lb)
    src = random_bytes(ub - lb + 16, 6)
    got = oracle.pack(t, src, src_offset=-lb)
    view = np.lib.stride_tricks.as_strided(src[-lb:], shape=(c, b * esz), strides=(S, 1))
    np.testing.assert_array_equal(got, view.reshape(-1))


def test_vector_negative_stride_order():
    """Typemap order, not address order (DESIGN R1): vector(3,2,-4) of double
    packs element displacements 0,8,-32,-24,-64,-56."""
    t = oracle.Type(("vector", 3, 2, -4, ("basic", "double")))
    d, _ = t.typemap()
    assert d.tolist() == [0, 8, -32, -24, -64, -56]
    assert t.extent() == (-64, 80)


# ------------------------------------------------------------ indexed / hindexed
@HSET
@given(st.data())
def test_indexed_matches_concatenation(data):
    n = data.draw(st.integers(1, 5))
    bl = [data.draw(st.integers(0, 4)) for _ in range(n)]
    dl = [data.draw(st.integers(-6, 12)) for _ in range(n)]
    h = data.draw(st.booleans())
    esz = 8
    if h:
        dl_b = [x * 4 for x in dl]  # byte displacements, not multiples of 8 in general
        t = oracle.Type(("hindexed", bl, dl_b, ("basic", "double")))
        starts = dl_b
    else:
        t = oracle.Type(("indexed", bl, dl, ("basic", "double")))
        starts = [x * esz for x in dl]
    nz = [(s, b) for s, b in zip(starts, bl) if b > 0]
    if nz:
        lb = min(s for s, _ in nz)
        ub = max(s + b * esz for s, b in nz)
    else:
        lb = ub = 0
    assert t.extent() == (lb, ub - lb)
    assert t.size == sum(bl) * esz
    src = random_bytes(256, 9)
    off = 80
    got = oracle.pack(t, src, src_offset=off)
    parts = [src[off + s: off + s + b * esz] for s, b in zip(starts, bl)]
    expect = np.concatenate(parts) if parts else np.zeros(0, np.uint8)
    np.testing.assert_array_equal(got, expect)


@HSET
@given(c=st.integers(1, 5), b=st.integers(1, 4), stride=st.integers(-5, 6), olb=st.integers(-24, 24),
       extra=st.integers(0, 24))
def test_vector_over_nonzero_lb_oldtype_closed_form(c, b, stride, olb, extra):
    """vector(c, b, stride, old) with old = resized(double, olb, E): the MPI
    closed form (SURVEY §8(c) pins) lb = min(0,(c-1)S) + min(0,(b-1)E) +
    lb(old), ub = max(0,(c-1)S) + max(0,(b-1)E) + ub(old), S = stride*E, with
    lb(old) = olb != 0; the entries (the double at offset 0 of every copy) pin
    the copy spacing through numpy's as_strided."""
    E = 8 + extra
    old = ("resized", ("basic", "double"), olb, E)
    t = oracle.Type(("vector", c, b, stride, old))
    lb, ub = _vector_closed_bounds(c, b, stride * E, E, olb=olb, oub=olb + E)
    assert t.extent() == (lb, ub - lb)
    lo = min(0, (c - 1) * stride * E)                      # lowest entry byte
    src = random_bytes(((c - 1) * abs(stride) + b) * E + 64, 13)
    off = -lo
    view = np.lib.stride_tricks.as_strided(src[off:], shape=(c, b, 8), strides=(stride * E, E, 1))
    np.testing.assert_array_equal(oracle.pack(t, src, src_offset=off), view.reshape(-1))


@HSET
@given(st.data())
def test_indexed_over_nonzero_lb_oldtype_closed_form(data):
    """indexed(B, D, old), old = resized(float, olb, E), blocks with B_i > 0:
    lb = min_i(D_i E + min(0,(B_i-1)E)) + lb(old), ub = max_i(D_i E +
    max(0,(B_i-1)E)) + ub(old) (SURVEY §8(c) pins), lb(old) != 0; the packed
    bytes are the concatenated blocks (numpy slicing)."""
    n = data.draw(st.integers(1, 5))
    bl = [data.draw(st.integers(0, 3)) for _ in range(n)]
    dl = [data.draw(st.integers(-4, 8)) for _ in range(n)]
    olb = data.draw(st.integers(-12, 12))
    E = 4 + data.draw(st.integers(0, 12))
    t = oracle.Type(("indexed", bl, dl, ("resized", ("basic", "float"), olb, E)))
    nz = [(d * E, b) for d, b in zip(dl, bl) if b > 0]
    if nz:
        lb = min(d + min(0, (b - 1) * E) for d, b in nz) + olb
        ub = max(d + max(0, (b - 1) * E) for d, b in nz) + olb + E
    else:
        lb = ub = 0
    assert t.extent() == (lb, ub - lb)
    src = random_bytes(512, 17)
    off = 200
    parts = [np.lib.stride_tricks.as_strided(src[off + d * E:], shape=(b, 4), strides=(E, 1)).reshape(-1)
             for d, b in zip(dl, bl)]
    expect = np.concatenate(parts) if parts else np.zeros(0, np.uint8)
    np.testing.assert_array_equal(oracle.pack(t, src, src_offset=off), expect)


def test_run_batch_shared_buffers_match_numpy():
    """oracle.run_batch (a fused batch executed request by request, SURVEY
    §8(c) step 5): packs of three layouts into disjoint slices of ONE packed
    buffer, then unpacks of the six faces of a 6x7x8 block from ONE packed
    buffer into ONE array -- pinned by numpy slicing / assignment."""
    a = random_bytes(6 * 7 * 8 * 8, 41).view(np.int64).reshape(6, 7, 8)
    specs = [("subarray", [6, 7, 8], [1, 5, 6], [0, 1, 1], "C", ("basic", "int64")),
             ("vector", 6, 1, 56, ("basic", "int64")),
             ("hindexed", [2, 1], [64, 8], ("basic", "int64"))]
    expect = [a[0:1, 1:6, 1:7].reshape(-1), a.reshape(-1)[0::56][:6], a.reshape(-1)[[8, 9, 1]]]
    types = [oracle.Type(sp) for sp in specs]
    packed = np.zeros(sum(t.size for t in types) + 16, np.uint8)
    reqs, o = [], 8
    for t in types:
        reqs.append(dict(op="pack", type=t, count=1, src=a, dst=packed, dst_offset=o))
        o += t.size
    oracle.run_batch(reqs)
    np.testing.assert_array_equal(packed[8:o].view(np.int64), np.concatenate(expect))
    assert not packed[:8].any() and not packed[o:].any()
    # unpack: the 6 interior faces of the block from consecutive packed slices
    faces = [(slice(0, 1), slice(1, 6), slice(1, 7)), (slice(5, 6), slice(1, 6), slice(1, 7)),
             (slice(1, 5), slice(0, 1), slice(1, 7)), (slice(1, 5), slice(6, 7), slice(1, 7)),
             (slice(1, 5), slice(1, 6), slice(0, 1)), (slice(1, 5), slice(1, 6), slice(7, 8))]
    fspecs = [("subarray", [6, 7, 8], [f.stop - f.start for f in fc], [f.start for f in fc], "C", ("basic", "int64"))
              for fc in faces]
    ftypes = [oracle.Type(sp) for sp in fspecs]
    src = random_bytes(sum(t.size for t in ftypes), 42)
    dst = np.full((6, 7, 8), -1, np.int64)
    reqs, o = [], 0
    for t in ftypes:
        reqs.append(dict(op="unpack", type=t, count=1, src=src, src_offset=o, dst=dst))
        o += t.size
    oracle.run_batch(reqs)
    ref = np.full((6, 7, 8), -1, np.int64)
    o = 0
    for fc, t in zip(faces, ftypes):
        blk = ref[fc]
        ref[fc] = src[o:o + t.size].view(np.int64).reshape(blk.shape)
        o += t.size
    np.testing.assert_array_equal(dst, ref)


def test_indexed_typemap_order():
    """indexed([2,1],[5,0]) of double packs displacements 40, 48, 0 (R1)."""
    t = oracle.Type(("indexed", [2, 1], [5, 0], ("basic", "double")))
    assert t.typemap()[0].tolist() == [40, 48, 0]
    assert t.extent() == (0, 56)
    assert t.true_extent() == (0, 56)


# ------------------------------------------------------------ nesting
@HSET
@given(c1=st.integers(1, 4), b1=st.integers(1, 3), s1=st.integers(1, 5),
       c2=st.integers(1, 3), b2=st.integers(1, 3), s2=st.integers(1, 4))
def test_nested_vector_matches_as_strided(c1, b1, s1, c2, b2, s2):
    """vector(c1,b1,s1, vector(c2,b2,s2,double)); the inner type's extent is
    ((c2-1)*s2 + b2)*8 (positive strides).  numpy's 4-D strided view pins both
    the outer displacement rule and the inner extent."""
    s2 = max(s2, b2)
    inner = ("vector", c2, b2, s2, ("basic", "double"))
    E = ((c2 - 1) * s2 + b2) * 8
    t = oracle.Type(("vector", c1, b1, s1, inner))
    nb = ((c1 - 1) * s1 + b1) * E + 64
    src = random_bytes(nb, 3)
    view = np.lib.stride_tricks.as_strided(src, shape=(c1, b1, c2, b2, 8),
                                           strides=(s1 * E, E, s2 * 8, 8, 1))
    np.testing.assert_array_equal(oracle.pack(t, src), view.reshape(-1))
    lb, ub = _vector_closed_bounds(c1, b1, s1 * E, E)
    assert t.extent() == (lb, ub - lb)


def test_subarray_of_subarray_uses_resized_extent():
    """A subarray oldtype has extent prod(sizes)*8 > its true extent; the outer
    constructor must step by the full (resized) extent (DESIGN R4)."""
    inner = ("subarray", [4, 5], [2, 2], [1, 3], "C", ("basic", "double"))  # extent 160 B
    t = oracle.Type(("vector", 3, 1, 2, inner))                            # copies at 0, 320, 640
    src = _labels(200)
    got = oracle.pack(t, src).view(np.int64) // 8
    a = np.arange(20).reshape(4, 5)[1:3, 3:5].reshape(-1)
    expect = np.concatenate([a + 40 * i for i in range(3)])
    np.testing.assert_array_equal(got, expect)
    inner_t = oracle.Type(inner)
    assert inner_t.extent() == (0, 160)
    assert inner_t.true_extent() == (8 * 8, (2 * 5 + 4 + 1 - 8) * 8)
    assert t.extent() == (0, 2 * 2 * 160 + 160)


def test_hindexed_of_vector_and_contiguous():
    inner = ("vector", 2, 1, 3, ("basic", "int32"))   # entries 0, 12 -> extent 16
    t = oracle.Type(("hindexed", [2, 1], [100, 4], inner))
    d, _ = t.typemap()
    assert d.tolist() == [100, 112, 116, 128, 4, 16]
    c = oracle.Type(("contiguous", 3, ("basic", "float")))
    assert c.extent() == (0, 12) and c.size == 12
    assert c.typemap()[0].tolist() == [0, 4, 8]


# ------------------------------------------------------------ empties
def test_empty_types():
    for spec in [("vector", 0, 3, 2, ("basic", "double")),
                 ("vector", 3, 0, 2, ("basic", "double")),
                 ("indexed", [0, 0], [4, 9], ("basic", "float")),
                 ("hindexed", [], [], ("basic", "float")),
                 ("contiguous", 0, ("basic", "int64"))]:
        t = oracle.Type(spec)
        assert t.size == 0 and t.extent() == (0, 0) and t.true_extent() == (0, 0)
        assert oracle.pack(t, np.zeros(8, np.uint8), count=3).nbytes == 0
    # zero-length blocks do not contribute to bounds
    t = oracle.Type(("indexed", [0, 2, 0], [-50, 3, 70], ("basic", "double")))
    assert t.extent() == (24, 16)


# ------------------------------------------------------------ count > 1, round trip
@HSET
@given(st.data())
def test_count_and_round_trip(data):
    kind = data.draw(st.sampled_from(["vector", "subarray", "hindexed"]))
    if kind == "vector":
        c, b = data.draw(st.integers(1, 4)), data.draw(st.integers(1, 3))
        stride = data.draw(st.sampled_from([-5, -3, 3, 4, 7]))
        spec = ("vector", c, b, stride, ("basic", "double"))
    elif kind == "subarray":
        spec = ("subarray", [3, 4, 5], [1, 2, 3], [2, 1, 1], data.draw(st.sampled_from("CF")), ("basic", "float"))
    else:
        spec = ("hindexed", [1, 3, 2], [40, 0, 13], ("basic", "byte"))
    count = data.draw(st.integers(1, 4))
    t = oracle.Type(spec)
    lb, ex = t.extent()
    src = random_bytes(4096, data.draw(st.integers(0, 99)))
    off = 1024
    packed = oracle.pack(t, src, count=count, src_offset=off)
    assert packed.nbytes == count * t.size
    # instance k is instance 0 shifted by k*extent
    for k in range(count):
        one = oracle.pack(t, src, count=1, src_offset=off + k * ex)
        np.testing.assert_array_equal(packed[k * t.size:(k + 1) * t.size], one)
    # round trip into a sentinel buffer
    dst = np.full(4096, SENTINEL, np.uint8)
    oracle.unpack(t, packed, dst, count=count, dst_offset=off)
    d, ln = t.typemap(count)
    mask = np.zeros(4096, bool)
    for a, n in zip(d.tolist(), ln.tolist()):
        mask[off + a: off + a + n] = True
    np.testing.assert_array_equal(dst[mask], src[mask])
    assert np.all(dst[~mask] == SENTINEL)


# ------------------------------------------------------------ workload recipes
def test_config3_and_config5_recipes_sizes():
    spec, nb = config3_spec(nblocks=1000, npoints=1 << 14)
    t = oracle.Type(spec)
    assert t.size == 12 * 1000
    src = random_bytes(nb, 1)
    got = oracle.pack(t, src)
    idx = np.array(spec[2]) // 12
    np.testing.assert_array_equal(got.reshape(-1, 12), src.reshape(-1, 12)[idx])
    for S in [64, 256, 1024, 65536]:
        spec, fp = config5_spec(S)
        t = oracle.Type(spec)
        assert t.size == S
        assert t.extent()[1] == fp


# ------------------------------------------------------------ halo exchange (configs 2, 4)
@pytest.mark.parametrize("P", [1, 2, 4, 8])
@pytest.mark.parametrize("faces_only", [False, True])
def test_oracle_exchange_matches_np_pad_wrap(P, faces_only):
    """After one exchange every rank's ghost cells equal numpy's periodic
    ('wrap') padding of the global array (SURVEY §8(c) 'Halo exchange' pin).
    Faces-only (config 2 shape): edge/corner ghosts stay sentinel."""
    from ddt_inputs import (halo_messages, padded_block, global_block, proc_grid, ghost_mask,
                            FACE_DIRS, ALL_DIRS)
    grid = proc_grid(P)
    local = (3, 4, 5)
    G = tuple(n * g for n, g in zip(local, grid))
    nvars = 2
    dirs = FACE_DIRS if faces_only else ALL_DIRS
    glob = [random_bytes(int(np.prod(G)) * 8, 100 + v).view(np.uint64).reshape(G) for v in range(nvars)]
    arrays = {}
    for r in range(P):
        for v in range(nvars):
            a = np.full((local[0] + 2, local[1] + 2, local[2] + 2), 0xA5A5A5A5A5A5A5A5, np.uint64)
            a[1:-1, 1:-1, 1:-1] = global_block(glob[v], r, P)
            arrays[(r, v)] = a
    msgs = []
    by_key = {}
    for r in range(P):
        for m in halo_messages(r, P, local, dirs=dirs, nvars=nvars):
            by_key[(r, m["recv_peer"], m["recv_tag"])] = m
    for r in range(P):
        for m in halo_messages(r, P, local, dirs=dirs, nvars=nvars):
            # the matching receive on the peer: recv from r with the same tag
            rm = by_key[(m["peer"], r, m["tag"])]
            assert rm["var"] == m["var"]
            msgs.append(dict(src_rank=r, dst_rank=m["peer"], var=m["var"],
                             send=oracle.Type(m["send_spec"]), recv=oracle.Type(rm["recv_spec"])))
    assert len(msgs) == P * nvars * len(dirs)
    oracle.exchange(arrays, msgs)
    gm = ghost_mask(local, dirs)
    for r in range(P):
        for v in range(nvars):
            exp = padded_block(glob[v], r, P)
            got = arrays[(r, v)]
            np.testing.assert_array_equal(got[gm], exp[gm])
            np.testing.assert_array_equal(got[1:-1, 1:-1, 1:-1], exp[1:-1, 1:-1, 1:-1])
            rest = ~gm
            rest[1:-1, 1:-1, 1:-1] = False
            assert np.all(got[rest] == 0xA5A5A5A5A5A5A5A5)


# ------------------------------------------------------------ struct / resized (MPI-3.1 §4.1.2, §4.1.7)
_NP = {"double": "<f8", "float": "<f4", "int32": "<i4", "int64": "<i8", "byte": "u1"}


@HSET
@given(st.data())
def test_struct_matches_numpy_aligned_structured_dtype(data):
    """A struct of basic blocks is a numpy structured dtype with explicit field
    offsets.  With ``align=True`` numpy lays records out like a C compiler:
    itemsize = the end of the last field rounded up to the largest field
    alignment -- MPI's alignment increment epsilon (MPI-3.1 §4.1: ub =
    max(disp + sizeof) + epsilon, rounding the extent to a multiple of max k_i;
    DESIGN R2).  numpy derives that itemsize itself; packing `count` records
    copies the fields in typemap (not address) order."""
    n = data.draw(st.integers(1, 4))
    names, formats, offsets, bl, d, olds = [], [], [], [], [], []
    pos = 0
    for i in range(n):
        base = data.draw(st.sampled_from(["double", "float", "int32", "int64", "byte"]))
        esz = oracle.BASIC_SIZES[base]
        b = data.draw(st.integers(1, 3))
        pos = (pos + esz - 1) // esz * esz          # natural alignment (numpy requires it with align=True)
        names.append(f"f{i}")
        formats.append((_NP[base], (b,)))
        offsets.append(pos)
        bl.append(b), d.append(pos), olds.append(("basic", base))
        pos += b * esz + data.draw(st.integers(0, 12))
    perm = data.draw(st.permutations(range(n)))          # typemap order != address order
    spec = ("struct", [bl[i] for i in perm], [d[i] for i in perm], [olds[i] for i in perm])
    t = oracle.Type(spec)
    rec = np.dtype({"names": names, "formats": formats, "offsets": offsets}, align=True)
    assert t.extent() == (0, rec.itemsize)
    hi = max(off + bb * oracle.BASIC_SIZES[o[1]] for off, bb, o in zip(d, bl, olds))
    assert t.true_extent() == (0, hi)
    count = data.draw(st.integers(1, 3))
    src = random_bytes(rec.itemsize * count + 16, 21)
    arr = np.frombuffer(src[: rec.itemsize * count].tobytes(), dtype=rec)
    packed_dt = np.dtype([(names[i], formats[i]) for i in perm])
    expect = np.empty(count, dtype=packed_dt)
    for i in perm:
        expect[names[i]] = arr[names[i]]
    got = oracle.pack(t, src, count)
    np.testing.assert_array_equal(got, expect.view(np.uint8))


def test_nested_struct_matches_numpy_nested_aligned_dtype():
    """A struct holding a struct: the inner record's itemsize (its rounded
    extent) is the spacing of its copies, and the outer alignment is the
    largest basic alignment anywhere inside (numpy nested align=True)."""
    inner_dt = np.dtype([("a", "<f8"), ("b", "u1")], align=True)                  # 16
    outer_dt = np.dtype([("c", "u1"), ("s", inner_dt, (2,)), ("e", "<i4")], align=True)
    inner = ("struct", [1, 1], [0, 8], [("basic", "double"), ("basic", "byte")])
    off = [outer_dt.fields[k][1] for k in ("c", "s", "e")]
    spec = ("struct", [1, 2, 1], off, [("basic", "byte"), inner, ("basic", "int32")])
    t = oracle.Type(spec)
    assert oracle.Type(inner).extent() == (0, inner_dt.itemsize)
    assert t.extent() == (0, outer_dt.itemsize)
    src = random_bytes(outer_dt.itemsize * 3, 77)
    arr = np.frombuffer(src.tobytes(), dtype=outer_dt)
    expect = b"".join(r["c"].tobytes() + b"".join(x["a"].tobytes() + x["b"].tobytes() for x in r["s"])
                      + r["e"].tobytes() for r in arr)
    assert oracle.pack(t, src, 3).tobytes() == expect


def test_struct_alignment_golden():
    """Hand-derived values (tests/golden/struct_alignment.json, each case cites
    its source): MPI-3.1 §4.1's own example {(double,0),(char,8)} has extent 16."""
    g = json.load(open(os.path.join(GOLD, "struct_alignment.json")))
    for case in g["cases"]:
        t = oracle.Type(_spec_from_json(case["spec"]))
        assert t.size == case["size"], case["name"]
        assert list(t.extent()) == [case["lb"], case["extent"]], case["name"]
        assert list(t.true_extent()) == [case["true_lb"], case["true_extent"]], case["name"]
        if "typemap_count2" in case:
            assert t.typemap(2)[0].tolist() == case["typemap_count2"], case["name"]


@HSET
@given(c=st.integers(1, 4), b=st.integers(1, 3), stride=st.integers(3, 6), lb=st.integers(-16, 16),
       extra=st.integers(0, 64), count=st.integers(1, 4))
def test_resized_steps_instances_by_the_new_extent(c, b, stride, lb, extra, count):
    inner = ("vector", c, b, stride, ("basic", "double"))
    E = ((c - 1) * stride + b) * 8 + extra
    t = oracle.Type(("resized", inner, lb, E))
    assert t.extent() == (lb, E)
    assert t.true_extent() == oracle.Type(inner).true_extent()
    src = random_bytes(E * count + 512, 8)
    got = oracle.pack(t, src, count)
    view = np.lib.stride_tricks.as_strided(src, shape=(count, c, b, 8), strides=(E, stride * 8, 8, 1))
    np.testing.assert_array_equal(got, view.reshape(-1))
    # a resized oldtype sets the copy spacing of its parent
    v = oracle.Type(("contiguous", 3, ("resized", ("basic", "double"), 0, 24)))
    assert v.typemap()[0].tolist() == [0, 24, 48]


def test_config3_cm_struct_on_indexed_matches_fancy_indexing():
    from ddt_inputs import config3_cm_spec
    spec, nb = config3_cm_spec(nblocks=2000, npoints=1 << 14)
    t = oracle.Type(spec)
    src = random_bytes(nb, 4)
    f = src.view(np.float32).reshape(3, -1)
    idx = np.array(spec[3][0][2])
    np.testing.assert_array_equal(oracle.pack(t, src), np.concatenate([f[0][idx], f[1][idx], f[2][idx]]).view(np.uint8))


def test_milc_nested_vector_matches_numpy():
    from ddt_inputs import milc_spec
    L = 4
    spec, fp = milc_spec(L)
    t = oracle.Type(spec)
    src = random_bytes(fp, 31)
    lat = src.view(np.float64).reshape(L, L, L, L, 6)          # [t][z][y][x][6]
    np.testing.assert_array_equal(oracle.pack(t, src).view(np.float64), lat[:, :, 0, :, :].reshape(-1))


def test_nas_mg_faces_match_numpy():
    """NAS_MG-style vector faces against numpy slicing of the
    (n3, n2, n1) C-order grid, x fastest."""
    from ddt_inputs import nas_mg_specs
    n1, n2, n3 = 6, 5, 7
    specs, fp = nas_mg_specs(n1, n2, n3)
    src = random_bytes(fp, 41)
    g = src.view(np.float64).reshape(n3, n2, n1)
    want = {"x": g[:, :, 0], "y": g[:, 0, :], "z": g[0, :, :]}
    for face, spec in specs.items():
        t = oracle.Type(spec)
        np.testing.assert_array_equal(oracle.pack(t, src).view(np.float64), want[face].reshape(-1), err_msg=face)
        assert t.size == want[face].size * 8
