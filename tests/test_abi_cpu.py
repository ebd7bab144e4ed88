"""CPU-only tests of the C ABI library: it loads, exports every symbol
include/ddt.h declares, and its host logic (closed-form type queries, the
flattener / layout cache) agrees with the oracle's enumeration.  No compute
calls (no GPU here)."""
import ctypes
import os
import re

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st, HealthCheck

import oracle
from ddt_inputs import config1_spec, config3_spec, config5_spec, halo_messages

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HSET = settings(max_examples=80, deadline=None, suppress_health_check=[HealthCheck.too_slow])


@pytest.fixture(scope="module")
def ddt():
    from paper_conf_cluster_chukzsp20_b200.build import build
    build()
    import paper_conf_cluster_chukzsp20_b200 as m
    return m


def test_exports_every_header_symbol(ddt):
    hdr = open(os.path.join(ROOT, "include", "ddt.h")).read()
    declared = set(re.findall(r"^\s*(?:ddt_status_t|int64_t|int32_t|void|const char\*)\s+(ddt_\w+)\s*\(", hdr, re.M))
    assert len(declared) >= 40
    L = ctypes.CDLL(os.path.join(ROOT, "paper_conf_cluster_chukzsp20_b200", "libddt.so"))
    missing = [s for s in declared if not hasattr(L, s)]
    assert not missing, missing
    from paper_conf_cluster_chukzsp20_b200._abi import PROTOTYPES
    assert declared == set(PROTOTYPES), declared ^ set(PROTOTYPES)
    assert ddt.lib().ddt_built_sm() == 100


def test_kernels_are_sm100a():
    import subprocess
    so = os.path.join(ROOT, "paper_conf_cluster_chukzsp20_b200", "libddt.so")
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-lelf", so], capture_output=True, text=True).stdout
    assert "sm_100a" in out, out


def test_queue_without_device_is_an_error(ddt):
    try:
        import torch
        if torch.cuda.is_available():
            pytest.skip("GPU present")
    except Exception:
        pass
    out = ctypes.c_void_p()
    rc = ddt.lib().ddt_queue_create(0, None, 0, ctypes.byref(out))
    assert rc == -11  # DDT_ERR_NODEV


def test_error_strings(ddt):
    for c in range(0, -12, -1):
        assert ddt.lib().ddt_strerror(c)


# ------------------------------------------------------- random type specs
def spec_strategy(depth=2):
    base = st.sampled_from([("basic", b) for b in ["byte", "int32", "int64", "float", "double"]])

    def extend(children):
        vec = st.tuples(st.just("vector"), st.integers(0, 4), st.integers(0, 3), st.integers(-6, 6), children)
        hvec = st.tuples(st.just("hvector"), st.integers(0, 4), st.integers(0, 3), st.integers(-40, 40), children)
        cont = st.tuples(st.just("contiguous"), st.integers(0, 4), children)
        idx = st.integers(1, 4).flatmap(lambda n: st.tuples(
            st.just("indexed"), st.lists(st.integers(0, 3), min_size=n, max_size=n),
            st.lists(st.integers(-5, 9), min_size=n, max_size=n), children))
        hidx = st.integers(1, 4).flatmap(lambda n: st.tuples(
            st.just("hindexed"), st.lists(st.integers(0, 3), min_size=n, max_size=n),
            st.lists(st.integers(-30, 60), min_size=n, max_size=n), children))
        sub = st.integers(1, 3).flatmap(lambda nd: st.lists(st.integers(1, 4), min_size=nd, max_size=nd).flatmap(
            lambda sizes: st.tuples(*[st.integers(1, s) for s in sizes]).flatmap(
                lambda subs: st.tuples(st.just("subarray"), st.just(list(sizes)), st.just(list(subs)),
                                       st.tuples(*[st.integers(0, s - b) for s, b in zip(sizes, subs)]).map(list),
                                       st.sampled_from(["C", "F"]), children))))
        strc = st.integers(1, 3).flatmap(lambda n: st.tuples(
            st.just("struct"), st.lists(st.integers(0, 3), min_size=n, max_size=n),
            st.lists(st.integers(-40, 80), min_size=n, max_size=n), st.lists(children, min_size=n, max_size=n)))
        rsz = st.tuples(st.just("resized"), children, st.integers(-24, 24), st.integers(0, 96))
        return st.one_of(vec, hvec, cont, idx, hidx, sub, strc, rsz)

    return st.recursive(base, extend, max_leaves=3)


def _merged(disp, ln):
    segs = []
    for a, b in zip(disp.tolist(), ln.tolist()):
        if segs and segs[-1][0] + segs[-1][1] == a:
            segs[-1][1] += b
        else:
            segs.append([a, b])
    return segs


def _bytes_of(segs):
    out = []
    for o, n in segs:
        out.extend(range(o, o + n))
    return out


@HSET
@given(spec=spec_strategy())
def test_closed_forms_match_oracle_enumeration(ddt, spec):
    t = ddt.Type.from_spec(spec)
    o = oracle.Type(spec)
    assert t.size == o.size
    assert t.extent() == o.extent(), spec
    assert t.true_extent() == o.true_extent(), spec
    # flattened segments (one instance, packed order) cover exactly the oracle's bytes in order
    offs, lens = t.segments()
    d, ln = o.typemap()
    assert _bytes_of(zip(offs.tolist(), lens.tolist())) == _bytes_of(zip(d.tolist(), ln.tolist()))
    assert t.num_segments == len(offs)
    # overlap flag == brute force over the oracle's entries
    b = _bytes_of(zip(d.tolist(), ln.tolist()))
    assert t.overlaps == (len(b) != len(set(b))), spec


def test_struct_alignment_golden_library(ddt):
    """The library's closed-form struct bounds (alignment epsilon, R2) against
    the hand-derived golden values (tests/golden/struct_alignment.json)."""
    import json
    from test_oracle_pins import _spec_from_json
    g = json.load(open(os.path.join(ROOT, "tests", "golden", "struct_alignment.json")))
    for case in g["cases"]:
        t = ddt.Type.from_spec(_spec_from_json(case["spec"]))
        assert t.size == case["size"], case["name"]
        assert list(t.extent()) == [case["lb"], case["extent"]], case["name"]
        assert list(t.true_extent()) == [case["true_lb"], case["true_extent"]], case["name"]


def test_layout_kinds(ddt):
    t = ddt.Type.from_spec(config1_spec())
    assert t.layout_kind == "strided" and t.num_segments == 16
    offs, lens = t.segments()
    assert offs.tolist() == [512 * i for i in range(16)] and set(lens.tolist()) == {32}
    spec, _ = config3_spec(nblocks=2000, npoints=1 << 14)
    t = ddt.Type.from_spec(spec)
    assert t.layout_kind == "uniform_list" and t.num_segments == 2000
    t = ddt.Type.from_spec(("indexed", [1, 2, 3], [0, 10, 20], ("basic", "double")))
    assert t.layout_kind == "general_list"
    # arithmetic indexed -> closed form
    t = ddt.Type.from_spec(("indexed", [2, 2, 2], [0, 5, 10], ("basic", "double")))
    assert t.layout_kind == "strided"
    t = ddt.Type.from_spec(("vector", 0, 2, 3, ("basic", "double")))
    assert t.layout_kind == "empty" and t.size == 0
    for S in (64, 4096, 1 << 20):
        t = ddt.Type.from_spec(config5_spec(S)[0])
        assert t.layout_kind == "strided"


def test_halo_face_types_are_closed_form(ddt):
    """Every config-2/4 message type flattens to <= 2 strided dims (no metadata)."""
    for m in halo_messages(0, 8, (128, 128, 128)):
        for spec in (m["send_spec"], m["recv_spec"]):
            t = ddt.Type.from_spec(spec)
            assert t.layout_kind == "strided"
            o = oracle.Type(spec)
            assert t.size == o.size and t.extent() == o.extent()


def test_overlapping_type_rejected_for_unpack_flag(ddt):
    t = ddt.Type.from_spec(("vector", 3, 2, 1, ("basic", "double")))  # blocks overlap
    assert t.overlaps
    t = ddt.Type.from_spec(("hindexed", [1, 1], [0, 4], ("basic", "double")))
    assert t.overlaps
    t = ddt.Type.from_spec(("vector", 3, 2, -2, ("basic", "double")))  # touching, not overlapping
    assert not t.overlaps


def test_invalid_arguments(ddt):
    from paper_conf_cluster_chukzsp20_b200 import DDTError
    d = ddt.Type.basic("double")
    with pytest.raises(DDTError):
        ddt.Type.vector(-1, 1, 1, d)
    with pytest.raises(DDTError):
        ddt.Type.subarray([4, 4], [5, 1], [0, 0], "C", d)
    with pytest.raises(DDTError):
        ddt.Type.subarray([4, 4], [2, 2], [3, 0], "C", d)
    with pytest.raises(DDTError):
        ddt.Type.indexed([1, -1], [0, 3], d)
    t = ddt.Type.vector(2, 1, 2, d)  # not committed
    with pytest.raises(DDTError):
        _ = t.num_segments
