"""GPU halo-exchange parity on one B200 (every message a self message at P=1):
after each ddt_exchange the ghost cells equal numpy's periodic padding of the
interior (SURVEY §8(c) 'Halo exchange' pin, an independent library routine),
the interior is untouched, and un-targeted ghosts keep the sentinel.  Both the
NCCL-mode plan (fused pack -> fused unpack) and the fused single-kernel P2P
plan (window + epoch flags, double-buffered by parity) are exercised over
several iterations, with and without CUDA-graph replay."""
import numpy as np
import pytest

from ddt_inputs import halo_messages, ghost_mask, FACE_DIRS, ALL_DIRS, random_bytes, seed

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ddt():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_cluster_chukzsp20_b200.build import build
    build()
    import paper_conf_cluster_chukzsp20_b200 as m
    return m


def _setup(ddt, local, dirs, nvars, mode, graph, cfg):
    import torch
    q = ddt.Queue()
    shape = tuple(n + 2 for n in local)
    arrs = []
    for v in range(nvars):
        a = torch.full(shape, 0, dtype=torch.int64, device="cuda")
        a.view(torch.uint8).fill_(0xA5)
        arrs.append(a)
    msgs = halo_messages(0, 1, local, dirs=dirs, nvars=nvars)
    types = {}

    def T(spec):
        key = repr(spec)
        if key not in types:
            types[key] = ddt.Type.from_spec(spec)
        return types[key]

    sends = [(m["peer"], m["tag"], T(m["send_spec"]), arrs[m["var"]], 1) for m in msgs]
    recvs = [(m["recv_peer"], m["recv_tag"], T(m["recv_spec"]), arrs[m["var"]], 1) for m in msgs]
    comm = ddt.Comm.single(torch.cuda.current_device())
    h = ddt.Halo(q, comm, sends, recvs, mode=mode, graph=graph)
    return q, arrs, h, comm


def _fill_interior(arrs, local, it, cfg):
    import torch
    for v, a in enumerate(arrs):
        n = int(np.prod(local))
        vals = random_bytes(n * 8, seed(cfg, 10 * it + v)).view(np.int64).reshape(local)
        a[1:-1, 1:-1, 1:-1] = torch.from_numpy(vals).cuda()


def _check(arrs, local, dirs, before=None):
    gm = ghost_mask(local, dirs)
    for i, a in enumerate(arrs):
        h = a.cpu().numpy()
        if before is not None:
            assert np.array_equal(h[1:-1, 1:-1, 1:-1], before[i]), "interior modified by the exchange"
        exp = np.pad(h[1:-1, 1:-1, 1:-1], 1, mode="wrap")
        assert np.array_equal(h[gm], exp[gm]), "ghost cells differ from np.pad(wrap)"
        rest = ~gm
        rest[1:-1, 1:-1, 1:-1] = False
        assert np.all(h.view(np.uint8).reshape(h.shape + (8,))[rest] == 0xA5)


@pytest.mark.parametrize("mode", ["nccl", "p2p", "p2p_direct"])
@pytest.mark.parametrize("graph", [False, True])
@pytest.mark.parametrize("local,dirs,nvars,cfg", [
    ((5, 6, 7), ALL_DIRS, 2, 4),
    ((9, 4, 3), FACE_DIRS, 1, 2),
])
@pytest.mark.parametrize("group", [False, True, "spread", "pair1"])
def test_halo_small(ddt, mode, graph, local, dirs, nvars, cfg, group, monkeypatch):
    """group=True: equal-size requests interleaved chunk by chunk even though the
    plan is one wave (the default only groups multi-wave plans); "spread": the
    multi-wave plain-plan form (explicit spread item table, one CTA per item,
    +x / -x style requests paired in the same items) forced on a small plan."""
    import torch
    if group == "spread":
        monkeypatch.setenv("DDT_SPREAD_ALWAYS", "1")
    elif group == "pair1":  # one-wave plan with its +x / -x requests paired (prefix form, in place / device table)
        monkeypatch.setenv("DDT_PAIR1", "1")
    elif group:
        monkeypatch.setenv("DDT_GROUP_ALWAYS", "1")
    q, arrs, h, comm = _setup(ddt, local, dirs, nvars, mode, graph, cfg)
    for it in range(4):
        _fill_interior(arrs, local, it, cfg)
        torch.cuda.synchronize()
        before = [a[1:-1, 1:-1, 1:-1].cpu().numpy() for a in arrs]
        h.exchange()
        torch.cuda.synchronize()
        _check(arrs, local, dirs, before)
    assert h.launches_per_exchange == 1  # P = 1: every message is a self message -> one DirectIPC launch
    h.destroy()
    comm.close()


@pytest.mark.parametrize("mode", ["nccl", "p2p"])
def test_config2_face_halo_full_size(ddt, mode):
    """BASELINE.json configs[1] per-rank size (128^3 doubles, 6 face messages),
    P = 1, as bench.py runs it (graph replay)."""
    import torch
    local = (128, 128, 128)
    q, arrs, h, comm = _setup(ddt, local, FACE_DIRS, 1, mode, True, 2)
    for it in range(3):
        _fill_interior(arrs, local, it, 2)
        torch.cuda.synchronize()
        before = [a[1:-1, 1:-1, 1:-1].cpu().numpy() for a in arrs]
        h.exchange()
        torch.cuda.synchronize()
        _check(arrs, local, FACE_DIRS, before)
    h.destroy()
    comm.close()


def test_config2_bench_launch_configuration(ddt):
    """bench.py's N = 1 launch configuration at full size: R independent 130^3
    arrays with one plan each (graph=False) on a side stream, K steps round
    robin captured into ONE CUDA graph, replayed; every replica's ghosts must
    equal np.pad(wrap) after each replay (sentinels reset in between)."""
    import torch
    local = (128, 128, 128)
    R, K = 3, 7
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        reps = [_setup(ddt, local, FACE_DIRS, 1, "p2p", False, 2) for _ in range(R)]
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for k in range(K):
                reps[k % R][2].exchange()
        for it in range(2):
            befores = []
            for r, (_, arrs, _, _) in enumerate(reps):
                arrs[0].view(torch.uint8).fill_(0xA5)
                _fill_interior(arrs, local, 10 * it + r, 2)
                befores.append([arrs[0][1:-1, 1:-1, 1:-1].cpu().numpy()])
            g.replay()
            torch.cuda.synchronize()
            for (_, arrs, _, _), before in zip(reps, befores):
                _check(arrs, local, FACE_DIRS, before)
        for q, _, h, comm in reps:
            h.destroy()
            comm.close()
            q.destroy()


def test_config4_comb_halo_full_size_p1(ddt):
    """BASELINE.json configs[3] at its 1-GPU point: 512^3 doubles, 4 variables,
    26 neighbours, 104 + 104 messages per iteration (one launch; the +x / -x
    faces paired); the full ghost mask of EVERY variable against np.pad(wrap)
    and every interior unchanged, over two exchanges."""
    import torch
    local = (512, 512, 512)
    q, arrs, h, comm = _setup(ddt, local, ALL_DIRS, 4, "p2p", True, 4)
    gm = ghost_mask(local, ALL_DIRS)
    g = torch.Generator(device="cuda")
    for it in range(2):
        g.manual_seed(seed(4, it))
        for a in arrs:
            a.random_(generator=g)  # ghosts random as well: a ghost the exchange misses is caught
        torch.cuda.synchronize()
        before = [a[1:-1, 1:-1, 1:-1].cpu().numpy() for a in arrs]
        h.exchange()
        torch.cuda.synchronize()
        for v, a in enumerate(arrs):
            got = a.cpu().numpy()
            assert np.array_equal(got[1:-1, 1:-1, 1:-1], before[v]), f"var {v}: interior modified"
            exp = np.pad(before[v], 1, mode="wrap")
            assert np.array_equal(got[gm], exp[gm]), f"it {it} var {v}: ghosts differ from np.pad(wrap)"
            del got, exp
        del before
    h.destroy()
    comm.close()
