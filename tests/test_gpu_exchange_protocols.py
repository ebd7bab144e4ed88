"""GPU parity of the multi-GPU exchange protocols, run on one B200.

The window protocol (pack -> peer window -> per-chunk release flag or LL word
-> acquire -> unpack, §IV-B) and the NCCL-mode staging path
normally carry only remote messages; the test hooks DDT_SELF_VIA_WINDOW=1 and
DDT_SELF_VIA_NCCL=1 (a 1-rank NCCL communicator, send/recv to self) route a
rank's self messages through them, so the exact code that runs between GPUs
runs here at the BASELINE.json sizes:

* configs[1] (128^3, 6 faces: LL words, or per-chunk flags with DDT_NO_LL=1);
* configs[3] at its 1-GPU point (512^3 x 4 variables, 26 directions: 2 MiB
  faces > 512 KB take the per-chunk flag protocol), every variable's full
  ghost mask checked;
* 4-B (float) layouts (flag protocol, 4-B vectors) and a receiver whose
  buffer sits at 4 mod 8 while the sender's does not (different vector widths
  on the two sides: the whole-message fan-out release + message counter);
* the exchange kernel completing while another stream's kernel holds all SM
  slots but a few (items are claimed by ticket: no co-residency needed);
* K exchanges captured into one CUDA graph (device-resident epoch).

Every check is against numpy's periodic padding (np.pad(..., mode="wrap")),
an independent library routine (SURVEY §8(c) "Halo exchange" pin)."""
import ctypes
import time

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


def _env(monkeypatch, **kv):
    from paper_conf_cluster_chukzsp20_b200 import reload_env
    for k, v in kv.items():
        monkeypatch.setenv(k, v)
    reload_env()


class Plan:
    """P = 1 halo plan whose sends read `src` arrays and whose receives write
    `dst` arrays (the same arrays for a true halo; distinct ones to give the
    two sides different alignments).  Arrays live in uint8 device buffers at
    byte offset `off` so the receive side can be misaligned on purpose."""

    def __init__(self, ddt, local, dirs, nvars, mode, graph=False, base="double", dst_off=None, comm=None):
        import torch
        self.local, self.dirs, self.nvars = local, dirs, nvars
        self.shape = tuple(n + 2 for n in local)
        self.esz = 8 if base == "double" else 4
        self.nbytes = int(np.prod(self.shape)) * self.esz
        self.q = ddt.Queue()
        self.src = [torch.empty(self.nbytes + 64, dtype=torch.uint8, device="cuda") for _ in range(nvars)]
        self.sep = dst_off is not None
        self.off = dst_off or 0
        self.dst = ([torch.empty(self.nbytes + 64, dtype=torch.uint8, device="cuda") for _ in range(nvars)]
                    if self.sep else self.src)
        for b in self.src + (self.dst if self.sep else []):
            b.fill_(0xA5)
        msgs = halo_messages(0, 1, local, dirs=dirs, nvars=nvars, base=base)
        cache = {}

        def T(spec):
            if repr(spec) not in cache:
                cache[repr(spec)] = ddt.Type.from_spec(spec)
            return cache[repr(spec)]
        sends = [(m["peer"], m["tag"], T(m["send_spec"]), self.src[m["var"]], 1) for m in msgs]
        recvs = [(m["recv_peer"], m["recv_tag"], T(m["recv_spec"]), (self.dst[m["var"]], self.off), 1)
                 for m in msgs]
        self.comm = comm or ddt.Comm.single(torch.cuda.current_device())
        self.h = ddt.Halo(self.q, self.comm, sends, recvs, mode=mode, graph=graph)
        self._types = cache

    def fill(self, it):
        """New random interiors (whole padded arrays: ghosts become random too,
        so a ghost the exchange misses is caught)."""
        import torch
        self.cur = []
        for v in range(self.nvars):
            a = random_bytes(self.nbytes, seed(7, 100 * it + v))
            self.src[v][:self.nbytes].copy_(torch.from_numpy(a))
            self.cur.append(a)
        if self.sep:
            for d in self.dst:
                d.fill_(0xA5)

    def check(self, what=""):
        import torch
        torch.cuda.synchronize()
        gm = ghost_mask(self.local, self.dirs)
        dt = np.int64 if self.esz == 8 else np.int32
        for v in range(self.nvars):
            src = self.cur[v].view(dt).reshape(self.shape)
            exp = np.pad(src[1:-1, 1:-1, 1:-1], 1, mode="wrap")
            got = self.dst[v][self.off:self.off + self.nbytes].cpu().numpy().view(dt).reshape(self.shape)
            assert np.array_equal(got[gm], exp[gm]), f"{what}: var {v} ghost cells differ from np.pad(wrap)"
            if not self.sep:
                assert np.array_equal(got[1:-1, 1:-1, 1:-1], src[1:-1, 1:-1, 1:-1]), f"{what}: interior modified"
            del got, exp

    def close(self):
        self.h.destroy()
        self.comm.close()
        self.q.destroy()


def _run(p, iters, what):
    for it in range(iters):
        p.fill(it)
        p.h.exchange()
        p.check(f"{what} it {it}")


@pytest.mark.parametrize("no_ll", [False, True])
@pytest.mark.parametrize("graph", [False, True])
def test_window_protocol_config1_full_size(ddt, monkeypatch, no_ll, graph):
    """configs[1] (128^3 doubles, 6 faces of 128 KiB) through the window path:
    LL words by default, per-chunk release/acquire flags with DDT_NO_LL=1."""
    _env(monkeypatch, DDT_SELF_VIA_WINDOW="1", **({"DDT_NO_LL": "1"} if no_ll else {}))
    p = Plan(ddt, (128, 128, 128), FACE_DIRS, 1, "p2p", graph=graph)
    _run(p, 3, f"cfg1 window no_ll={no_ll} graph={graph}")
    p.close()


@pytest.mark.timeout(900)
def test_window_protocol_comb_full_size_every_variable(ddt, monkeypatch):
    """configs[3] at its 1-GPU point through the window path: 512^3 doubles x 4
    variables, 26 directions (104 + 104 messages); 2 MiB faces take the
    per-chunk flag protocol, edges / corners LL words.  The full ghost mask of
    EVERY variable is checked, over two exchanges (both window halves)."""
    import torch
    _env(monkeypatch, DDT_SELF_VIA_WINDOW="1")
    local = (512, 512, 512)
    shape = tuple(n + 2 for n in local)
    q = ddt.Queue()
    arrs = [torch.empty(shape, dtype=torch.int64, device="cuda") for _ in range(4)]
    msgs = halo_messages(0, 1, local, dirs=ALL_DIRS, nvars=4)
    cache = {}

    def T(spec):
        if repr(spec) not in cache:
            cache[repr(spec)] = ddt.Type.from_spec(spec)
        return cache[repr(spec)]
    sends = [(m["peer"], m["tag"], T(m["send_spec"]), arrs[m["var"]], 1) for m in msgs]
    recvs = [(m["recv_peer"], m["recv_tag"], T(m["recv_spec"]), arrs[m["var"]], 1) for m in msgs]
    comm = ddt.Comm.single(0)
    h = ddt.Halo(q, comm, sends, recvs, mode="p2p", graph=False)
    g = torch.Generator(device="cuda")
    gm = ghost_mask(local, ALL_DIRS)
    for it in range(2):
        g.manual_seed(seed(4, it))
        for a in arrs:
            a.random_(generator=g)  # ghosts random too: a missed ghost cell is caught
        torch.cuda.synchronize()
        h.exchange()
        torch.cuda.synchronize()
        for v, a in enumerate(arrs):
            got = a.cpu().numpy()
            exp = np.pad(got[1:-1, 1:-1, 1:-1], 1, mode="wrap")
            assert np.array_equal(got[gm], exp[gm]), f"COMB window it {it} var {v}: ghosts differ from np.pad(wrap)"
            del got, exp
    h.destroy()
    comm.close()
    q.destroy()


@pytest.mark.parametrize("local,dirs", [((40, 36, 30), ALL_DIRS), ((4, 260, 260), FACE_DIRS)])
def test_window_protocol_float_layouts(ddt, monkeypatch, local, dirs):
    """4-B elements: rows start at 4 mod 16, vectors are 4 B, LL does not apply
    -> every message takes the per-chunk flag protocol (1 vector per thread
    per item up to 512 KB, 2 above; (4, 260, 260) floats: 264 KiB z faces)."""
    _env(monkeypatch, DDT_SELF_VIA_WINDOW="1")
    p = Plan(ddt, local, dirs, 2, "p2p", base="float")
    _run(p, 3, f"float {local}")
    p.close()


@pytest.mark.parametrize("no_ll", [False, True])
def test_window_protocol_mismatched_widths_fan_out(ddt, monkeypatch, no_ll):
    """Sender arrays 16-B aligned, receiver arrays at byte offset 4: the pack
    side moves 8-B (or phased) vectors, the unpack side 4-B ones, so sender and
    receiver chunk differently -> the message is released as a whole (fan-out
    of all the receiver's chunk flags after the per-message counter reaches
    its item count)."""
    _env(monkeypatch, DDT_SELF_VIA_WINDOW="1", **({"DDT_NO_LL": "1"} if no_ll else {}))
    p = Plan(ddt, (24, 40, 72), ALL_DIRS, 2, "p2p", dst_off=4)
    _run(p, 3, "mismatched widths")
    p.close()


@pytest.mark.parametrize("base,no_ll", [("double", False), ("double", True), ("float", False)])
def test_window_protocol_exchange_pairs(ddt, monkeypatch, base, no_ll):
    """Exchange pairs (+x / -x packs in one item, both ghost ends unpacked in
    one item: two flags waited, two signalled, or two LL words polled
    together), forced on a small 26-direction plan (multi-wave plans pair by
    default), direct and captured in a graph."""
    import torch
    env = {"DDT_SELF_VIA_WINDOW": "1", "DDT_XPAIR_ALWAYS": "1"}
    if no_ll:
        env["DDT_NO_LL"] = "1"
    _env(monkeypatch, **env)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):  # the plan's queue (and the capture) on a side stream
        p = Plan(ddt, (10, 14, 18), ALL_DIRS, 2, "p2p", base=base)
        _run(p, 3, f"exchange pairs {base} no_ll={no_ll}")
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(3):
                p.h.exchange()
        p.fill(7)
        g.replay()
        p.check("exchange pairs graph")
    p.close()


def test_window_protocol_large_faces_graph(ddt, monkeypatch):
    """(4, 260, 260) doubles: 528 KiB z faces (> the LL limit) -> per-chunk
    flags at 2 vectors per thread per item, replayed from a captured graph."""
    _env(monkeypatch, DDT_SELF_VIA_WINDOW="1")
    p = Plan(ddt, (4, 260, 260), FACE_DIRS, 2, "p2p", graph=True)
    _run(p, 4, "large faces graph")
    p.close()


@pytest.mark.parametrize("local,dirs,nvars", [((128, 128, 128), FACE_DIRS, 1), ((10, 12, 14), ALL_DIRS, 2)])
@pytest.mark.parametrize("graph", [False, True])
@pytest.mark.parametrize("mode", ["nccl", "nccl_early"])
def test_nccl_mode_staging_and_sendrecv(ddt, monkeypatch, local, dirs, nvars, graph, mode):
    """NCCL mode with every message through the remote path: fused pack into
    per-peer staging, grouped ncclSend/ncclRecv (here: to self, over a 1-rank
    NCCL communicator), fused unpack from the receive staging.  nccl_early:
    the peer's send/recv group runs on its own stream once the pack kernel's
    per-message completion counters (device memory, stream-waited) show its
    messages packed; the counters are re-armed each exchange (4 iterations,
    direct and graph-replayed)."""
    import torch
    _env(monkeypatch, DDT_SELF_VIA_NCCL="1")
    comm = ddt.Comm.single(torch.cuda.current_device(), nccl=True)
    p = Plan(ddt, local, dirs, nvars, mode, graph=graph, comm=comm)
    assert p.h.launches_per_exchange == 2  # pack batch + unpack batch (NCCL between them)
    _run(p, 4, f"{mode} self {local}")
    p.close()


def test_exchange_completes_while_another_kernel_holds_the_sms(ddt, monkeypatch):
    """A kernel on another stream holds two 1024-thread CTAs on every SM but
    one (so at most a few exchange CTAs are ever resident) until released.
    The window-protocol exchange (more items than its resident grid would
    hold, pack items before the unpack items that wait for them) must finish
    while that kernel is still running: items are claimed by ticket in item
    order, so a waiting CTA never holds back an unclaimed signalling item.
    (The occupier runs with the maximum shared-memory carveout: an SM only
    takes CTAs of a kernel whose carveout it can serve, so an occupier at the
    minimum carveout would keep the exchange off its last SM regardless of
    the item order -- measured: no item ran until the occupier ended.)"""
    import torch
    from gpu_util import occupier
    _env(monkeypatch, DDT_SELF_VIA_WINDOW="1", DDT_NO_LL="1")
    occ = occupier()
    nsm = torch.cuda.get_device_properties(0).multi_processor_count
    p = Plan(ddt, (64, 128, 128), ALL_DIRS, 2, "p2p")
    p.h.set_timeout(5.0)
    # one exchange first: CUDA loads kernels lazily at their first launch, and a
    # module load issued while another kernel holds the GPU can stall behind it
    p.fill(0)
    p.h.exchange()
    p.check("before occupancy")
    p.fill(1)
    torch.cuda.synchronize()
    stop = torch.zeros(1, dtype=torch.int32).pin_memory()
    s_occ = torch.cuda.Stream()
    ctas = 2 * nsm - 1
    started = torch.zeros(ctas, dtype=torch.int32).pin_memory()  # one slot per occupier CTA
    rc = occ.occupy_launch(ctypes.c_void_p(s_occ.cuda_stream), ctas, 1024, ctypes.c_void_p(stop.data_ptr()),
                           ctypes.c_void_p(started.data_ptr()), int(20e9))
    assert rc == 0
    t0 = time.time()
    while int(started.sum()) < ctas and time.time() - t0 < 10:
        time.sleep(0.001)
    assert int(started.sum()) == ctas, "occupier did not become resident"
    p.h.exchange()  # on the queue's stream (the current stream at Plan creation)
    done_stream = torch.cuda.current_stream()
    t0 = time.time()
    finished = False
    while time.time() - t0 < 15:
        if done_stream.query():
            finished = True
            break
        time.sleep(0.002)
    still_occupied = s_occ.query() is False
    stop[0] = 1
    torch.cuda.synchronize()
    assert finished, "exchange did not complete while the SMs were held"
    assert still_occupied, "the occupier finished first: the test did not constrain the exchange"
    p.check("exchange under occupancy")
    p.h.exchange()  # the plan stays usable (epoch from the tickets)
    p.fill(2)
    p.h.exchange()
    p.check("after occupancy")
    p.close()


def test_k_exchanges_captured_in_one_graph(ddt, monkeypatch):
    """The device-resident epoch makes a flagged P2P plan capturable: K = 5
    exchanges of the window protocol in ONE captured graph, replayed twice;
    parity alternates inside the graph (odd K), results exact each time."""
    import torch
    _env(monkeypatch, DDT_SELF_VIA_WINDOW="1")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        p = Plan(ddt, (20, 24, 28), ALL_DIRS, 2, "p2p")
        g = torch.cuda.CUDAGraph()
        p.fill(0)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=s):
            for _ in range(5):
                p.h.exchange()
        for it in range(1, 3):
            p.fill(it)
            g.replay()
            p.check(f"graph replay {it}")
        p.close()


@pytest.mark.parametrize("local,dirs,nvars,base,dst_off", [
    ((128, 128, 128), FACE_DIRS, 1, "double", None),   # configs[1]
    ((10, 14, 18), ALL_DIRS, 2, "double", None),
    ((12, 20, 36), ALL_DIRS, 2, "float", 4),            # receiver at 4 mod 8: 4-B vectors on that side
    ((256, 256, 256), ALL_DIRS, 1, "double", None),     # multi-wave (resident grid claiming chunks)
])
@pytest.mark.parametrize("graph", [False, True])
def test_direct_protocol_pack_free(ddt, monkeypatch, local, dirs, nvars, base, dst_off, graph):
    """P2P_DIRECT (pack-free, §IV-B's DirectIPC path between GPUs):
    with DDT_SELF_VIA_DIRECT=1 the self messages take the remote protocol --
    the receiver's ready flag, the sender's gather straight into the
    "peer's" receive layout (no staging), the per-message done flag the
    receiver waits on -- the one-GPU stand-in for the IPC-mapped peer."""
    _env(monkeypatch, DDT_SELF_VIA_DIRECT="1")
    p = Plan(ddt, local, dirs, nvars, "p2p_direct", graph=graph, base=base, dst_off=dst_off)
    _run(p, 4, f"direct {local} {base} graph={graph}")
    p.close()


def test_direct_protocol_k_exchanges_in_one_graph(ddt, monkeypatch):
    """K = 5 pack-free exchanges (ready / done flags, device-resident epoch)
    captured in one graph, replayed twice."""
    import torch
    _env(monkeypatch, DDT_SELF_VIA_DIRECT="1")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        p = Plan(ddt, (20, 24, 28), ALL_DIRS, 2, "p2p_direct")
        g = torch.cuda.CUDAGraph()
        p.fill(0)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=s):
            for _ in range(5):
                p.h.exchange()
        for it in range(1, 3):
            p.fill(it)
            g.replay()
            p.check(f"direct graph replay {it}")
        p.close()


@pytest.mark.parametrize("dst_off", [None, 4])
def test_window_protocol_multiwave_chunk_flags(ddt, monkeypatch, dst_off):
    """A multi-wave plan (resident grid claiming chunks) with every message on
    per-chunk flags (DDT_NO_LL=1): messages <= 512 KB keep their 1-vector
    items (xub_for, the chunking the receiver's flags assume) -- a regression
    test for the multi-wave table build once resetting every item size to the
    plan's; dst_off = 4: different vector widths on the two sides, the
    whole-message release through the per-message counter."""
    _env(monkeypatch, DDT_SELF_VIA_WINDOW="1", DDT_NO_LL="1")
    p = Plan(ddt, (200, 200, 200), ALL_DIRS, 1, "p2p", dst_off=dst_off)
    _run(p, 3, f"multi-wave flags dst_off={dst_off}")
    p.close()
