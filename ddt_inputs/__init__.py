"""Seeded synthetic inputs and workload recipes shared by the oracle side and the
CUDA side.  This module holds NO datatype arithmetic: it never packs, unpacks,
flattens or computes a size/extent.  It only produces

* random byte buffers (PCG64 via numpy.random.default_rng, SURVEY §8(d) "Inputs"),
* datatype *spec tuples* (the neutral constructor language both sides parse
  independently; see oracle/__init__.py for the grammar),
* halo-exchange message recipes (which subarray goes to which neighbour, with
  which tag) for BASELINE.json configs 2 and 4.

Seeds: ``seed = 20200914 + 1000*config + var``.
"""
from __future__ import annotations

import itertools

import numpy as np

SEED0 = 20200914
SENTINEL = 0xA5


def seed(config: int, var: int = 0) -> int:
    return SEED0 + 1000 * int(config) + int(var)


def random_bytes(nbytes: int, s: int) -> np.ndarray:
    """`nbytes` random bytes (random 64-bit patterns: NaN/Inf/denormal/-0 included
    when viewed as float)."""
    n64 = (int(nbytes) + 7) // 8
    a = np.random.default_rng(s).integers(0, 2**64, size=n64, dtype=np.uint64, endpoint=False)
    return a.view(np.uint8)[: int(nbytes)].copy()


def sentinel_bytes(nbytes: int) -> np.ndarray:
    return np.full(int(nbytes), SENTINEL, dtype=np.uint8)


# ----------------------------------------------------------------- config 1
def config1_spec():
    """BASELINE.json configs[0]: MPI_Type_vector(count=16, blocklen=4, stride=64) of double."""
    return ("vector", 16, 4, 64, ("basic", "double"))


# ----------------------------------------------------------------- config 3
def config3_spec(nblocks: int = 100_000, npoints: int = 1 << 20, s: int | None = None,
                 shuffled: bool = False):
    """BASELINE.json configs[2]: specfem3D-like sparse hindexed layout: `nblocks`
    blocks of 3 floats (12 B) at byte displacement 12*idx, idx a sorted random
    subset of `npoints` points.  Returns (spec, src_bytes)."""
    rng = np.random.default_rng(seed(3) if s is None else s)
    idx = np.sort(rng.choice(npoints, size=nblocks, replace=False)).astype(np.int64)
    if shuffled:
        idx = rng.permutation(idx)
    spec = ("hindexed", [3] * nblocks, (12 * idx).tolist(), ("basic", "float"))
    return spec, 12 * npoints


def config3_cm_spec(nblocks: int = 100_000, npoints: int = 1 << 20, s: int | None = None):
    """specfem3D_cm-style struct-on-indexed layout (SURVEY
    W2): three float field arrays of `npoints` each (x, y, z stored one after the
    other), one indexed(1-float blocks at idx) type per component, combined by a
    struct at the arrays' byte offsets.  Returns (spec, src_bytes)."""
    rng = np.random.default_rng(seed(3, 7) if s is None else s)
    idx = np.sort(rng.choice(npoints, size=nblocks, replace=False)).astype(np.int64).tolist()
    comp = ("indexed", [1] * nblocks, idx, ("basic", "float"))
    spec = ("struct", [1, 1, 1], [0, 4 * npoints, 8 * npoints], [comp, comp, comp])
    return spec, 12 * npoints


def milc_spec(L: int = 16):
    """MILC-style nested vector ("nested vectors (MILC)"; SURVEY
    D2/W4): the y = 0 face of an L^4 lattice of su3 vectors (3 complex doubles =
    6 doubles per site, x fastest): an hvector over t of a vector over z of
    x-rows.  Returns (spec, footprint_bytes)."""
    row = L * 6                                   # doubles per x-row
    inner = ("vector", L, row, L * row, ("basic", "double"))          # z rows at stride L*L sites
    spec = ("hvector", L, 1, L ** 3 * 6 * 8, inner)                   # t planes at stride L^3 sites
    return spec, L ** 4 * 48


def nas_mg_specs(n1: int = 34, n2: int = 34, n3: int = 34):
    """NAS_MG-style face types ("vectors (NAS_MG)"; ddtbench's
    MG kernel): the three boundary faces of an n1 x n2 x n3 grid of doubles, x
    (extent n1) fastest, each face at its first index (i = 0, j = 0, k = 0):
      x face: vector(n2*n3, 1, n1)        -- one element per x-row
      y face: vector(n3, n1, n1*n2)       -- one x-row per plane
      z face: contiguous(n1*n2)           -- one whole plane
    Returns ({"x": spec, "y": spec, "z": spec}, footprint_bytes)."""
    d = ("basic", "double")
    specs = {"x": ("vector", n2 * n3, 1, n1, d),
             "y": ("vector", n3, n1, n1 * n2, d),
             "z": ("contiguous", n1 * n2, d)}
    return specs, n1 * n2 * n3 * 8


# ----------------------------------------------------------------- config 5
def config5_spec(S: int):
    """BASELINE.json configs[4]: dense vector of doubles, block = min(S, 256 B),
    count = S/block, stride = 2*block (50% density).  Returns (spec, footprint)."""
    blk = min(S, 256)
    assert S % blk == 0 and blk % 8 == 0
    count = S // blk
    b = blk // 8
    spec = ("vector", count, b, 2 * b, ("basic", "double"))
    footprint = ((count - 1) * 2 * b + b) * 8
    return spec, footprint


CONFIG5_SIZES = [64 * 4**k for k in range(11)]          # 64 B .. 64 MiB
CONFIG5_BATCHES = [1, 4, 16, 64, 256, 1024]


# ----------------------------------------------------- halo (configs 2, 4)
def proc_grid(P: int):
    """Periodic Cartesian process grid (pz, py, px), slowest dim split first."""
    return {1: (1, 1, 1), 2: (2, 1, 1), 4: (2, 2, 1), 8: (2, 2, 2)}[int(P)]


def rank_of(coords, grid):
    cz, cy, cx = coords
    return (cz * grid[1] + cy) * grid[2] + cx


def coords_of(rank, grid):
    pz, py, px = grid
    return (rank // (py * px), (rank // px) % py, rank % px)


FACE_DIRS = [d for d in itertools.product((-1, 0, 1), repeat=3) if sum(map(abs, d)) == 1]
ALL_DIRS = [d for d in itertools.product((-1, 0, 1), repeat=3) if d != (0, 0, 0)]


def dir_index(d):
    """0..26 index of a direction (dz,dy,dx) in {-1,0,1}^3 (13 = self, unused)."""
    return (d[0] + 1) * 9 + (d[1] + 1) * 3 + (d[2] + 1)


def _region(n, side, ghost: bool):
    """(start, subsize) along one axis of a (n+2)-long ghosted axis."""
    if side == 0:
        return 1, n
    if ghost:
        return (0, 1) if side < 0 else (n + 1, 1)
    return (1, 1) if side < 0 else (n, 1)


def halo_messages(rank: int, P: int, local, dirs=ALL_DIRS, nvars: int = 1, base="double"):
    """Messages of one rank for one halo exchange (Alg 3: one
    Isend and one Irecv per boundary buffer; COMB-style 3-D decomposition [33]).

    local: interior shape (nz, ny, nx); arrays are (nz+2, ny+2, nx+2), C order,
    ghost width 1, periodic.  Returns a list of dicts
      {peer, tag, var, dir, send_spec, recv_peer, recv_tag, recv_spec}
    where the send goes to `peer` with `tag` and the receive (filling the ghost
    on side `dir`) comes from `recv_peer` with `recv_tag`.  Tags:
    dir_index(sender's direction) * nvars + var."""
    grid = proc_grid(P)
    c = coords_of(rank, grid)
    nz, ny, nx = local
    sizes = [nz + 2, ny + 2, nx + 2]
    out = []
    for var in range(nvars):
        for d in dirs:
            peer_c = tuple((c[k] + d[k]) % grid[k] for k in range(3))
            src_c = tuple((c[k] + d[k]) % grid[k] for k in range(3))  # ghost side d filled by neighbour at c+d
            send = [_region(n, s, ghost=False) for n, s in zip(local, d)]
            recv = [_region(n, s, ghost=True) for n, s in zip(local, d)]
            neg = tuple(-x for x in d)
            out.append(dict(
                var=var, dir=d,
                peer=rank_of(peer_c, grid), tag=dir_index(d) * nvars + var,
                send_spec=("subarray", sizes, [r[1] for r in send], [r[0] for r in send], "C", ("basic", base)),
                recv_peer=rank_of(src_c, grid), recv_tag=dir_index(neg) * nvars + var,
                recv_spec=("subarray", sizes, [r[1] for r in recv], [r[0] for r in recv], "C", ("basic", base)),
            ))
    return out


def global_block(global_arr: np.ndarray, rank: int, P: int):
    """The rank's interior block of a global (Z, Y, X) array."""
    grid = proc_grid(P)
    c = coords_of(rank, grid)
    Z, Y, X = global_arr.shape
    nz, ny, nx = Z // grid[0], Y // grid[1], X // grid[2]
    return global_arr[c[0] * nz:(c[0] + 1) * nz, c[1] * ny:(c[1] + 1) * ny, c[2] * nx:(c[2] + 1) * nx]


def padded_block(global_arr: np.ndarray, rank: int, P: int):
    """Expected post-exchange local array (26-neighbour case): the rank's block
    +-1 cell of numpy's periodic ('wrap') padding of the global array."""
    grid = proc_grid(P)
    c = coords_of(rank, grid)
    Z, Y, X = global_arr.shape
    nz, ny, nx = Z // grid[0], Y // grid[1], X // grid[2]
    g = np.pad(global_arr, 1, mode="wrap")
    return g[c[0] * nz:(c[0] + 1) * nz + 2, c[1] * ny:(c[1] + 1) * ny + 2, c[2] * nx:(c[2] + 1) * nx + 2]


def ghost_mask(local, dirs):
    """Boolean mask over the (nz+2, ny+2, nx+2) array of the ghost cells that the
    given directions fill."""
    nz, ny, nx = local
    m = np.zeros((nz + 2, ny + 2, nx + 2), dtype=bool)
    for d in dirs:
        sl = []
        for n, s in zip(local, d):
            a, b = _region(n, s, ghost=True)
            sl.append(slice(a, a + b))
        m[tuple(sl)] = True
    return m
