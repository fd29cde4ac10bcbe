"""Seeded synthetic graphs shaped like the paper's input families.

PAPER.md §4 (Table 2): inputs are undirected, stored in CSR
with both directions of every edge (P:329 fn 2), cleaned of self-loops and
multi-edges, with integer weights (random where the source graph had none).
The five BASELINE.json configs mirror Table 2's families; the recipes are
stated in DESIGN.md §"Input recipe" and in SURVEY.md §8(d):

  grid     C1  512x512 4-neighbour lattice, uniform int weights in [0, 2^31)
  road     C2  6000x4000 jittered lattice, all horizontal + 20% vertical
               edges, weight = round(1000 * Euclidean length)  (heavy ties)
  rgg      C3  random geometric graph, 2^24 points, expected degree 6,
               weight = round(dist / r * 2^30), ids in spatial cell order
  rmat     C4  Graph500 RMAT scale 24, edge factor 16, (.57,.19,.19,.05),
               random vertex permutation, uniform int weights
  uniform  C5  G(n, m): 2^26 vertices, 1e9 uniform pairs, uniform weights

All randomness is counter-based (synth.rng), so a graph is a pure function of
its parameters and seed on any device.  Generators return torch tensors on the
requested device; nothing here computes anything about spanning forests.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import torch

from . import rng

# stream ids (fixed forever: changing one changes every graph)
_S_W = 1        # weights
_S_X, _S_Y = 2, 3
_S_EDGE = 4     # edge keep / draw
_S_PERM = 5
_S_U, _S_V = 6, 7


@dataclass
class Graph:
    """CSR graph: row u owns entries nindex[u] .. nindex[u+1]-1."""
    n: int
    nindex: torch.Tensor   # int64 [n+1]
    nlist: torch.Tensor    # int32 [M]
    eweight: torch.Tensor  # int32 [M]
    name: str = ""
    meta: dict = field(default_factory=dict)

    @property
    def M(self) -> int:
        return int(self.nlist.numel())

    def to(self, device) -> "Graph":
        return Graph(self.n, self.nindex.to(device), self.nlist.to(device),
                     self.eweight.to(device), self.name, dict(self.meta))

    def numpy(self):
        return (self.n, self.nindex.cpu().numpy(), self.nlist.cpu().numpy(),
                self.eweight.cpu().numpy())

    def stats(self) -> dict:
        """Table-2-style columns that need no graph algorithm."""
        deg = (self.nindex[1:] - self.nindex[:-1]) if self.n else self.nindex[:0]
        return {"name": self.name, "n": self.n, "M": self.M,
                "d_avg": (self.M / self.n) if self.n else 0.0,
                "d_max": int(deg.max()) if self.n and self.M else 0}


# ----------------------------------------------------------------------------
# CSR builders
# ----------------------------------------------------------------------------

def csr_from_entries(n: int, src: torch.Tensor, dst: torch.Tensor, w: torch.Tensor,
                     name: str = "") -> Graph:
    """CSR from an explicit directed entry list (kept as is: self-loops,
    multi-edges and missing mirrors survive).  Rows sorted by (src, dst,
    original position) so the result is deterministic."""
    src = src.to(torch.int64)
    dst = dst.to(torch.int64)
    dev = src.device
    M = src.numel()
    if M:
        key = src * max(n, 1) + dst
        order = torch.sort(key, stable=True).indices
        src, dst, w = src[order], dst[order], w[order]
    counts = torch.bincount(src, minlength=n) if M else torch.zeros(n, dtype=torch.int64, device=dev)
    nindex = torch.zeros(n + 1, dtype=torch.int64, device=dev)
    if n:
        nindex[1:] = torch.cumsum(counts, 0)
    return Graph(n, nindex, dst.to(torch.int32), w.to(torch.int32), name)


def csr_from_undirected(n: int, u: torch.Tensor, v: torch.Tensor, w: torch.Tensor,
                        name: str = "") -> Graph:
    """Symmetric CSR (both directions, same weight) from an undirected list."""
    return csr_from_entries(n, torch.cat([u, v]), torch.cat([v, u]), torch.cat([w, w]), name)


def csr_from_pairs(n: int, u: torch.Tensor, v: torch.Tensor, wfn, name: str = "",
                   chunk: int = 1 << 28) -> Graph:
    """Symmetric, cleaned CSR from candidate pairs: self-loops and duplicate
    pairs are dropped, back edges are added.  Weights
    come from wfn(a, b) with a < b, so both directions agree and the builder
    never has to carry weights through the sort.
    """
    u = u.to(torch.int64)
    v = v.to(torch.int64)
    keep = u != v
    u, v = u[keep], v[keep]
    keys = torch.minimum(u, v) * n + torch.maximum(u, v)
    del u, v, keep
    return csr_from_keys(n, keys, wfn, name, chunk)


def csr_from_keys(n: int, keys: torch.Tensor, wfn, name: str = "", chunk: int = 1 << 28) -> Graph:
    """As csr_from_pairs, from canonical keys a*n + b (a < b, duplicates allowed).
    Works in chunks so a 1e9-edge graph fits comfortably in one GPU."""
    dev = keys.device
    canon = torch.unique(keys)          # sorted, deduplicated canonical pairs
    del keys
    m = canon.numel()
    mirror = torch.empty_like(canon)
    for s in range(0, m, chunk):
        a = canon[s:s + chunk] // n
        mirror[s:s + chunk] = (canon[s:s + chunk] - a * n) * n + a
    allk = _sorted_union(canon, mirror)  # both directions, sorted by (src, dst)
    del canon, mirror
    M = allk.numel()
    counts = torch.zeros(n, dtype=torch.int64, device=dev)
    nlist = torch.empty(M, dtype=torch.int32, device=dev)
    eweight = torch.empty(M, dtype=torch.int32, device=dev)
    for s in range(0, M, chunk):
        k = allk[s:s + chunk]
        src = k // n
        dst = k - src * n
        counts += torch.bincount(src, minlength=n)
        nlist[s:s + chunk] = dst.to(torch.int32)
        eweight[s:s + chunk] = wfn(torch.minimum(src, dst), torch.maximum(src, dst)).to(torch.int32)
        del k, src, dst
    del allk
    nindex = torch.zeros(n + 1, dtype=torch.int64, device=dev)
    nindex[1:] = torch.cumsum(counts, 0)
    g = Graph(n, nindex, nlist, eweight, name)
    g.meta["m_undirected"] = int(m)
    return g


def _sorted_union(a: torch.Tensor, b: torch.Tensor, buckets: int = 8) -> torch.Tensor:
    """Sorted concatenation of two disjoint sorted int64 tensors (key-range
    buckets keep every individual sort well below 2^31 elements)."""
    total = a.numel() + b.numel()
    if total <= (1 << 29):
        return torch.sort(torch.cat([a, b])).values
    lo = min(int(a[0]), int(b.min()))
    hi = max(int(a[-1]), int(b.max())) + 1
    step = (hi - lo + buckets - 1) // buckets
    out = torch.empty(total, dtype=a.dtype, device=a.device)
    pos = 0
    for i in range(buckets):
        x0, x1 = lo + i * step, lo + (i + 1) * step
        ia0, ia1 = torch.searchsorted(a, torch.tensor([x0, x1], device=a.device)).tolist()
        part_b = b[(b >= x0) & (b < x1)]
        part = torch.sort(torch.cat([a[ia0:ia1], part_b])).values
        out[pos:pos + part.numel()] = part
        pos += part.numel()
        del part, part_b
    assert pos == total
    return out


def _hash_weight(seed: int, n: int):
    def wfn(a, b):
        return rng.uniform_int31(seed, _S_W, a * n + b)
    return wfn


# ----------------------------------------------------------------------------
# the five families
# ----------------------------------------------------------------------------

def grid2d(width: int = 512, height: int = 512, seed: int = 1, device="cpu") -> Graph:
    """C1: 4-neighbour grid (Table 2 '2d-2e20.sym'); id = y*width + x."""
    n = width * height
    ids = torch.arange(n, dtype=torch.int64, device=device)
    x = ids % width
    y = ids // width
    hu = ids[x < width - 1]
    vu = ids[y < height - 1]
    u = torch.cat([hu, vu])
    v = torch.cat([hu + 1, vu + width])
    g = csr_from_pairs(n, u, v, _hash_weight(seed, n), name=f"grid{width}x{height}")
    g.meta.update(family="grid", seed=seed, width=width, height=height)
    return g


def road_like(width: int = 6000, height: int = 4000, p_vertical: float = 0.2,
              jitter: float = 0.35, seed: int = 2, device="cpu") -> Graph:
    """C2: road-network-like graph (Table 2 'USA-road-d.*').

    Jittered lattice points; every horizontal neighbour pair is an edge, each
    vertical pair w.p. p_vertical (avg degree ~2.4, max 4, long diameter);
    weight = round(1000 * Euclidean distance) -> integers ~[300, 1700] with
    heavy ties.  Row-major ids keep spatial locality like DIMACS road maps.
    """
    n = width * height
    ids = torch.arange(n, dtype=torch.int64, device=device)
    gx = (ids % width).to(torch.float64)
    gy = (ids // width).to(torch.float64)
    px = gx + (rng.uniform_f64(seed, _S_X, ids) * 2.0 - 1.0) * jitter
    py = gy + (rng.uniform_f64(seed, _S_Y, ids) * 2.0 - 1.0) * jitter
    x = ids % width
    y = ids // width
    hu = ids[x < width - 1]
    vcand = ids[y < height - 1]
    vu = vcand[rng.bernoulli(seed, _S_EDGE, vcand, p_vertical)]
    u = torch.cat([hu, vu])
    v = torch.cat([hu + 1, vu + width])

    def wfn(a, b):
        dx = px[a] - px[b]
        dy = py[a] - py[b]
        return torch.round(torch.sqrt(dx * dx + dy * dy) * 1000.0).to(torch.int64)

    g = csr_from_pairs(n, u, v, wfn, name=f"road{width}x{height}")
    g.meta.update(family="road", seed=seed, width=width, height=height, p_vertical=p_vertical)
    return g


def rgg2d(n: int = 1 << 24, avg_degree: float = 6.0, seed: int = 3, device="cpu") -> Graph:
    """C3: 2D random geometric graph standing in for 'delaunay_n24'.

    n uniform points in the unit square, edge iff distance < r with
    r = sqrt(avg_degree / (pi n)); vertex ids follow the spatial cell order;
    weight = round(dist / r * 2^30).  Unlike a triangulation it has many small
    components (an MSF input).
    """
    ids = torch.arange(n, dtype=torch.int64, device=device)
    x = rng.uniform_f64(seed, _S_X, ids)
    y = rng.uniform_f64(seed, _S_Y, ids)
    r = math.sqrt(avg_degree / (math.pi * n))
    G = max(1, int(math.floor(1.0 / r)))
    cx = torch.clamp((x * G).to(torch.int64), max=G - 1)
    cy = torch.clamp((y * G).to(torch.int64), max=G - 1)
    cell = cy * G + cx
    order = torch.sort(cell, stable=True).indices
    x, y, cx, cy, cell = x[order], y[order], cx[order], cy[order], cell[order]
    del order
    counts = torch.bincount(cell, minlength=G * G)
    start = torch.zeros(G * G + 1, dtype=torch.int64, device=device)
    start[1:] = torch.cumsum(counts, 0)
    maxocc = int(counts.max())
    r2 = r * r
    us, vs = [], []
    for dx, dy in ((0, 0), (1, 0), (-1, 1), (0, 1), (1, 1)):
        ncx = cx + dx
        ncy = cy + dy
        ok = (ncx >= 0) & (ncx < G) & (ncy < G)
        src = ids[ok]
        nc = ncy[ok] * G + ncx[ok]
        s = start[nc]
        e = start[nc + 1]
        for k in range(maxocc):
            j = s + k
            valid = j < e
            if not bool(valid.any()):
                break
            if dx == 0 and dy == 0:
                valid &= j > src
            i_v = src[valid]
            j_v = j[valid]
            ddx = x[i_v] - x[j_v]
            ddy = y[i_v] - y[j_v]
            close = (ddx * ddx + ddy * ddy) < r2
            us.append(i_v[close])
            vs.append(j_v[close])
    u = torch.cat(us) if us else ids[:0]
    v = torch.cat(vs) if vs else ids[:0]
    del us, vs

    def wfn(a, b):
        ddx = x[a] - x[b]
        ddy = y[a] - y[b]
        return torch.round(torch.sqrt(ddx * ddx + ddy * ddy) / r * float(1 << 30)).to(torch.int64)

    g = csr_from_pairs(n, u, v, wfn, name=f"rgg{n}")
    g.meta.update(family="rgg", seed=seed, avg_degree=avg_degree, radius=r)
    return g


def _random_permutation(n: int, seed: int, device) -> torch.Tensor:
    ids = torch.arange(n, dtype=torch.int64, device=device)
    h = rng.hash_u64(seed, _S_PERM, ids)
    order = torch.sort(h, stable=True).indices
    newid = torch.empty_like(order)
    newid[order] = ids
    return newid


def rmat(scale: int = 24, edge_factor: int = 16, a: float = 0.57, b: float = 0.19,
         c: float = 0.19, seed: int = 4, device="cpu", chunk: int = 1 << 24) -> Graph:
    """C4: Graph500-style RMAT/Kronecker graph (Table 2 'rmat22.sym',
    'kron_g500-logn21'): power-law degrees, many isolated vertices
    and components; random vertex permutation; uniform int weights."""
    n = 1 << scale
    m_draws = edge_factor * n
    tA = int(a * (1 << 53))
    tAB = int((a + b) * (1 << 53))
    tABC = int((a + b + c) * (1 << 53))
    perm = _random_permutation(n, seed, device)
    parts = []
    for s0 in range(0, m_draws, chunk):
        d = torch.arange(s0, min(m_draws, s0 + chunk), dtype=torch.int64, device=device)
        u = torch.zeros_like(d)
        v = torch.zeros_like(d)
        for lvl in range(scale):
            r = rng._srl(rng.hash_u64(seed, _S_EDGE, d * scale + lvl), 11)
            ub = (r >= tAB).to(torch.int64)
            vb = (((r >= tA) & (r < tAB)) | (r >= tABC)).to(torch.int64)
            u = u | (ub << (scale - 1 - lvl))
            v = v | (vb << (scale - 1 - lvl))
        u = perm[u]
        v = perm[v]
        keep = u != v
        u, v = u[keep], v[keep]
        parts.append(torch.minimum(u, v) * n + torch.maximum(u, v))
        del d, u, v, keep
    del perm
    keys = torch.cat(parts)
    del parts
    g = csr_from_keys(n, keys, _hash_weight(seed, n), name=f"rmat{scale}")
    g.meta.update(family="rmat", seed=seed, scale=scale, edge_factor=edge_factor)
    return g


def uniform_random(n: int = 1 << 26, m_draws: int = 1_000_000_000, seed: int = 5,
                   device="cpu", chunk: int = 1 << 27) -> Graph:
    """C5: uniform random graph G(n, m) (Table 2 'r4-2e23.sym')."""
    parts = []
    for s0 in range(0, m_draws, chunk):
        d = torch.arange(s0, min(m_draws, s0 + chunk), dtype=torch.int64, device=device)
        u = rng.below(seed, _S_U, d, n)
        v = rng.below(seed, _S_V, d, n)
        keep = u != v
        u, v = u[keep], v[keep]
        parts.append(torch.minimum(u, v) * n + torch.maximum(u, v))
        del d, u, v, keep
    keys = torch.cat(parts)
    del parts
    g = csr_from_keys(n, keys, _hash_weight(seed, n), name=f"uniform{n}")
    g.meta.update(family="uniform", seed=seed, m_draws=m_draws)
    return g


# ----------------------------------------------------------------------------
# small structured / adversarial graphs for tests
# ----------------------------------------------------------------------------

def _weights(kind: str, seed: int, idx: torch.Tensor) -> torch.Tensor:
    """Weight distributions for adversarial tests."""
    h = rng.hash_u64(seed, _S_W, idx)
    if kind == "uniform":
        return rng._srl(h, 33)                      # [0, 2^31)
    if kind == "full":                              # all of int32, incl. extremes
        w = (h >> 32)                               # arithmetic: [-2^31, 2^31)
        ext = rng._srl(h, 1) % 8
        w = torch.where(ext == 0, torch.full_like(w, -(1 << 31)), w)
        w = torch.where(ext == 1, torch.full_like(w, (1 << 31) - 1), w)
        return w
    if kind == "ties":                              # [-3, 3): tie-heavy, negative
        return rng._srl(h, 1) % 6 - 3
    if kind == "equal":
        return torch.full_like(idx, 7)
    if kind == "two":                               # mostly 7, a few 0
        return torch.where(rng._srl(h, 1) % 25 == 0, torch.zeros_like(idx), torch.full_like(idx, 7))
    raise ValueError(kind)


def random_small(n: int, m: int, seed: int = 0, weights: str = "ties",
                 multi: bool = False, self_loops: bool = False, device="cpu") -> Graph:
    """Random undirected (multi)graph with n vertices and m edge draws,
    symmetric CSR.  With multi=False duplicates and self-loops are removed."""
    d = torch.arange(m, dtype=torch.int64, device=device)
    u = rng.below(seed, _S_U, d, max(n, 1))
    v = rng.below(seed, _S_V, d, max(n, 1))
    w = _weights(weights, seed, d)
    if not self_loops:
        keep = u != v
        u, v, w, d = u[keep], v[keep], w[keep], d[keep]
    if not multi:
        a = torch.minimum(u, v)
        b = torch.maximum(u, v)
        key = a * max(n, 1) + b
        _, inv = torch.unique(key, return_inverse=True)
        first = torch.full((int(inv.max()) + 1 if inv.numel() else 0,), m, dtype=torch.int64, device=device)
        first.scatter_reduce_(0, inv, torch.arange(inv.numel(), device=device), reduce="amin")
        u, v, w = u[first], v[first], w[first]
    g = csr_from_undirected(n, u, v, w, name=f"small{n}_{m}_{weights}")
    g.meta.update(family="small", seed=seed, weights=weights)
    return g


def complete_graph(n: int, seed: int = 0, weights: str = "uniform", device="cpu") -> Graph:
    a, b = torch.triu_indices(n, n, 1, device=device)
    a = a.to(torch.int64)
    b = b.to(torch.int64)
    w = _weights(weights, seed, a * n + b)
    g = csr_from_undirected(n, a, b, w, name=f"K{n}")
    g.meta.update(family="complete", seed=seed)
    return g


def path_graph(n: int, weights: torch.Tensor | None = None, device="cpu") -> Graph:
    a = torch.arange(max(n - 1, 0), dtype=torch.int64, device=device)
    w = a.clone() if weights is None else weights.to(torch.int64)
    return csr_from_undirected(n, a, a + 1, w, name=f"path{n}")


def cycle_graph(n: int, seed: int = 0, weights: str = "uniform", device="cpu") -> Graph:
    a = torch.arange(n, dtype=torch.int64, device=device)
    b = (a + 1) % n
    w = _weights(weights, seed, a)
    return csr_from_undirected(n, a, b, w, name=f"cycle{n}")


def star_graph(n: int, seed: int = 0, weights: str = "uniform", device="cpu") -> Graph:
    """Hub 0 joined to every other vertex (one very high-degree row)."""
    b = torch.arange(1, n, dtype=torch.int64, device=device)
    a = torch.zeros_like(b)
    w = _weights(weights, seed, b)
    return csr_from_undirected(n, a, b, w, name=f"star{n}")


# ----------------------------------------------------------------------------
# named configs (BASELINE.json "configs", in order)
# ----------------------------------------------------------------------------

CONFIGS = {
    # name: (builder, full-size kwargs, small kwargs for CPU-oracle parity)
    "grid": (grid2d, dict(width=512, height=512, seed=1), dict(width=100, height=37, seed=1)),
    "road": (road_like, dict(width=6000, height=4000, seed=2), dict(width=300, height=211, seed=2)),
    "rgg": (rgg2d, dict(n=1 << 24, seed=3), dict(n=(1 << 15) + 123, seed=3)),
    "rmat": (rmat, dict(scale=24, edge_factor=16, seed=4), dict(scale=14, edge_factor=16, seed=4)),
    "uniform": (uniform_random, dict(n=1 << 26, m_draws=1_000_000_000, seed=5),
                dict(n=(1 << 14) + 7, m_draws=1 << 18, seed=5)),
}


def make_config(name: str, size: str = "full", device="cpu", **overrides) -> Graph:
    fn, full, small = CONFIGS[name]
    kw = dict(full if size == "full" else small)
    kw.update(overrides)
    g = fn(device=device, **kw)
    g.meta["config"] = name
    g.meta["size"] = size
    return g
