"""Pins for the CPU oracle (oracle/kruskal.c) -- no GPU needed.

Each test checks the oracle against something other than itself: brute force,
an independent Prim, the lighter-edge connectivity characterisation, scipy's
MST weight, structural invariants, closed forms, and Frieze's zeta(3) limit.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from synth import graphs as G
from tests import refs
from tests.fixtures import asymmetric_graph, empty_graph, load_fig2


def run(g):
    return oracle.kruskal_graph(g)


# --- brute force on tiny graphs (all weight regimes, multigraphs, loops) ---

@pytest.mark.parametrize("seed", range(60))
def test_brute_force_tiny(seed):
    kinds = ["ties", "equal", "two", "full", "uniform"]
    n = 2 + seed % 6
    m = 3 + (seed * 7) % 10
    g = G.random_small(n, m, seed=seed, weights=kinds[seed % 5],
                       multi=(seed % 3 == 0), self_loops=(seed % 4 == 0))
    mask, total, count = run(g)
    bmask, btotal, k, bmin = refs.brute_force_msf(*g.numpy())
    assert np.array_equal(mask, bmask)
    assert total == btotal == bmin           # unique (w,id)-MSF also minimises sum w
    assert count == k


# --- independent Prim and the cycle-property characterisation ---

@pytest.mark.parametrize("seed,weights,multi", [
    (s, w, mu) for s in range(4) for w in ("ties", "two", "full", "uniform") for mu in (False, True)])
def test_prim_and_characterisation(seed, weights, multi):
    g = G.random_small(40 + seed, 160, seed=100 + seed, weights=weights, multi=multi, self_loops=multi)
    mask, total, count = run(g)
    pmask, ptotal, pcount = refs.prim_msf(*g.numpy())
    assert np.array_equal(mask, pmask)
    assert (total, count) == (ptotal, pcount)
    cmask = refs.lighter_path_msf(*g.numpy())
    assert np.array_equal(mask, cmask)


@pytest.mark.parametrize("name", list(synth.CONFIGS))
def test_config_shapes_prim_invariants(name):
    """Small instances of the five BASELINE configs: Prim + invariants."""
    g = synth.make_config(name, "small")
    mask, total, count = run(g)
    pmask, ptotal, _ = refs.prim_msf(*g.numpy())
    assert np.array_equal(mask, pmask)
    assert total == ptotal
    inv = refs.check_forest(*g.numpy(), mask)
    assert all(inv.values()), inv


def test_scipy_weight_crosscheck():
    scipy_sparse = pytest.importorskip("scipy.sparse")
    csgraph = pytest.importorskip("scipy.sparse.csgraph")
    for seed, weights in [(1, "uniform"), (2, "ties"), (3, "full")]:
        g = G.random_small(300, 2000, seed=seed, weights=weights)
        n, nindex, nlist, eweight = g.numpy()
        u, v, w, _ = refs.canonical_edges(n, nindex, nlist, eweight)
        mask, total, count = oracle.kruskal(n, nindex, nlist, eweight)
        # every spanning forest has n - #CC edges, so a constant shift that
        # makes all weights positive (scipy drops zeros) preserves the optimum
        shift = 1 - int(w.min())
        A = scipy_sparse.coo_matrix(((w + shift).astype(np.float64), (u, v)), shape=(n, n)).tocsr()
        T = csgraph.minimum_spanning_tree(A)
        ncc, _ = csgraph.connected_components(A, directed=False)
        assert count == n - ncc
        assert int(round(T.sum())) - shift * count == total


# --- closed forms and special cases ---

def test_fig2_reconstruction():
    g, ids, mst, weight = load_fig2()
    mask, total, count = run(g)
    assert total == weight
    assert {lab for lab, j in ids.items() if mask[j]} == mst
    assert count == 3


def test_tree_input_keeps_every_edge():
    for seed in range(5):
        n = 200
        parent = synth.rng.below(seed, 9, torch.arange(1, n), 1 << 30) % torch.arange(1, n)
        child = torch.arange(1, n)
        w = synth.rng.uniform_int31(seed, 1, child) - (1 << 30)
        g = G.csr_from_undirected(n, parent, child, w)
        mask, total, count = run(g)
        assert count == n - 1 and total == int(w.sum())
        n_, nindex, nlist, _ = g.numpy()
        u, v, _, ids = refs.canonical_edges(n_, nindex, nlist, g.eweight.numpy())
        assert mask.sum() == n - 1 and np.all(mask[ids] == 1)


def test_cycle_drops_exactly_the_max():
    for seed, weights in [(0, "uniform"), (1, "ties"), (2, "equal")]:
        g = G.cycle_graph(57, seed=seed, weights=weights)
        n, nindex, nlist, eweight = g.numpy()
        u, v, w, ids = refs.canonical_edges(n, nindex, nlist, eweight)
        mask, total, count = run(g)
        worst = max(range(len(ids)), key=lambda i: (int(w[i]), int(ids[i])))
        expect = np.zeros_like(mask)
        expect[ids] = 1
        expect[ids[worst]] = 0
        assert np.array_equal(mask, expect)
        assert total == int(w.sum()) - int(w[worst])


def test_equal_weights_is_index_order():
    """All weights equal: the (w, id) order is the id order, so edge id j is
    in the MSF iff its ends are not joined by edges with smaller ids."""
    g = G.random_small(30, 120, seed=5, weights="equal")
    mask, _, _ = run(g)
    assert np.array_equal(mask, refs.lighter_path_msf(*g.numpy()))


def test_offset_preserves_mask_relabel_preserves_total():
    g = G.random_small(80, 400, seed=11, weights="uniform")
    mask, total, count = run(g)
    g2 = G.Graph(g.n, g.nindex, g.nlist, (g.eweight.to(torch.int64) - 12345).to(torch.int32))
    mask2, total2, _ = run(g2)
    assert np.array_equal(mask, mask2) and total2 == total - 12345 * count
    # relabel vertices by a permutation: total weight is invariant
    n, nindex, nlist, eweight = g.numpy()
    u, v, w, _ = refs.canonical_edges(n, nindex, nlist, eweight)
    perm = torch.from_numpy(np.random.default_rng(3).permutation(n))
    g3 = G.csr_from_undirected(n, perm[torch.from_numpy(u)], perm[torch.from_numpy(v)], torch.from_numpy(w))
    _, total3, count3 = run(g3)
    assert (total3, count3) == (total, count)


def test_disjoint_union_is_union_of_forests():
    a = G.random_small(50, 200, seed=21, weights="ties")
    b = G.random_small(70, 300, seed=22, weights="ties")
    ma, ta, ca = run(a)
    mb, tb, cb = run(b)
    nindex = torch.cat([a.nindex, b.nindex[1:] + a.M])
    nlist = torch.cat([a.nlist, b.nlist + a.n])
    eweight = torch.cat([a.eweight, b.eweight])
    u = G.Graph(a.n + b.n, nindex, nlist, eweight)
    mu, tu, cu = run(u)
    assert np.array_equal(mu, np.concatenate([ma, mb]))
    assert (tu, cu) == (ta + tb, ca + cb)


def test_frieze_zeta3():
    """K_n with i.i.d. U[0,1) weights: E[W_MST] -> zeta(3) (Frieze 1985)."""
    g = G.complete_graph(1000, seed=7, weights="uniform")
    _, total, count = run(g)
    assert count == 999
    assert abs(total / 2.0 ** 31 - 1.2020569) < 0.15


def test_asymmetric_selfloop_multiedge_semantics():
    g = asymmetric_graph()
    mask, total, count = run(g)
    bmask, btotal, k, _ = refs.brute_force_msf(*g.numpy())
    assert np.array_equal(mask, bmask) and total == btotal and count == k
    n, nindex, nlist, _ = g.numpy()
    rows = np.repeat(np.arange(n), np.diff(nindex))
    assert np.all(mask[rows >= nlist] == 0)      # mirror slots and loops never marked


def test_degenerate_sizes():
    for n in (0, 1, 5):
        mask, total, count = run(empty_graph(n))
        assert mask.size == 0 and total == 0 and count == 0
    g = G.path_graph(2, weights=torch.tensor([-(1 << 31)]))
    mask, total, count = run(g)
    assert total == -(1 << 31) and count == 1 and mask.tolist() == [1, 0]


def test_rejects_invalid_csr():
    with pytest.raises(ValueError):
        oracle.kruskal(2, np.array([0, 1, 2]), np.array([1, 5], dtype=np.int32), np.array([1, 1], dtype=np.int32))
    with pytest.raises(ValueError):
        oracle.kruskal(2, np.array([0, 2, 1]), np.array([1, 0], dtype=np.int32), np.array([1, 1], dtype=np.int32))


def test_rng_matches_scalar_splitmix():
    idx = torch.arange(0, 1000, 37)
    h = synth.hash_u64(12, 5, idx)
    for i, x in zip(idx.tolist(), h.tolist()):
        assert (x & ((1 << 64) - 1)) == synth.rng.hash_u64_py(12, 5, i)
    assert synth.splitmix64_py(0) == 0xE220A8397B1DCDAF   # published splitmix64 first output


# --- the per-edge and component helpers used for full-size (sampled) checks ---

@pytest.mark.parametrize("seed", range(6))
def test_edge_in_msf_and_components_agree_with_pins(seed):
    kinds = ["ties", "two", "full", "uniform", "equal", "ties"]
    g = G.random_small(60 + seed, 150, seed=300 + seed, weights=kinds[seed], multi=seed % 2 == 0,
                       self_loops=seed % 3 == 0)
    n, nindex, nlist, eweight = g.numpy()
    u, v, w, ids = refs.canonical_edges(n, nindex, nlist, eweight)
    cmask = refs.lighter_path_msf(n, nindex, nlist, eweight)     # independent BFS characterisation
    for j in ids.tolist():
        assert oracle.edge_in_msf(n, nindex, nlist, eweight, j) == bool(cmask[j])
    ncc, _ = refs.components(n, u, v)
    assert oracle.components(n, nindex, nlist) == ncc
    with pytest.raises(ValueError):
        rows = np.repeat(np.arange(n), np.diff(nindex))
        mirror = int(np.nonzero(rows > nlist)[0][0])
        oracle.edge_in_msf(n, nindex, nlist, eweight, mirror)
