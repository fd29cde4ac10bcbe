"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, bit-exact.

The in_mst byte mask and the int64 total weight must equal the oracle's on
the same seeded inputs (BASELINE.json north_star).
"""
import math

import numpy as np
import pytest
import torch

import oracle
import synth
from synth import graphs as G
from tests.fixtures import asymmetric_graph, empty_graph, load_fig2

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def eclmst():
    import paper_conf_sc_fallingsb23_b200 as m
    m.load()
    return m


def gpu_run(m, g, **opts):
    dev = torch.device("cuda:0")
    gd = g.to(dev)
    o = m.default_options(**opts) if opts else None
    mask, total, ws = m.ecl_mst_device(gd.n, gd.nindex, gd.nlist, gd.eweight, options=o)
    stats = m.ecl_mst_read_stats(ws)
    return mask.cpu().numpy(), int(total.item()), stats


def assert_parity(m, g, **opts):
    omask, ototal, ocount = oracle.kruskal_graph(g)
    mask, total, stats = gpu_run(m, g, **opts)
    assert stats["status"] == 0
    assert total == ototal, (total, ototal)
    if not np.array_equal(mask, omask):
        diff = np.nonzero(mask != omask)[0]
        raise AssertionError(f"{len(diff)} mask mismatches, first ids {diff[:10]}")
    assert stats["msf_edges"] == ocount
    return stats


def check_round_bound(g, stats):
    """<= ceil(log2 n) + 1 rounds per phase incl. the final empty pass A; a
    crowded-round split (opts.refilter) adds one sub-phase of as many."""
    bound = (math.ceil(math.log2(max(g.n, 2))) + 1) * (1 + stats["refilters"])
    r = stats["rounds"]
    p2 = stats["phase2_round"]
    if p2 < 0:
        assert r <= bound + 1, (r, bound)
    else:
        assert p2 <= bound + 1 and r - p2 <= bound + 1, (r, p2, bound)


def test_fig2(eclmst):
    g, ids, mst, weight = load_fig2()
    mask, total, stats = gpu_run(eclmst, g)
    assert total == weight
    assert {lab for lab, j in ids.items() if mask[j]} == mst
    # two iterations that join edges, then the empty final pass
    assert stats["winners"][:2] == [2, 1]


@pytest.mark.parametrize("seed", range(40))
def test_tiny_adversarial(eclmst, seed):
    kinds = ["ties", "equal", "two", "full", "uniform"]
    g = G.random_small(2 + seed % 9, 3 + (seed * 7) % 40, seed=seed, weights=kinds[seed % 5],
                       multi=seed % 3 == 0, self_loops=seed % 4 == 0)
    assert_parity(eclmst, g)
    assert_parity(eclmst, g, relabel=1, refilter=seed % 2, filter=seed % 3 - 1)


@pytest.mark.parametrize("weights", ["ties", "two", "full", "uniform", "equal"])
@pytest.mark.parametrize("n,m", [(1000, 6000), (5000, 2000), (20000, 200000)])
def test_random_multi_tile(eclmst, weights, n, m):
    g = G.random_small(n, m, seed=n + m, weights=weights, multi=True, self_loops=True)
    stats = assert_parity(eclmst, g)
    check_round_bound(g, stats)
    stats = assert_parity(eclmst, g, relabel=1)
    check_round_bound(g, stats)
    if m > n:
        assert stats["relabels"] >= 1


@pytest.mark.parametrize("name", list(synth.CONFIGS))
def test_config_small(eclmst, name):
    g = synth.make_config(name, "small")
    stats = assert_parity(eclmst, g)
    check_round_bound(g, stats)


@pytest.mark.parametrize("opts", [
    dict(filter=0), dict(filter=1), dict(filter=1, threshold_mode=1, threshold=-(1 << 31)),
    dict(filter=1, threshold_mode=1, threshold=(1 << 31) - 1), dict(filter=1, threshold_mode=1, threshold=0),
    dict(seed=1), dict(seed=12345), dict(path_halving=0), dict(max_ctas=1), dict(max_ctas=7),
    dict(atomic_guards=0), dict(atomic_guards=1), dict(flatten=0), dict(flatten=0, path_halving=0), dict(trace=1),
    dict(threshold_samples=20), dict(threshold_samples=4096, seed=7),
    dict(populate_order=1), dict(populate_order=2), dict(populate_order=3), dict(populate_order=2, max_ctas=3),
    dict(populate_order=1, max_ctas=2),
    dict(refilter=0), dict(refilter=1), dict(refilter=1, max_ctas=3), dict(refilter=1, atomic_guards=0),
    dict(refilter=1, filter=0), dict(refilter=1, path_halving=0, flatten=0),
    dict(filter_c=2), dict(filter_c=3), dict(filter_c=1, refilter=1), dict(filter_c=64),
    # the largest-set bitmap of phase 2 (auto only at n >= 2^25): forced on at small n
    dict(giant_bitmap=1), dict(giant_bitmap=0), dict(giant_bitmap=1, refilter=1),
    dict(giant_bitmap=1, filter=1, threshold_mode=1, threshold=0), dict(giant_bitmap=1, max_ctas=3),
    dict(giant_bitmap=1, atomic_guards=0), dict(giant_bitmap=1, flatten=0),
    # exact-quantile threshold (NEXT-3)
    dict(threshold_mode=2), dict(threshold_mode=2, filter=1, filter_c=1), dict(threshold_mode=2, filter_c=64),
    # contraction to dense set ids (auto only for levels of >= 2M sets): forced at every halving
    dict(relabel=1), dict(relabel=0), dict(relabel=1, refilter=1), dict(relabel=1, giant_bitmap=1),
    dict(relabel=1, max_ctas=3), dict(relabel=1, path_halving=0), dict(relabel=1, filter=0),
    dict(relabel=1, refilter=1, filter=1, filter_c=1, giant_bitmap=1), dict(relabel=1, atomic_guards=1),
    # contraction inside phase 2 (threshold 0: nearly every edge is heavy) and with no phase 2 at all
    dict(relabel=1, filter=1, threshold_mode=1, threshold=0), dict(relabel=1, filter=1, threshold_mode=1,
                                                                   threshold=(1 << 31) - 1),
    dict(relabel=1, max_ctas=1), dict(relabel=1, threshold_mode=2, giant_bitmap=1),
    # the Table-5 de-optimisations, one at a time and all together
    dict(populate_mode=1), dict(both_directions=1), dict(tuple_layout=1), dict(drive=1), dict(drive=2),
    dict(populate_mode=1, both_directions=1, tuple_layout=1, drive=2, atomic_guards=0, filter=0, path_halving=0,
         flatten=0),
    dict(tuple_layout=1, refilter=1, relabel=1, giant_bitmap=1), dict(both_directions=1, refilter=1, relabel=1),
    dict(drive=1, tuple_layout=1, both_directions=1), dict(populate_mode=1, relabel=1, max_ctas=3),
])
@pytest.mark.parametrize("name", ["rmat", "uniform", "road"])
def test_knobs_give_identical_msf(eclmst, name, opts):
    g = synth.make_config(name, "small")
    assert_parity(eclmst, g, **opts)


@pytest.mark.parametrize("weights", ["ties", "two", "equal", "uniform"])
@pytest.mark.parametrize("n,m", [(3000, 60000), (20000, 400000)])
def test_refilter_forced(eclmst, weights, n, m):
    """Crowded-round splits (opts.refilter = 1): light part first, deferred
    part filtered afterwards -- the MSF must not change (P:143 argument)."""
    g = G.random_small(n, m, seed=n ^ m, weights=weights, multi=True, self_loops=True)
    stats = assert_parity(eclmst, g, refilter=1)
    check_round_bound(g, stats)
    stats = assert_parity(eclmst, g, refilter=1, giant_bitmap=1)   # phase 2 through the bitmap
    check_round_bound(g, stats)
    # without the two-phase filter the rounds crowd for sure
    stats = assert_parity(eclmst, g, refilter=1, filter=0)
    check_round_bound(g, stats)
    if weights == "uniform":
        assert stats["refilters"] >= 1


@pytest.mark.parametrize("seed", range(24))
def test_tiny_adversarial_refilter(eclmst, seed):
    kinds = ["ties", "equal", "two", "full", "uniform"]
    g = G.random_small(3 + seed % 13, 10 + (seed * 11) % 90, seed=1000 + seed, weights=kinds[seed % 5],
                       multi=True, self_loops=seed % 2 == 0)
    assert_parity(eclmst, g, refilter=1, filter=seed % 3 - 1)


def test_two_valued_weights_nontrivial_phase1(eclmst):
    """Reading Q2: phase 2 must keep canonical ids/directions (tie-heavy)."""
    for seed in range(6):
        g = G.random_small(3000, 40000, seed=seed, weights="two")
        assert_parity(eclmst, g, filter=1, threshold_mode=1, threshold=1)


@pytest.mark.parametrize("relabel", [-1, 1])
def test_special_graphs(eclmst, relabel):
    kw = dict(relabel=relabel)
    assert_parity(eclmst, G.star_graph(1_000_001, seed=1), **kw)         # one 1M-degree row
    assert_parity(eclmst, G.path_graph(200_000), **kw)                  # monotone: deep chain
    assert_parity(eclmst, G.path_graph(200_000, weights=-torch.arange(199_999)), **kw)
    assert_parity(eclmst, G.complete_graph(700, seed=2, weights="ties"), **kw)
    assert_parity(eclmst, G.cycle_graph(99_999, seed=3, weights="ties"), **kw)
    assert_parity(eclmst, asymmetric_graph(), **kw)
    # exactly M = 4n: the filter boundary
    n = 50_000
    a = torch.arange(n, dtype=torch.int64)
    u = torch.cat([a, a])
    v = torch.cat([(a + 1) % n, (a + 2) % n])
    w = synth.rng.uniform_int31(4, 1, torch.arange(2 * n))
    g = G.csr_from_undirected(n, u, v, w)
    assert g.M == 4 * n
    st = assert_parity(eclmst, g, **kw)
    assert st["filtered"]


def test_many_components_and_isolated(eclmst):
    g = G.random_small(100_000, 30_000, seed=8, weights="ties")  # mostly isolated vertices
    assert_parity(eclmst, g)
    g = G.rmat(scale=16, edge_factor=4, seed=8)
    assert_parity(eclmst, g)


def test_degenerate(eclmst):
    for n in (0, 1, 17):
        g = empty_graph(n)
        if n == 0:
            mask, total, _ = gpu_run(eclmst, g)
            assert mask.size == 0 and total == 0
        else:
            assert_parity(eclmst, g)
    assert_parity(eclmst, G.path_graph(2, weights=torch.tensor([(1 << 31) - 1])))
    assert_parity(eclmst, G.random_small(2, 50, seed=1, weights="full", multi=True, self_loops=True))


def test_deterministic_and_reusable_workspace(eclmst):
    g = synth.make_config("rmat", "small").to("cuda:0")
    a, ta, ws = eclmst.ecl_mst_device(g.n, g.nindex, g.nlist, g.eweight)
    a = a.clone()
    ta = int(ta.item())
    for _ in range(3):
        b, tb, ws = eclmst.ecl_mst_device(g.n, g.nindex, g.nlist, g.eweight, workspace=ws)
        assert torch.equal(a, b) and int(tb.item()) == ta


@pytest.mark.parametrize("name", ["grid", "rmat", "uniform", "rgg"])
def test_host_api_staged_upload(eclmst, name):
    """The host path uploads the CSR in pieces under the populate (NEXT-1):
    same MSF as the oracle for filtered (eweight sampled first) and
    unfiltered graphs, pinned and pageable host buffers."""
    g = synth.make_config(name, "small")
    omask, ototal, _ = oracle.kruskal_graph(g)
    for pin in (True, False):
        out = torch.empty(g.M, dtype=torch.uint8)
        args = (g.nindex, g.nlist, g.eweight)
        if pin:
            out = out.pin_memory()
            args = tuple(a.pin_memory() for a in args)
        total = eclmst.ecl_mst(g.n, *args, out)
        assert total == ototal
        assert np.array_equal(out.numpy(), omask)


def _star(leaves, seed=3):
    # vertex 0 joined to every leaf: row 0 has `leaves` entries
    n = leaves + 1
    g = torch.Generator().manual_seed(seed)
    w = torch.randint(0, 1000, (leaves,), generator=g, dtype=torch.int32)   # ties on purpose
    nindex = torch.empty(n + 1, dtype=torch.int64)
    nindex[0] = 0
    nindex[1] = leaves
    nindex[2:] = leaves + torch.arange(1, n, dtype=torch.int64)
    nlist = torch.cat([torch.arange(1, n, dtype=torch.int32), torch.zeros(leaves, dtype=torch.int32)])
    eweight = torch.cat([w, w])
    return n, nindex, nlist, eweight


@pytest.mark.parametrize("leaves", [300, 70000])   # a hub row below and above 2^16 entries
def test_host_api_hub_rows(eclmst, leaves):
    """A star (one row holding every edge) through the host path, pinned and
    pageable: the staged upload's pieces split inside the hub row."""
    n, nindex, nlist, eweight = _star(leaves)
    omask, ototal, ocount = oracle.kruskal(n, nindex.numpy(), nlist.numpy(), eweight.numpy())
    assert ocount == leaves
    for pin in (True, False):
        args = (nindex, nlist, eweight)
        out = torch.empty(nlist.numel(), dtype=torch.uint8)
        if pin:
            args = tuple(a.pin_memory() for a in args)
            out = out.pin_memory()
        total = eclmst.ecl_mst(n, *args, out)
        assert total == ototal
        assert np.array_equal(out.numpy(), omask)


def test_host_api_non_monotone_offsets(eclmst):
    """Decreasing row offsets through the host path: the device validation
    reports the inconsistent CSR."""
    g = synth.make_config("grid", "small")
    bad = g.nindex.clone()
    bad[10], bad[11] = bad[11].item(), bad[10].item()
    out = torch.empty(g.M, dtype=torch.uint8)
    with pytest.raises(eclmst.EclMstError):
        eclmst.ecl_mst(g.n, bad, g.nlist, g.eweight, out)


def test_host_api_memcpy_variant(eclmst):
    g = synth.make_config("road", "small")
    omask, ototal, _ = oracle.kruskal_graph(g)
    out = torch.empty(g.M, dtype=torch.uint8).pin_memory()
    total = eclmst.ecl_mst(g.n, g.nindex.pin_memory(), g.nlist.pin_memory(), g.eweight.pin_memory(), out)
    assert total == ototal
    assert np.array_equal(out.numpy(), omask)
    # invalid CSR (neighbour out of range) is reported, not crashed on
    bad = g.nlist.clone()
    bad[5] = g.n + 3
    with pytest.raises(eclmst.EclMstError):
        eclmst.ecl_mst(g.n, g.nindex, bad, g.eweight, out)


@pytest.mark.parametrize("weights", ["uniform", "full", "ties", "equal", "two"])
@pytest.mark.parametrize("c", [1, 3, 4, 1000])
def test_exact_quantile_threshold(eclmst, weights, c):
    """threshold_mode 2 puts T at the entry of rank min(c n, M - 1) of all M
    weights (numpy's partition decides the rank independently); the MSF is
    the oracle's whatever T is."""
    g = G.random_small(3000 + c, 50_000, seed=c, weights=weights, multi=True, self_loops=True)
    st = assert_parity(eclmst, g, threshold_mode=2, filter=1, filter_c=c)
    w = g.eweight.numpy()
    k = min(c * g.n, g.M - 1)
    assert st["threshold"] == int(np.partition(w, k)[k])
    assert st["heavy_edges"] == int(np.count_nonzero(w[oracle_canonical(g)] >= st["threshold"]))


def oracle_canonical(g):
    """Boolean mask of the canonical (u < v) CSR entries."""
    idx = g.nindex.numpy()
    rows = np.repeat(np.arange(g.n), np.diff(idx))
    return rows < g.nlist.numpy()


DEOPTS = [dict(populate_mode=1), dict(both_directions=1), dict(tuple_layout=1), dict(drive=1), dict(drive=2),
          dict(populate_mode=1, both_directions=1, tuple_layout=1, drive=2)]


@pytest.mark.parametrize("opts", DEOPTS)
@pytest.mark.parametrize("seed", range(6))
def test_deopts_adversarial(eclmst, opts, seed):
    """Every de-optimisation of Table 5 (NEXT-2) on tie-heavy multigraphs with
    loops, both filter settings, a star row and a monotone path."""
    kinds = ["ties", "two", "equal", "full", "uniform", "ties"]
    g = G.random_small(300 + 97 * seed, 4000 + 500 * seed, seed=5000 + seed, weights=kinds[seed], multi=True,
                       self_loops=True)
    for filt in (-1, 0, 1):
        assert_parity(eclmst, g, filter=filt, **opts)
    if seed == 0:
        assert_parity(eclmst, G.star_graph(5000, seed=1), **opts)
        assert_parity(eclmst, G.path_graph(3000), **opts)


@pytest.mark.parametrize("seed", range(12))
def test_giant_bitmap_forced_adversarial(eclmst, seed):
    """The n >= 2^25 phase-2 filter (largest-set bitmap) at small n: tie-heavy
    multigraphs whose light edges percolate, so a largest set exists and most
    heavy edges are filtered through its bitmap."""
    kinds = ["ties", "two", "equal", "full", "uniform", "ties"]
    n = 500 + 331 * seed
    g = G.random_small(n, 12 * n, seed=4000 + seed, weights=kinds[seed % 6], multi=True, self_loops=True)
    for opts in (dict(giant_bitmap=1), dict(giant_bitmap=1, filter=1, filter_c=2),
                 dict(giant_bitmap=1, refilter=1, threshold_samples=20, seed=seed),
                 dict(giant_bitmap=1, relabel=1, refilter=seed % 2)):
        assert_parity(eclmst, g, **opts)


@pytest.mark.parametrize("case", ["last_short", "last_long", "first_nonzero", "negative", "beyond_M"])
@pytest.mark.parametrize("name", ["grid", "rmat"])
def test_device_rejects_bad_offsets(eclmst, name, case):
    """nindex errors the device can only see: flagged as
    ERR_INPUT with no out-of-range access; the context stays usable."""
    g = synth.make_config(name, "small").to("cuda:0")
    bad = g.nindex.clone()
    if case == "last_short":
        bad[-1] -= 300                  # nindex[n] < M: the last chunks have no row
    elif case == "last_long":
        bad[-1] += 300
    elif case == "first_nonzero":
        bad[0] = 7
    elif case == "negative":
        bad[3] = -1000
    else:
        bad[g.n // 2] = g.M + (1 << 40)
    mask, total, ws = eclmst.ecl_mst_device(g.n, bad, g.nlist, g.eweight)
    st = eclmst.ecl_mst_read_stats(ws)
    assert st["status"] == -5 and int(total.item()) == -(1 << 63)
    h = eclmst.ecl_mst_dist_init(None, 0, 1)
    try:
        _, total2, ws2 = eclmst.ecl_mst_dist_device(h, g.n, bad, g.nlist, g.eweight, local_shards=2)
        assert eclmst.ecl_mst_read_stats(ws2)["status"] == -5 and int(total2.item()) == -(1 << 63)
    finally:
        eclmst.ecl_mst_dist_finalize(h)
    torch.cuda.synchronize()
    assert_parity(eclmst, synth.make_config(name, "small"))   # no sticky error


def test_host_api_checks_sizes(eclmst):
    """The host call checks array sizes before the library reads nindex[n] entries."""
    g = synth.make_config("grid", "small")
    out = torch.empty(g.M, dtype=torch.uint8)
    with pytest.raises(ValueError):
        eclmst.ecl_mst(g.n, g.nindex[:-1].contiguous(), g.nlist, g.eweight, out)
    with pytest.raises(ValueError):
        eclmst.ecl_mst(g.n, g.nindex, g.nlist[:-5].contiguous(), g.eweight, out)
    with pytest.raises(ValueError):
        eclmst.ecl_mst(g.n, g.nindex, g.nlist, g.eweight, out[:-1])


def test_device_detects_inconsistent_csr(eclmst):
    g = synth.make_config("grid", "small").to("cuda:0")
    bad = g.nindex.clone()
    bad[-1] += 1   # nindex[n] != M
    mask, total, ws = eclmst.ecl_mst_device(g.n, bad, g.nlist, g.eweight)
    st = eclmst.ecl_mst_read_stats(ws)
    assert st["status"] == -5 and int(total.item()) == -(1 << 63)


@pytest.mark.parametrize("name", ["grid", "road"])
def test_full_size_exact(eclmst, name):
    """BASELINE configs C1/C2 at full size, whole mask vs the oracle."""
    g = synth.make_config(name, "full", device="cuda:0").to("cpu")
    stats = assert_parity(eclmst, g)
    check_round_bound(g, stats)


@pytest.mark.slow
@pytest.mark.parametrize("name", ["rgg", "rmat"])
def test_full_size_exact_large(eclmst, name):
    """BASELINE configs C3/C4 at full size (100M / 521M CSR entries), whole
    mask vs the oracle (the C4 oracle run takes about a minute)."""
    g = synth.make_config(name, "full", device="cuda:0").to("cpu")
    stats = assert_parity(eclmst, g)
    check_round_bound(g, stats)


@pytest.mark.slow
def test_full_size_c5_exact(eclmst):
    """C5 at full size (n = 2^26, M = 2.0e9), the only config whose default
    run takes the n >= 2^25 branches (largest-set bitmap, guards in every
    round): the whole mask and the total against one serial Kruskal over the
    same arrays ("verifies the solution ... serial Kruskal"; about 5
    minutes and 40 GB of host memory).  Cheap invariants run first."""
    gd = synth.make_config("uniform", "full", device="cuda:0")
    mask_d, total_d, ws = eclmst.ecl_mst_device(gd.n, gd.nindex, gd.nlist, gd.eweight)
    st = eclmst.ecl_mst_read_stats(ws)
    assert st["status"] == 0
    assert st["filtered"] and st["phase2_round"] > 0
    n = gd.n
    nindex = gd.nindex.cpu().numpy()
    nlist = gd.nlist.cpu().numpy()
    eweight = gd.eweight.cpu().numpy()
    mask = mask_d.cpu().numpy()
    total = int(total_d.item())
    del gd, mask_d, ws
    torch.cuda.empty_cache()
    marked = np.flatnonzero(mask)
    assert len(marked) == st["msf_edges"]
    assert int(eweight[marked].astype(np.int64).sum()) == total
    heavy = int(np.count_nonzero(eweight[marked] >= st["threshold"]))
    assert heavy > 0                                  # phase 2 added MSF edges (P:152 path exercised)
    omask, ototal, ocount = oracle.kruskal(n, nindex, nlist, eweight)
    assert total == ototal
    assert ocount == st["msf_edges"]
    if not np.array_equal(mask, omask):
        diff = np.nonzero(mask != omask)[0]
        raise AssertionError(f"{len(diff)} mask mismatches, first ids {diff[:10]}")


@pytest.mark.slow
def test_ids_above_2_31():
    """Reading Q13: M up to 2^32 - 1, so edge ids above 2^31 must order as
    unsigned.  A ring of n = 2^20 vertices whose every neighbour pair is
    joined by k = 1100 parallel edges of one weight (M = 2.31e9 CSR entries):
    ties inside a pair go to the smallest id, so the MSF is, by construction,
    the smallest canonical id of every pair except the pair whose
    (weight, smallest id) is largest -- the one that closes the ring."""
    import paper_conf_sc_fallingsb23_b200 as m
    dev = torch.device("cuda:0")
    n, k = 1 << 20, 1100
    M = 2 * n * k
    assert (1 << 31) < M < (1 << 32) - 1
    r = torch.arange(n, device=dev, dtype=torch.int64)
    lo = torch.where(r == 0, 1, torch.where(r == n - 1, 0, r - 1))
    hi = torch.where(r == 0, n - 1, torch.where(r == n - 1, n - 2, r + 1))
    # pair (a, a + 1) is pair a; the wrap pair (n - 1, 0) is pair n - 1
    def pair(a, b):
        return torch.where((a - b).abs() == 1, torch.minimum(a, b), torch.full_like(a, n - 1))
    wp = synth.rng.uniform_int31(13, 1, torch.arange(n, device=dev)).to(torch.int32) % 1000   # ties across pairs too
    nindex = (torch.arange(n + 1, device=dev, dtype=torch.int64) * (2 * k))
    nlist = torch.empty(M, dtype=torch.int32, device=dev)
    eweight = torch.empty(M, dtype=torch.int32, device=dev)
    nlist.view(n, 2, k)[:, 0, :] = lo.to(torch.int32)[:, None]
    nlist.view(n, 2, k)[:, 1, :] = hi.to(torch.int32)[:, None]
    eweight.view(n, 2, k)[:, 0, :] = wp[pair(r, lo)][:, None]
    eweight.view(n, 2, k)[:, 1, :] = wp[pair(r, hi)][:, None]
    # smallest canonical id of every pair: row a holds a + 1 as its `hi`
    # neighbour (ids a*2k + k ...), except row 0 where 1 is `lo` (id 0) and
    # the wrap pair (0, n - 1) sits at row 0's `hi` (id k)
    first = r * (2 * k) + k
    first[0] = 0
    first[n - 1] = k
    key = wp.to(torch.int64) * (1 << 32) + first
    drop = int(torch.argmax(key))
    mask, total, ws = m.ecl_mst_device(n, nindex, nlist, eweight)
    st = m.ecl_mst_read_stats(ws)
    assert st["status"] == 0
    expect_ids = torch.cat([first[:drop], first[drop + 1:]])
    assert int(total.item()) == int(wp.to(torch.int64).sum()) - int(wp[drop])
    assert st["msf_edges"] == n - 1
    got = torch.nonzero(mask).flatten()
    assert got.numel() == n - 1
    assert torch.equal(got, torch.sort(expect_ids).values)
    assert int(got.max()) > (1 << 31)      # ids beyond the signed range were marked


@pytest.mark.parametrize("seed", range(8))
def test_contraction_levels(eclmst, seed):
    """Forced contraction on graphs that need many rounds (long paths of
    tie-heavy cycles joined into a ring, heavy-tailed degrees): many closed
    levels in both phases, the flatten walking all of them, stats consistent."""
    kinds = ["ties", "two", "uniform", "full"]
    n = 2000 + 700 * seed
    g = G.random_small(n, 3 * n, seed=7000 + seed, weights=kinds[seed % 4], multi=True, self_loops=True)
    for opts in (dict(relabel=1), dict(relabel=1, filter=1, filter_c=1), dict(relabel=1, filter=1, filter_c=2,
                                                                            refilter=1)):
        st = assert_parity(eclmst, g, **opts)
        check_round_bound(g, st)
        assert st["relabels"] >= 1, opts
    st = assert_parity(eclmst, G.path_graph(50_000), relabel=1)     # monotone path: one hook chain
    assert st["relabels"] >= 1


@pytest.mark.parametrize("both", [0, 1])
@pytest.mark.parametrize("seed", [0, 1])
def test_populate_dynamic_tail_full_regions(eclmst, both, seed):
    """The phase-2 populate's dynamic tail (ECL_POP_DYN) when every entry is
    kept: a one-direction CSR (only u < v entries, reading Q11) whose edges
    are all heavy (threshold below every weight), so phase 1 hooks nothing
    and phase 2 emits a tuple per entry (two with both_directions).  Regions
    fill up, and a warp that claims batches must stop at its room (rcap) --
    every chunk still gets processed exactly once."""
    gen = torch.Generator().manual_seed(4100 + seed)
    n, m = 1 << 20, 4_300_000
    u = torch.randint(0, n, (m,), generator=gen)
    v = torch.randint(0, n, (m,), generator=gen)
    lo, hi = torch.minimum(u, v), torch.maximum(u, v)
    w = torch.randint(-(1 << 30), 1 << 30, (m,), generator=gen)
    g = G.csr_from_entries(n, lo, hi, w, name=f"onedir{seed}")
    stats = assert_parity(eclmst, g, filter=1, threshold_mode=1, threshold=-(1 << 31), both_directions=both)
    assert stats["filtered"] == 1 and stats["phase2_round"] >= 0
    # phase 2 kept every canonical entry but the self-loops
    assert stats["live"][stats["phase2_round"]] == int((lo != hi).sum()) * (1 + both)


@pytest.mark.parametrize("offset", [0, 4, 8, 12])
def test_in_mst_alignment_and_poison(eclmst, offset):
    """in_mst is written from the MSF bit marks at the end (k_expand): every
    byte, 16 at a time where the output is 16-byte aligned and 4 at a time
    otherwise (the C ABI asks for 4-byte alignment), plus a ragged tail
    (M not a multiple of 16).  The output starts poisoned."""
    g = G.random_small(3000, 40_001, seed=77, weights="ties", multi=True, self_loops=True)
    omask, ototal, _ = oracle.kruskal_graph(g)
    dev = torch.device("cuda:0")
    gd = g.to(dev)
    M = int(gd.nlist.numel())
    assert M % 16 != 0
    buf = torch.full((M + 64,), 0xAB, dtype=torch.uint8, device=dev)
    out = buf[offset: offset + M]
    mask, total, ws = eclmst.ecl_mst_device(gd.n, gd.nindex, gd.nlist, gd.eweight, in_mst_out=out)
    assert int(total.item()) == ototal
    assert np.array_equal(out.cpu().numpy(), omask)
    assert (buf[:offset] == 0xAB).all() and (buf[offset + M:] == 0xAB).all()   # nothing outside
