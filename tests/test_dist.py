"""Edge-sharded multi-GPU path.

CPU (gloo, world size 2): the host logic -- NCCL unique-id rendezvous over
torch.distributed and the chunk ownership partition.
GPU (one B200): the sharded algorithm with virtual shards on one device
(on-device min-reduction instead of the allreduce) and with a real one-rank
NCCL communicator, bit-exact against the oracle.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as tdist
import torch.multiprocessing as mp

import oracle
import synth
from synth import graphs as G


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _gloo_worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_fallingsb23_b200 import _native, dist
        uid = dist.unique_id_from_group()
        res = {"uid": uid}
        owned = {}
        for M in (0, 1, 127, 128, 129, 10_000, 1_046_528, 2_000_000_000):
            owned[M] = _native.ecl_mst_dist_shard_chunks(M, rank, world)
        res["owned"] = owned
        out[rank] = res
    finally:
        tdist.destroy_process_group()


def test_gloo_rendezvous_and_partition():
    world = 2
    port = _free_port()
    with mp.Manager() as mgr:
        out = mgr.dict()
        mp.spawn(_gloo_worker, args=(world, port, out), nprocs=world, join=True)
        res = dict(out)
    assert res[0]["uid"] == res[1]["uid"] and len(res[0]["uid"]) == 128
    for M in res[0]["owned"]:
        nchunks = (M + 127) // 128
        total = sum(res[r]["owned"][M] for r in range(world))
        assert total == nchunks
        assert abs(res[0]["owned"][M] - res[1]["owned"][M]) <= 1


def test_shard_partition_is_exact_cover():
    from paper_conf_sc_fallingsb23_b200 import _native
    for M in (5, 1000, 99_999):
        for P in (1, 2, 3, 8):
            nchunks = (M + 127) // 128
            counts = [_native.ecl_mst_dist_shard_chunks(M, s, P) for s in range(P)]
            # shard s owns s, s+P, ...: the counts are those of a round-robin deal
            assert counts == [len(range(s, nchunks, P)) for s in range(P)]


# ------------------------------------------------------------------- GPU ---

@pytest.fixture(scope="module")
def ecl():
    import paper_conf_sc_fallingsb23_b200 as m
    m.load()
    return m


def dist_run(m, g, handle, shards, **opts):
    gd = g.to("cuda:0")
    o = m.default_options(**opts) if opts else None
    mask, total, ws = m.ecl_mst_dist_device(handle, gd.n, gd.nindex, gd.nlist, gd.eweight,
                                            local_shards=shards, options=o)
    st = m.ecl_mst_read_stats(ws)
    return mask.cpu().numpy(), int(total.item()), st


@pytest.mark.gpu
@pytest.mark.parametrize("shards", [1, 2, 3, 5])
@pytest.mark.parametrize("name", list(synth.CONFIGS))
def test_virtual_shards_parity(ecl, name, shards):
    g = synth.make_config(name, "small")
    h = ecl.ecl_mst_dist_init(None, 0, 1)
    try:
        mask, total, st = dist_run(ecl, g, h, shards)
    finally:
        ecl.ecl_mst_dist_finalize(h)
    omask, ototal, ocount = oracle.kruskal_graph(g)
    assert st["status"] == 0
    assert total == ototal
    assert np.array_equal(mask, omask)
    assert st["msf_edges"] == ocount


@pytest.mark.gpu
@pytest.mark.parametrize("seed", range(8))
def test_virtual_shards_adversarial(ecl, seed):
    kinds = ["ties", "two", "full", "equal"]
    g = G.random_small(300 + 50 * seed, 3000, seed=seed, weights=kinds[seed % 4], multi=True, self_loops=True)
    h = ecl.ecl_mst_dist_init(None, 0, 1)
    try:
        for shards, opts in ((2, {}), (4, dict(filter=1, threshold_mode=1, threshold=0)), (7, dict(filter=0))):
            mask, total, st = dist_run(ecl, g, h, shards, **opts)
            omask, ototal, _ = oracle.kruskal_graph(g)
            assert total == ototal and np.array_equal(mask, omask), (shards, opts)
    finally:
        ecl.ecl_mst_dist_finalize(h)


@pytest.mark.gpu
def test_sharded_matches_single_gpu_rounds(ecl):
    """Same hooking rule: per-round winners summed over shards equal the
    single-GPU kernel's, and so do the round counts."""
    g = synth.make_config("rmat", "small")
    gd = g.to("cuda:0")
    # (the sharded rounds never split a crowded round: compare without splits)
    _, _, ws = ecl.ecl_mst_device(gd.n, gd.nindex, gd.nlist, gd.eweight, options=ecl.default_options(refilter=0))
    single = ecl.ecl_mst_read_stats(ws)
    h = ecl.ecl_mst_dist_init(None, 0, 1)
    try:
        _, _, st = dist_run(ecl, g, h, 3, refilter=0)
    finally:
        ecl.ecl_mst_dist_finalize(h)
    assert st["rounds"] == single["rounds"]
    assert st["winners"] == single["winners"]
    assert st["live"] == single["live"]


@pytest.mark.gpu
def test_one_rank_nccl_communicator(ecl):
    """World of one, but through a real NCCL communicator and ncclAllReduce."""
    uid = ecl.ecl_mst_dist_unique_id()
    h = ecl.ecl_mst_dist_init(uid, 0, 1)
    try:
        for name in ("uniform", "road"):
            g = synth.make_config(name, "small")
            mask, total, st = dist_run(ecl, g, h, 1)
            omask, ototal, _ = oracle.kruskal_graph(g)
            assert total == ototal and np.array_equal(mask, omask)
    finally:
        ecl.ecl_mst_dist_finalize(h)


@pytest.mark.gpu
@pytest.mark.parametrize("shards", [1, 2, 5])
@pytest.mark.parametrize("weights", ["ties", "two", "equal", "uniform"])
def test_virtual_shards_refilter_forced(ecl, weights, shards):
    """Crowded-round splits on the sharded path (opts.refilter = 1): the
    threshold is agreed by an allreduce(min) over shards, light tuples run to
    completion, deferred ones are drained and filtered -- same MSF."""
    g = G.random_small(5000, 120000, seed=77 + shards, weights=weights, multi=True, self_loops=True)
    omask, ototal, _ = oracle.kruskal_graph(g)
    h = ecl.ecl_mst_dist_init(None, 0, 1)
    try:
        for opts in (dict(refilter=1), dict(refilter=1, filter=0), dict(refilter=1, filter_c=1)):
            mask, total, st = dist_run(ecl, g, h, shards, **opts)
            assert st["status"] == 0
            assert total == ototal and np.array_equal(mask, omask), (shards, opts)
            if weights == "uniform" and opts.get("filter") == 0:
                assert st["refilters"] >= 1
    finally:
        ecl.ecl_mst_dist_finalize(h)


@pytest.mark.gpu
@pytest.mark.parametrize("name", ["rmat", "uniform"])
def test_one_rank_nccl_refilter(ecl, name):
    """Splits through a real NCCL communicator (the candidate allreduce)."""
    uid = ecl.ecl_mst_dist_unique_id()
    h = ecl.ecl_mst_dist_init(uid, 0, 1)
    try:
        g = synth.make_config(name, "small")
        omask, ototal, _ = oracle.kruskal_graph(g)
        for opts in (dict(refilter=1), dict(refilter=1, filter=0)):
            mask, total, st = dist_run(ecl, g, h, 1, **opts)
            assert total == ototal and np.array_equal(mask, omask), opts
    finally:
        ecl.ecl_mst_dist_finalize(h)


@pytest.mark.gpu
@pytest.mark.parametrize("seed", range(16))
def test_virtual_shards_fuzz(ecl, seed):
    """Random multigraphs with loops and tie-heavy weights through every
    sharded-path mechanism at once: 2-4 virtual shards (rep pass 1 sliced
    over them), forced crowded-round splits with drains, both phases."""
    kinds = ["ties", "two", "equal", "full", "uniform"]
    n = 50 + 97 * seed
    g = G.random_small(n, 6 * n + 11 * seed, seed=900 + seed, weights=kinds[seed % 5], multi=True,
                       self_loops=seed % 2 == 0)
    omask, ototal, ocount = oracle.kruskal_graph(g)
    h = ecl.ecl_mst_dist_init(None, 0, 1)
    try:
        for opts in (dict(refilter=1), dict(refilter=1, filter=1, threshold_mode=1, threshold=0),
                     dict(refilter=1, filter=0, filter_c=1), dict(refilter=0),
                     dict(giant_bitmap=1), dict(giant_bitmap=1, refilter=1, filter=1, filter_c=2)):
            mask, total, st = dist_run(ecl, g, h, 2 + seed % 3, **opts)
            assert st["status"] == 0, opts
            assert total == ototal and np.array_equal(mask, omask), opts
            assert st["msf_edges"] == ocount, opts
    finally:
        ecl.ecl_mst_dist_finalize(h)


# ---------------------------------------------- device-initiated round loop ---

@pytest.mark.gpu
@pytest.mark.parametrize("shards", [1, 2, 3, 5])
@pytest.mark.parametrize("name", list(synth.CONFIGS))
def test_device_loop_parity(ecl, name, shards):
    """opts.dist_loop 1 (NEXT-4): every round of a phase inside one persistent
    kernel -- exchange (device-side min over the shards' key arrays), rep
    passes, compaction, pass A -- bit-exact against the oracle."""
    g = synth.make_config(name, "small")
    h = ecl.ecl_mst_dist_init(None, 0, 1)
    try:
        mask, total, st = dist_run(ecl, g, h, shards, dist_loop=1)
    finally:
        ecl.ecl_mst_dist_finalize(h)
    omask, ototal, ocount = oracle.kruskal_graph(g)
    assert st["status"] == 0
    assert total == ototal and np.array_equal(mask, omask)
    assert st["msf_edges"] == ocount


@pytest.mark.gpu
@pytest.mark.parametrize("seed", range(10))
def test_device_loop_fuzz(ecl, seed):
    kinds = ["ties", "two", "equal", "full", "uniform"]
    n = 40 + 131 * seed
    g = G.random_small(n, 7 * n + 13 * seed, seed=1900 + seed, weights=kinds[seed % 5], multi=True,
                       self_loops=seed % 2 == 1)
    omask, ototal, ocount = oracle.kruskal_graph(g)
    h = ecl.ecl_mst_dist_init(None, 0, 1)
    try:
        for opts in (dict(), dict(filter=1, threshold_mode=1, threshold=0), dict(filter=0), dict(giant_bitmap=1),
                     dict(filter=1, filter_c=1, max_ctas=3)):
            mask, total, st = dist_run(ecl, g, h, 1 + seed % 4, dist_loop=1, **opts)
            assert st["status"] == 0, opts
            assert total == ototal and np.array_equal(mask, omask), opts
            assert st["msf_edges"] == ocount, opts
    finally:
        ecl.ecl_mst_dist_finalize(h)


@pytest.mark.gpu
def test_device_loop_matches_host_loop_rounds(ecl):
    """Same hook rule and data flow: the device loop's per-round winners, live
    counts and round count equal the host-driven loop's and the single-GPU
    kernel's (no crowded-round splits in either)."""
    g = synth.make_config("rmat", "small")
    gd = g.to("cuda:0")
    _, _, ws = ecl.ecl_mst_device(gd.n, gd.nindex, gd.nlist, gd.eweight, options=ecl.default_options(refilter=0))
    single = ecl.ecl_mst_read_stats(ws)
    h = ecl.ecl_mst_dist_init(None, 0, 1)
    try:
        _, _, host = dist_run(ecl, g, h, 3, refilter=0)
        _, _, dev = dist_run(ecl, g, h, 3, dist_loop=1)
    finally:
        ecl.ecl_mst_dist_finalize(h)
    for st in (host, dev):
        assert st["rounds"] == single["rounds"]
        assert st["winners"] == single["winners"]
        assert st["live"] == single["live"]
