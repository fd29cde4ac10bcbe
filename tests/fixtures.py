"""Small shared test inputs (test-only)."""
from __future__ import annotations

import os

import torch

from synth.graphs import csr_from_entries, csr_from_undirected

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_fig2():
    """Fig. 2 reconstruction -> (Graph, {label: canonical CSR id}, mst labels, weight)."""
    n = None
    edges = []
    mst, weight = None, None
    with open(os.path.join(GOLDEN, "fig2_reconstruction.txt")) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            tok = line.split()
            if tok[0] == "n":
                n = int(tok[1])
            elif tok[0] == "edge":
                edges.append((tok[1], int(tok[2]), int(tok[3]), int(tok[4])))
            elif tok[0] == "mst":
                mst = set(tok[1:])
            elif tok[0] == "weight":
                weight = int(tok[1])
    u = torch.tensor([e[1] for e in edges], dtype=torch.int64)
    v = torch.tensor([e[2] for e in edges], dtype=torch.int64)
    w = torch.tensor([e[3] for e in edges], dtype=torch.int64)
    g = csr_from_undirected(n, u, v, w, name="fig2")
    ids = {}
    nindex = g.nindex.tolist()
    nlist = g.nlist.tolist()
    for lab, a, b, _ in edges:
        lo, hi = min(a, b), max(a, b)
        for j in range(nindex[lo], nindex[lo + 1]):
            if nlist[j] == hi:
                ids[lab] = j
    return g, ids, mst, weight


def asymmetric_graph():
    """CSR with a missing mirror, a mirror-only entry, a self-loop and a
    multi-edge whose copies carry different weights (reading Q11)."""
    src = torch.tensor([0, 1, 1, 2, 2, 3, 3, 3, 4, 0, 0], dtype=torch.int64)
    dst = torch.tensor([1, 0, 2, 1, 2, 4, 4, 0, 3, 3, 3], dtype=torch.int64)
    w = torch.tensor([5, 5, 2, 9, 1, 7, 3, 0, 3, 8, 6], dtype=torch.int64)
    return csr_from_entries(5, src, dst, w, name="asym")


def empty_graph(n):
    return csr_from_entries(n, torch.zeros(0, dtype=torch.int64), torch.zeros(0, dtype=torch.int64),
                            torch.zeros(0, dtype=torch.int64), name=f"empty{n}")
