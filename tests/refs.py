"""Independent reference checks used to PIN the oracle (test-only).

Nothing here imports oracle/ or the CUDA package.  Each function is a
different route to the same mathematical object as the oracle's Kruskal:

* brute_force_msf  -- enumerate every edge subset of size n - #CC, keep the
                      acyclic ones, minimise the sum of (w, id)-ranks.
* prim_msf         -- Prim's algorithm with (w, id) keys, restarted in
                      every component.
* lighter_path_msf -- the characterisation "edge e is in the MSF iff its ends
                      are NOT connected by edges that precede e in the (w, id)
                      order" (cycle property), checked by BFS per edge.
* check_forest     -- structural invariants (|F| = n - #CC, acyclic, spanning,
                      cycle property via binary lifting).
"""
from __future__ import annotations

import heapq
import itertools
from collections import deque

import numpy as np


def canonical_edges(n, nindex, nlist, eweight):
    """(u, v, w, id) for CSR entries with u < nlist[id] (Alg. 2 L4)."""
    nindex = np.asarray(nindex, dtype=np.int64)
    nlist = np.asarray(nlist, dtype=np.int64)
    eweight = np.asarray(eweight, dtype=np.int64)
    M = nlist.shape[0]
    rows = np.repeat(np.arange(n, dtype=np.int64), np.diff(nindex)) if n else np.zeros(0, np.int64)
    ids = np.arange(M, dtype=np.int64)
    sel = rows < nlist
    return rows[sel], nlist[sel], eweight[sel], ids[sel]


def components(n, us, vs):
    adj = [[] for _ in range(n)]
    for a, b in zip(us, vs):
        adj[a].append(b)
        adj[b].append(a)
    comp = [-1] * n
    c = 0
    for s in range(n):
        if comp[s] >= 0:
            continue
        comp[s] = c
        dq = deque([s])
        while dq:
            x = dq.popleft()
            for y in adj[x]:
                if comp[y] < 0:
                    comp[y] = c
                    dq.append(y)
        c += 1
    return c, comp


def brute_force_msf(n, nindex, nlist, eweight):
    u, v, w, ids = canonical_edges(n, nindex, nlist, eweight)
    m = len(u)
    order = sorted(range(m), key=lambda i: (int(w[i]), int(ids[i])))
    rank = [0] * m
    for r, i in enumerate(order):
        rank[i] = r
    ncc, _ = components(n, u, v)
    k = n - ncc
    best, best_set, best_w = None, None, None
    min_w_any = None
    for comb in itertools.combinations(range(m), k):
        parent = list(range(n))

        def f(x):
            while parent[x] != x:
                x = parent[x]
            return x
        ok = True
        for i in comb:
            a, b = f(int(u[i])), f(int(v[i]))
            if a == b:
                ok = False
                break
            parent[a] = b
        if not ok:
            continue
        s = sum(rank[i] for i in comb)
        sw = sum(int(w[i]) for i in comb)
        min_w_any = sw if min_w_any is None else min(min_w_any, sw)
        if best is None or s < best:
            best, best_set, best_w = s, comb, sw
    mask = np.zeros(len(nlist), dtype=np.uint8)
    for i in best_set or ():
        mask[int(ids[i])] = 1
    return mask, (best_w or 0), k, (min_w_any or 0)


def prim_msf(n, nindex, nlist, eweight):
    u, v, w, ids = canonical_edges(n, nindex, nlist, eweight)
    adj = [[] for _ in range(n)]
    for a, b, ww, j in zip(u.tolist(), v.tolist(), w.tolist(), ids.tolist()):
        adj[a].append((ww, j, b))
        adj[b].append((ww, j, a))
    seen = [False] * n
    mask = np.zeros(len(nlist), dtype=np.uint8)
    total = 0
    count = 0
    for s in range(n):
        if seen[s]:
            continue
        seen[s] = True
        heap = list(adj[s])
        heapq.heapify(heap)
        while heap:
            ww, j, x = heapq.heappop(heap)
            if seen[x]:
                continue
            seen[x] = True
            mask[j] = 1
            total += ww
            count += 1
            for e in adj[x]:
                if not seen[e[2]]:
                    heapq.heappush(heap, e)
    return mask, total, count


def lighter_path_msf(n, nindex, nlist, eweight):
    """e in MSF  <=>  ends not connected using only edges preceding e."""
    u, v, w, ids = canonical_edges(n, nindex, nlist, eweight)
    keys = list(zip(w.tolist(), ids.tolist()))
    mask = np.zeros(len(nlist), dtype=np.uint8)
    for i in range(len(u)):
        ki = keys[i]
        adj = [[] for _ in range(n)]
        for t in range(len(u)):
            if keys[t] < ki:
                adj[int(u[t])].append(int(v[t]))
                adj[int(v[t])].append(int(u[t]))
        target = int(v[i])
        seen = {int(u[i])}
        dq = deque([int(u[i])])
        found = False
        while dq and not found:
            x = dq.popleft()
            for y in adj[x]:
                if y == target:
                    found = True
                    break
                if y not in seen:
                    seen.add(y)
                    dq.append(y)
        if not found:
            mask[int(ids[i])] = 1
    return mask


def check_forest(n, nindex, nlist, eweight, mask):
    """Invariants of the unique MSF under the (w, id) order.

    Returns a dict of booleans; all must be True.  Uses numpy binary lifting
    for the cycle property: every non-forest canonical edge must be the
    (w, id)-maximum of the cycle it closes in the forest.
    """
    u, v, w, ids = canonical_edges(n, nindex, nlist, eweight)
    mask = np.asarray(mask)
    res = {}
    canon = np.zeros(len(nlist), dtype=bool)
    canon[ids] = True
    res["only_canonical_slots"] = bool(np.all(mask[~canon] == 0))
    inF = mask[ids].astype(bool)
    fu, fv, fw, fid = u[inF], v[inF], w[inF], ids[inF]
    ncc, comp = components(n, u, v)
    res["edge_count"] = len(fu) == n - ncc
    # acyclic + spanning: forest components must equal graph components
    fcc, fcomp = components(n, fu, fv)
    res["spanning_acyclic"] = (fcc == ncc) and (len(fu) == n - fcc)
    if not res["spanning_acyclic"]:
        res["cycle_property"] = False
        return res
    # total order rank over all canonical edges
    order = np.lexsort((ids, w))
    rank = np.empty(len(ids), dtype=np.int64)
    rank[order] = np.arange(len(ids))
    frank = rank[inF]
    # root the forest by BFS
    adj = [[] for _ in range(n)]
    for a, b, r in zip(fu.tolist(), fv.tolist(), frank.tolist()):
        adj[a].append((b, r))
        adj[b].append((a, r))
    par = np.full(n, -1, dtype=np.int64)
    pr = np.full(n, -1, dtype=np.int64)
    depth = np.zeros(n, dtype=np.int64)
    seen = np.zeros(n, dtype=bool)
    for s in range(n):
        if seen[s]:
            continue
        seen[s] = True
        par[s] = s
        dq = deque([s])
        while dq:
            x = dq.popleft()
            for y, r in adj[x]:
                if not seen[y]:
                    seen[y] = True
                    par[y] = x
                    pr[y] = r
                    depth[y] = depth[x] + 1
                    dq.append(y)
    LOG = max(1, int(depth.max()).bit_length() + 1) if n else 1
    up = [par]
    mx = [pr]
    for _ in range(1, LOG):
        p = up[-1]
        up.append(p[p])
        mx.append(np.maximum(mx[-1], mx[-1][p]))
    nf = ~inF
    qa, qb, qr = u[nf].copy(), v[nf].copy(), rank[nf]
    best = np.full(len(qa), -1, dtype=np.int64)
    # lift deeper endpoint
    swap = depth[qa] < depth[qb]
    qa[swap], qb[swap] = qb[swap], qa[swap].copy()
    diff = depth[qa] - depth[qb]
    for k in range(LOG):
        sel = (diff >> k) & 1 == 1
        best[sel] = np.maximum(best[sel], mx[k][qa[sel]])
        qa[sel] = up[k][qa[sel]]
    for k in range(LOG - 1, -1, -1):
        sel = up[k][qa] != up[k][qb]
        best[sel] = np.maximum(best[sel], np.maximum(mx[k][qa[sel]], mx[k][qb[sel]]))
        qa[sel] = up[k][qa[sel]]
        qb[sel] = up[k][qb[sel]]
    last = qa != qb
    best[last] = np.maximum(best[last], np.maximum(pr[qa[last]], pr[qb[last]]))
    res["cycle_property"] = bool(np.all(best < qr))
    return res
