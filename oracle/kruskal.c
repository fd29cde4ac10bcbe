/*
 * oracle/kruskal.c -- CPU reference for the minimum spanning forest.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this code.  It
 * shares nothing with the CUDA path (no headers, helpers or constants).
 *
 * What it computes (the plain definition):
 *   Edge set   E = { (u, v = nlist[j], w = eweight[j], id = j) :
 *                    nindex[u] <= j < nindex[u+1], u < v }
 *              -- one direction only, "if v < n" (Alg. 2 L4);
 *              the edge ID is the CSR index of that entry (reading Q1).
 *   Order      by (w as signed 32-bit integer, then id) -- the weight in the
 *              most significant bits, the edge ID as deterministic tie breaker
 *              (P:140).  Under this strict total order the MSF is unique.
 *   Algorithm  Kruskal (the paper verifies every run against a
 *              serial Kruskal): sort E, scan in order, keep an edge iff
 *              its endpoints lie in different sets of a disjoint-set forest,
 *              then union them.
 *   Output     mask[j] = 1 for the ids of the forest edges, 0 elsewhere
 *              ("MST_id <- true"); total = sum of their weights (int64);
 *              count = number of forest edges.
 *
 * Pins: tests/test_oracle.py (brute force, Prim, lighter-edge connectivity
 * characterisation, scipy weights, cycle/cut properties, closed forms).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
    int32_t w;
    uint32_t id;
    int32_t u;
    int32_t v;
} oracle_edge;

static int cmp_edge(const void *pa, const void *pb)
{
    const oracle_edge *a = (const oracle_edge *)pa;
    const oracle_edge *b = (const oracle_edge *)pb;
    if (a->w != b->w) return a->w < b->w ? -1 : 1;
    if (a->id != b->id) return a->id < b->id ? -1 : 1;
    return 0;
}

/* textbook disjoint-set forest: find with path halving, union by size */
static int32_t ds_find(int32_t *parent, int32_t x)
{
    while (parent[x] != x) {
        parent[x] = parent[parent[x]];
        x = parent[x];
    }
    return x;
}

/*
 * Returns 0 on success, -1 on invalid arguments, -2 on allocation failure.
 * Arrays: nindex[n+1] (int64, nindex[0] = 0, non-decreasing), nlist[M] and
 * eweight[M] with M = nindex[n]; mask_out[M] written completely.
 */
int oracle_kruskal(int32_t n, const int64_t *nindex, const int32_t *nlist,
                   const int32_t *eweight, uint8_t *mask_out,
                   int64_t *total_out, int64_t *count_out)
{
    if (n < 0 || (n > 0 && !nindex)) return -1;
    int64_t M = n > 0 ? nindex[n] : 0;
    if (M < 0 || (M > 0 && (!nlist || !eweight || !mask_out))) return -1;
    if (M > 0xFFFFFFFFLL) return -1;
    if (n > 0 && nindex[0] != 0) return -1;
    for (int32_t u = 0; u < n; ++u)
        if (nindex[u + 1] < nindex[u]) return -1;
    for (int64_t j = 0; j < M; ++j)
        if (nlist[j] < 0 || nlist[j] >= n) return -1;

    if (M > 0) memset(mask_out, 0, (size_t)M);

    /* 1. canonical edges: entries j of row u with u < nlist[j] */
    int64_t m = 0;
    for (int32_t u = 0; u < n; ++u)
        for (int64_t j = nindex[u]; j < nindex[u + 1]; ++j)
            if (u < nlist[j]) ++m;
    oracle_edge *E = (oracle_edge *)malloc((size_t)(m > 0 ? m : 1) * sizeof(oracle_edge));
    int32_t *parent = (int32_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int32_t));
    int32_t *size = (int32_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int32_t));
    if (!E || !parent || !size) { free(E); free(parent); free(size); return -2; }
    int64_t k = 0;
    for (int32_t u = 0; u < n; ++u)
        for (int64_t j = nindex[u]; j < nindex[u + 1]; ++j)
            if (u < nlist[j]) {
                E[k].w = eweight[j];
                E[k].id = (uint32_t)j;
                E[k].u = u;
                E[k].v = nlist[j];
                ++k;
            }

    /* 2. sort by (w, id) */
    qsort(E, (size_t)m, sizeof(oracle_edge), cmp_edge);

    /* 3. scan with a disjoint-set forest */
    for (int32_t v = 0; v < n; ++v) { parent[v] = v; size[v] = 1; }
    int64_t total = 0, count = 0;
    for (int64_t i = 0; i < m; ++i) {
        int32_t a = ds_find(parent, E[i].u);
        int32_t b = ds_find(parent, E[i].v);
        if (a == b) continue;
        if (size[a] < size[b]) { int32_t t = a; a = b; b = t; }
        parent[b] = a;
        size[a] += size[b];
        mask_out[E[i].id] = 1;
        total += E[i].w;
        ++count;
    }
    free(E); free(parent); free(size);
    if (total_out) *total_out = total;
    if (count_out) *count_out = count;
    return 0;
}

/*
 * Connected components of the graph (all canonical edges), by one scan of the
 * CSR with the same disjoint-set forest.  Returns the number of components
 * (>= 0) or -1 on invalid input.  An MSF has exactly n - #CC edges (P:63 fn 1).
 */
int64_t oracle_components(int32_t n, const int64_t *nindex, const int32_t *nlist)
{
    if (n < 0 || (n > 0 && !nindex)) return -1;
    int32_t *parent = (int32_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int32_t));
    if (!parent) return -1;
    for (int32_t v = 0; v < n; ++v) parent[v] = v;
    int64_t comps = n;
    for (int32_t u = 0; u < n; ++u)
        for (int64_t j = nindex[u]; j < nindex[u + 1]; ++j) {
            const int32_t v = nlist[j];
            if (v < 0 || v >= n) { free(parent); return -1; }
            if (!(u < v)) continue;
            int32_t a = ds_find(parent, u), b = ds_find(parent, v);
            if (a == b) continue;
            if (a < b) { int32_t t = a; a = b; b = t; }
            parent[a] = b;
            --comps;
        }
    free(parent);
    return comps;
}

/*
 * Is canonical edge `id` in the MSF?  The cycle-property characterisation
 * written out: e = (u, v, w, id) is in the unique MSF under the (w, id) order
 * iff u and v are NOT connected by canonical edges that precede e in that
 * order.  One scan of the CSR unioning exactly those edges.  Returns 1, 0, or
 * -1 if `id` is not a canonical entry / the input is invalid.
 */
int oracle_edge_in_msf(int32_t n, const int64_t *nindex, const int32_t *nlist,
                       const int32_t *eweight, int64_t id)
{
    if (n <= 0 || !nindex || id < 0 || id >= nindex[n]) return -1;
    int32_t eu = -1;
    for (int32_t u = 0; u < n; ++u)               /* row of entry id (linear: plain) */
        if (nindex[u] <= id && id < nindex[u + 1]) { eu = u; break; }
    const int32_t ev = nlist[id];
    if (eu < 0 || !(eu < ev)) return -1;
    const int32_t ew = eweight[id];
    int32_t *parent = (int32_t *)malloc((size_t)n * sizeof(int32_t));
    if (!parent) return -1;
    for (int32_t v = 0; v < n; ++v) parent[v] = v;
    for (int32_t u = 0; u < n; ++u)
        for (int64_t j = nindex[u]; j < nindex[u + 1]; ++j) {
            const int32_t v = nlist[j];
            if (!(u < v)) continue;
            const int32_t w = eweight[j];
            const int lighter = (w < ew) || (w == ew && (uint64_t)j < (uint64_t)id);
            if (!lighter) continue;
            int32_t a = ds_find(parent, u), b = ds_find(parent, v);
            if (a != b) parent[a] = b;
        }
    const int in = ds_find(parent, eu) != ds_find(parent, ev);
    free(parent);
    return in;
}
