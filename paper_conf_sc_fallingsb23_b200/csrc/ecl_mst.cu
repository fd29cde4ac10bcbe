// ecl_mst.cu -- B200 (sm_100a) implementation of the ECL-MST hot path behind
// the C ABI in include/ecl_mst.h.
//
// One MSF = one stream-ordered sequence of kernels, no host round-trip:
//
//   k_init        Alg. 1: parent[v] = v, key[v] = inf; chunk start
//                 rows (so populate needs no search); block 0 draws the filter
//                 threshold and checks nindex.
//   k_populate<1> Alg. 2 L1-11 fused with round 0 of L14-21: one warp per
//                 128-entry CSR chunk (edge-centric, high occupancy).  Emits
//                 <u,v,w,id> for u < v (L4) meeting the threshold (L6) into
//                 one of G arenas (round-robin by CTA, so every arena samples
//                 the whole CSR evenly) and atomicMins the key into both
//                 endpoints (all endpoints are roots in round 0).
//   k_rounds      persistent cooperative kernel, CTA b owns arena b:
//                 while (live > 0) { pass B ; pass A } with grid barriers.
//                 pass B  L27-31: an edge whose key won at endpoint p hooks p
//                         under the other endpoint (Boruvka hooking: each
//                         representative is written by exactly one edge, no
//                         CAS; a mutual pair keeps its smaller end as root),
//                         marks in_mst[id], adds its weight, and resets
//                         key[p] (L34-37 fused: an edge that lost at p compares
//                         unequal to the old minimum and to inf alike).
//                 pass A  L14-23: find (implicit path compression L15-18),
//                         drop p == q, compact <p,q,w,id> into the other
//                         worklist, atomicMin the key into both sets.
//   k_flatten     phase 2 only: parent[v] = find(v), so every vertex points
//                 at its root.
//   k_populate<2> P:152: heavy edges, endpoints replaced by set(u), set(v)
//                 (one load each after flattening), intra-set edges filtered.
//   k_rounds      phase 2 rounds (exits at once when there is no phase 2).
//   k_finalize    total weight / status -> caller's output.
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <climits>
#include <cstdarg>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <dlfcn.h>

#include <algorithm>
#include <mutex>
#include <string>
#include <vector>

#include "device.cuh"
#include "ecl_mst.h"

namespace cg = cooperative_groups;

namespace eclmst {

constexpr int kMaxGrid = 4096;                 // CTAs of k_rounds (= arenas), upper bound
constexpr int kPopWarps = 8;                   // warps per k_populate CTA (one chunk each)
constexpr int kPopBlock = 32 * kPopWarps;
constexpr int kMaxPopWarps = 65536;            // populate warps (= worklist regions), upper bound
constexpr int kMaxRegionsPerCta = 256;         // regions a k_rounds CTA starts from
constexpr int kTraceSlots = 2 * ECL_MST_MAX_ROUNDS + 4;
constexpr int kMaxSamples = 4096;              // threshold sample size cap
static_assert(kMaxGrid == ECL_MST_TRACE_CTAS, "trace layout");

struct Internal {
    unsigned long long reps;           // distributed path: sets with a finite key this round
    unsigned int done;                 // unused ticket
    int g_cur;                         // first global round of the running phase
    int g_end;                         // last global round of the finished phase
    int giant;                         // root of the largest set after phase 1 (-1: none)
    int pad0;
};

struct Layout {
    size_t stats, internal, trace, rowstart, region, giant, key, parent, wl0, wl1, total;
    long long wl_cap;                  // tuples per worklist buffer
};

static inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

static inline long long ceil_div(long long a, long long b) { return (a + b - 1) / b; }

// worklist tuples needed for W populate regions of ceil(nchunks/W)*kChunk
// tuples, for any W <= min(kMaxPopWarps, nchunks)
static inline long long wl_capacity(long long M) {
    const long long nchunks = ceil_div(M, kChunk);
    const long long wmax = nchunks < kMaxPopWarps ? nchunks : kMaxPopWarps;
    return (nchunks + wmax) * (long long)kChunk;
}

static inline Layout layout_for(int64_t n, int64_t M) {
    Layout L;
    size_t off = 0;
    const long long nchunks = ceil_div(M, kChunk);
    L.wl_cap = wl_capacity(M);
    L.stats = off;    off = align_up(off + sizeof(ecl_mst_stats), 256);
    L.internal = off; off = align_up(off + sizeof(Internal), 256);
    L.trace = off;    off = align_up(off + sizeof(long long) * kTraceSlots * kMaxGrid, 256);
    L.rowstart = off; off = align_up(off + sizeof(int) * (size_t)(nchunks + 1), 256);
    L.region = off;   off = align_up(off + sizeof(int4) * (size_t)kMaxPopWarps, 256);
    L.giant = off;    off = align_up(off + sizeof(unsigned) * (size_t)((n + 31) / 32 + 1), 256);
    L.key = off;      off = align_up(off + sizeof(long long) * (size_t)n, 256);
    L.parent = off;   off = align_up(off + sizeof(int) * (size_t)n, 256);
    L.wl0 = off;      off = align_up(off + sizeof(int4) * (size_t)L.wl_cap, 256);
    L.wl1 = off;      off = align_up(off + sizeof(int4) * (size_t)L.wl_cap, 256);
    L.total = off;
    return L;
}

struct Params {
    int n;
    long long M;
    long long nchunks;                // ceil(M / kChunk)
    int G;                            // k_rounds CTAs = arenas
    long long cap;                    // tuples per arena (k_rounds worklists)
    int W;                            // populate warps = regions of wl0
    long long rcap;                   // tuples per region
    const long long* __restrict__ nindex;
    const int* __restrict__ nlist;
    const int* __restrict__ eweight;
    unsigned char* in_mst;
    long long* total_out;
    ecl_mst_stats* st;
    Internal* in;
    long long* trace;                 // [kTraceSlots][kMaxGrid] or null
    int* rowstart;                    // row of CSR entry c*kChunk, per chunk
    int4* region;                     // per populate warp: {tuples, canonical, heavy, 0}
    unsigned* giant_bits;             // bit v: v is in the largest set after phase 1 (or null)
    long long* key;
    int* parent;
    int4* wl0;
    int4* wl1;
    unsigned long long seed;
    int filter_mode;
    int threshold_mode;
    int threshold_value;
    int samples;
    int halving;
    int guards;                       // -1 auto, 0 off, 1 on
    int flatten;
    // edge sharding (distributed path; single GPU: shard 0 of 1)
    int shard;                        // global shard id
    int nshards;                      // total shards
    long long nlocal;                 // chunks of this shard: shard, shard + nshards, ...
    int zero_mst;                     // populate phase 1 zeroes its chunks of in_mst
    int* acnt;                        // per arena tuple count (distributed pass A)
    int* tgt;                         // per vertex hook target (distributed rep pass)
    long long* const* keys_all;       // virtual shards: every shard's key array
    int nkeys;
};

__device__ __forceinline__ DS ds_of(const Params& P) {
    DS D;
    D.parent = P.parent;
    D.key = P.key;
    return D;
}

__device__ __forceinline__ void stamp(const Params& P, int slot) {
    if (blockIdx.x == 0 && threadIdx.x == 0 && slot < kTraceSlots)
        P.st->t_ns[slot] = (long long)globaltimer_ns();
}

// per-CTA end of a stage (diagnostics; P.trace is null unless opts.trace)
__device__ __forceinline__ void trace_cta(const Params& P, int slot) {
    if (P.trace && slot < kTraceSlots) {
        __syncthreads();
        if (threadIdx.x == 0) P.trace[(long long)slot * kMaxGrid + blockIdx.x] = (long long)globaltimer_ns();
    }
}

// phase 2 runs iff filtering is on and phase 1 deferred at least one edge
// (read-only within the kernels that ask: one L1 line per SM, not one L2
// slice hammered by every warp of the grid)
__device__ __forceinline__ bool phase2_needed(const Params& P) {
    return __ldg(&P.st->filtered) != 0 && __ldg(&P.st->heavy_edges) != 0;
}

// ---------------------------------------------------------------------------
// k_init: Alg. 1 + chunk start rows + threshold
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_init(Params P) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const long long stride = (long long)gridDim.x * blockDim.x;
    const long long i0 = (long long)blockIdx.x * blockDim.x + tid;
    bool err = false;
    for (long long v = i0; v < P.n; v += stride) {
        P.parent[v] = (int)v;                       // every vertex its own set
        if (P.keys_all) {                           // no minimum edge recorded
            for (int s2 = 0; s2 < P.nkeys; ++s2) P.keys_all[s2][v] = kInf;
        } else {
            P.key[v] = kInf;
        }
        // chunk starts inside row v: rowstart[c] = v for c*kChunk in [s, e)
        const long long s = P.nindex[v], e = P.nindex[v + 1];
        if (e < s) err = true;
        for (long long c = (s + kChunk - 1) / kChunk; c * kChunk < e && c < P.nchunks; ++c) P.rowstart[c] = (int)v;
    }
    if (blockIdx.x == 0) {
        ecl_mst_stats* st = P.st;   // zeroed by a memset node just before this kernel
        __shared__ int s_w[kMaxSamples];
        __shared__ int s_T;
        // filter decision (readings Q5-Q7): estimate the
        // weight of the c|V| lightest of the M entries (c = 4) from S random
        // entries: T = the sample of rank floor(S * 4n / M)
        const bool filtered = P.filter_mode < 0 ? (P.M >= 4LL * P.n) : (P.filter_mode != 0);
        if (tid == 0) s_T = (filtered && P.threshold_mode == 1) ? P.threshold_value : INT_MAX;
        if (filtered && P.threshold_mode == 0) {
            const int S = P.samples;
            for (int i = tid; i < S; i += blockDim.x) {
                const unsigned long long h = splitmix64(P.seed * 0x100000001B3ull + (unsigned long long)i);
                s_w[i] = P.eweight[(long long)(h % (unsigned long long)P.M)];
            }
            __syncthreads();
            long long kpos = ((long long)S * 4LL * P.n) / P.M;
            if (kpos > S - 1) kpos = S - 1;
            for (int i = tid; i < S; i += blockDim.x) {
                const int wi = s_w[i];
                int rank = 0;
                for (int t = 0; t < S; ++t) {
                    const int wt = s_w[t];
                    rank += (wt < wi) || (wt == wi && t < i);
                }
                if (rank == (int)kpos) s_T = wi;
            }
        }
        __syncthreads();
        if (tid == 0) {
            st->t_ns[0] = (long long)globaltimer_ns();
            st->filtered = filtered ? 1 : 0;
            st->threshold = s_T;
            st->grid = P.G;
            st->block = kBlock;
            st->phase2_round = -1;
            if (P.nindex[0] != 0 || P.nindex[P.n] != P.M) err = true;
            P.in->g_cur = 0;
            P.in->g_end = 0;
            P.in->done = 0;
            P.in->giant = -1;
        }
    }
    if (err) atomicExch(&P.st->status, ECL_MST_ERR_INPUT);
}

// ---------------------------------------------------------------------------
// k_populate<PH>: one warp per 128-entry CSR chunk
// ---------------------------------------------------------------------------
template <int PH>
#ifndef ECL_DEEP_PH1
#define ECL_DEEP_PH1 0
#endif
#ifndef ECL_DEEP_PH2
#define ECL_DEEP_PH2 1
#endif
#ifndef ECL_GIANT_MIN_N
#define ECL_GIANT_MIN_N (32LL << 20)   // parent[] larger than ~half the L2
#endif
#ifndef ECL_POP_MINB
#define ECL_POP_MINB 4
#endif
__global__ void __launch_bounds__(kPopBlock, ECL_POP_MINB) k_populate(Params P) {
    __shared__ int s_mark[kPopWarps][kChunk];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (PH == 2 && !phase2_needed(P)) return;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        if (PH == 1) P.st->t_ns[1] = (long long)globaltimer_ns();   // init done
        else P.st->t_ns[3] = (long long)globaltimer_ns();           // flatten done
    }
    const bool filtered = __ldg(&P.st->filtered) != 0;
    const int T = __ldg(&P.st->threshold);
    const bool guard = (P.guards > 0) || (P.guards < 0 && PH == 2);
    const DS D = ds_of(P);
    // warp w takes chunks w, w + W, ... (an even sample of the whole CSR, so
    // every region -- and every k_rounds CTA -- gets the same mix even where
    // the density of u < v entries drifts along the rows) and appends its
    // tuples densely to its own region: no atomics, no CTA barrier.
    const int w = blockIdx.x * kPopWarps + warp;
    if (w >= P.W) return;
    int4* const out = P.wl0 + (long long)w * P.rcap;
    int cnt = 0, canon_cnt = 0, heavy_cnt = 0;
    bool err = false;
    const int p0 = lane * kItems;
    // CSR entries of chunk c (lane owns entries p0 .. p0+3), streaming loads
    auto load_entries = [&](long long c, int (&vv)[kItems], int (&ww)[kItems]) {
        const long long c0 = c * kChunk;
        const int len = (int)(min(c0 + (long long)kChunk, P.M) - c0);
        if (p0 + kItems <= len) {
            const int4 a = __ldcs(reinterpret_cast<const int4*>(P.nlist + c0 + p0));
            const int4 b = __ldcs(reinterpret_cast<const int4*>(P.eweight + c0 + p0));
            vv[0] = a.x; vv[1] = a.y; vv[2] = a.z; vv[3] = a.w;
            ww[0] = b.x; ww[1] = b.y; ww[2] = b.z; ww[3] = b.w;
        } else {
#pragma unroll
            for (int k = 0; k < kItems; ++k) {
                const bool ok = p0 + k < len;
                vv[k] = ok ? __ldcs(P.nlist + c0 + p0 + k) : -1;
                ww[k] = ok ? __ldcs(P.eweight + c0 + p0 + k) : 0;
            }
        }
    };
    // software pipeline (edge sharding: this shard owns chunks shard,
    // shard + nshards, ...; lc indexes them, c is the global chunk).  While
    // chunk i is processed, chunk i+1's CSR entries and its first 64 row
    // starts, and chunk i+2's row bracket, are in flight; at the end of
    // chunk i the phase-2 membership bits of chunk i+1's far ends are
    // requested (their entries have arrived by then).
    const int giant = (PH == 2 && P.flatten && P.giant_bits) ? __ldg(&P.in->giant) : -1;
    // deep: also prefetch the next chunk's row starts (phase 2, where the
    // bitmap / parent loads already lengthen each chunk's chain)
    constexpr bool deep = PH == 1 ? ECL_DEEP_PH1 : ECL_DEEP_PH2;
    auto bracket = [&](long long lc, int& r0, int& rl) {
        const long long c = P.shard + lc * P.nshards;
        r0 = __ldg(P.rowstart + c);
        rl = (c + 1 < P.nchunks) ? __ldg(P.rowstart + c + 1) : P.n - 1;
    };
    auto starts = [&](int r0, int rl, long long& sa, long long& sz) {
        const int ra = r0 + 1 + lane, rz = r0 + 33 + lane;
        sa = ra <= rl ? __ldg(P.nindex + ra) : LLONG_MAX;
        sz = rz <= rl ? __ldg(P.nindex + rz) : LLONG_MAX;
    };
    auto vbits = [&](const int (&vv)[kItems]) {
        unsigned b = 0;
        if (PH == 2 && giant >= 0) {
#pragma unroll
            for (int k = 0; k < kItems; ++k)
                if ((unsigned)vv[k] < (unsigned)P.n)
                    b |= ((__ldg(P.giant_bits + (vv[k] >> 5)) >> (vv[k] & 31)) & 1u) << k;
        }
        return b;
    };
    int nr0 = 0, nrl = 0, n2r0 = 0, n2rl = 0, nv[kItems], nw[kItems];
    long long nsa = LLONG_MAX, nsz = LLONG_MAX;
    unsigned nvb = 0;
    if (w < P.nlocal) {
        bracket(w, nr0, nrl);
        load_entries(P.shard + (long long)w * P.nshards, nv, nw);
        if (deep) {
            starts(nr0, nrl, nsa, nsz);
            if (w + P.W < P.nlocal) bracket(w + P.W, n2r0, n2rl);
        }
        nvb = vbits(nv);
    }
    for (long long lc = w; lc < P.nlocal; lc += P.W) {
    const long long c = P.shard + lc * P.nshards;
    bool keep[kItems];
    int4 t[kItems];
#pragma unroll
    for (int k = 0; k < kItems; ++k) keep[k] = false;
    {
        const long long c0 = c * kChunk;
        const long long c1 = min(c0 + (long long)kChunk, P.M);
        const int len = (int)(c1 - c0);
        // rows of this chunk: r0 = row of entry c0; rows r0+1 .. r_last start inside
        const int r0 = nr0, r_last = nrl;
        const long long sa = nsa, sz = nsz;
        const unsigned vb = nvb;
        int vv[kItems], ww[kItems];
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            vv[k] = nv[k];
            ww[k] = nw[k];
        }
        const long long lcn = lc + P.W;
        if (lcn < P.nlocal) {
            load_entries(P.shard + lcn * P.nshards, nv, nw);
            if (deep) {
                nr0 = n2r0;
                nrl = n2rl;
                starts(nr0, nrl, nsa, nsz);
                if (lcn + P.W < P.nlocal) bracket(lcn + P.W, n2r0, n2rl);
            } else {
                bracket(lcn, nr0, nrl);
            }
        }
        int* mark = s_mark[warp];
#pragma unroll
        for (int i = lane; i < kChunk; i += 32) mark[i] = -1;
        __syncwarp();
        if (deep) {   // the first 64 row starts arrived with the prefetch
            const int ra = r0 + 1 + lane, rz = r0 + 33 + lane;
            if (sa >= c0 && sa < c1) atomicMax(&mark[sa - c0], ra);
            else if (sa < c0) err = true;
            if (sz >= c0 && sz < c1) atomicMax(&mark[sz - c0], rz);
            else if (sz < c0) err = true;
        }
        for (int rb = r0 + (deep ? 65 : 1); rb <= r_last; rb += 64) {   // (further) row starts
            const int ra = rb + lane, rz = rb + 32 + lane;
            const long long ta = ra <= r_last ? __ldg(P.nindex + ra) : LLONG_MAX;
            const long long tz = rz <= r_last ? __ldg(P.nindex + rz) : LLONG_MAX;
            if (ta >= c0 && ta < c1) atomicMax(&mark[ta - c0], ra);
            else if (ta < c0) err = true;
            if (tz >= c0 && tz < c1) atomicMax(&mark[tz - c0], rz);
            else if (tz < c0) err = true;
        }
        __syncwarp();
        int row[kItems];
#pragma unroll
        for (int k = 0; k < kItems; ++k) row[k] = mark[p0 + k];
        // inclusive max-scan over the warp's 128 positions
#pragma unroll
        for (int k = 1; k < kItems; ++k) row[k] = max(row[k], row[k - 1]);
        int incl = row[kItems - 1];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(kFull, incl, o);
            if (lane >= o) incl = max(incl, y);
        }
        int excl = __shfl_up_sync(kFull, incl, 1);
        if (lane == 0) excl = r0;                 // position 0 belongs to row r0
#pragma unroll
        for (int k = 0; k < kItems; ++k) row[k] = max(row[k], max(excl, r0));

        if (PH == 1 && P.zero_mst) {   // every in_mst byte is written once, here (Alg. 1 "not in MST")
            if (p0 + kItems <= len) {
                __stcs(reinterpret_cast<unsigned*>(P.in_mst + c0 + p0), 0u);
            } else {
#pragma unroll
                for (int k = 0; k < kItems; ++k)
                    if (p0 + k < len) P.in_mst[c0 + p0 + k] = 0;
            }
        }
        bool cand[kItems];
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            const bool valid = p0 + k < len;
            const bool in_range = (unsigned)vv[k] < (unsigned)P.n;
            if (valid && !in_range) err = true;
            const bool canon = valid && in_range && row[k] < vv[k];   // L4: one direction only
            const bool heavy = filtered && ww[k] >= T;                // L6 threshold condition
            if (PH == 1) {
                canon_cnt += canon;
                heavy_cnt += (canon && heavy);
                cand[k] = canon && !heavy;
            } else {
                cand[k] = canon && heavy;
            }
        }
        int pk[kItems], qk[kItems];
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            pk[k] = row[k];
            qk[k] = vv[k];
        }
        if (PH == 2) {   // set(v), set(n): one load each after k_flatten
#pragma unroll
            for (int k = 0; k < kItems; ++k) {
                if (cand[k] && giant >= 0 && ((vb >> k) & 1u) &&
                    ((__ldg(P.giant_bits + (row[k] >> 5)) >> (row[k] & 31)) & 1)) {
                    pk[k] = qk[k] = giant;                    // both ends in the largest set: filtered
                } else if (cand[k]) {
                    pk[k] = (k > 0 && cand[k - 1] && row[k] == row[k - 1]) ? -1 : __ldca(D.par(row[k]));
                    qk[k] = __ldca(D.par(vv[k]));
                }
            }
#pragma unroll
            for (int k = 1; k < kItems; ++k)
                if (pk[k] == -1) pk[k] = pk[k - 1];
            if (!P.flatten) {
#pragma unroll
                for (int k = 0; k < kItems; ++k) {
                    if (cand[k]) {
                        pk[k] = find_root(D, pk[k], P.halving != 0);
                        qk[k] = find_root(D, qk[k], P.halving != 0);
                    }
                }
            }
        }
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            const long long j = c0 + p0 + k;
            t[k] = make_int4(pk[k], qk[k], ww[k], (int)(unsigned)j);
            keep[k] = cand[k] && pk[k] != qk[k];                  // phase 2: the filter
        }
        // L19-21: the lane's entries come in row order, so merge equal p first
        long long best = kInf;
        int bp = -1;
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            if (!keep[k]) continue;
            const long long key = make_key(t[k].z, (unsigned)t[k].w);   // L19 val <- e_w : e_id
            if (t[k].x != bp) {
                if (bp >= 0) record_min(D.k(bp), best, guard);
                bp = t[k].x;
                best = key;
            } else {
                best = min(best, key);
            }
        }
        if (bp >= 0) record_min(D.k(bp), best, guard);
#pragma unroll
        for (int k = 0; k < kItems; ++k)
            if (keep[k]) record_min(D.k(t[k].y), make_key(t[k].z, (unsigned)t[k].w), guard);
    }
    if (PH == 2 && lc + P.W < P.nlocal) nvb = vbits(nv);   // next chunk's far-end bits
    // L7: append the chunk's tuples to the warp's region
    unsigned m[kItems];
    int off[kItems];
    int tot = 0;
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
        m[i] = __ballot_sync(kFull, keep[i]);
        off[i] = tot;
        tot += __popc(m[i]);
    }
    const unsigned lt = (1u << lane) - 1u;
#pragma unroll
    for (int i = 0; i < kItems; ++i)
        if (keep[i]) __stcg(out + cnt + off[i] + __popc(m[i] & lt), t[i]);
    cnt += tot;
    }
    if (err) atomicExch(&P.st->status, ECL_MST_ERR_INPUT);
    if (PH == 1) {   // |E| and the deferred count of this warp's chunks
        canon_cnt = warp_sum(canon_cnt);
        heavy_cnt = warp_sum(heavy_cnt);
    }
    if (lane == 0) P.region[w] = make_int4(cnt, canon_cnt, heavy_cnt, 0);
}

// ---------------------------------------------------------------------------
// k_flatten: parent[v] = find(v) before the phase-2 populate, so the phase-2
// populate can use parent[x] as set(x) with one load.  Two launches: stage 1
// compresses with path halving from every vertex (fast, but a halving store
// of one thread can land after another thread's final root store and leave
// a vertex one or two hops from its root); stage 2 finishes exactly with
// owner-only pointer jumping (each slot written by the thread that owns it,
// reads through L2 to see the others' progress), cheap on the short paths
// stage 1 leaves.  Roots never change here.
// ---------------------------------------------------------------------------
template <int STAGE>
__global__ void __launch_bounds__(256) k_flatten(Params P) {
    if (!phase2_needed(P) || !P.flatten) return;
    const long long stride = (long long)gridDim.x * blockDim.x;
    const DS D = ds_of(P);
    const int lane = threadIdx.x & 31;
    const int giant = (STAGE == 2 && P.giant_bits) ? __ldcg(&P.in->giant) : -1;
    // warps walk 32 consecutive vertices together (stage 2 ballots the bitmap)
    for (long long base = (long long)blockIdx.x * blockDim.x + threadIdx.x - lane; base < P.n; base += stride) {
        const long long v = base + lane;
        const bool valid = v < P.n;
        if (STAGE == 1) {
            // fast, racy compression: path halving by everybody (ends close
            // to, but not always exactly at, one hop)
            if (valid) {
                const int r = find_root(D, (int)v, true);
                if (r != (int)v) *D.par(v) = r;
            }
        } else {
            // exact: owner-only pointer jumping over the now-short paths
            int p = valid ? __ldcg(D.par(v)) : -1;
            while (valid) {
                const int pp = __ldcg(D.par(p));
                if (pp == p) break;
                __stcg(D.par(v), pp);
                p = pp;
            }
            if (P.giant_bits) {
                const unsigned bits = __ballot_sync(kFull, valid && p == giant);
                if (lane == 0) P.giant_bits[base >> 5] = bits;
            }
        }
    }
}

// After phase 1 most vertices of a graph whose light edges percolate (C3-C5)
// sit in ONE set.  Find its root by a majority vote over sampled vertices;
// k_flatten<2> then writes a bitmap of its members, and the phase-2 populate
// filters an edge with both ends in it from the bitmap (n/8 bytes, L2
// resident) instead of two random parent loads.
__global__ void __launch_bounds__(256) k_giant(Params P) {
    __shared__ int s_r[1024];
    if (!phase2_needed(P) || !P.flatten || !P.giant_bits) return;
    const DS D = ds_of(P);
    for (int i = threadIdx.x; i < 1024; i += blockDim.x) {
        const long long v = (long long)(splitmix64(0x6A09E667F3BCC909ull + (unsigned long long)i) % (unsigned long long)P.n);
        s_r[i] = find_root(D, (int)v, false);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        int cand = -1, votes = 0;                 // Boyer-Moore majority vote
        for (int i = 0; i < 1024; ++i) {
            if (votes == 0) { cand = s_r[i]; votes = 1; }
            else votes += (s_r[i] == cand) ? 1 : -1;
        }
        int cnt = 0;
        for (int i = 0; i < 1024; ++i) cnt += s_r[i] == cand;
        P.in->giant = cnt >= 256 ? cand : -1;     // worth a bitmap only if it holds >= 1/4
    }
}

// ---------------------------------------------------------------------------
// rounds: pass A / pass B over the CTA's arena
// ---------------------------------------------------------------------------

// A CTA's worklist as a sequence of 128-tuple chunks.  Right after populate
// it is the CTA's share of the populate regions (regions b, b+G, ..., each a
// dense run of region[w].x tuples; chunk j maps to a region by a binary
// search over the shared prefix s_pre) -- RegionSrc; after a pass A it is one
// compact run of cnt tuples -- CompactSrc.  Two types, so each pass is
// compiled once per mode and carries only the registers that mode needs.
struct CompactSrc {
    const int4* base;
    int cnt;
    int nloc;
    __device__ __forceinline__ const int4* get(const Params&, int j, int& count) const {
        count = min(kChunk, cnt - j * kChunk);
        return base + (long long)j * kChunk;
    }
};

struct RegionSrc {
    const int* s_pre;   // shared memory: chunk prefix per region (nreg + 1)
    const int* s_rcnt;  // shared memory: tuples per region
    int nreg;
    int nloc;
    int first_w;
    __device__ __forceinline__ const int4* get(const Params& P, int j, int& count) const {
        int lo = 0, hi = nreg;
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (s_pre[mid] <= j) lo = mid;
            else hi = mid;
        }
        const int off = j - s_pre[lo];
        count = min(kChunk, s_rcnt[lo] - off * kChunk);
        return P.wl0 + (long long)(first_w + lo * P.G) * P.rcap + (long long)off * kChunk;
    }
};

__device__ __forceinline__ CompactSrc compact_src(const int4* base, int cnt) {
    CompactSrc S;
    S.base = base;
    S.cnt = cnt;
    S.nloc = (cnt + kChunk - 1) / kChunk;
    return S;
}

// the populate output of CTA b: regions w = b, b + G, ...  Loads the region
// counts into shared memory, builds the chunk prefix, and adds the kept,
// canonical and deferred counts to the stats (phase 1 counters only if
// count_phase1).  Every thread of the CTA must call it.
__device__ __forceinline__ RegionSrc region_src(const Params& P, int b, int* s_pre, int* s_rcnt,
                                                long long (*s_red)[kWarps], int64_t* live_slot,
                                                bool count_phase1) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    RegionSrc R;
    R.s_pre = s_pre;
    R.s_rcnt = s_rcnt;
    R.nreg = b < P.W ? (P.W - b + P.G - 1) / P.G : 0;
    R.first_w = b;
    long long canon = 0, heavy = 0;
    for (int k = tid; k < R.nreg; k += kBlock) {
        const int4 r = P.region[b + k * P.G];
        s_rcnt[k] = r.x;
        canon += r.y;
        heavy += r.z;
    }
    canon = warp_sum(canon);
    heavy = warp_sum(heavy);
    if (lane == 0) {
        s_red[1][warp] = canon;
        s_red[2][warp] = heavy;
    }
    __syncthreads();
    if (tid == 0) {
        long long kept = 0;
        int pre = 0;
        for (int k = 0; k < R.nreg; ++k) {
            s_pre[k] = pre;
            pre += (s_rcnt[k] + kChunk - 1) / kChunk;
            kept += s_rcnt[k];
        }
        s_pre[R.nreg] = pre;
        canon = heavy = 0;
        for (int w2 = 0; w2 < kWarps; ++w2) {
            canon += s_red[1][w2];
            heavy += s_red[2][w2];
        }
        if (kept) atomicAdd(reinterpret_cast<unsigned long long*>(live_slot), (unsigned long long)kept);
        if (count_phase1) {
            if (canon) atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->canonical_edges), (unsigned long long)canon);
            if (heavy) atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->heavy_edges), (unsigned long long)heavy);
        }
    }
    __syncthreads();
    R.nloc = s_pre[R.nreg];
    return R;
}

// L14-23 of one round over the CTA's worklist: S -> out (compact).
template <class SRC>
__device__ __forceinline__ void passA(const Params& P, const SRC& S, int4* __restrict__ out, int* s_out,
                                      bool guard) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const bool halving = P.halving != 0;
    const DS D = ds_of(P);
    for (int k = warp; k < S.nloc; k += kWarps) {
        int count;
        const int4* __restrict__ in = S.get(P, k, count);
        int4 t[kItems];
        bool keep[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            const int idx = i * 32 + lane;
            keep[i] = idx < count;
            t[i] = keep[i] ? __ldcs(in + idx) : make_int4(0, 0, 0, 0);
        }
        int px[kItems], qx[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (keep[i]) {
                px[i] = __ldca(D.par(t[i].x));
                qx[i] = __ldca(D.par(t[i].y));
            }
        }
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (keep[i]) {
                const int p = find_from(D, t[i].x, px[i], halving);        // L15
                const int q = find_from(D, t[i].y, qx[i], halving);        // L16
                keep[i] = p != q;                                          // L17
                t[i].x = p;                                                // L18: implicit
                t[i].y = q;                                                //      path compression
            }
        }
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (keep[i]) {
                const long long key = make_key(t[i].z, (unsigned)t[i].w); // L19
                record_min(D.k(t[i].x), key, guard);                      // L20
                record_min(D.k(t[i].y), key, guard);                      // L21
            }
        }
        warp_emit(t, keep, out, s_out);                                   // L18
    }
}

// L27-31 (+ L34-37): check, join, mark over the CTA's worklist.
template <class SRC>
__device__ __forceinline__ void passB(const Params& P, const SRC& S, long long& wsum, long long& wcnt) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const DS D = ds_of(P);
    for (int k = warp; k < S.nloc; k += kWarps) {
        int count;
        const int4* __restrict__ in = S.get(P, k, count);
        int4 t[kItems];
        bool ok[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            const int idx = i * 32 + lane;
            ok[i] = idx < count;
            t[i] = ok[i] ? __ldcg(in + idx) : make_int4(0, 0, 0, 0);
        }
        // Only the id half of each slot is compared: ids are unique per
        // edge, so id equality is key equality (and inf's id half, 2^32-1,
        // is never a valid id).  L1 is fine: K[p] only changes when p's own
        // winner resets it.
        unsigned kp[kItems], kq[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (ok[i]) {
                kp[i] = __ldca(reinterpret_cast<const unsigned*>(D.k(t[i].x)));
                kq[i] = __ldca(reinterpret_cast<const unsigned*>(D.k(t[i].y)));
            }
        }
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (!ok[i]) continue;
            const bool wp = kp[i] == (unsigned)t[i].w, wq = kq[i] == (unsigned)t[i].w;   // L29
            if (wp || wq) {
                const int p = t[i].x, q = t[i].y;
                // L30 join: each set hooks along its own lightest edge;
                // a mutual pair keeps the smaller representative as root.
                if (wp && !(wq && p < q)) __stcg(D.par(p), q);
                if (wq && !(wp && q < p)) __stcg(D.par(q), p);
                if (wp) __stcg(D.k(p), kInf);                          // L35
                if (wq) __stcg(D.k(q), kInf);                          // L36
                P.in_mst[(unsigned)t[i].w] = 1;                        // L31
                wsum += t[i].z;
                wcnt += 1;
            }
        }
    }
}

// guard policy for pass A.  "auto" guards when edges crowd onto few
// sets -- each set with a live edge produced exactly one winner last round
// (mutual pairs: one for two sets), so live / winners estimates the number of
// edges per set that would atomicMin the same slot -- or when the key array
// is far larger than L2 (n >= 2^25: every unguarded atomic on a random slot
// is a DRAM read-modify-write, a guard miss only a read).  Measured: C5 and
// C4 gain, C2/C3 lose with guards in every round.
__device__ __forceinline__ bool use_guard(const Params& P, long long live, long long winners) {
    if (P.guards >= 0) return P.guards != 0;
    return live > 8 * winners || P.n >= (1 << 25);
}

template <int PH>
__global__ void __launch_bounds__(kBlock, ECL_R_MINB) k_rounds(Params P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ int s_out;
    __shared__ long long s_red[3][kWarps];
    __shared__ int s_pre[kMaxRegionsPerCta + 1];
    __shared__ int s_rcnt[kMaxRegionsPerCta];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const bool b0 = blockIdx.x == 0;
    ecl_mst_stats* st = P.st;
    if (PH == 2 && !phase2_needed(P)) return;
    int g = (PH == 1) ? 0 : __ldcg(&P.in->g_end) + 1;
    if (g >= ECL_MST_MAX_ROUNDS) {
        if (b0 && tid == 0) atomicExch(&st->status, ECL_MST_ERR_INPUT);
        return;
    }
    stamp(P, 4 + 2 * g);                      // populate done
    const int b = blockIdx.x;
    int4* wl[2] = {P.wl0 + (long long)b * P.cap, P.wl1 + (long long)b * P.cap};
    // the populate output of this CTA: regions w = b, b + G, ... (region mode)
    const RegionSrc R = region_src(P, b, s_pre, s_rcnt, s_red, &st->live[g], PH == 1);
    if (b0 && tid == 0 && PH == 2) st->phase2_round = g;
    trace_cta(P, 4 + 2 * g);
    grid.sync();
    long long wsum = 0, wcnt = 0;
    int cur = 0;
    bool overflow = false;
    long long L = __ldcg(&st->live[g]);
    CompactSrc C = compact_src(wl[0], 0);
    // one round: pass B over S, then pass A from S into the other worklist
    auto round = [&](const auto& S) {
        const long long w0 = wcnt;
        passB(P, S, wsum, wcnt);
        const long long d = warp_sum(wcnt - w0);
        if (lane == 0 && d) atomicAdd(reinterpret_cast<unsigned long long*>(&st->winners[g]), (unsigned long long)d);
        if (tid == 0) s_out = 0;
        trace_cta(P, 5 + 2 * g);
        grid.sync();
        stamp(P, 5 + 2 * g);
        if (g + 1 >= ECL_MST_MAX_ROUNDS) {
            overflow = true;
            return false;
        }
        const bool guard = use_guard(P, L, __ldcg(&st->winners[g]));
        ++g;
        passA(P, S, wl[cur ^ 1], &s_out, guard);
        cur ^= 1;
        __syncthreads();
        C = compact_src(wl[cur], s_out);
        if (tid == 0 && C.cnt) atomicAdd(reinterpret_cast<unsigned long long*>(&st->live[g]), (unsigned long long)C.cnt);
        trace_cta(P, 4 + 2 * g);
        grid.sync();
        stamp(P, 4 + 2 * g);
        L = __ldcg(&st->live[g]);
        return true;
    };
    if (L > 0 && round(R))
        while (L > 0 && round(C)) {
        }
    const long long s = warp_sum(wsum), c = warp_sum(wcnt);
    if (lane == 0) {
        if (s) atomicAdd(reinterpret_cast<unsigned long long*>(&st->total_weight), (unsigned long long)s);
        if (c) atomicAdd(reinterpret_cast<unsigned long long*>(&st->msf_edges), (unsigned long long)c);
    }
    if (b0 && tid == 0) {
        P.in->g_end = g;
        st->rounds = g + 1;
        if (overflow) atomicExch(&st->status, ECL_MST_ERR_INPUT);
    }
}

__global__ void k_finalize(Params P) {
    if (threadIdx.x == 0) {
        ecl_mst_stats* st = P.st;
        st->t_ns[2] = (long long)globaltimer_ns();
        const int status = *reinterpret_cast<volatile int*>(&st->status);
        *P.total_out = status ? LLONG_MIN : *reinterpret_cast<volatile long long*>(&st->total_weight);
    }
}


// ---------------------------------------------------------------------------
// Distributed (edge-sharded) MSF -- SURVEY §8(e).  Every rank holds the full
// CSR, a replicated union-find and a full key array; it owns the CSR chunks
// c = shard, shard + P, ... and the tuples they produce.  Per round:
//   allreduce(key, min) over the ranks  ->  every rank knows each set's
//   lightest edge;  rep-centric pass B, identical on every rank (each set
//   with a finite key hooks along its edge, looked up by id in the CSR);
//   local pass A over the rank's own tuples.
// ---------------------------------------------------------------------------

// row of CSR entry j: binary search inside the rows of j's chunk
__device__ __forceinline__ int row_of_entry(const Params& P, long long j) {
    const long long c = j / kChunk;
    int lo = __ldg(P.rowstart + c);
    int hi = (c + 1 < P.nchunks) ? __ldg(P.rowstart + c + 1) : P.n - 1;
    while (lo < hi) {   // largest r in [lo, hi] with nindex[r] <= j
        const int mid = lo + ((hi - lo + 1) >> 1);
        if (__ldg(P.nindex + mid) <= j) lo = mid;
        else hi = mid - 1;
    }
    return lo;
}

// virtual shards on one GPU: the "allreduce" is an elementwise min over the
// shards' key arrays, written back to every copy (as NCCL would)
__global__ void __launch_bounds__(256) k_vreduce(Params P) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < P.n; v += stride) {
        long long m = kInf;
        for (int s2 = 0; s2 < P.nkeys; ++s2) m = min(m, P.keys_all[s2][v]);
        for (int s2 = 0; s2 < P.nkeys; ++s2) P.keys_all[s2][v] = m;
    }
}

// rep pass 1: for every set x with a finite (reduced) key, the other end's set
// q of its lightest edge, and whether that edge is q's lightest too (mutual)
__global__ void __launch_bounds__(256) k_dist_reps1(Params P) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    unsigned long long found = 0;
    for (long long x = (long long)blockIdx.x * blockDim.x + threadIdx.x; x < P.n; x += stride) {
        const long long kx = P.key[x];   // distributed path: own arrays (stride 1)
        if (kx == kInf) continue;
        ++found;
        const unsigned j = (unsigned)(kx & 0xffffffffll);
        const int u = row_of_entry(P, (long long)j);
        const int v = __ldg(P.nlist + j);
        const DS D = ds_of(P);
        const int pu = find_root(D, u, false), pv = find_root(D, v, false);
        const int q = (pu == (int)x) ? pv : pu;
        const bool mutual = P.key[q] == kx;
        P.tgt[x] = q | (mutual ? (int)0x80000000 : 0);
    }
    found = warp_sum(found);
    if ((threadIdx.x & 31) == 0 && found) atomicAdd(reinterpret_cast<unsigned long long*>(&P.in->reps), found);
}

// rep pass 2 (L30-31, L34-37): hook, mark, sum, reset -- the same rule as the
// tuple-centric pass B, so the partition after each round is the same
__global__ void __launch_bounds__(256) k_dist_reps2(Params P, int g) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    long long wsum = 0, wcnt = 0;
    for (long long x = (long long)blockIdx.x * blockDim.x + threadIdx.x; x < P.n; x += stride) {
        const long long kx = P.key[x];
        if (kx == kInf) continue;
        const int t = P.tgt[x];
        const int q = t & 0x7fffffff;
        const bool mutual = t < 0;
        if (!mutual || (int)x > q) P.parent[x] = q;
        if (!mutual || (int)x < q) {
            P.in_mst[(unsigned)(kx & 0xffffffffll)] = 1;
            wsum += (int)(kx >> 32);
            wcnt += 1;
        }
        for (int s2 = 0; s2 < P.nkeys; ++s2) P.keys_all[s2][x] = kInf;
    }
    wsum = warp_sum(wsum);
    wcnt = warp_sum(wcnt);
    if ((threadIdx.x & 31) == 0 && wcnt) {
        atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->total_weight), (unsigned long long)wsum);
        atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->msf_edges), (unsigned long long)wcnt);
        atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->winners[g]), (unsigned long long)wcnt);
    }
}

// local pass A of shard P.shard: CTA b reads arena b (FIRST: its populate
// regions), compacts the survivors into the other worklist
template <bool FIRST>
__global__ void __launch_bounds__(kBlock, 2) k_dist_passA(Params P, int g, int cur) {
    __shared__ int s_out;
    __shared__ long long s_red[3][kWarps];
    __shared__ int s_pre[kMaxRegionsPerCta + 1];
    __shared__ int s_rcnt[kMaxRegionsPerCta];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int b = blockIdx.x;
    int4* wl[2] = {P.wl0 + (long long)b * P.cap, P.wl1 + (long long)b * P.cap};
    if (tid == 0) s_out = 0;
    if (FIRST) {
        const RegionSrc R = region_src(P, b, s_pre, s_rcnt, s_red, &P.st->live[g - 1], g - 1 == 0);
        passA(P, R, wl[cur ^ 1], &s_out, P.guards != 0);
    } else {
        __syncthreads();
        passA(P, compact_src(wl[cur], P.acnt[b]), wl[cur ^ 1], &s_out, P.guards != 0);
    }
    __syncthreads();
    if (tid == 0) {
        P.acnt[b] = s_out;
        if (s_out) atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->live[g]), (unsigned long long)s_out);
    }
}

// ---------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------

static thread_local std::string g_last_error;

static int fail(int code, const char* fmt, ...) __attribute__((format(printf, 2, 3)));
static int fail(int code, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_last_error = buf;
    return code;
}

struct DevInfo {
    int sms = 0;
    int occ = 0;       // resident k_rounds CTAs per SM
    int pop_occ = 0;   // resident k_populate CTAs per SM
};

static std::mutex g_dev_mu;
static DevInfo g_dev[64];

// per-thread CUDA events bracketing the kernels of the last timed call
constexpr int kTimedStages = 7;   // init, populate1, rounds1, flatten, populate2, rounds2, finalize
struct Timing {
    bool ready = false;
    bool valid = false;
    cudaEvent_t ev[kTimedStages + 1];
};
static thread_local Timing g_timing;

static int device_info(DevInfo* out) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "cudaGetDevice: %s", cudaGetErrorString(e));
    if (dev < 0 || dev >= 64) return fail(ECL_MST_ERR_CUDA, "device index %d out of range", dev);
    std::lock_guard<std::mutex> lk(g_dev_mu);
    if (g_dev[dev].sms == 0) {
        int sms = 0, coop = 0, occ = 0;
        e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (e == cudaSuccess) e = cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, dev);
        if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_rounds<1>, kBlock, 0);
        int pop_occ = 0;
        if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&pop_occ, k_populate<1>, kPopBlock, 0);
        g_dev[dev].pop_occ = pop_occ > 0 ? pop_occ : 1;
        if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "device query: %s", cudaGetErrorString(e));
        if (!coop || occ < 1) return fail(ECL_MST_ERR_CUDA, "cooperative launch unsupported (coop=%d occ=%d)", coop, occ);
        g_dev[dev].sms = sms;
        g_dev[dev].occ = occ;
    }
    *out = g_dev[dev];
    return ECL_MST_OK;
}

}  // namespace eclmst

using namespace eclmst;

extern "C" {

int ecl_mst_abi_version(void) { return ECL_MST_ABI_VERSION; }

const char* ecl_mst_last_error(void) { return g_last_error.c_str(); }

void ecl_mst_default_options(ecl_mst_options* o) {
    if (!o) return;
    std::memset(o, 0, sizeof *o);
    o->filter = -1;
    o->threshold_mode = 0;
    o->threshold = 0;
    o->path_halving = 1;
    o->atomic_guards = -1;
    o->flatten = 1;
    o->max_ctas = 0;
    o->trace = 0;
    o->seed = 0x5eedull;
    o->threshold_samples = 1024;
}

size_t ecl_mst_workspace_bytes(int64_t n, int64_t M) {
    if (n < 0 || n > INT32_MAX || M < 0 || M > (int64_t)0xFFFFFFFFLL) return 0;
    return layout_for(n, M).total;
}

int ecl_mst_device(int32_t n, int64_t M, const int64_t* nindex, const int32_t* nlist, const int32_t* eweight,
                   uint8_t* in_mst_out, int64_t* total_weight_out, void* workspace, size_t workspace_bytes,
                   const ecl_mst_options* opts, void* stream) {
    g_last_error.clear();
    if (n < 0 || M < 0) return fail(ECL_MST_ERR_INVALID, "negative n or M");
    if (M > (int64_t)0xFFFFFFFFLL) return fail(ECL_MST_ERR_TOO_LARGE, "M = %lld exceeds 2^32-1", (long long)M);
    if (!total_weight_out || !workspace) return fail(ECL_MST_ERR_INVALID, "null total_weight_out or workspace");
    if (n > 0 && !nindex) return fail(ECL_MST_ERR_INVALID, "null nindex");
    if (M > 0 && (!nlist || !eweight || !in_mst_out)) return fail(ECL_MST_ERR_INVALID, "null CSR or output array");
    if (M > 0 && n == 0) return fail(ECL_MST_ERR_INVALID, "M > 0 with n = 0");
    const Layout L = layout_for(n, M);
    if (workspace_bytes < L.total) return fail(ECL_MST_ERR_WORKSPACE, "workspace %zu < %zu bytes", workspace_bytes, L.total);
    if (reinterpret_cast<uintptr_t>(workspace) % 256) return fail(ECL_MST_ERR_WORKSPACE, "workspace not 256-byte aligned");
    ecl_mst_options o;
    ecl_mst_default_options(&o);
    if (opts) o = *opts;
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    char* ws = static_cast<char*>(workspace);
    if (M == 0) {
        // no edges: empty forest.  Clear the stats so read_stats is meaningful.
        cudaError_t e = cudaMemsetAsync(ws + L.stats, 0, sizeof(ecl_mst_stats), s);
        if (e == cudaSuccess) e = cudaMemsetAsync(total_weight_out, 0, sizeof(int64_t), s);
        if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "memset: %s", cudaGetErrorString(e));
        return ECL_MST_OK;
    }
    DevInfo di;
    int rc = device_info(&di);
    if (rc) return rc;
    const long long nchunks = ceil_div(M, kChunk);
    long long G = (long long)di.sms * di.occ;
    if (o.max_ctas > 0 && G > o.max_ctas) G = o.max_ctas;
    if (G > nchunks) G = nchunks;                 // small graphs: fewer, fuller arenas
    if (G > kMaxGrid) G = kMaxGrid;
    if (G < 1) G = 1;
    // populate: one pass of the GPU, every warp a region; W a multiple of G
    // so that every k_rounds CTA starts from the same number of regions
    long long W = (long long)di.sms * di.pop_occ * kPopWarps;
    if (W > nchunks) W = nchunks;
    if (W > kMaxPopWarps) W = kMaxPopWarps;
    if (W > G * kMaxRegionsPerCta) W = G * kMaxRegionsPerCta;
    W = std::max<long long>(1, W / G) * G;
    const long long rcap = ceil_div(nchunks, W) * kChunk;
    if (W * rcap > L.wl_cap) return fail(ECL_MST_ERR_WORKSPACE, "internal: regions exceed worklist capacity");
    // k_rounds arenas: the worklist of CTA b never exceeds its first input,
    // the W / G regions b, b + G, ...  (arenas in wl0 overlay the regions;
    // they are first written after every CTA has consumed its regions)
    const long long cap = (W / G) * rcap;
    if (cap >= (1LL << 30)) return fail(ECL_MST_ERR_TOO_LARGE, "arena of %lld tuples too large", cap);

    Params P;
    P.n = n;
    P.M = M;
    P.nchunks = nchunks;
    P.G = (int)G;
    P.cap = cap;
    P.W = (int)W;
    P.rcap = rcap;
    P.nindex = reinterpret_cast<const long long*>(nindex);
    P.nlist = nlist;
    P.eweight = eweight;
    P.in_mst = in_mst_out;
    P.total_out = reinterpret_cast<long long*>(total_weight_out);
    P.st = reinterpret_cast<ecl_mst_stats*>(ws + L.stats);
    P.in = reinterpret_cast<Internal*>(ws + L.internal);
    P.trace = o.trace ? reinterpret_cast<long long*>(ws + L.trace) : nullptr;
    P.rowstart = reinterpret_cast<int*>(ws + L.rowstart);
    P.region = reinterpret_cast<int4*>(ws + L.region);
    // the largest-set bitmap only pays when parent[] does not fit the L2
    P.giant_bits = (long long)n >= ECL_GIANT_MIN_N ? reinterpret_cast<unsigned*>(ws + L.giant) : nullptr;
    P.key = reinterpret_cast<long long*>(ws + L.key);
    P.parent = reinterpret_cast<int*>(ws + L.parent);
    P.wl0 = reinterpret_cast<int4*>(ws + L.wl0);
    P.wl1 = reinterpret_cast<int4*>(ws + L.wl1);
    P.seed = o.seed;
    P.filter_mode = o.filter < 0 ? -1 : (o.filter ? 1 : 0);
    P.threshold_mode = o.threshold_mode;
    P.threshold_value = o.threshold;
    P.samples = o.threshold_samples > 0 ? std::min(o.threshold_samples, kMaxSamples) : 20;
    P.halving = o.path_halving ? 1 : 0;
    P.guards = o.atomic_guards < 0 ? -1 : (o.atomic_guards ? 1 : 0);
    P.flatten = o.flatten ? 1 : 0;
    P.shard = 0;
    P.nshards = 1;
    P.nlocal = nchunks;
    P.zero_mst = 1;
    P.acnt = nullptr;
    P.tgt = nullptr;
    P.keys_all = nullptr;
    P.nkeys = 1;
    if ((reinterpret_cast<uintptr_t>(nlist) | reinterpret_cast<uintptr_t>(eweight)) % 16 ||
        reinterpret_cast<uintptr_t>(in_mst_out) % 4)
        return fail(ECL_MST_ERR_INVALID, "nlist/eweight must be 16-byte and in_mst 4-byte aligned");

    const long long init_blocks = std::min<long long>(ceil_div((long long)n, 256), (long long)di.sms * 8);
    const long long pop_blocks = ceil_div(W, kPopWarps);
    if (pop_blocks > INT_MAX) return fail(ECL_MST_ERR_TOO_LARGE, "too many populate CTAs");
    void* args[] = {&P};
    // opts.trace bit 1: CUDA events between the kernels (ecl_mst_kernel_times)
    const bool timing = (o.trace & 2) != 0;
    if (timing && !g_timing.ready) {
        for (int i = 0; i < kTimedStages + 1; ++i) {
            cudaError_t e0 = cudaEventCreate(&g_timing.ev[i]);
            if (e0 != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "cudaEventCreate: %s", cudaGetErrorString(e0));
        }
        g_timing.ready = true;
    }
    g_timing.valid = false;
    int ev_i = 0;
    auto mark = [&]() -> cudaError_t {
        return timing ? cudaEventRecord(g_timing.ev[ev_i++], s) : cudaSuccess;
    };
    const unsigned flat_blocks = (unsigned)std::max<long long>(init_blocks, 1);
    cudaError_t e = mark();
    if (e == cudaSuccess) e = cudaMemsetAsync(P.st, 0, sizeof(ecl_mst_stats), s);
    if (e == cudaSuccess) {
        k_init<<<flat_blocks, 256, 0, s>>>(P);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = mark();
    if (e == cudaSuccess) {
        k_populate<1><<<(unsigned)pop_blocks, kPopBlock, 0, s>>>(P);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = mark();
    if (e == cudaSuccess)
        e = cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(k_rounds<1>), dim3((unsigned)G), dim3(kBlock), args, 0, s);
    if (e == cudaSuccess) e = mark();
    // phase 2 can only happen when filtering is on; with the automatic rule
    // (M >= 4n) the host knows that already and skips the three launches
    const bool maybe_phase2 = P.filter_mode > 0 || (P.filter_mode < 0 && M >= 4LL * n);
    if (e == cudaSuccess && maybe_phase2) {
        k_flatten<1><<<flat_blocks, 256, 0, s>>>(P);
        k_giant<<<1, 256, 0, s>>>(P);
        k_flatten<2><<<flat_blocks, 256, 0, s>>>(P);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = mark();
    if (e == cudaSuccess && maybe_phase2) {
        k_populate<2><<<(unsigned)pop_blocks, kPopBlock, 0, s>>>(P);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = mark();
    if (e == cudaSuccess && maybe_phase2)
        e = cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(k_rounds<2>), dim3((unsigned)G), dim3(kBlock), args, 0, s);
    if (e == cudaSuccess) e = mark();
    if (e == cudaSuccess) {
        k_finalize<<<1, 32, 0, s>>>(P);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = mark();
    if (e == cudaSuccess && timing) g_timing.valid = true;
    if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "launch (G=%lld): %s", G, cudaGetErrorString(e));
    return ECL_MST_OK;
}

int ecl_mst_kernel_times(float* ms_out, int32_t max_stages) {
    g_last_error.clear();
    if (!ms_out) return fail(ECL_MST_ERR_INVALID, "null argument");
    if (!g_timing.valid) return fail(ECL_MST_ERR_INVALID, "no timed run on this thread (opts.trace & 2)");
    cudaError_t e = cudaEventSynchronize(g_timing.ev[kTimedStages]);
    int n = 0;
    for (; e == cudaSuccess && n < kTimedStages && n < max_stages; ++n)
        e = cudaEventElapsedTime(&ms_out[n], g_timing.ev[n], g_timing.ev[n + 1]);
    if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "kernel_times: %s", cudaGetErrorString(e));
    return n;
}

int ecl_mst_read_stats(const void* workspace, ecl_mst_stats* out, void* stream) {
    g_last_error.clear();
    if (!workspace || !out) return fail(ECL_MST_ERR_INVALID, "null argument");
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    cudaError_t e = cudaMemcpyAsync(out, workspace, sizeof(ecl_mst_stats), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "read_stats: %s", cudaGetErrorString(e));
    return ECL_MST_OK;
}

int ecl_mst_read_trace(const void* workspace, int64_t* out, size_t max_entries, void* stream) {
    g_last_error.clear();
    if (!workspace || !out) return fail(ECL_MST_ERR_INVALID, "null argument");
    const Layout L = layout_for(0, 0);
    size_t count = (size_t)kTraceSlots * kMaxGrid;
    if (count > max_entries) count = max_entries;
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    cudaError_t e = cudaMemcpyAsync(out, static_cast<const char*>(workspace) + L.trace, count * sizeof(int64_t),
                                    cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "read_trace: %s", cudaGetErrorString(e));
    return ECL_MST_OK;
}

// ---- host convenience path ("ECL-MST memcpy") ----
static std::mutex g_pool_mu;
static void* g_pool = nullptr;
static size_t g_pool_cap = 0;
static int g_pool_dev = -1;
static cudaStream_t g_pool_stream = nullptr;

void ecl_mst_release_host_cache(void) {
    std::lock_guard<std::mutex> lk(g_pool_mu);
    if (g_pool) cudaFree(g_pool);
    if (g_pool_stream) cudaStreamDestroy(g_pool_stream);
    g_pool = nullptr;
    g_pool_cap = 0;
    g_pool_stream = nullptr;
    g_pool_dev = -1;
}

int64_t ecl_mst(int32_t n, const int64_t* nindex, const int32_t* nlist, const int32_t* eweight, uint8_t* in_mst_out) {
    g_last_error.clear();
    if (n < 0 || (n > 0 && !nindex)) {
        fail(ECL_MST_ERR_INVALID, "invalid n or null nindex");
        return INT64_MIN;
    }
    const int64_t M = n > 0 ? nindex[n] : 0;
    if (n > 0 && nindex[0] != 0) {
        fail(ECL_MST_ERR_INVALID, "nindex[0] != 0");
        return INT64_MIN;
    }
    if (M < 0 || M > (int64_t)0xFFFFFFFFLL) {
        fail(ECL_MST_ERR_TOO_LARGE, "M out of range");
        return INT64_MIN;
    }
    if (M > 0 && (!nlist || !eweight || !in_mst_out)) {
        fail(ECL_MST_ERR_INVALID, "null CSR or output array");
        return INT64_MIN;
    }
    if (M == 0) return 0;
    std::lock_guard<std::mutex> lk(g_pool_mu);
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    const size_t b_idx = align_up(sizeof(int64_t) * ((size_t)n + 1), 256);
    const size_t b_list = align_up(sizeof(int32_t) * (size_t)M, 256);
    const size_t b_mst = align_up((size_t)M, 256);
    const size_t b_tot = 256;
    const size_t b_ws = ecl_mst_workspace_bytes(n, M);
    const size_t need = b_idx + 2 * b_list + b_mst + b_tot + b_ws;
    if (e == cudaSuccess && (g_pool_dev != dev || g_pool_cap < need)) {
        if (g_pool) cudaFree(g_pool);
        g_pool = nullptr;
        g_pool_cap = 0;
        if (g_pool_stream && g_pool_dev != dev) {
            cudaStreamDestroy(g_pool_stream);
            g_pool_stream = nullptr;
        }
        e = cudaMalloc(&g_pool, need);
        if (e == cudaSuccess) {
            g_pool_cap = need;
            g_pool_dev = dev;
        }
    }
    if (e == cudaSuccess && !g_pool_stream) e = cudaStreamCreateWithFlags(&g_pool_stream, cudaStreamNonBlocking);
    if (e != cudaSuccess) {
        fail(ECL_MST_ERR_CUDA, "host path setup: %s", cudaGetErrorString(e));
        return INT64_MIN;
    }
    char* base = static_cast<char*>(g_pool);
    int64_t* d_idx = reinterpret_cast<int64_t*>(base);
    int32_t* d_list = reinterpret_cast<int32_t*>(base + b_idx);
    int32_t* d_w = reinterpret_cast<int32_t*>(base + b_idx + b_list);
    uint8_t* d_mst = reinterpret_cast<uint8_t*>(base + b_idx + 2 * b_list);
    int64_t* d_tot = reinterpret_cast<int64_t*>(base + b_idx + 2 * b_list + b_mst);
    void* d_ws = base + b_idx + 2 * b_list + b_mst + b_tot;
    cudaStream_t s = g_pool_stream;
    e = cudaMemcpyAsync(d_idx, nindex, sizeof(int64_t) * ((size_t)n + 1), cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(d_list, nlist, sizeof(int32_t) * (size_t)M, cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(d_w, eweight, sizeof(int32_t) * (size_t)M, cudaMemcpyHostToDevice, s);
    if (e != cudaSuccess) {
        fail(ECL_MST_ERR_CUDA, "H2D: %s", cudaGetErrorString(e));
        return INT64_MIN;
    }
    int rc = ecl_mst_device(n, M, d_idx, d_list, d_w, d_mst, d_tot, d_ws, b_ws, nullptr, s);
    if (rc) return INT64_MIN;
    int64_t total = INT64_MIN;
    e = cudaMemcpyAsync(in_mst_out, d_mst, (size_t)M, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(&total, d_tot, sizeof total, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) {
        fail(ECL_MST_ERR_CUDA, "D2H/run: %s", cudaGetErrorString(e));
        return INT64_MIN;
    }
    if (total == INT64_MIN) fail(ECL_MST_ERR_INPUT, "device found an inconsistent CSR");
    return total;
}

}  // extern "C"

// ===========================================================================
// distributed (edge-sharded) path: host side
// ===========================================================================
namespace eclmst {

// NCCL is taken from the process at run time (torch's libnccl.so.2 when torch
// is loaded), so the single-GPU library has no NCCL dependency.
struct NcclUid {
    char internal[128];
};
typedef void* NcclComm;
struct NcclApi {
    bool ok = false;
    int (*getUniqueId)(NcclUid*) = nullptr;
    int (*commInitRank)(NcclComm*, int, NcclUid, int) = nullptr;
    int (*allReduce)(const void*, void*, size_t, int, int, NcclComm, cudaStream_t) = nullptr;
    int (*commDestroy)(NcclComm) = nullptr;
    const char* (*getErrorString)(int) = nullptr;
};
constexpr int kNcclInt64 = 4, kNcclSum = 0, kNcclMin = 3;
static NcclApi g_nccl;
static std::mutex g_nccl_mu;

static int load_nccl() {
    std::lock_guard<std::mutex> lk(g_nccl_mu);
    if (g_nccl.ok) return ECL_MST_OK;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    const char* env = getenv("ECLMST_NCCL_LIB");
    if (!h && env) h = dlopen(env, RTLD_NOW);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW);
    if (!h) return fail(ECL_MST_ERR_CUDA, "libnccl.so.2 not found: %s", dlerror());
    g_nccl.getUniqueId = reinterpret_cast<int (*)(NcclUid*)>(dlsym(h, "ncclGetUniqueId"));
    g_nccl.commInitRank = reinterpret_cast<int (*)(NcclComm*, int, NcclUid, int)>(dlsym(h, "ncclCommInitRank"));
    g_nccl.allReduce = reinterpret_cast<int (*)(const void*, void*, size_t, int, int, NcclComm, cudaStream_t)>(
        dlsym(h, "ncclAllReduce"));
    g_nccl.commDestroy = reinterpret_cast<int (*)(NcclComm)>(dlsym(h, "ncclCommDestroy"));
    g_nccl.getErrorString = reinterpret_cast<const char* (*)(int)>(dlsym(h, "ncclGetErrorString"));
    if (!g_nccl.getUniqueId || !g_nccl.commInitRank || !g_nccl.allReduce || !g_nccl.commDestroy)
        return fail(ECL_MST_ERR_CUDA, "libnccl.so.2 lacks the needed symbols");
    g_nccl.ok = true;
    return ECL_MST_OK;
}

struct DistHandle {
    int rank = 0, world = 1;
    NcclComm comm = nullptr;
    long long* h_pin = nullptr;   // pinned host word for the per-round set count
};

struct DistLayout {
    size_t stats, internal, rowstart, parent, tgt, keyptrs, shard0, shard_bytes, total;
    size_t region, acnt, key, wl0, wl1;   // offsets inside one shard block
    long long wl_cap, nlocal_max;
};

static inline DistLayout dist_layout(int64_t n, int64_t M, int S, int world) {
    DistLayout L;
    const long long nchunks = ceil_div(M, kChunk);
    const long long P = (long long)S * world;
    L.nlocal_max = ceil_div(nchunks, P);
    const long long wmax = L.nlocal_max < kMaxPopWarps ? L.nlocal_max : kMaxPopWarps;
    L.wl_cap = (L.nlocal_max + wmax) * kChunk;
    size_t off = 0;
    L.stats = off;    off = align_up(off + sizeof(ecl_mst_stats), 256);
    L.internal = off; off = align_up(off + sizeof(Internal), 256);
    L.rowstart = off; off = align_up(off + sizeof(int) * (size_t)(nchunks + 1), 256);
    L.parent = off;   off = align_up(off + sizeof(int) * (size_t)n, 256);
    L.tgt = off;      off = align_up(off + sizeof(int) * (size_t)n, 256);
    L.keyptrs = off;  off = align_up(off + sizeof(long long*) * (size_t)S, 256);
    size_t so = 0;
    L.region = so; so = align_up(so + sizeof(int4) * (size_t)kMaxPopWarps, 256);
    L.acnt = so;   so = align_up(so + sizeof(int) * (size_t)kMaxGrid, 256);
    L.key = so;    so = align_up(so + sizeof(long long) * (size_t)n, 256);
    L.wl0 = so;    so = align_up(so + sizeof(int4) * (size_t)L.wl_cap, 256);
    L.wl1 = so;    so = align_up(so + sizeof(int4) * (size_t)L.wl_cap, 256);
    L.shard_bytes = so;
    L.shard0 = off;
    off += so * (size_t)S;
    L.total = off;
    return L;
}

}  // namespace eclmst

extern "C" {

int ecl_mst_dist_unique_id(void* uid_out) {
    g_last_error.clear();
    if (!uid_out) return fail(ECL_MST_ERR_INVALID, "null argument");
    int rc = load_nccl();
    if (rc) return rc;
    int r = g_nccl.getUniqueId(reinterpret_cast<NcclUid*>(uid_out));
    if (r) return fail(ECL_MST_ERR_CUDA, "ncclGetUniqueId: %d", r);
    return ECL_MST_OK;
}

int ecl_mst_dist_init(const void* uid, int32_t rank, int32_t world, void** handle_out) {
    g_last_error.clear();
    if (!handle_out || world < 1 || rank < 0 || rank >= world) return fail(ECL_MST_ERR_INVALID, "bad rank/world");
    DistHandle* h = new DistHandle;
    h->rank = rank;
    h->world = world;
    cudaError_t e = cudaHostAlloc(reinterpret_cast<void**>(&h->h_pin), sizeof(long long) * 4, cudaHostAllocDefault);
    if (e != cudaSuccess) {
        delete h;
        return fail(ECL_MST_ERR_CUDA, "cudaHostAlloc: %s", cudaGetErrorString(e));
    }
    if (world > 1 || uid) {   // world 1 with a uid: a one-rank NCCL communicator (tests the NCCL path)
        if (!uid) {
            cudaFreeHost(h->h_pin);
            delete h;
            return fail(ECL_MST_ERR_INVALID, "world > 1 needs an NCCL unique id");
        }
        int rc = load_nccl();
        NcclUid id;
        if (!rc) {
            std::memcpy(id.internal, uid, sizeof id.internal);
            const int r = g_nccl.commInitRank(&h->comm, world, id, rank);
            if (r) rc = fail(ECL_MST_ERR_CUDA, "ncclCommInitRank: %s", g_nccl.getErrorString ? g_nccl.getErrorString(r) : "?");
        }
        if (rc) {
            cudaFreeHost(h->h_pin);
            delete h;
            return rc;
        }
    }
    *handle_out = h;
    return ECL_MST_OK;
}

int ecl_mst_dist_finalize(void* handle) {
    g_last_error.clear();
    DistHandle* h = static_cast<DistHandle*>(handle);
    if (!h) return ECL_MST_OK;
    if (h->comm && g_nccl.ok) g_nccl.commDestroy(h->comm);
    if (h->h_pin) cudaFreeHost(h->h_pin);
    delete h;
    return ECL_MST_OK;
}

int64_t ecl_mst_dist_shard_chunks(int64_t M, int32_t shard, int32_t nshards) {
    if (M < 0 || nshards < 1 || shard < 0 || shard >= nshards) return -1;
    const long long nchunks = ceil_div(M, kChunk);
    return shard < nchunks ? (nchunks - shard + nshards - 1) / nshards : 0;
}

size_t ecl_mst_dist_workspace_bytes(int64_t n, int64_t M, int32_t local_shards, int32_t world) {
    if (n < 0 || n > INT32_MAX || M < 0 || M > (int64_t)0xFFFFFFFFLL || local_shards < 1 || world < 1) return 0;
    return dist_layout(n, M, local_shards, world).total;
}

int ecl_mst_dist_device(void* handle, int32_t local_shards, int32_t n, int64_t M, const int64_t* nindex,
                        const int32_t* nlist, const int32_t* eweight, uint8_t* in_mst_out,
                        int64_t* total_weight_out, void* workspace, size_t workspace_bytes,
                        const ecl_mst_options* opts, void* stream) {
    g_last_error.clear();
    DistHandle* h = static_cast<DistHandle*>(handle);
    if (!h) return fail(ECL_MST_ERR_INVALID, "null handle (ecl_mst_dist_init)");
    const int S = local_shards, world = h->world, rank = h->rank;
    if (S < 1 || S > 64) return fail(ECL_MST_ERR_INVALID, "local_shards must be in [1, 64]");
    if (world > 1 && S != 1) return fail(ECL_MST_ERR_INVALID, "local_shards > 1 only without NCCL (world 1)");
    if (n < 0 || M < 0) return fail(ECL_MST_ERR_INVALID, "negative n or M");
    if (M > (int64_t)0xFFFFFFFFLL) return fail(ECL_MST_ERR_TOO_LARGE, "M exceeds 2^32-1");
    if (!total_weight_out || !workspace || (n > 0 && !nindex) || (M > 0 && (!nlist || !eweight || !in_mst_out)))
        return fail(ECL_MST_ERR_INVALID, "null argument");
    if (M > 0 && n == 0) return fail(ECL_MST_ERR_INVALID, "M > 0 with n = 0");
    const DistLayout L = dist_layout(n, M, S, world);
    if (workspace_bytes < L.total) return fail(ECL_MST_ERR_WORKSPACE, "workspace %zu < %zu bytes", workspace_bytes, L.total);
    if (reinterpret_cast<uintptr_t>(workspace) % 256) return fail(ECL_MST_ERR_WORKSPACE, "workspace not 256-byte aligned");
    if ((reinterpret_cast<uintptr_t>(nlist) | reinterpret_cast<uintptr_t>(eweight)) % 16 ||
        reinterpret_cast<uintptr_t>(in_mst_out) % 4)
        return fail(ECL_MST_ERR_INVALID, "nlist/eweight must be 16-byte and in_mst 4-byte aligned");
    ecl_mst_options o;
    ecl_mst_default_options(&o);
    if (opts) o = *opts;
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    char* ws = static_cast<char*>(workspace);
    ecl_mst_stats* st = reinterpret_cast<ecl_mst_stats*>(ws + L.stats);
    Internal* in = reinterpret_cast<Internal*>(ws + L.internal);
    if (M == 0) {
        cudaError_t e = cudaMemsetAsync(st, 0, sizeof(ecl_mst_stats), s);
        if (e == cudaSuccess) e = cudaMemsetAsync(total_weight_out, 0, sizeof(int64_t), s);
        if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "memset: %s", cudaGetErrorString(e));
        return ECL_MST_OK;
    }
    DevInfo di;
    int rc = device_info(&di);
    if (rc) return rc;
    const long long nchunks = ceil_div(M, kChunk);
    const long long Pt = (long long)S * world;

    // per-shard launch geometry and parameters
    std::vector<Params> sp(S);
    std::vector<long long*> keyptr(S);
    for (int k = 0; k < S; ++k) keyptr[k] = reinterpret_cast<long long*>(ws + L.shard0 + k * L.shard_bytes + L.key);
    long long** d_keyptrs = reinterpret_cast<long long**>(ws + L.keyptrs);
    cudaError_t e = cudaMemcpyAsync(d_keyptrs, keyptr.data(), sizeof(long long*) * S, cudaMemcpyHostToDevice, s);
    for (int k = 0; k < S; ++k) {
        Params& P = sp[k];
        std::memset(&P, 0, sizeof P);
        const int shard = rank * S + k;
        const long long nlocal = shard < nchunks ? (nchunks - shard + Pt - 1) / Pt : 0;
        long long G = (long long)di.sms * di.occ;
        if (G > std::max<long long>(nlocal, 1)) G = std::max<long long>(nlocal, 1);
        if (G > kMaxGrid) G = kMaxGrid;
        long long W = (long long)di.sms * di.pop_occ * kPopWarps;
        if (W > std::max<long long>(nlocal, 1)) W = std::max<long long>(nlocal, 1);
        if (W > kMaxPopWarps) W = kMaxPopWarps;
        if (W > G * kMaxRegionsPerCta) W = G * kMaxRegionsPerCta;
        W = std::max<long long>(1, W / G) * G;
        const long long rcap = std::max<long long>(1, ceil_div(nlocal, W)) * kChunk;
        const long long cap = (W / G) * rcap;
        if (W * rcap > L.wl_cap || cap >= (1LL << 30)) return fail(ECL_MST_ERR_TOO_LARGE, "shard worklist too large");
        char* sb = ws + L.shard0 + k * L.shard_bytes;
        P.n = n;
        P.M = M;
        P.nchunks = nchunks;
        P.G = (int)G;
        P.cap = cap;
        P.W = (int)W;
        P.rcap = rcap;
        P.nindex = reinterpret_cast<const long long*>(nindex);
        P.nlist = nlist;
        P.eweight = eweight;
        P.in_mst = in_mst_out;
        P.total_out = reinterpret_cast<long long*>(total_weight_out);
        P.st = st;
        P.in = in;
        P.trace = nullptr;
        P.rowstart = reinterpret_cast<int*>(ws + L.rowstart);
        P.region = reinterpret_cast<int4*>(sb + L.region);
        P.key = keyptr[k];
        P.parent = reinterpret_cast<int*>(ws + L.parent);
        P.wl0 = reinterpret_cast<int4*>(sb + L.wl0);
        P.wl1 = reinterpret_cast<int4*>(sb + L.wl1);
        P.seed = o.seed;
        P.filter_mode = o.filter < 0 ? -1 : (o.filter ? 1 : 0);
        P.threshold_mode = o.threshold_mode;
        P.threshold_value = o.threshold;
        P.samples = o.threshold_samples > 0 ? std::min(o.threshold_samples, kMaxSamples) : 20;
        P.halving = o.path_halving ? 1 : 0;
        P.guards = o.atomic_guards == 0 ? 0 : 1;
        P.flatten = o.flatten ? 1 : 0;
        P.shard = shard;
        P.nshards = (int)Pt;
        P.nlocal = nlocal;
        P.zero_mst = 0;
        P.acnt = reinterpret_cast<int*>(sb + L.acnt);
        P.tgt = reinterpret_cast<int*>(ws + L.tgt);
        P.keys_all = d_keyptrs;
        P.nkeys = S;
    }
    Params& P0 = sp[0];
    const unsigned vblocks = (unsigned)std::max<long long>(1, std::min<long long>(ceil_div((long long)n, 256), (long long)di.sms * 8));
    auto check = [&](const char* what) -> int {
        cudaError_t e2 = cudaGetLastError();
        if (e2 != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e2));
        return ECL_MST_OK;
    };
    auto allreduce = [&](void* buf, size_t count, int op) -> int {
        if (!h->comm) return ECL_MST_OK;
        const int r = g_nccl.allReduce(buf, buf, count, kNcclInt64, op, h->comm, s);
        if (r) return fail(ECL_MST_ERR_CUDA, "ncclAllReduce: %s", g_nccl.getErrorString ? g_nccl.getErrorString(r) : "?");
        return ECL_MST_OK;
    };
    auto read_word = [&](const void* dptr, long long* out) -> int {
        cudaError_t e2 = cudaMemcpyAsync(h->h_pin, dptr, sizeof(long long), cudaMemcpyDeviceToHost, s);
        if (e2 == cudaSuccess) e2 = cudaStreamSynchronize(s);
        if (e2 != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "sync: %s", cudaGetErrorString(e2));
        *out = *h->h_pin;
        return ECL_MST_OK;
    };

    if (e == cudaSuccess) e = cudaMemsetAsync(st, 0, sizeof(ecl_mst_stats), s);
    if (e == cudaSuccess) e = cudaMemsetAsync(in_mst_out, 0, (size_t)M, s);   // every rank returns the full mask
    if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "memset: %s", cudaGetErrorString(e));
    k_init<<<vblocks, 256, 0, s>>>(P0);
    if ((rc = check("k_init"))) return rc;
    int g = 0;
    for (int ph = 1; ph <= 2; ++ph) {
        if (ph == 2) {
            // the phase-2 decision needs the global deferred count
            if ((rc = allreduce(&st->canonical_edges, 2, kNcclSum))) return rc;
            long long filtered = 0, heavy = 0;
            if ((rc = read_word(&st->heavy_edges, &heavy))) return rc;
            if ((rc = read_word(&st->filtered, &filtered))) return rc;
            if (!(filtered & 0xffffffffll) || heavy == 0) break;
            k_flatten<1><<<vblocks, 256, 0, s>>>(P0);
            k_flatten<2><<<vblocks, 256, 0, s>>>(P0);
            ++g;
            if (g >= ECL_MST_MAX_ROUNDS) return fail(ECL_MST_ERR_INPUT, "round limit");
            e = cudaMemcpyAsync(&st->phase2_round, &g, sizeof(int), cudaMemcpyHostToDevice, s);
            if (e == cudaSuccess) e = cudaStreamSynchronize(s);   // &g is a host stack value
            if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "phase2: %s", cudaGetErrorString(e));
        }
        for (int k = 0; k < S; ++k) {
            if (ph == 1) k_populate<1><<<(unsigned)ceil_div(sp[k].W, kPopWarps), kPopBlock, 0, s>>>(sp[k]);
            else k_populate<2><<<(unsigned)ceil_div(sp[k].W, kPopWarps), kPopBlock, 0, s>>>(sp[k]);
        }
        if ((rc = check("populate"))) return rc;
        bool first = true;
        int cur = 0;
        while (true) {
            // allreduce(min) of the best-edge keys over all shards
            if (S > 1) k_vreduce<<<vblocks, 256, 0, s>>>(P0);
            if ((rc = allreduce(P0.key, (size_t)n, kNcclMin))) return rc;
            e = cudaMemsetAsync(&in->reps, 0, sizeof(in->reps), s);
            if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "memset: %s", cudaGetErrorString(e));
            k_dist_reps1<<<vblocks, 256, 0, s>>>(P0);
            long long reps = 0;
            if ((rc = read_word(&in->reps, &reps))) return rc;
            if (reps == 0) {
                if (first)
                    for (int k = 0; k < S; ++k) k_dist_passA<true><<<sp[k].G, kBlock, 0, s>>>(sp[k], g + 1, cur);
                break;   // no set has a live edge anywhere: the phase is done
            }
            k_dist_reps2<<<vblocks, 256, 0, s>>>(P0, g);
            if (g + 1 >= ECL_MST_MAX_ROUNDS) return fail(ECL_MST_ERR_INPUT, "round limit");
            ++g;
            for (int k = 0; k < S; ++k) {
                if (first) k_dist_passA<true><<<sp[k].G, kBlock, 0, s>>>(sp[k], g, cur);
                else k_dist_passA<false><<<sp[k].G, kBlock, 0, s>>>(sp[k], g, cur);
            }
            cur ^= 1;
            first = false;
            if ((rc = check("rounds"))) return rc;
        }
    }
    const int rounds = g + 1;
    e = cudaMemcpyAsync(&st->rounds, &rounds, sizeof(int), cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "stats: %s", cudaGetErrorString(e));
    k_finalize<<<1, 32, 0, s>>>(P0);
    if ((rc = check("finalize"))) return rc;
    return ECL_MST_OK;
}

}  // extern "C"
