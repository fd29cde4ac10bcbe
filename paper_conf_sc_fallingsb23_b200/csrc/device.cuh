// device.cuh -- device building blocks of the ECL-MST hot path (sm_100a).
//
// Union-find with implicit path compression (Alg. 2 L15-18),
// the packed 64-bit (weight:id) best-edge key, guarded 64-bit
// atomicMin, and warp-level worklist compaction (ballot + one shared
// atomicAdd per warp and chunk, replacing the paper's per-edge atomicAdd of
// P:154 "Lines 7 and 18").
#pragma once

#include <cstdint>
#include <climits>
#include <cuda_runtime.h>

namespace eclmst {

#ifndef ECL_R_BLOCK
#define ECL_R_BLOCK 512
#endif
#ifndef ECL_R_MINB
#define ECL_R_MINB 2
#endif
constexpr int kBlock = ECL_R_BLOCK;          // threads per k_rounds CTA
constexpr int kWarps = kBlock / 32;
constexpr int kItems = 4;                    // tuples / CSR entries per lane per warp chunk
constexpr int kChunk = 32 * kItems;          // 128 per warp chunk
constexpr long long kInf = LLONG_MAX;        // "no edge recorded" (reading Q4)
constexpr unsigned kFull = 0xffffffffu;

// View of the per-vertex state: disjoint-set parent and best-edge key
// (minEdge), two arrays.  (Interleaving them into 16-byte records was
// measured slower on every config: C5 86.9 vs 73.9 ms, road 2.92 vs 2.38 ms.)
struct DS {
    int* parent;
    long long* key;
    __device__ __forceinline__ int* par(long long v) const { return parent + v; }
    __device__ __forceinline__ long long* k(long long v) const { return key + v; }
};

// (weight:id) key, weight in the most significant bits: signed order
// of the key == lexicographic order of (weight as int32, id as uint32).
__device__ __forceinline__ long long make_key(int w, unsigned id) {
    return (long long)(((unsigned long long)(long long)w << 32) | (unsigned long long)id);
}

__device__ __forceinline__ unsigned long long globaltimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// ---------------------------------------------------------------------------
// disjoint sets.  Within one stage of the persistent kernel parent[] only
// changes by path halving (a vertex re-pointed to one of its ancestors) or,
// in pass B, by hooking roots -- and pass B never reads it.  Every grid
// barrier ends with a gpu-scope fence, which invalidates L1 (CCTL.IVALL), so a
// find() may read parent[] through L1 (ld.global.ca): a stale cached pointer
// is still an ancestor, and roots cannot change while finds run.  Hot roots
// (one giant set touched by millions of edges) are then served by L1 instead
// of one L2 slice.
// ---------------------------------------------------------------------------

// Continue a find() from x whose parent px is already loaded.  With halving
// on, every visited non-root is re-pointed to its grandparent (path halving;
// a benign race: the stored value is always an ancestor).
__device__ __forceinline__ int find_from(const DS& D, int x, int px, bool halving) {
    while (px != x) {
        const int ppx = __ldca(D.par(px));
        if (ppx == px) return px;
        if (halving) *D.par(x) = ppx;
        x = ppx;
        px = __ldca(D.par(x));
    }
    return x;
}

__device__ __forceinline__ int find_root(const DS& D, int x, bool halving) {
    return find_from(D, x, __ldca(D.par(x)), halving);
}

// find() in a CLOSED contraction level (opts.relabel): every root r stores
// ~label(r), its id in the next level, so the walk ends at the first negative
// entry and returns that label.  Halving re-points x to its grandparent as
// above (only non-negative ancestors are ever stored).
__device__ __forceinline__ int find_label_from(int* par, int x, int px, bool halving) {
    while (px >= 0) {
        const int ppx = __ldca(par + px);
        if (ppx < 0) return ~ppx;
        if (halving) par[x] = ppx;
        x = ppx;
        px = __ldca(par + x);
    }
    return ~px;
}

// 64-bit atomicMin (L20-21) with the paper's optional guard: a plain
// load first, skipping the atomic when it cannot lower the slot.  The guard
// may read through L1: slots only decrease during a pass, so a stale value is
// >= the current one and a skipped atomic could never have lowered the slot.
__device__ __forceinline__ void record_min(long long* slot, long long key, bool guard) {
    if (!guard || __ldca(slot) > key) atomicMin(slot, key);
}

// ---------------------------------------------------------------------------
// Worklist tuple storage.  The default is the paper's 16-byte 4-tuple
// <p, q, w, id>, one vector access per tuple.  SOA is the "No
// Tuples" de-optimisation: the four items in four int planes
// `stride` tuples apart.  A tuple pointer is the int4* of a range's first
// tuple (AoS) or the address of that tuple's plane-0 int, cast to int4*
// (SoA); tadd() moves it by tuples either way.
// ---------------------------------------------------------------------------
template <bool SOA>
__device__ __forceinline__ int4* tadd(int4* p, long long n) {
    return SOA ? reinterpret_cast<int4*>(reinterpret_cast<int*>(p) + n) : p + n;
}
template <bool SOA>
__device__ __forceinline__ const int4* tadd(const int4* p, long long n) {
    return SOA ? reinterpret_cast<const int4*>(reinterpret_cast<const int*>(p) + n) : p + n;
}
// streaming load (read once), L2 load, L2 store, and the weight alone
template <bool SOA>
__device__ __forceinline__ int4 tld_cs(const int4* p, long long i, long long stride) {
    if (!SOA) return __ldcs(p + i);
    const int* q = reinterpret_cast<const int*>(p) + i;
    return make_int4(__ldcs(q), __ldcs(q + stride), __ldcs(q + 2 * stride), __ldcs(q + 3 * stride));
}
template <bool SOA>
__device__ __forceinline__ int4 tld_cg(const int4* p, long long i, long long stride) {
    if (!SOA) return __ldcg(p + i);
    const int* q = reinterpret_cast<const int*>(p) + i;
    return make_int4(__ldcg(q), __ldcg(q + stride), __ldcg(q + 2 * stride), __ldcg(q + 3 * stride));
}
template <bool SOA>
__device__ __forceinline__ void tst_cg(int4* p, long long i, int4 t, long long stride) {
    if (!SOA) {
        __stcg(p + i, t);
        return;
    }
    int* q = reinterpret_cast<int*>(p) + i;
    __stcg(q, t.x);
    __stcg(q + stride, t.y);
    __stcg(q + 2 * stride, t.z);
    __stcg(q + 3 * stride, t.w);
}
template <bool SOA>
__device__ __forceinline__ int tld_w(const int4* p, long long i, long long stride) {
    return SOA ? __ldcg(reinterpret_cast<const int*>(p) + i + 2 * stride) : __ldcg(&p[i].z);
}

// Warp-level compaction of one chunk (kItems tuples per lane, any order):
// one shared-memory atomicAdd per warp reserves the output range.
template <bool SOA = false>
__device__ __forceinline__ int warp_emit(const int4 (&t)[kItems], const bool (&keep)[kItems],
                                         int4* __restrict__ out, int* s_out, long long stride = 0) {
    const int lane = threadIdx.x & 31;
    unsigned m[kItems];
    int off[kItems];
    int tot = 0;
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
        m[i] = __ballot_sync(kFull, keep[i]);
        off[i] = tot;
        tot += __popc(m[i]);
    }
    int base = 0;
    if (lane == 0 && tot) base = atomicAdd(s_out, tot);
    base = __shfl_sync(kFull, base, 0);
    const unsigned lt = (1u << lane) - 1u;
#pragma unroll
    for (int i = 0; i < kItems; ++i)
        if (keep[i]) tst_cg<SOA>(out, base + off[i] + __popc(m[i] & lt), t[i], stride);
    return tot;
}

// Same, for the tuples a crowded-round split defers: they fill the arena from
// its end downwards ([end - total, end) after the pass, contiguous).
template <bool SOA = false>
__device__ __forceinline__ void warp_emit_back(const int4 (&t)[kItems], const bool (&keep)[kItems],
                                               int4* __restrict__ end, int* s_cnt, long long stride = 0) {
    const int lane = threadIdx.x & 31;
    unsigned m[kItems];
    int off[kItems];
    int tot = 0;
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
        m[i] = __ballot_sync(kFull, keep[i]);
        off[i] = tot;
        tot += __popc(m[i]);
    }
    if (!tot) return;
    int base = 0;
    if (lane == 0) base = atomicAdd(s_cnt, tot);
    base = __shfl_sync(kFull, base, 0);
    int4* dst = tadd<SOA>(end, -(long long)(base + tot));
    const unsigned lt = (1u << lane) - 1u;
#pragma unroll
    for (int i = 0; i < kItems; ++i)
        if (keep[i]) tst_cg<SOA>(dst, off[i] + __popc(m[i] & lt), t[i], stride);
}

// warp-cooperative 32-ary search: largest r in [0, n) with nindex[r] <= x.
// Requires nindex[0] <= x; about log32(n) dependent 8-byte loads.
__device__ __forceinline__ int warp_row_of(const long long* __restrict__ nindex, int n, long long x) {
    const int lane = threadIdx.x & 31;
    long long lo = 0, hi = n;
    while (hi - lo > 1) {
        const long long step = (hi - lo + 31) / 32;
        const long long r = lo + lane * step;
        const bool ok = (r < hi) && (__ldg(nindex + r) <= x);
        const unsigned b = __ballot_sync(kFull, ok);
        const int k = b ? 31 - __clz(b) : 0;
        lo = lo + k * step;
        hi = min(hi, lo + step);
    }
    return (int)lo;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
    return v;
}

__device__ __forceinline__ unsigned long long splitmix64(unsigned long long x) {
    unsigned long long z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

}  // namespace eclmst
