// device.cuh -- device building blocks of the ECL-MST hot path (sm_100a).
//
// Union-find with implicit path compression (Alg. 2 L15-18),
// the packed 64-bit (weight:id) best-edge key, lock-free CAS
// union ("Line 30 ... atomicCAS"), and block-level worklist
// compaction (warp ballot + one block scan, replacing the paper's per-edge
// atomicAdd of P:154 "Lines 7 and 18").
#pragma once

#include <cstdint>
#include <climits>
#include <cuda_runtime.h>

namespace eclmst {

constexpr int kBlock = 512;                  // threads per CTA
constexpr int kItems = 4;                    // worklist tuples / CSR entries per thread per tile
constexpr int kTile = kBlock * kItems;       // 2048 per CTA tile
constexpr int kWarps = kBlock / 32;
constexpr int kScanSlots = kItems * kWarps;  // per-(item, warp) counts of one tile
static_assert(kScanSlots == 64, "block_compact scans 64 slots with one warp (2 per lane)");
constexpr long long kInf = LLONG_MAX;        // "no edge recorded" (reading Q4)
constexpr unsigned kFull = 0xffffffffu;

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
// disjoint sets.  parent[] is read through L2 (ld.global.cg): other SMs hook
// roots with atomicCAS during the check/join pass, and L1 is not coherent.
// ---------------------------------------------------------------------------

// Continue a find() from x whose parent px is already loaded.  With halving
// on, every visited non-root is re-pointed to its grandparent (path halving;
// benign race: the stored value is always an ancestor, and roots are never
// written except by the CAS in join()).
__device__ __forceinline__ int find_from(int* __restrict__ parent, int x, int px, bool halving) {
    while (px != x) {
        const int ppx = __ldcg(parent + px);
        if (ppx == px) return px;
        if (halving) __stcg(parent + x, ppx);
        x = ppx;
        px = __ldcg(parent + x);
    }
    return x;
}

__device__ __forceinline__ int find_root(int* __restrict__ parent, int x, bool halving) {
    return find_from(parent, x, __ldcg(parent + x), halving);
}

// Lock-free union: hook the larger root under the smaller with
// atomicCAS, retrying from the new parent if another thread hooked it first.
// The root of every set is therefore its minimum vertex id (reading Q3).
__device__ __forceinline__ void join(int* __restrict__ parent, int a, int b, bool halving) {
    while (true) {
        a = find_root(parent, a, halving);
        b = find_root(parent, b, halving);
        if (a == b) return;
        const int lo = min(a, b), hi = max(a, b);
        const int old = atomicCAS(parent + hi, hi, lo);
        if (old == hi) return;
        a = lo;
        b = old;
    }
}

// Guarded 64-bit atomicMin ("atomic guards"): plain L2 load first,
// skip the atomic if it cannot lower the slot.
__device__ __forceinline__ void guarded_min(long long* slot, long long key) {
    if (__ldcg(slot) > key) atomicMin(slot, key);
}

// ---------------------------------------------------------------------------
// block-level compaction of one tile: kItems tuples per thread, any order.
// Returns the number kept (block-uniform) and writes them to out[0, kept).
// s_cnt must hold kScanSlots + 1 ints.
// ---------------------------------------------------------------------------
__device__ __forceinline__ int block_compact(const int4 (&t)[kItems], const bool (&keep)[kItems],
                                             int4* __restrict__ out, int* s_cnt) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    unsigned mask[kItems];
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
        mask[i] = __ballot_sync(kFull, keep[i]);
        if (lane == 0) s_cnt[i * kWarps + warp] = __popc(mask[i]);
    }
    __syncthreads();
    if (warp == 0) {
        const int a = s_cnt[2 * lane], b = s_cnt[2 * lane + 1];
        const int s = a + b;
        int incl = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(kFull, incl, o);
            if (lane >= o) incl += y;
        }
        const int excl = incl - s;
        s_cnt[2 * lane] = excl;
        s_cnt[2 * lane + 1] = excl + a;
        if (lane == 31) s_cnt[kScanSlots] = incl;
    }
    __syncthreads();
    const unsigned lt = (1u << lane) - 1u;
#pragma unroll
    for (int i = 0; i < kItems; ++i)
        if (keep[i]) __stcg(out + s_cnt[i * kWarps + warp] + __popc(mask[i] & lt), t[i]);
    const int kept = s_cnt[kScanSlots];
    __syncthreads();
    return kept;
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
