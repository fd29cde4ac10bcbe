// rounds.cuh -- the round loop: k_flatten / k_giant (before phase 2), the
// worklist views, pass A (Alg. 2 L14-23), pass B (L27-31 + L34-37), the
// persistent cooperative k_rounds kernel and k_finalize.
#pragma once

#include <type_traits>

#include "common.cuh"

namespace eclmst {

#ifndef ECL_WARP_CLAIM
#define ECL_WARP_CLAIM 1   // k_rounds' warps take their CTA's chunks by a shared ticket (next_chunk)
#endif

// ---------------------------------------------------------------------------
// k_flatten: set(v) for every vertex before the phase-2 populate, so
// that populate reads each endpoint's set with one load.
//   stage 0: with two or more closed contraction levels (opts.relabel), the
//            final set of every id of the closed levels above the vertices,
//            kept in that id's (dead) best-edge slot: each walk climbs the
//            small upper levels once instead of once per vertex.
//   stage 1: setid[v] = the root of v's set: a walk in the vertices' level,
//            then its label's final set (stage 0, or a find in the open level
//            when it is the only one above).  With no closed level it also
//            points v at its root (compression for the phase-2 rounds' finds).
//            Roots never change here, so every walk ends at v's root whatever
//            the other threads' halving stores do.
//   stage 2: the largest set's membership bitmap (P.giant_bits) from setid.
// ---------------------------------------------------------------------------
template <int STAGE>
__global__ void __launch_bounds__(256) k_flatten(Params P) {
    if (!phase2_needed(P) || !P.flatten) return;
    if (STAGE == 2 && !P.giant_bits) return;
    const int nlev = __ldcg(&P.in->nlev);
    if (STAGE == 0 && nlev < 2) return;
    const long long stride = (long long)gridDim.x * blockDim.x;
    const int lane = threadIdx.x & 31;
    const DS D = ds_of(P);
    const long long open = __ldcg(&P.in->lv_base);   // first id of the open level
    if (STAGE == 0) {
        for (long long x = P.n + (long long)blockIdx.x * blockDim.x + threadIdx.x; x < open; x += stride) {
            int y = (int)x;
            while (y < open) y = find_label_from(P.parent, y, __ldca(P.parent + y), true);
            __stcg(P.key + x, (long long)find_root(D, y, true));
        }
        return;
    }
    if (STAGE == 1) {
        // a warp takes 128 consecutive vertices, four per lane in flight (the
        // walks are chains of dependent loads; C3 flatten 0.145 -> 0.114 ms,
        // C4 0.108 -> 0.094, C5 0.95 -> 0.90), and v keeps its parent entry
        // when it already names its label
        for (long long b4 = ((long long)blockIdx.x * blockDim.x + threadIdx.x - lane) * 4; b4 < P.n; b4 += 4 * stride) {
            int px[4], lab[4];
#pragma unroll
            for (int a = 0; a < 4; ++a) {
                const long long v = b4 + 32 * a + lane;
                px[a] = v < P.n ? __ldca(P.parent + v) : 0;
            }
#pragma unroll
            for (int a = 0; a < 4; ++a) {
                const long long v = b4 + 32 * a + lane;
                if (v >= P.n) continue;
                if (nlev == 0) {
                    lab[a] = find_from(D, (int)v, px[a], true);
                    if (lab[a] != (int)v) *D.par(v) = lab[a];
                } else {
                    lab[a] = find_label_from(P.parent, (int)v, px[a], true);
                    if (px[a] != ~lab[a]) P.parent[v] = ~lab[a];   // v now names its label directly
                }
            }
            if (nlev >= 2) {   // the label's final set, kept by stage 0 in its dead key slot
#pragma unroll
                for (int a = 0; a < 4; ++a)
                    if (b4 + 32 * a + lane < P.n) lab[a] = (int)__ldcg(P.key + lab[a]);
            } else if (nlev == 1) {
#pragma unroll
                for (int a = 0; a < 4; ++a)
                    if (b4 + 32 * a + lane < P.n) lab[a] = find_root(D, lab[a], true);
            }
#pragma unroll
            for (int a = 0; a < 4; ++a) {
                const long long v = b4 + 32 * a + lane;
                if (v < P.n) __stcg(P.setid + v, lab[a]);
            }
        }
        return;
    }
    const int giant = STAGE == 2 ? __ldcg(&P.in->giant) : -1;
    // warps walk 32 consecutive vertices together (stage 2 ballots the bitmap)
    for (long long base = (long long)blockIdx.x * blockDim.x + threadIdx.x - lane; base < P.n; base += stride) {
        const long long v = base + lane;
        const bool valid = v < P.n;
        if (STAGE == 1) {
            if (valid) {
                int r;
                if (nlev == 0) {
                    r = find_root(D, (int)v, true);
                    if (r != (int)v) *D.par(v) = r;
                } else {
                    const int lab = find_label_from(P.parent, (int)v, __ldca(P.parent + v), true);
                    P.parent[v] = ~lab;   // v now names its label directly
                    r = nlev == 1 ? find_root(D, lab, true) : (int)__ldcg(P.key + lab);
                }
                __stcg(P.setid + v, r);
            }
        } else {
            const int sv = valid ? __ldcg(P.setid + v) : -1;
            const unsigned bits = __ballot_sync(kFull, valid && sv == giant);
            if (lane == 0) P.giant_bits[base >> 5] = bits;
        }
    }
}

// After phase 1 most vertices of a graph whose light edges percolate (C3-C5)
// sit in ONE set.  Find its root as the mode of 256 sampled vertices' roots.
// The phase-2 populate keeps that set's key minimum per warp (it is the hot
// slot almost every kept edge touches), and for n >= 2^25 k_flatten<2> writes
// a bitmap of its members, so that populate filters an edge with both ends in
// it from the bitmap (n/8 bytes, L2 resident) instead of two random parent
// loads.
__global__ void __launch_bounds__(256) k_giant(Params P) {
    constexpr int kS = 256;   // samples (one per thread)
    __shared__ int s_r[kS];
    __shared__ int s_c[kS];
    if (!phase2_needed(P) || !P.flatten) return;
    const int i = threadIdx.x;
    const long long v = (long long)(splitmix64(0x6A09E667F3BCC909ull + (unsigned long long)i) % (unsigned long long)P.n);
    s_r[i] = __ldcg(P.setid + v);   // k_flatten<1> ran
    __syncthreads();
    // the mode of the samples, exactly (a majority vote misses a set holding
    // less than half of them, e.g. RMAT's giant among many isolated vertices)
    int c = 0;
    for (int t = 0; t < kS; ++t) c += s_r[t] == s_r[i];
    s_c[i] = c;
    __syncthreads();
    if (i == 0) {
        int best = 0;
        for (int t = 1; t < kS; ++t)
            if (s_c[t] > s_c[best] || (s_c[t] == s_c[best] && s_r[t] < s_r[best])) best = t;
        P.in->giant = s_c[best] >= kS / 8 ? s_r[best] : -1;   // worth it only if it holds >= 1/8
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
// (SOA: the tuples are stored as four planes, opts.tuple_layout; see tadd.)
template <bool SOA_ = false>
struct CompactSrcT {
    static constexpr bool SOA = SOA_;
    const int4* base;
    int cnt;
    int nloc;
    __device__ __forceinline__ const int4* get(const Params&, int j, int& count) const {
        count = min(kChunk, cnt - j * kChunk);
        return tadd<SOA>(base, (long long)j * kChunk);
    }
};
using CompactSrc = CompactSrcT<false>;

template <bool SOA_ = false>
struct RegionSrcT {
    static constexpr bool SOA = SOA_;
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
        return tadd<SOA>(P.wl0, (long long)(first_w + lo * P.G) * P.rcap + (long long)off * kChunk);
    }
};
using RegionSrc = RegionSrcT<false>;

// pass B's view of the one list a vertex-centric pass A appends to (opts.drive
// 2): CTA b reads the list's chunks b, b + G, ...
template <bool SOA_ = false>
struct GlobalSrcT {
    static constexpr bool SOA = SOA_;
    const int4* base;
    long long cnt;
    int nloc;
    __device__ __forceinline__ const int4* get(const Params&, int j, int& count) const {
        const long long c = blockIdx.x + (long long)j * gridDim.x;
        count = (int)min((long long)kChunk, cnt - c * kChunk);
        return tadd<SOA>(base, c * kChunk);
    }
};

template <bool SOA = false>
__device__ __forceinline__ GlobalSrcT<SOA> global_src(const int4* base, long long cnt) {
    GlobalSrcT<SOA> S;
    S.base = base;
    S.cnt = cnt;
    const long long nch = (cnt + kChunk - 1) / kChunk;
    S.nloc = blockIdx.x < nch ? (int)((nch - blockIdx.x + gridDim.x - 1) / gridDim.x) : 0;
    return S;
}

template <class T>
struct is_compact_src : std::false_type {};
template <bool S2>
struct is_compact_src<CompactSrcT<S2>> : std::true_type {};

template <bool SOA = false>
__device__ __forceinline__ CompactSrcT<SOA> compact_src(const int4* base, int cnt) {
    CompactSrcT<SOA> S;
    S.base = base;
    S.cnt = cnt;
    S.nloc = (cnt + kChunk - 1) / kChunk;
    return S;
}

// the populate output of CTA b: regions w = b, b + G, ...  Loads the region
// counts into shared memory, builds the chunk prefix, and adds the kept,
// canonical and deferred counts to the stats (phase 1 counters only if
// count_phase1).  Every thread of the CTA must call it.
template <bool SOA = false>
__device__ __forceinline__ RegionSrcT<SOA> region_src(const Params& P, int b, int* s_pre, int* s_rcnt,
                                                      long long (*s_red)[kWarps], int64_t* live_slot,
                                                      bool count_phase1) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    RegionSrcT<SOA> R;
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
        if (kept && live_slot) atomicAdd(reinterpret_cast<unsigned long long*>(live_slot), (unsigned long long)kept);
        if (count_phase1) {
            if (canon) atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->canonical_edges), (unsigned long long)canon);
            if (heavy) atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->heavy_edges), (unsigned long long)heavy);
        }
    }
    __syncthreads();
    R.nloc = s_pre[R.nreg];
    return R;
}

// L14-23 of one round over the CTA's worklist: S -> out (compact).  With a
// split threshold T < INT_MAX (a crowded round, see split_threshold) only the
// tuples with w < T record their key and go to the front of `out`; the others
// are deferred to the back of the arena (ending at out_end, count in *s_def).
//
// MAP: a relabel opened a new contraction
// level right before this pass, so the tuples still hold ids of the level
// below, now closed: find() ends at the root's label, its id in the new level
// (where nothing has hooked yet).  The tuples leave with the new level's ids.
// Chunk order within the CTA (ECL_WARP_CLAIM): with a shared ticket counter
// (s_tk, zero at the start of the pass) each warp takes the CTA's next chunk
// when it is free, so the CTA's warps finish together instead of waiting at
// the barrier for the one that drew the slow chunks; without it, warp w takes
// chunks w, w + kWarps, ...  first_chunk/next_chunk return the next index or
// a value >= nloc.
__device__ __forceinline__ int next_chunk(int* s_tk, int k) {
    if (!s_tk) return k + kWarps;
    int t = 0;
    if ((threadIdx.x & 31) == 0) t = atomicAdd(s_tk, 1);
    return __shfl_sync(kFull, t, 0);
}
__device__ __forceinline__ int first_chunk(int* s_tk) { return s_tk ? next_chunk(s_tk, 0) : (int)(threadIdx.x >> 5); }

template <bool SPLIT = false, bool MAP = false, class SRC>
__device__ __forceinline__ void passA(const Params& P, const DS& D, const SRC& S, int4* __restrict__ out,
                                      int* s_out, bool guard, int T = INT_MAX, int4* out_end = nullptr,
                                      int* s_def = nullptr, int* s_tk = nullptr) {
    const int lane = threadIdx.x & 31;
    const bool halving = P.halving != 0;
    for (int k = first_chunk(s_tk); k < S.nloc; k = next_chunk(s_tk, k)) {
        int count;
        const int4* __restrict__ in = S.get(P, k, count);
        int4 t[kItems];
        bool keep[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            const int idx = i * 32 + lane;
            keep[i] = idx < count;
            t[i] = keep[i] ? tld_cs<SRC::SOA>(in, idx, P.wlcap) : make_int4(0, 0, 0, 0);
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
                const int p = MAP ? find_label_from(D.parent, t[i].x, px[i], halving)   // L15
                                  : find_from(D, t[i].x, px[i], halving);
                const int q = MAP ? find_label_from(D.parent, t[i].y, qx[i], halving)   // L16
                                  : find_from(D, t[i].y, qx[i], halving);
                keep[i] = p != q;                                          // L17
                t[i].x = p;                                                // L18: implicit
                t[i].y = q;                                                //      path compression
            }
        }
        if (SPLIT) {   // crowded round: defer w >= T (they record no key)
            bool heavy[kItems];
#pragma unroll
            for (int i = 0; i < kItems; ++i) {
                heavy[i] = keep[i] && t[i].z >= T;
                keep[i] = keep[i] && t[i].z < T;
            }
            warp_emit_back<SRC::SOA>(t, heavy, out_end, s_def, P.wlcap);
        }
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (keep[i]) {
                const long long key = make_key(t[i].z, (unsigned)t[i].w); // L19
                record_min(D.k(t[i].x), key, guard);                      // L20
                record_min(D.k(t[i].y), key, guard);                      // L21
            }
        }
        warp_emit<SRC::SOA>(t, keep, out, s_out, P.wlcap);                // L18
    }
}

// opts.drive 2, "Vertex-Centric": pass A as one thread per vertex
// walking its CSR row in every round -- topology-driven, all edges of the
// phase: p = find(u) once per vertex, q = find(v) per edge (no tuple carries
// representatives between rounds); live edges record their key (L19-21) and
// are appended to one list (global atomicAdd) that pass B reads.
template <int PH, bool SOA>
__device__ __forceinline__ void passA_vc(const Params& P, const DS& D, unsigned long long* cnt, bool guard) {
    const bool filtered = __ldg(&P.st->filtered) != 0;
    const int T = __ldg(&P.st->threshold);
    const bool halving = P.halving != 0;
    const long long stride = (long long)gridDim.x * kBlock;
    for (long long u = (long long)blockIdx.x * kBlock + threadIdx.x; u < P.n; u += stride) {
        const long long s0 = __ldg(P.nindex + u), s1 = __ldg(P.nindex + u + 1);
        int pu = -1;
        for (long long j = s0; j < s1; ++j) {
            const int v = __ldg(P.nlist + j);
            if ((unsigned)v >= (unsigned)P.n || !((int)u < v)) continue;          // L4
            const int w = __ldg(P.eweight + j);
            const bool hv = filtered && w >= T;
            if (PH == 1 ? hv : !hv) continue;                                     // this phase's edges
            if (pu < 0) pu = find_root(D, (int)u, halving);                      // L15
            const int q = find_root(D, v, halving);                              // L16
            if (pu == q) continue;                                               // L17
            const long long key = make_key(w, (unsigned)j);                      // L19
            record_min(D.k(pu), key, guard);                                     // L20
            record_min(D.k(q), key, guard);                                      // L21
            const unsigned long long at = atomicAdd(cnt, 1ull + P.both);
            tst_cg<SOA>(P.wl1, (long long)at, make_int4(pu, q, w, (int)(unsigned)j), P.wlcap);
            if (P.both) tst_cg<SOA>(P.wl1, (long long)at + 1, make_int4(q, pu, w, (int)(unsigned)j), P.wlcap);
        }
    }
}

#ifndef ECL_B_REVERSE
#define ECL_B_REVERSE 1   // C2 2.319 -> 2.281 ms, C3 2.86 -> 2.83 ms, C4 -0.2%, C1 +-0
#endif
// L27-31 (+ L34-37): check, join, mark over the CTA's worklist.
// The MSF weight and edge count go to this warp's shared accumulators once per
// chunk (acc[0] += weights, acc[1] += edges): no 64-bit running sums held in
// registers across the loop (k_rounds is register-capped; they spilled).
// NORESET: a relabel is expected right after this pass, which abandons this
// level's best-edge slots, so the winners leave them as they are (k_rounds
// refills them should the relabel not happen after all).
template <bool NORESET = false, class SRC>
__device__ __forceinline__ void passB(const Params& P, const DS& D, const SRC& S, long long* acc,
                                      int* s_tk = nullptr) {
    const int lane = threadIdx.x & 31;
    for (int kk = first_chunk(s_tk); kk < S.nloc; kk = next_chunk(s_tk, kk)) {
        // (ECL_B_REVERSE: walk the chunks back to front, so pass B starts on the
        // tuples the last pass wrote most recently, still in L2, and the next
        // pass A, walking front to back, starts on the ones pass B read last)
        const int k = ECL_B_REVERSE ? S.nloc - 1 - kk : kk;
        int count;
        const int4* __restrict__ in = S.get(P, k, count);
        int4 t[kItems];
        bool ok[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            const int idx = i * 32 + lane;
            ok[i] = idx < count;
            t[i] = ok[i] ? tld_cg<SRC::SOA>(in, idx, P.wlcap) : make_int4(0, 0, 0, 0);
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
        long long csum = 0;
        int ccnt = 0;
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
                if (!NORESET && wp) __stcg(D.k(p), kInf);              // L35
                if (!NORESET && wq) __stcg(D.k(q), kInf);              // L36
                mark_msf(P, (unsigned)t[i].w);                         // L31
                // (both_directions: the edge's two copies make the same
                // hooks and marks; only the p < q copy counts it)
                if (!P.both || p < q) {
                    csum += t[i].z;
                    ccnt += 1;
                }
            }
        }
        ccnt = warp_sum(ccnt);
        if (ccnt) {
            csum = warp_sum(csum);
            if (lane == 0) {
                acc[0] += csum;
                acc[1] += ccnt;
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
#ifndef ECL_GUARD_SLOTS
#define ECL_GUARD_SLOTS (1 << 24)
#endif
__device__ __forceinline__ bool use_guard(const Params& P, long long live, long long winners, long long slots) {
    if (P.guards >= 0) return P.guards != 0;
    // (huge graphs, n >= 2^25: guard while the open level holds > 2^24 slots
    // (> 128 MB, beyond the L2); measured: C2's 24M-vertex level with guards
    // 1.68 -> 1.93 ms, C5's relabelled 19.7M-slot level without them +0.8 ms)
    return live > 8 * winners || (P.n >= (1 << 25) && slots > ECL_GUARD_SLOTS);
}

// ---------------------------------------------------------------------------
// crowded rounds.  Once a giant set forms (RMAT, uniform graphs), most live
// edges join a handful of huge sets: C5 keeps ~78 M live tuples for six
// rounds that add 77 K, 11 K, ..., 3 MSF edges.  Every such round rereads all
// of them to find one minimum per set.  The paper's own remedy for the whole
// graph -- process the edges below a sampled threshold first, then filter the
// rest by set(u) != set(v) -- applies to the live worklist as
// well: the light part runs to completion, then the deferred part is
// filtered once.  Light edges precede heavy ones in the (w, id) order, so
// the MSF is unchanged (the argument of P:143 for the two phases).
// ---------------------------------------------------------------------------
#ifndef ECL_CROWD_RATIO
#define ECL_CROWD_RATIO 6    // auto: split when live > this x last round's MSF edges (C5: 56.8 -> 54.6 ms vs 16)
#endif
#ifndef ECL_DRAIN_FLAT
#define ECL_DRAIN_FLAT 1
#endif
#ifndef ECL_PREFLAT
#define ECL_PREFLAT 1    // flatten a small open level before pass A when live >= this x its ids (0: never)
#endif
#ifndef ECL_DRAIN_FLAT_MAX
#define ECL_DRAIN_FLAT_MAX (1LL << 22)   // open levels up to this many ids
#endif
#ifndef ECL_SPLIT_C
#define ECL_SPLIT_C 2        // light part: about this many edges per MSF edge of the last round
                             // (4 -> 2: C4 7.18 -> 7.10 ms, C2 2.283 -> 2.262 ms, C5 -0.5%, C3 +-0)
#endif
__device__ __forceinline__ bool crowded(const Params& P, long long live, long long winners, int g) {
    // a split opens a sub-phase of up to round_bound rounds and the phase
    // itself may still need as many: only split while both fit the slots
    if (P.refilter == 0 || __ldcg(&P.in->splits) >= 16 || g + 2 * P.round_bound + 2 >= ECL_MST_MAX_ROUNDS)
        return false;
    if (P.refilter > 0) return live > 4 * winners;
    return live >= (1LL << 20) && live > ECL_CROWD_RATIO * winners;
}

// T' such that about c = ECL_SPLIT_C live edges per set (c x last round's MSF edges,
// P:143's c applied to the contracted graph; 2, the low end of its range) have w < T':
// every CTA samples its own worklist evenly, then every CTA ranks the same
// samples (identical result everywhere).  INT_MAX: no useful split.  All
// threads of all CTAs must call it (one grid barrier).
template <class CSRC>
__device__ __forceinline__ int split_threshold(const Params& P, const CSRC& S, long long live,
                                               long long winners, cg::grid_group& grid, int* s_w) {
    const int tid = threadIdx.x;
    const int ks = max(1, kSplitSamples / P.G);
    const int ctas = min(P.G, kSplitSampleSlots / ks);   // samples from the first CTAs only
    if ((int)blockIdx.x < ctas)
    for (int i = tid; i < ks; i += kBlock) {
        int w = INT_MAX;   // an empty arena votes "heavy"
        if (S.cnt > 0) w = tld_w<CSRC::SOA>(S.base, (long long)(2 * i + 1) * S.cnt / (2 * ks), P.wlcap);
        P.samp[blockIdx.x * ks + i] = w;
    }
    grid.sync();
    const int N = ks * ctas;
    for (int i = tid; i < N; i += kBlock) s_w[i] = __ldcg(&P.samp[i]);
    if (tid == 0) s_w[N] = INT_MAX;
    __syncthreads();
    long long k = (long long)N * ECL_SPLIT_C * winners / max(live, 1LL);
    if (k < 1) k = 1;
    if (k >= N) return INT_MAX;
    for (int i = tid; i < N; i += kBlock) {
        const int wi = s_w[i];
        int less = 0, rank = 0;
        for (int t = 0; t < N; ++t) {
            const int wt = s_w[t];
            less += wt < wi;
            rank += (wt < wi) || (wt == wi && t < i);
        }
        // T' = the sample of rank k, if some sample lies below it (else the
        // light part could be empty: no split)
        if (rank == (int)k) s_w[N + 1] = (less > 0 && wi != INT_MAX) ? wi : INT_MAX;
    }
    __syncthreads();
    const int T = s_w[N + 1];
    __syncthreads();
    return T;
}

// ---------------------------------------------------------------------------
// Contraction (opts.relabel).  After pass B the surviving sets of
// a round are the roots of the open level.  When they are few, they get dense
// ids 0..R'-1 in a new level: each root r of the old level stores ~label(r)
// (the level closes), the new level's parent array starts as the identity,
// and from the next pass A on (which maps the tuples' ids, see passA MAP) the
// rounds' random accesses -- finds, best-edge slots, hooks -- hit arrays of
// R' entries instead of n, which stay in L2 once R' is a few million.  The
// partition, hence every decision of the algorithm, is unchanged: only the
// names of the sets change.
//
// The new level takes the next free id range of parent[] / key[]; its slots
// start as the identity and inf.  Every CTA
// scans a contiguous slice of the old level twice -- count the roots, then
// assign labels in order -- with one grid barrier between the scans and one
// after.  Returns R' (the same in every CTA).
// ---------------------------------------------------------------------------
#ifndef ECL_RELABEL_MIN
#define ECL_RELABEL_MIN (1 << 21)    // auto: only levels of >= 2M ids (>= 24 MB of key + parent) ...
#endif
#ifndef ECL_RELABEL_FIRST
#define ECL_RELABEL_FIRST (1 << 21)  // ... the vertices' level included (measured with the 256-id
                                     // scans: C2 2.261 -> 2.129 ms, C3 2.875 -> 2.810, C4 +-0, C1 +-0;
                                     // the first, one-id-per-lane scans had cost C2 +0.1 ms)
#endif
#ifndef ECL_RELABEL_FLAT
#define ECL_RELABEL_FLAT 1
#endif
constexpr int kRlItems = 8;                     // ids per lane per step of a relabel scan
constexpr int kRlStep = 32 * kRlItems;          // 256 ids per warp step
__device__ __forceinline__ long long relabel(const Params& P, long long base, long long size, long long nbase,
                                             cg::grid_group& grid, int* s_wc, long long (*s_red)[kWarps]) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int G = gridDim.x, b = blockIdx.x;
    // contiguous steps of 256 ids per warp, in (CTA, warp) order; each lane
    // keeps 8 independent loads in flight (ids lane, lane + 32, ...)
    const long long steps = (size + kRlStep - 1) / kRlStep;
    const long long nw = (long long)G * kWarps, gw = (long long)b * kWarps + warp;
    const long long s0 = steps * gw / nw, s1 = steps * (gw + 1) / nw;
    const long long end = base + size;
    int c = 0;
    for (long long st = s0; st < s1; ++st) {
        const long long x0 = base + st * kRlStep + lane;
        int v[kRlItems];
#pragma unroll
        for (int i = 0; i < kRlItems; ++i) v[i] = x0 + 32 * i < end ? __ldcg(P.parent + x0 + 32 * i) : -1;
#pragma unroll
        for (int i = 0; i < kRlItems; ++i) c += v[i] == (int)(x0 + 32 * i);
    }
    c = warp_sum(c);
    if (lane == 0) s_wc[warp] = c;
    __syncthreads();
    if (tid == 0) {
        int t = 0;
        for (int w = 0; w < kWarps; ++w) t += s_wc[w];
        P.lvcnt[b] = t;
    }
    grid.sync();
    long long before = 0, total = 0;
    for (int k = tid; k < G; k += kBlock) {
        const long long v = __ldcg(P.lvcnt + k);
        total += v;
        if (k < b) before += v;
    }
    before = warp_sum(before);
    total = warp_sum(total);
    if (lane == 0) {
        s_red[0][warp] = before;
        s_red[1][warp] = total;
    }
    __syncthreads();
    long long at = nbase, tot = 0;
    for (int w = 0; w < kWarps; ++w) {
        at += s_red[0][w];
        tot += s_red[1][w];
    }
    for (int w = 0; w < warp; ++w) at += s_wc[w];
    const unsigned lt = (1u << lane) - 1u;
    for (long long st = s0; st < s1; ++st) {
        const long long x0 = base + st * kRlStep + lane;
        int v[kRlItems];
#pragma unroll
        for (int i = 0; i < kRlItems; ++i) v[i] = x0 + 32 * i < end ? __ldcg(P.parent + x0 + 32 * i) : -1;
#pragma unroll
        for (int i = 0; i < kRlItems; ++i) {   // labels in id order: item i covers ids x0 + 32 i
            const long long x = x0 + 32 * i;
            const bool root = v[i] == (int)x;
            const unsigned m = __ballot_sync(kFull, root);
            if (root) {
                const int l = (int)(at + __popc(m & lt));
                __stcg(P.parent + x, ~l);
                __stcg(P.parent + l, l);
                __stcg(P.key + l, kInf);
            }
            at += __popc(m);
        }
    }
    grid.sync();
#if ECL_RELABEL_FLAT
    // Flatten the closed level: every non-root id takes its root's label
    // directly (~label, the root's own encoding), so the next pass A's finds
    // from it -- and the flatten before phase 2 -- take one load.  Walks run
    // concurrently; a walker meeting an id already rewritten stops there with
    // the right label.  Four ids per thread in flight.
    const long long gstride = (long long)G * kBlock;
    for (long long x0 = base + (long long)b * kBlock + tid; x0 < end; x0 += 4 * gstride) {
        int px[4];
#pragma unroll
        for (int a = 0; a < 4; ++a) px[a] = x0 + a * gstride < end ? __ldcg(P.parent + x0 + a * gstride) : -1;
#pragma unroll
        for (int a = 0; a < 4; ++a) {
            if (px[a] >= 0) {
                const long long x = x0 + a * gstride;
                const int lab = find_label_from(P.parent, (int)x, px[a], false);
                __stcg(P.parent + x, ~lab);
            }
        }
    }
    grid.sync();
#endif
    return tot;
}

// SOA: opts.tuple_layout 1; DRIVE: opts.drive (compile-time, so the default
// instantiation carries none of the de-optimisations' code or registers)
template <int PH, bool SOA = false, int DRIVE = 0>
__global__ void __launch_bounds__(kBlock, ECL_R_MINB) k_rounds(Params P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ int s_out, s_def;
    __shared__ long long s_red[3][kWarps];
    // region prefix/counts (first round only) and split samples (later rounds) share one buffer
    __shared__ int s_buf[kSplitSampleSlots + 2];
    static_assert(2 * kMaxRegionsPerCta + 1 <= kSplitSampleSlots + 2, "shared buffer");
    int* const s_pre = s_buf;
    int* const s_rcnt = s_buf + kMaxRegionsPerCta + 1;
    int* const s_w = s_buf;
    const int tid = threadIdx.x, lane = tid & 31;
    const bool b0 = blockIdx.x == 0;
    ecl_mst_stats* st = P.st;
    if (!input_ok(P) || (PH == 2 && !phase2_needed(P))) return;
    int g = (PH == 1) ? 0 : __ldcg(&P.in->g_end) + 1;
    if (g >= ECL_MST_MAX_ROUNDS) {
        if (b0 && tid == 0) atomicExch(&st->status, ECL_MST_ERR_ROUNDS);
        return;
    }
    stamp(P, 4 + 2 * g);                      // populate done
    const int b = blockIdx.x;
    int4* wl[2] = {tadd<SOA>(P.wl0, (long long)b * P.cap), tadd<SOA>(P.wl1, (long long)b * P.cap)};
    // opts.drive 1, "Topology-Driven": every pass A reads the phase's
    // whole edge list again (the populate output, never overwritten: pass A
    // always writes buffer 1) instead of the last round's survivors
    constexpr bool topo = DRIVE == 1;
    constexpr bool vc = DRIVE == 2;
    // the populate output of this CTA: regions w = b, b + G, ... (region mode)
    const RegionSrcT<SOA> R = region_src<SOA>(P, b, s_pre, s_rcnt, s_red, &st->live[g], PH == 1);
    if (b0 && tid == 0 && PH == 2) st->phase2_round = g;
    if (P.trace && tid == 0 && PH == 1) {   // diagnostics: this CTA's SM and its first pass's chunks
        unsigned sm;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
        P.trace[b] = sm;
        P.trace[kMaxGrid + b] = R.nloc;
    }
    trace_cta(P, 4 + 2 * g);
    grid.sync();
    __shared__ long long s_acc[kWarps][2];   // per warp: MSF weight, MSF edges (pass B)
    if (lane == 0) s_acc[tid >> 5][0] = s_acc[tid >> 5][1] = 0;
    long long* const acc = s_acc[tid >> 5];
    int cur = 0;
    bool overflow = false;
    long long L = __ldcg(&st->live[g]);
    CompactSrcT<SOA> C = compact_src<SOA>(wl[0], 0);
    // deferred tuples of a crowded-round split: at the back of this CTA's
    // arena in buffer hb (-1: none pending), hcnt of them (per CTA; hb is the
    // same in every CTA because every split decision is)
    int hb = -1, hcnt = 0;
    // the open contraction level (opts.relabel): first id, ids, roots, next
    // level's first id -- identical in every CTA, touched once per round
    // only, so kept in shared memory rather than in (capped) registers
    __shared__ int s_wc[kWarps];
    __shared__ long long s_lv[4];
    __shared__ int s_lev;
    const DS D = ds_of(P);
    // per-pass chunk tickets of this CTA's warps (next_chunk): pass i counts
    // in s_tk[i & 1] and clears the other one, last used a barrier ago
    __shared__ int s_tk[2];
    int tkp = 0;
    auto tk = [&]() -> int* {
        if (!ECL_WARP_CLAIM) return nullptr;
        int* c = &s_tk[tkp & 1];
        if (tid == 0) s_tk[(tkp + 1) & 1] = 0;
        ++tkp;
        return c;
    };
    if (tid == 0) {
        s_tk[0] = 0;
        s_lev = __ldcg(&P.in->nlev);
        s_lv[0] = __ldcg(&P.in->lv_base);
        s_lv[1] = __ldcg(&P.in->lv_size);
        s_lv[2] = __ldcg(&P.in->lv_roots);
        s_lv[3] = __ldcg(&P.in->lv_next);
    }
    __syncthreads();
    // one round: pass B over S, then pass A from S into the other worklist
    // every relabel condition that does not depend on this round's winners
    // (the decision itself follows pass B); see passB NORESET
    auto may_relabel = [&]() {
        const long long lv_size = s_lv[1];
        return P.relabel != 0 && hb < 0 && s_lev + 1 < kMaxLevels && L > 0 &&
               (P.relabel > 0 || (lv_size >= ECL_RELABEL_MIN && 4 * L >= lv_size &&
                                  (s_lev > 0 || lv_size >= ECL_RELABEL_FIRST)));
    };
    auto round = [&](const auto& S) {
        const long long w0 = acc[1];
        const bool noreset = may_relabel();
        // (both_directions: an edge's two copies must see the same slots, so
        // no copy resets them in pass B; the paper's separate reset kernel,
        // L34-37, follows instead)
        int* const tkB = tk();
        if (noreset || P.both) passB<true>(P, D, S, acc, tkB);
        else passB(P, D, S, acc, tkB);
        const long long d = acc[1] - w0;
        if (lane == 0 && d) atomicAdd(reinterpret_cast<unsigned long long*>(&st->winners[g]), (unsigned long long)d);
        if (tid == 0) s_out = s_def = 0;
        trace_cta(P, 5 + 2 * g);
        grid.sync();
        stamp(P, 5 + 2 * g);
        if (g + 1 >= ECL_MST_MAX_ROUNDS) {
            overflow = true;
            return false;
        }
        if (P.both && !noreset) {   // L34-37 as its own pass over the tuples (both_directions)
            for (int k = threadIdx.x >> 5; k < S.nloc; k += kWarps) {
                int count;
                const int4* in = S.get(P, k, count);
                for (int i = lane; i < count; i += 32) {
                    const int4 t = tld_cg<std::decay_t<decltype(S)>::SOA>(in, i, P.wlcap);
                    __stcg(D.k(t.x), kInf);
                    __stcg(D.k(t.y), kInf);
                }
            }
            grid.sync();
        }
        const long long win = __ldcg(&st->winners[g]);
        ++g;
        // every winner hooked exactly one root of the open level
        const long long lv_size = s_lv[1], lv_roots = s_lv[2] - win;
        // contraction: never while deferred tuples (which keep this level's
        // ids) wait for their drain
        // (uniform: every input is the same in every thread of every CTA)
        const bool mapped = noreset && 2 * lv_roots <= lv_size && s_lv[3] + lv_roots <= 2LL * P.n;
        const long long nb = s_lv[3];
        long long tot = 0;
        if (mapped) {
            tot = relabel(P, s_lv[0], lv_size, nb, grid, s_wc, s_red);
        } else if (noreset) {   // the level stays open: restore its slots to inf
            const long long stride = (long long)gridDim.x * kBlock;
            for (long long x = s_lv[0] + (long long)blockIdx.x * kBlock + tid; x < s_lv[0] + lv_size; x += stride)
                __stcg(P.key + x, kInf);
            grid.sync();
        }
        // one barrier, one writer: every thread has read s_lv above
        __syncthreads();
        if (tid == 0) {
            if (mapped) {
                ++s_lev;
                s_lv[0] = nb;
                s_lv[1] = s_lv[2] = tot;
                s_lv[3] = nb + tot;
            } else {
                s_lv[2] = lv_roots;
            }
        }
        __syncthreads();
#if ECL_PREFLAT
        // a small open level found by many more tuples than it has ids, after
        // a round that hooked (chains of hooks make long finds): compress it
        // first, every id in parallel, so that pass A's finds take one hop
        if (!mapped && win > 0 && s_lv[1] <= ECL_DRAIN_FLAT_MAX && L >= ECL_PREFLAT * s_lv[1]) {
            const long long lo = s_lv[0], hi = s_lv[0] + s_lv[1];
            for (long long x = lo + (long long)blockIdx.x * kBlock + tid; x < hi; x += (long long)gridDim.x * kBlock) {
                const int r = find_root(D, (int)x, true);
                if (r != (int)x) __stcg(D.par(x), r);
            }
            grid.sync();
        }
#endif
        const bool guard = use_guard(P, L, win, s_lv[1]);
        // a split defers to the back of the output arena; with tuples already
        // deferred (hb >= 0) only when that is the same buffer, below them --
        // the deferred set is then one run, drained together (any union of
        // deferred parts is heavier than the light part still running)
        int T = INT_MAX;
        if constexpr (is_compact_src<std::decay_t<decltype(S)>>::value) {
            if (!mapped && (hb < 0 || hb == (cur ^ 1)) && crowded(P, L, win, g)) {
                T = split_threshold(P, S, L, win, grid, s_w);
                if (tid == 0) s_def = hb < 0 ? 0 : hcnt;
                __syncthreads();
            }
        }
        unsigned long long* const vcnt = &P.in->vc_cnt[g % 3];
        int* const tkA = tk();
        (void)tkA;
        if constexpr (vc) {
            if (b0 && tid == 0) P.in->vc_cnt[(g + 1) % 3] = 0;   // next round's list counter (read 2 rounds ago)
            passA_vc<PH, SOA>(P, D, vcnt, guard);
        } else if constexpr (topo) {
            passA(P, D, R, wl[1], &s_out, guard, INT_MAX, nullptr, nullptr, tkA);
        } else if (T != INT_MAX)
            passA<true>(P, D, S, wl[cur ^ 1], &s_out, guard, T, tadd<SOA>(wl[cur ^ 1], P.cap), &s_def, tkA);
        else if (mapped) passA<false, true>(P, D, S, wl[cur ^ 1], &s_out, guard, INT_MAX, nullptr, nullptr, tkA);
        else passA(P, D, S, wl[cur ^ 1], &s_out, guard, INT_MAX, nullptr, nullptr, tkA);
        cur = topo ? 1 : cur ^ 1;
        __syncthreads();
        C = compact_src<SOA>(wl[cur], s_out);
        if (T != INT_MAX) {
            hb = cur;
            hcnt = s_def;
            if (b0 && tid == 0) atomicAdd(&P.in->splits, 1);
        }
        if (!vc && tid == 0 && C.cnt) atomicAdd(reinterpret_cast<unsigned long long*>(&st->live[g]), (unsigned long long)C.cnt);
        trace_cta(P, 4 + 2 * g);
        grid.sync();
        stamp(P, 4 + 2 * g);
        if (vc) {
            L = (long long)__ldcg(vcnt);
            if (b0 && tid == 0) st->live[g] = L;
        } else {
            L = __ldcg(&st->live[g]);
        }
        return true;
    };
    // the light part of a split is done: filter the deferred tuples (find,
    // drop set(u) == set(v), record, compact) -- a pass A with no pass B
    // before it, since every key is inf again after the last (empty) round
    auto drain = [&]() {
        if (g + 1 >= ECL_MST_MAX_ROUNDS) {
            overflow = true;
            return false;
        }
        const CompactSrcT<SOA> H = compact_src<SOA>(tadd<SOA>(wl[hb], P.cap - hcnt), hcnt);
        const int ob = hb ^ 1;
        hb = -1;
        hcnt = 0;
        ++g;
        if (tid == 0) s_out = 0;
        __syncthreads();
#if ECL_DRAIN_FLAT
        // the deferred tuples' ends have not been found since the split, while
        // the light part's rounds hooked chains of sets above them: compress
        // the open level first (every id to its root, all ids in parallel),
        // so that the drain's finds take one hop
        if (s_lv[1] <= ECL_DRAIN_FLAT_MAX) {
            const long long lo = s_lv[0], hi = s_lv[0] + s_lv[1];
            for (long long x = lo + (long long)blockIdx.x * kBlock + tid; x < hi; x += (long long)gridDim.x * kBlock) {
                const int r = find_root(D, (int)x, true);
                if (r != (int)x) __stcg(D.par(x), r);
            }
            grid.sync();
        }
#endif
        passA(P, D, H, wl[ob], &s_out, true, INT_MAX, nullptr, nullptr, tk());
        cur = ob;
        __syncthreads();
        C = compact_src<SOA>(wl[cur], s_out);
        if (tid == 0 && C.cnt) atomicAdd(reinterpret_cast<unsigned long long*>(&st->live[g]), (unsigned long long)C.cnt);
        trace_cta(P, 4 + 2 * g);
        grid.sync();
        stamp(P, 4 + 2 * g);
        L = __ldcg(&st->live[g]);
        return true;
    };
    if (L > 0 && round(R)) {
        for (;;) {
            if (L > 0) {
                if constexpr (vc) {
                    if (!round(global_src<SOA>(P.wl1, L))) break;
                } else {
                    if (!round(C)) break;
                }
            } else if (hb >= 0) {
                if (!drain()) break;
            } else {
                break;
            }
        }
    }
    const long long s = acc[0], c = acc[1];
    if (lane == 0) {
        if (s) atomicAdd(reinterpret_cast<unsigned long long*>(&st->total_weight), (unsigned long long)s);
        if (c) atomicAdd(reinterpret_cast<unsigned long long*>(&st->msf_edges), (unsigned long long)c);
    }
    if (b0 && tid == 0) {
        P.in->g_end = g;
        P.in->nlev = s_lev;
        P.in->lv_base = s_lv[0];
        P.in->lv_size = s_lv[1];
        P.in->lv_roots = s_lv[2];
        P.in->lv_next = s_lv[3];
        st->relabels = s_lev;
        st->rounds = g + 1;
        st->refilters = __ldcg(&P.in->splits);
        if (overflow) atomicExch(&st->status, ECL_MST_ERR_ROUNDS);
    }
}

// in_mst from the bit marks (P.mbits): 16 bytes per thread (4 where in_mst is
// not 16-byte aligned), coalesced.  Every byte of in_mst is written here, once
// (Alg. 1's "not in MST" included).
__device__ __forceinline__ unsigned expand4(unsigned b) {   // 4 bits -> 4 bytes 0/1
    return (b & 1u) | ((b & 2u) << 7) | ((b & 4u) << 14) | ((b & 8u) << 21);
}
__global__ void __launch_bounds__(256) k_expand(Params P) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    const long long t0 = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    long long done = 0;   // bytes written by the vector loop
    if ((reinterpret_cast<uintptr_t>(P.in_mst) & 15) == 0) {
        const long long n16 = P.M / 16;
        for (long long i = t0; i < n16; i += stride) {
            const unsigned b = (__ldg(P.mbits + (i >> 1)) >> ((i & 1) * 16)) & 0xFFFFu;
            __stcs(reinterpret_cast<uint4*>(P.in_mst) + i,
                   make_uint4(expand4(b), expand4(b >> 4), expand4(b >> 8), expand4(b >> 12)));
        }
        done = n16 * 16;
    } else {
        const long long n4 = P.M / 4;
        for (long long i = t0; i < n4; i += stride) {
            const unsigned b = (__ldg(P.mbits + (i >> 3)) >> ((i & 7) * 4)) & 0xFu;
            __stcs(reinterpret_cast<unsigned*>(P.in_mst) + i, expand4(b));
        }
        done = n4 * 4;
    }
    if (blockIdx.x == 0 && threadIdx.x < P.M - done) {
        const long long j = done + threadIdx.x;
        P.in_mst[j] = (unsigned char)((P.mbits[j >> 5] >> (j & 31)) & 1u);
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


}  // namespace eclmst
