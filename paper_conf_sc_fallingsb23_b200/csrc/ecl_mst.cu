// ecl_mst.cu -- B200 (sm_100a) implementation of the ECL-MST hot path behind
// the C ABI in include/ecl_mst.h.
//
// One persistent cooperative kernel per MSF (no host round-trips per round,
// replacing the paper's host while-loop with a cudaMemcpy per iteration,
// P:86-88).  Grid = SMs x resident CTAs; every warp owns a contiguous
// range of CSR entries, every CTA the union of its warps' ranges and the same
// slice of the two worklists.  Warps work independently (warp-level
// compaction, no CTA barriers inside a pass); stages are separated by grid
// barriers:
//
//   init      Alg. 1: parent[v] = v, key[v] = inf; block 0 draws the
//             filter threshold; each warp finds the row of its
//             first CSR entry.
//   populate  Alg. 2 L1-11 over the warp's CSR range (edge-balanced), FUSED
//             with round 0 of L14-21 (all endpoints are roots then, so the
//             find is the identity and nothing is dropped): emit <u,v,w,id>
//             for u < v (L4) meeting the threshold (L6), atomicMin the key
//             into both endpoints.  Phase 2 re-reads the CSR for the
//             heavy edges, replaces endpoints by set(u), set(v), drops
//             intra-set edges (the filter) and records keys the same way.
//   pass B    L27-31: an edge whose key won at endpoint p hooks p under the
//             other endpoint (Boruvka hooking: each representative is written
//             by exactly one edge, so no CAS is needed; a mutual pair keeps
//             its smaller end as root), marks in_mst[id] and adds its weight.
//             The winning edge of p also resets key[p] (L34-37 fused: an edge
//             that lost at p compares unequal to both the old minimum and to
//             inf, so the early reset cannot change any decision).
//   pass A    L14-23 of the next round: find (implicit path compression,
//             L15-18), drop p == q, keep <p,q,w,id> in the other worklist,
//             atomicMin the key into both representatives.
//   flatten   before phase 2: parent[v] = find(v) for every v.
//
// Loop per phase: populate ; while (live > 0) { B ; A }.
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <climits>
#include <cstdarg>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <string>

#include "device.cuh"
#include "ecl_mst.h"

namespace cg = cooperative_groups;

namespace eclmst {

constexpr int kMaxGrid = 4096;

struct Internal {
    unsigned int done;      // end-of-kernel ticket
    unsigned int pad[63];
};

constexpr int kTraceSlots = 2 * ECL_MST_MAX_ROUNDS + 4;
static_assert(kMaxGrid == ECL_MST_TRACE_CTAS, "trace layout");

struct Layout {
    size_t stats, internal, trace, key, parent, wl0, wl1, total;
};

static inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

static inline Layout layout_for(int64_t n, int64_t M) {
    Layout L;
    size_t off = 0;
    L.stats = off;    off = align_up(off + sizeof(ecl_mst_stats), 256);
    L.internal = off; off = align_up(off + sizeof(Internal), 256);
    L.trace = off;    off = align_up(off + sizeof(long long) * kTraceSlots * kMaxGrid, 256);
    L.key = off;      off = align_up(off + sizeof(long long) * (size_t)n, 256);
    L.parent = off;   off = align_up(off + sizeof(int) * (size_t)n, 256);
    L.wl0 = off;      off = align_up(off + sizeof(int4) * (size_t)M, 256);
    L.wl1 = off;      off = align_up(off + sizeof(int4) * (size_t)M, 256);
    L.total = off;
    return L;
}

struct Params {
    int n;
    long long M;
    long long sub;                    // CSR entries per warp (multiple of kItems)
    const long long* __restrict__ nindex;
    const int* __restrict__ nlist;
    const int* __restrict__ eweight;
    unsigned char* in_mst;
    long long* total_out;
    ecl_mst_stats* st;
    Internal* in;
    long long* trace;                 // [kTraceSlots][kMaxGrid] or null
    long long* key;
    int* parent;
    int4* wl0;
    int4* wl1;
    unsigned long long seed;
    int filter_mode;
    int threshold_mode;
    int threshold_value;
    int halving;
    int guards;
    int flatten;
    int vec_ok;
};

// inclusive max-scan over a warp's chunk (kItems consecutive values per lane)
__device__ __forceinline__ void warp_max_scan(int (&m)[kItems]) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int k = 1; k < kItems; ++k) m[k] = max(m[k], m[k - 1]);
    int incl = m[kItems - 1];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(kFull, incl, o);
        if (lane >= o) incl = max(incl, y);
    }
    int excl = __shfl_up_sync(kFull, incl, 1);
    if (lane == 0) excl = INT_MIN;
#pragma unroll
    for (int k = 0; k < kItems; ++k) m[k] = max(m[k], excl);
}

// Alg. 2 L1-11 (+ round 0 of L14-21) over one warp's CSR range [wb, we).
// PH = 1: light edges; PH = 2: heavy edges with set() endpoints and the
// cycle filter.
template <int PH>
__device__ __forceinline__ void populate(const Params& P, long long wb, long long we, int r_first,
                                         bool filtered, int T, int* s_mark, int4* __restrict__ out, int* s_out,
                                         long long& canon_cnt, long long& heavy_cnt, int& err) {
    const int lane = threadIdx.x & 31;
    const bool halving = P.halving != 0, guard = P.guards != 0;
    long long* __restrict__ K = P.key;
    int r_cur = r_first;
    // software pipeline: the next chunk's CSR entries are in flight while the
    // current chunk searches rows, records keys and emits tuples
    int nv[kItems], nw[kItems];
    auto load_chunk = [&](long long c0, int (&vv)[kItems], int (&ww)[kItems]) {
        const long long c1 = min(c0 + (long long)kChunk, we);
        const int len = (int)(c1 - c0);
        const int p0 = lane * kItems;
        if (P.vec_ok && p0 + kItems <= len) {
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
    if (wb < we) load_chunk(wb, nv, nw);
    for (long long c0 = wb; c0 < we; c0 += kChunk) {
        const long long c1 = min(c0 + (long long)kChunk, we);
        const int len = (int)(c1 - c0);
        const bool need_carry = c1 < we;
        const int p0 = lane * kItems;
        const bool full = p0 + kItems <= len;
        int vv[kItems], ww[kItems];
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            vv[k] = nv[k];
            ww[k] = nw[k];
        }
        if (c1 < we) load_chunk(c1, nv, nw);

        // row of every entry: mark row starts inside the chunk, then max-scan
#pragma unroll
        for (int i = lane; i < kChunk; i += 32) s_mark[i] = (i == 0) ? r_cur : -1;
        __syncwarp();
        int carry = r_cur;
        for (long long rb = (long long)r_cur + 1;; rb += 32) {
            const long long r = rb + lane;
            bool active = false;
            if (r < P.n) {
                const long long s = __ldg(P.nindex + r);
                if (s < c1) {
                    active = true;
                    if (s >= c0) atomicMax(&s_mark[s - c0], (int)r);
                    else err = 1;   // nindex decreasing
                } else if (s == c1 && need_carry) {
                    active = true;
                }
            }
            const int na = __popc(__ballot_sync(kFull, active));
            if (na > 0) carry = (int)(rb + na - 1);
            if (na < 32) break;
        }
        __syncwarp();
        int row[kItems];
#pragma unroll
        for (int k = 0; k < kItems; ++k) row[k] = s_mark[p0 + k];
        __syncwarp();
        warp_max_scan(row);

        if (PH == 1) {   // every in_mst byte is written once, here (Alg. 1 "not in MST")
            if (P.vec_ok && full) {
                __stcs(reinterpret_cast<unsigned*>(P.in_mst + c0 + p0), 0u);
            } else {
#pragma unroll
                for (int k = 0; k < kItems; ++k)
                    if (p0 + k < len) P.in_mst[c0 + p0 + k] = 0;
            }
        }

        int4 t[kItems];
        bool keep[kItems];
        int prev_u = -1, prev_p = -1;
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            const long long j = c0 + p0 + k;
            const bool valid = p0 + k < len;
            const int u = row[k], v = vv[k], w = ww[k];
            const bool in_range = (unsigned)v < (unsigned)P.n;
            if (valid && !in_range) err = 1;
            const bool canon = valid && in_range && u < v;       // L4: one direction only
            int p = u, q = v;
            bool kk = false;
            if (PH == 1) {
                const bool heavy = filtered && w >= T;            // L6 threshold condition
                canon_cnt += canon;
                heavy_cnt += (canon && heavy);
                kk = canon && !heavy;
            } else if (canon && filtered && w >= T) {
                p = (u == prev_u) ? prev_p : find_root(P.parent, u, halving);   // set(v)
                prev_u = u;
                prev_p = p;
                q = find_root(P.parent, v, halving);                            // set(n)
                kk = p != q;                                      // filtered out otherwise
            }
            t[k] = make_int4(p, q, w, (int)(unsigned)j);
            keep[k] = kk;
        }
        // L20: the lane's entries come in row order, so merge equal p first
        long long best = kInf;
        int bp = -1;
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            if (!keep[k]) continue;
            const long long key = make_key(t[k].z, (unsigned)t[k].w);   // L19 val <- e_w : e_id
            if (t[k].x != bp) {
                if (bp >= 0) record_min(K + bp, best, guard);
                bp = t[k].x;
                best = key;
            } else {
                best = min(best, key);
            }
        }
        if (bp >= 0) record_min(K + bp, best, guard);
#pragma unroll
        for (int k = 0; k < kItems; ++k)                          // L21
            if (keep[k]) record_min(K + t[k].y, make_key(t[k].z, (unsigned)t[k].w), guard);
        warp_emit(t, keep, out, s_out);                          // L7
        r_cur = carry;
    }
}

// L14-23 of one round over the CTA's worklist slice: in[0, cnt) -> out.
__device__ __forceinline__ void passA(const Params& P, const int4* __restrict__ in, int cnt,
                                      int4* __restrict__ out, int* s_out) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const bool halving = P.halving != 0, guard = P.guards != 0;
    int* __restrict__ parent = P.parent;
    long long* __restrict__ K = P.key;
    for (int c = warp * kChunk; c < cnt; c += kWarps * kChunk) {
        int4 t[kItems];
        bool keep[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            const int idx = c + i * 32 + lane;
            keep[i] = idx < cnt;
            t[i] = keep[i] ? __ldcs(in + idx) : make_int4(0, 0, 0, 0);
        }
        int px[kItems], qx[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (keep[i]) {
                px[i] = __ldca(parent + t[i].x);
                qx[i] = __ldca(parent + t[i].y);
            }
        }
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (keep[i]) {
                const int p = find_from(parent, t[i].x, px[i], halving);   // L15
                const int q = find_from(parent, t[i].y, qx[i], halving);   // L16
                keep[i] = p != q;                                          // L17
                t[i].x = p;                                                // L18: implicit
                t[i].y = q;                                                //      path compression
            }
        }
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (keep[i]) {
                const long long key = make_key(t[i].z, (unsigned)t[i].w); // L19
                record_min(K + t[i].x, key, guard);                       // L20
                record_min(K + t[i].y, key, guard);                       // L21
            }
        }
        warp_emit(t, keep, out, s_out);                                   // L18
    }
}

// L27-31 (+ L34-37): check, join, mark over the CTA's worklist slice.
__device__ __forceinline__ void passB(const Params& P, const int4* __restrict__ wl, int cnt,
                                      long long& wsum, long long& wcnt) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    int* __restrict__ parent = P.parent;
    long long* __restrict__ K = P.key;
    for (int c = warp * kChunk; c < cnt; c += kWarps * kChunk) {
        int4 t[kItems];
        bool ok[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            const int idx = c + i * 32 + lane;
            ok[i] = idx < cnt;
            t[i] = ok[i] ? __ldcg(wl + idx) : make_int4(0, 0, 0, 0);
        }
        // Only the id half of each slot is compared: ids are unique per
        // edge, so id equality is key equality (and inf's id half, 2^32-1,
        // is never a valid id).  L1 is fine: K[p] only changes when p's own
        // winner resets it.
        const unsigned* __restrict__ Kid = reinterpret_cast<const unsigned*>(K);
        unsigned kp[kItems], kq[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (ok[i]) {
                kp[i] = __ldca(Kid + 2 * (long long)t[i].x);
                kq[i] = __ldca(Kid + 2 * (long long)t[i].y);
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
                if (wp && !(wq && p < q)) __stcg(parent + p, q);
                if (wq && !(wp && q < p)) __stcg(parent + q, p);
                if (wp) __stcg(K + p, kInf);                           // L35
                if (wq) __stcg(K + q, kInf);                           // L36
                P.in_mst[(unsigned)t[i].w] = 1;                        // L31
                wsum += t[i].z;
                wcnt += 1;
            }
        }
    }
}

// per-CTA end of a stage (diagnostics; P.trace is null unless opts.trace)
__device__ __forceinline__ void trace_cta(const Params& P, int slot) {
    if (P.trace && slot < kTraceSlots) {
        __syncthreads();
        if (threadIdx.x == 0) P.trace[(long long)slot * kMaxGrid + blockIdx.x] = (long long)globaltimer_ns();
    }
}

__device__ __forceinline__ void stamp(const Params& P, int slot) {
    if (blockIdx.x == 0 && threadIdx.x == 0 && slot < 2 * ECL_MST_MAX_ROUNDS + 4)
        P.st->t_ns[slot] = (long long)globaltimer_ns();
}

__global__ void __launch_bounds__(kBlock, 2) mst_persistent(Params P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ int s_mark[kWarps][kChunk];
    __shared__ int s_out;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const bool b0 = blockIdx.x == 0;
    ecl_mst_stats* st = P.st;
    const long long t_start = (b0 && tid == 0) ? (long long)globaltimer_ns() : 0;
    const long long cta_begin = min(P.M, (long long)blockIdx.x * kWarps * P.sub);
    const long long wb = min(P.M, cta_begin + warp * P.sub);
    const long long we = min(P.M, wb + P.sub);
    int err = 0;

    // ---------------- init (Alg. 1) ----------------
    for (long long v = (long long)blockIdx.x * kBlock + tid; v < P.n; v += (long long)gridDim.x * kBlock) {
        P.parent[v] = (int)v;
        P.key[v] = kInf;
    }
    const int r_first = (wb < we) ? warp_row_of(P.nindex, P.n, wb) : 0;
    if (b0) {
        long long* words = reinterpret_cast<long long*>(st);
        for (int i = tid; i < (int)(sizeof(ecl_mst_stats) / 8); i += kBlock) words[i] = 0;
        __syncthreads();
        if (warp == 1) {
            // filter decision (readings Q5-Q7)
            const bool filtered = P.filter_mode < 0 ? (P.M >= 4LL * P.n) : (P.filter_mode != 0);
            int T = INT_MAX;
            if (filtered) {
                if (P.threshold_mode == 1) {
                    T = P.threshold_value;
                } else {
                    int w = INT_MAX;
                    if (lane < 20) {
                        const unsigned long long h = splitmix64(P.seed * 0x100000001B3ull + (unsigned long long)lane);
                        w = __ldg(P.eweight + (long long)(h % (unsigned long long)P.M));
                    }
                    int rank = 0;
                    for (int s = 0; s < 20; ++s) {
                        const int ws = __shfl_sync(kFull, w, s);
                        if (lane < 20 && (ws < w || (ws == w && s < lane))) ++rank;
                    }
                    long long kpos = (80LL * P.n) / P.M;   // c|V| lightest of M entries: 20 * 4n / M
                    if (kpos > 19) kpos = 19;
                    const unsigned b = __ballot_sync(kFull, lane < 20 && rank == (int)kpos);
                    T = __shfl_sync(kFull, w, __ffs(b) - 1);
                }
            }
            if (lane == 0) {
                st->filtered = filtered ? 1 : 0;
                st->threshold = T;
                st->grid = gridDim.x;
                st->block = kBlock;
                st->phase2_round = -1;
                if (P.nindex[0] != 0 || P.nindex[P.n] != P.M) err = 1;
            }
        }
        if (tid == 0) P.in->done = 0u;
    }
    trace_cta(P, 1);
    grid.sync();
    const bool filtered = __ldcg(&st->filtered) != 0;
    const int T = __ldcg(&st->threshold);
    if (b0 && tid == 0) {
        st->t_ns[0] = t_start;
        st->t_ns[1] = (long long)globaltimer_ns();
    }

    long long canon_cnt = 0, heavy_cnt = 0, wsum = 0, wcnt = 0;
    int4* wl[2] = {P.wl0 + cta_begin, P.wl1 + cta_begin};
    int cur = 0, g = 0, cnt = 0;
    bool overflow = false;
    for (int ph = 1; ph <= 2 && !overflow; ++ph) {
        if (ph == 2) {
            if (!filtered || __ldcg(&st->heavy_edges) == 0) break;
            if (g + 1 >= ECL_MST_MAX_ROUNDS) { overflow = true; break; }
            if (P.flatten) {   // compress every path once: phase-2 finds become one hop
                for (long long v = (long long)blockIdx.x * kBlock + tid; v < P.n; v += (long long)gridDim.x * kBlock) {
                    const int r = find_root(P.parent, (int)v, true);
                    if (r != (int)v) P.parent[v] = r;
                }
                trace_cta(P, 3);
                grid.sync();
                stamp(P, 3);
            }
            ++g;
            if (b0 && tid == 0) st->phase2_round = g;
        }
        if (tid == 0) s_out = 0;
        __syncthreads();
        if (ph == 1)
            populate<1>(P, wb, we, r_first, filtered, T, s_mark[warp], wl[cur], &s_out, canon_cnt, heavy_cnt, err);
        else
            populate<2>(P, wb, we, r_first, filtered, T, s_mark[warp], wl[cur], &s_out, canon_cnt, heavy_cnt, err);
        __syncthreads();
        cnt = s_out;
        if (tid == 0 && cnt) atomicAdd(reinterpret_cast<unsigned long long*>(&st->live[g]), (unsigned long long)cnt);
        if (ph == 1) {
            const long long c = warp_sum(canon_cnt), h = warp_sum(heavy_cnt);
            if (lane == 0 && c) atomicAdd(reinterpret_cast<unsigned long long*>(&st->canonical_edges), (unsigned long long)c);
            if (lane == 0 && h) atomicAdd(reinterpret_cast<unsigned long long*>(&st->heavy_edges), (unsigned long long)h);
        }
        trace_cta(P, 4 + 2 * g);
        grid.sync();
        stamp(P, 4 + 2 * g);
        long long L = __ldcg(&st->live[g]);
        while (L > 0) {
            const long long w0 = wcnt;
            passB(P, wl[cur], cnt, wsum, wcnt);
            const long long d = warp_sum(wcnt - w0);
            if (lane == 0 && d) atomicAdd(reinterpret_cast<unsigned long long*>(&st->winners[g]), (unsigned long long)d);
            if (tid == 0) s_out = 0;
            trace_cta(P, 5 + 2 * g);
            grid.sync();
            stamp(P, 5 + 2 * g);
            if (g + 1 >= ECL_MST_MAX_ROUNDS) { overflow = true; break; }
            ++g;
            passA(P, wl[cur], cnt, wl[cur ^ 1], &s_out);
            cur ^= 1;
            __syncthreads();
            cnt = s_out;
            if (tid == 0 && cnt) atomicAdd(reinterpret_cast<unsigned long long*>(&st->live[g]), (unsigned long long)cnt);
            trace_cta(P, 4 + 2 * g);
            grid.sync();
            stamp(P, 4 + 2 * g);
            L = __ldcg(&st->live[g]);
        }
    }
    if (overflow) err = 1;

    // ---------------- finalise ----------------
    const long long s = warp_sum(wsum), c = warp_sum(wcnt);
    if (lane == 0) {
        if (s) atomicAdd(reinterpret_cast<unsigned long long*>(&st->total_weight), (unsigned long long)s);
        if (c) atomicAdd(reinterpret_cast<unsigned long long*>(&st->msf_edges), (unsigned long long)c);
    }
    if (err) atomicExch(&st->status, ECL_MST_ERR_INPUT);
    __threadfence();
    __syncthreads();
    if (tid == 0) {
        if (b0) {
            st->rounds = g + 1;
            st->t_ns[2] = (long long)globaltimer_ns();
        }
        const unsigned ticket = atomicAdd(&P.in->done, 1u);
        if (ticket == gridDim.x - 1) {
            __threadfence();
            const long long tot = *reinterpret_cast<volatile long long*>(&st->total_weight);
            const int status = *reinterpret_cast<volatile int*>(&st->status);
            *P.total_out = status ? LLONG_MIN : tot;
        }
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
    int occ = 0;
};

static std::mutex g_dev_mu;
static DevInfo g_dev[64];

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
        if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, mst_persistent, kBlock, 0);
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
    o->atomic_guards = 1;
    o->flatten = 1;
    o->max_ctas = 0;
    o->trace = 0;
    o->seed = 0x5eedull;
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
    const long long max_g = (long long)di.sms * di.occ;
    long long G = max_g;
    const long long chunks = (M + kChunk - 1) / kChunk;
    if (G * kWarps > chunks) G = (chunks + kWarps - 1) / kWarps;   // small graphs: fewer CTAs
    if (o.max_ctas > 0 && G > o.max_ctas) G = o.max_ctas;
    if (G > kMaxGrid) G = kMaxGrid;
    if (G < 1) G = 1;
    long long sub = (M + G * kWarps - 1) / (G * kWarps);
    sub = (sub + kItems - 1) / kItems * kItems;
    // per-CTA worklist counts are int: keep a CTA's slice below 2^30 entries
    while (sub * kWarps >= (1LL << 30)) {
        if (G >= max_g) return fail(ECL_MST_ERR_TOO_LARGE, "graph needs more CTAs than fit");
        ++G;
        sub = (M + G * kWarps - 1) / (G * kWarps);
        sub = (sub + kItems - 1) / kItems * kItems;
    }

    Params P;
    P.n = n;
    P.M = M;
    P.sub = sub;
    P.nindex = reinterpret_cast<const long long*>(nindex);
    P.nlist = nlist;
    P.eweight = eweight;
    P.in_mst = in_mst_out;
    P.total_out = reinterpret_cast<long long*>(total_weight_out);
    P.st = reinterpret_cast<ecl_mst_stats*>(ws + L.stats);
    P.in = reinterpret_cast<Internal*>(ws + L.internal);
    P.trace = o.trace ? reinterpret_cast<long long*>(ws + L.trace) : nullptr;
    P.key = reinterpret_cast<long long*>(ws + L.key);
    P.parent = reinterpret_cast<int*>(ws + L.parent);
    P.wl0 = reinterpret_cast<int4*>(ws + L.wl0);
    P.wl1 = reinterpret_cast<int4*>(ws + L.wl1);
    P.seed = o.seed;
    P.filter_mode = o.filter < 0 ? -1 : (o.filter ? 1 : 0);
    P.threshold_mode = o.threshold_mode;
    P.threshold_value = o.threshold;
    P.halving = o.path_halving ? 1 : 0;
    P.guards = o.atomic_guards ? 1 : 0;
    P.flatten = o.flatten ? 1 : 0;
    P.vec_ok = (reinterpret_cast<uintptr_t>(nlist) % 16 == 0) && (reinterpret_cast<uintptr_t>(eweight) % 16 == 0) &&
               (reinterpret_cast<uintptr_t>(in_mst_out) % 4 == 0);
    void* args[] = {&P};
    cudaError_t e = cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(mst_persistent), dim3((unsigned)G),
                                                dim3(kBlock), args, 0, s);
    if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "cooperative launch (grid %lld): %s", G, cudaGetErrorString(e));
    return ECL_MST_OK;
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
