// ecl_mst.cu -- B200 (sm_100a) implementation of the ECL-MST hot path behind
// the C ABI in include/ecl_mst.h.
//
// One persistent cooperative kernel per MSF (no host round-trips per round,
// replacing the paper's host while-loop with a cudaMemcpy per iteration,
// P:86-88).  Grid = SMs x resident CTAs; CTA b owns CSR entries
// [b*chunk, (b+1)*chunk) and the same slice of the worklist, which it
// compacts in place round after round.  Stages, separated by grid barriers:
//
//   init      Alg. 1: parent[v] = v, both best-edge buffers = inf;
//             block 0 draws the filter threshold.
//   populate  Alg. 2 L1-11 over the CTA's CSR range (edge-balanced), FUSED
//             with round 0 of L14-21 (all endpoints are roots then, so the
//             find is the identity and nothing is dropped): emit <u,v,w,id>
//             for u < v (L4) meeting the threshold (L6), atomicMin the key
//             into both endpoints.  Phase 2 re-reads the CSR for the
//             heavy edges, replaces endpoints by set(u), set(v), drops
//             intra-set edges (the filter) and records keys the same way.
//   pass B    L27-31: edge whose key won at either endpoint -> join (CAS),
//             mark in_mst[id], add its weight.
//   pass A    L14-23 of the next round: find (implicit path compression,
//             L15-18), drop p == q, keep <p,q,w,id>, guarded atomicMin into
//             the OTHER key buffer; also resets the previous buffer at the
//             tuple's stored endpoints, which are exactly the slots written
//             last round (L34-37 fused away).
//
// Loop: populate ; while (live > 0) { B ; A } per phase.
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <climits>
#include <cstdint>
#include <cstdarg>
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

struct Layout {
    size_t stats, internal, parent, key0, key1, wl, total;
};

static inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

static inline Layout layout_for(int64_t n, int64_t M) {
    Layout L;
    size_t off = 0;
    L.stats = off;    off = align_up(off + sizeof(ecl_mst_stats), 256);
    L.internal = off; off = align_up(off + sizeof(Internal), 256);
    L.key0 = off;     off = align_up(off + sizeof(long long) * (size_t)n, 256);
    L.key1 = off;     off = align_up(off + sizeof(long long) * (size_t)n, 256);
    L.parent = off;   off = align_up(off + sizeof(int) * (size_t)n, 256);
    L.wl = off;       off = align_up(off + sizeof(int4) * (size_t)M, 256);
    L.total = off;
    return L;
}

struct Params {
    int n;
    long long M;
    long long chunk;                  // CSR entries per CTA (multiple of kItems)
    const long long* __restrict__ nindex;
    const int* __restrict__ nlist;
    const int* __restrict__ eweight;
    unsigned char* in_mst;
    long long* total_out;
    ecl_mst_stats* st;
    Internal* in;
    int* parent;
    long long* key0;
    long long* key1;
    int4* wl;
    unsigned long long seed;
    int filter_mode;
    int threshold_mode;
    int threshold_value;
    int halving;
    int vec_ok;
};

// inclusive max-scan of a blocked tile (kItems consecutive values per thread)
__device__ __forceinline__ void block_max_scan(int (&m)[kItems], int* s_warp) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
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
    if (lane == 31) s_warp[warp] = incl;
    __syncthreads();
    int pre = excl;
    for (int w = 0; w < warp; ++w) pre = max(pre, s_warp[w]);
#pragma unroll
    for (int k = 0; k < kItems; ++k) m[k] = max(m[k], pre);
    __syncthreads();
}

// Alg. 2 L1-11 (+ round 0 of L14-21).  PH = 1: light edges; PH = 2: heavy
// edges with set() endpoints and the cycle filter.
template <int PH>
__device__ __forceinline__ int populate(const Params& P, long long j_begin, long long j_end, int r_first,
                                        long long* __restrict__ Kc, bool filtered, int T, int* s_mark,
                                        int* s_cnt, long long& canon_cnt, long long& heavy_cnt, int& err) {
    const int tid = threadIdx.x;
    const bool halving = P.halving != 0;
    int4* seg = P.wl + j_begin;
    int cnt = 0;
    int r_cur = r_first;
    for (long long t0 = j_begin; t0 < j_end; t0 += kTile) {
        const long long t1 = min(t0 + (long long)kTile, j_end);
        const int len = (int)(t1 - t0);
        const bool need_carry = t1 < j_end;

        // --- row of every entry: mark row starts inside the tile, then max-scan
        for (int i = tid; i < kTile; i += kBlock) s_mark[i] = (i == 0) ? r_cur : -1;
        __syncthreads();
        int carry = r_cur;
        for (long long rb = (long long)r_cur + 1;; rb += kBlock) {
            const long long r = rb + tid;
            bool active = false;
            if (r < P.n) {
                const long long s = __ldg(P.nindex + r);
                if (s < t1) {
                    active = true;
                    if (s >= t0) atomicMax(&s_mark[s - t0], (int)r);
                    else err = 1;   // nindex decreasing
                } else if (s == t1 && need_carry) {
                    active = true;
                }
            }
            const int na = __syncthreads_count(active);
            if (na > 0) carry = (int)(rb + na - 1);
            if (na < kBlock) break;
        }

        const int p0 = tid * kItems;
        int vv[kItems], ww[kItems];
        const bool full = p0 + kItems <= len;
        if (P.vec_ok && full) {
            const int4 a = __ldcs(reinterpret_cast<const int4*>(P.nlist + t0 + p0));
            const int4 b = __ldcs(reinterpret_cast<const int4*>(P.eweight + t0 + p0));
            vv[0] = a.x; vv[1] = a.y; vv[2] = a.z; vv[3] = a.w;
            ww[0] = b.x; ww[1] = b.y; ww[2] = b.z; ww[3] = b.w;
        } else {
#pragma unroll
            for (int k = 0; k < kItems; ++k) {
                const bool ok = p0 + k < len;
                vv[k] = ok ? __ldcs(P.nlist + t0 + p0 + k) : -1;
                ww[k] = ok ? __ldcs(P.eweight + t0 + p0 + k) : 0;
            }
        }
        if (PH == 1) {   // every in_mst byte is written once, here (Alg. 1 "not in MST")
            if (P.vec_ok && full) {
                __stcs(reinterpret_cast<unsigned*>(P.in_mst + t0 + p0), 0u);
            } else {
#pragma unroll
                for (int k = 0; k < kItems; ++k)
                    if (p0 + k < len) P.in_mst[t0 + p0 + k] = 0;
            }
        }
        int row[kItems];
#pragma unroll
        for (int k = 0; k < kItems; ++k) row[k] = s_mark[p0 + k];
        block_max_scan(row, s_cnt);

        int4 t[kItems];
        bool keep[kItems];
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            const long long j = t0 + p0 + k;
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
                p = find_root(P.parent, u, halving);              // set(v), set(n)
                q = find_root(P.parent, v, halving);
                kk = p != q;                                      // filtered out otherwise
            }
            if (kk) {
                const long long key = make_key(w, (unsigned)j);   // L19 val <- e_w : e_id
                guarded_min(Kc + p, key);                         // L20
                guarded_min(Kc + q, key);                         // L21
            }
            t[k] = make_int4(p, q, w, (int)(unsigned)j);
            keep[k] = kk;
        }
        cnt += block_compact(t, keep, seg + cnt, s_cnt);         // L7 / L18
        r_cur = carry;
    }
    return cnt;
}

// L14-23 of round g (> 0 within a phase), with L34-37 of round g-1 fused in.
__device__ __forceinline__ int passA(const Params& P, int4* __restrict__ seg, int cnt,
                                     long long* __restrict__ Kc, long long* __restrict__ Kp, int* s_cnt) {
    const bool halving = P.halving != 0;
    int* __restrict__ parent = P.parent;
    int wp = 0;
    for (int base = 0; base < cnt; base += kTile) {
        int4 t[kItems];
        bool keep[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            const int idx = base + i * kBlock + (int)threadIdx.x;
            keep[i] = idx < cnt;
            t[i] = keep[i] ? __ldcg(seg + idx) : make_int4(0, 0, 0, 0);
        }
        int px[kItems], qx[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (keep[i]) {
                px[i] = __ldcg(parent + t[i].x);
                qx[i] = __ldcg(parent + t[i].y);
            }
        }
#pragma unroll
        for (int i = 0; i < kItems; ++i) {   // reset last round's slots (L35-36)
            if (keep[i]) {
                if (__ldcg(Kp + t[i].x) != kInf) __stcg(Kp + t[i].x, kInf);
                if (__ldcg(Kp + t[i].y) != kInf) __stcg(Kp + t[i].y, kInf);
            }
        }
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (keep[i]) {
                const int p = find_from(parent, t[i].x, px[i], halving);   // L15
                const int q = find_from(parent, t[i].y, qx[i], halving);   // L16
                keep[i] = p != q;                                          // L17
                if (keep[i]) {
                    const long long key = make_key(t[i].z, (unsigned)t[i].w);
                    guarded_min(Kc + p, key);
                    guarded_min(Kc + q, key);
                    t[i].x = p;    // L18: implicit path compression
                    t[i].y = q;
                }
            }
        }
        wp += block_compact(t, keep, seg + wp, s_cnt);
    }
    return wp;
}

// L27-31: check, join, mark.
__device__ __forceinline__ void passB(const Params& P, const int4* __restrict__ seg, int cnt,
                                      const long long* __restrict__ Kc, long long& wsum, long long& wcnt) {
    const bool halving = P.halving != 0;
    for (int base = 0; base < cnt; base += kTile) {
        int4 t[kItems];
        bool ok[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            const int idx = base + i * kBlock + (int)threadIdx.x;
            ok[i] = idx < cnt;
            t[i] = ok[i] ? __ldcg(seg + idx) : make_int4(0, 0, 0, 0);
        }
        long long kp[kItems], kq[kItems];
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (ok[i]) {
                kp[i] = __ldcg(Kc + t[i].x);
                kq[i] = __ldcg(Kc + t[i].y);
            }
        }
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            if (ok[i]) {
                const long long key = make_key(t[i].z, (unsigned)t[i].w);
                if (kp[i] == key || kq[i] == key) {               // L29
                    join(P.parent, t[i].x, t[i].y, halving);      // L30
                    P.in_mst[(unsigned)t[i].w] = 1;               // L31
                    wsum += t[i].z;
                    wcnt += 1;
                }
            }
        }
    }
}

__device__ __forceinline__ void stamp(const Params& P, int slot) {
    if (blockIdx.x == 0 && threadIdx.x == 0 && slot < 2 * ECL_MST_MAX_ROUNDS + 4)
        P.st->t_ns[slot] = (long long)globaltimer_ns();
}

__global__ void __launch_bounds__(kBlock, 2) mst_persistent(Params P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ int s_mark[kTile];
    __shared__ int s_cnt[kScanSlots + 1];
    __shared__ int s_row;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const bool b0 = blockIdx.x == 0;
    ecl_mst_stats* st = P.st;
    const long long t_start = (b0 && tid == 0) ? (long long)globaltimer_ns() : 0;
    const long long j_begin = min(P.M, (long long)blockIdx.x * P.chunk);
    const long long j_end = min(P.M, j_begin + P.chunk);
    int err = 0;

    // ---------------- init (Alg. 1) ----------------
    for (long long v = (long long)blockIdx.x * kBlock + tid; v < P.n; v += (long long)gridDim.x * kBlock) {
        P.parent[v] = (int)v;
        P.key0[v] = kInf;
        P.key1[v] = kInf;
    }
    if (warp == 0) {
        const int r = (j_begin < j_end) ? warp_row_of(P.nindex, P.n, j_begin) : 0;
        if (lane == 0) s_row = r;
    }
    if (b0) {
        long long* words = reinterpret_cast<long long*>(st);
        for (int i = tid; i < (int)(sizeof(ecl_mst_stats) / 8); i += kBlock) words[i] = 0;
        __syncthreads();
        if (warp == 1) {
            // filter decision (readings Q5-Q7)
            bool filtered = P.filter_mode < 0 ? (P.M >= 4LL * P.n) : (P.filter_mode != 0);
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
    grid.sync();
    const int r_first = s_row;
    const bool filtered = __ldcg(&st->filtered) != 0;
    const int T = __ldcg(&st->threshold);
    if (b0 && tid == 0) {
        st->t_ns[0] = t_start;
        st->t_ns[1] = (long long)globaltimer_ns();
    }

    long long canon_cnt = 0, heavy_cnt = 0, wsum = 0, wcnt = 0;
    int4* seg = P.wl + j_begin;
    int g = 0, cnt = 0;
    bool overflow = false;
    for (int ph = 1; ph <= 2 && !overflow; ++ph) {
        if (ph == 2) {
            if (!filtered || __ldcg(&st->heavy_edges) == 0) break;
            if (g + 1 >= ECL_MST_MAX_ROUNDS) { overflow = true; break; }
            ++g;
            if (b0 && tid == 0) st->phase2_round = g;
        }
        long long* Kc = (g & 1) ? P.key1 : P.key0;
        if (ph == 1)
            cnt = populate<1>(P, j_begin, j_end, r_first, Kc, filtered, T, s_mark, s_cnt, canon_cnt, heavy_cnt, err);
        else
            cnt = populate<2>(P, j_begin, j_end, r_first, Kc, filtered, T, s_mark, s_cnt, canon_cnt, heavy_cnt, err);
        if (tid == 0 && cnt) atomicAdd(reinterpret_cast<unsigned long long*>(&st->live[g]), (unsigned long long)cnt);
        if (ph == 1) {
            const long long c = warp_sum(canon_cnt), h = warp_sum(heavy_cnt);
            if (lane == 0 && c) atomicAdd(reinterpret_cast<unsigned long long*>(&st->canonical_edges), (unsigned long long)c);
            if (lane == 0 && h) atomicAdd(reinterpret_cast<unsigned long long*>(&st->heavy_edges), (unsigned long long)h);
        }
        grid.sync();
        stamp(P, 4 + 2 * g);
        long long L = __ldcg(&st->live[g]);
        while (L > 0) {
            const long long w0 = wcnt;
            passB(P, seg, cnt, Kc, wsum, wcnt);
            const long long d = warp_sum(wcnt - w0);
            if (lane == 0 && d) atomicAdd(reinterpret_cast<unsigned long long*>(&st->winners[g]), (unsigned long long)d);
            grid.sync();
            stamp(P, 5 + 2 * g);
            if (g + 1 >= ECL_MST_MAX_ROUNDS) { overflow = true; break; }
            ++g;
            long long* Kp = Kc;
            Kc = (g & 1) ? P.key1 : P.key0;
            cnt = passA(P, seg, cnt, Kc, Kp, s_cnt);
            if (tid == 0 && cnt) atomicAdd(reinterpret_cast<unsigned long long*>(&st->live[g]), (unsigned long long)cnt);
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
    o->max_ctas = 0;
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
    long long G = (long long)di.sms * di.occ;
    const long long tiles = (M + kTile - 1) / kTile;
    if (G > tiles) G = tiles;
    if (o.max_ctas > 0 && G > o.max_ctas) G = o.max_ctas;
    if (G > kMaxGrid) G = kMaxGrid;
    if (G < 1) G = 1;
    // per-CTA counts are int: keep a CTA's slice below 2^30 entries
    const long long min_g = (M + (1LL << 30) - 1) >> 30;
    if (G < min_g) G = min_g;
    if (G > (long long)di.sms * di.occ) return fail(ECL_MST_ERR_TOO_LARGE, "graph needs more CTAs than fit");
    long long chunk = (M + G - 1) / G;
    chunk = (chunk + kItems - 1) / kItems * kItems;

    Params P;
    P.n = n;
    P.M = M;
    P.chunk = chunk;
    P.nindex = reinterpret_cast<const long long*>(nindex);
    P.nlist = nlist;
    P.eweight = eweight;
    P.in_mst = in_mst_out;
    P.total_out = reinterpret_cast<long long*>(total_weight_out);
    P.st = reinterpret_cast<ecl_mst_stats*>(ws + L.stats);
    P.in = reinterpret_cast<Internal*>(ws + L.internal);
    P.parent = reinterpret_cast<int*>(ws + L.parent);
    P.key0 = reinterpret_cast<long long*>(ws + L.key0);
    P.key1 = reinterpret_cast<long long*>(ws + L.key1);
    P.wl = reinterpret_cast<int4*>(ws + L.wl);
    P.seed = o.seed;
    P.filter_mode = o.filter < 0 ? -1 : (o.filter ? 1 : 0);
    P.threshold_mode = o.threshold_mode;
    P.threshold_value = o.threshold;
    P.halving = o.path_halving ? 1 : 0;
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
