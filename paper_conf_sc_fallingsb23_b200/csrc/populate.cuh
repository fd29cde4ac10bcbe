// populate.cuh -- k_init (Alg. 1, chunk start rows, threshold sample) and
// k_populate (Alg. 2 L1-11 fused with round 0 of L14-21; phase 2 with the
// cycle filter).
#pragma once

#include <type_traits>

#include "common.cuh"

namespace eclmst {


// ---------------------------------------------------------------------------
// k_init: Alg. 1 + chunk start rows + threshold
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_init(Params P) {
    const int tid = threadIdx.x;
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
        // chunk starts inside row v: rowstart[c] = v for c*kChunk in [s, e).
        // A row outside [0, M] or running backwards is an input error; it
        // writes nothing (every later kernel then exits at once, see
        // input_ok), so invalid offsets never index rowstart[] out of range.
        const long long s = P.nindex[v], e = P.nindex[v + 1];
        if (s < 0 || e < s || e > P.M) {
            err = true;
            continue;
        }
        for (long long c = (s + kChunk - 1) / kChunk; c * kChunk < e && c < P.nchunks; ++c) P.rowstart[c] = (int)v;
    }
    if (P.mbits)   // no edge in the MSF yet (the bit marks of mark_msf)
        for (long long i = i0; i < (P.M + 31) / 32; i += stride) P.mbits[i] = 0u;
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
            long long kpos = ((long long)S * P.filter_c * P.n) / P.M;   // c|V| lightest
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
            P.in->pop_ctr[0] = P.in->pop_ctr[1] = 0;
            P.in->giant = -1;
            P.in->splits = 0;
            P.in->tcount = P.in->tcanon = P.in->theavy = 0;
            P.in->vc_cnt[0] = P.in->vc_cnt[1] = P.in->vc_cnt[2] = 0;
            // exact quantile (threshold_mode 2): the entry of rank c|V| (0-based,
            // at most M - 1) among all M, found by k_qhist / k_qselect below
            long long k = (long long)P.filter_c * P.n;
            P.in->q_rank = k < P.M ? k : P.M - 1;
            P.in->q_prefix = 0;
            P.in->nlev = 0;                   // level 0 open: n sets, all roots
            P.in->lv_base = 0;
            P.in->lv_size = P.n;
            P.in->lv_roots = P.n;
            P.in->lv_next = P.n;
        }
        if (P.threshold_mode == 2)
            for (int i = tid; i < kQBins; i += blockDim.x) P.qhist[i] = 0;
    }
    if (err) atomicExch(&P.st->status, ECL_MST_ERR_INPUT);
}

// ---------------------------------------------------------------------------
// Exact-quantile threshold (threshold_mode 2): the weight
// of rank c|V| among all M CSR entries -- the target P:143's 20 samples
// estimate -- by a radix select over the order key u = w ^ 0x80000000 (signed
// order as unsigned): pass 1 histograms the top 11 bits of every entry, pass
// 2 the next 11 bits of the entries under the chosen 11-bit prefix, pass 3
// the last 10 bits under the chosen 22-bit prefix.  k_qselect<PASS> turns a
// histogram into the next prefix and the rank left below it.
// ---------------------------------------------------------------------------
template <int PASS>
__device__ __forceinline__ void q_bits(int& shift, unsigned& mask) {
    shift = PASS == 1 ? 21 : PASS == 2 ? 10 : 0;
    mask = PASS == 3 ? 0x3FFu : 0x7FFu;
}

template <int PASS>
__global__ void __launch_bounds__(256) k_qhist(Params P) {
    __shared__ unsigned h[kQBins];
    if (!input_ok(P) || __ldg(&P.st->filtered) == 0) return;
    for (int i = threadIdx.x; i < kQBins; i += blockDim.x) h[i] = 0;
    __syncthreads();
    int shift;
    unsigned mask;
    q_bits<PASS>(shift, mask);
    const unsigned prefix = __ldg(&P.in->q_prefix);   // bits above this pass's digit
    auto add = [&](int w) {
        const unsigned u = (unsigned)w ^ 0x80000000u;
        if (PASS == 1 || (u >> (shift + (PASS == 2 ? 11 : 10))) == prefix) atomicAdd(&h[(u >> shift) & mask], 1u);
    };
    const long long nq = P.M / 4;
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nq; i += stride) {
        const int4 w4 = __ldcs(reinterpret_cast<const int4*>(P.eweight) + i);
        add(w4.x);
        add(w4.y);
        add(w4.z);
        add(w4.w);
    }
    for (long long j = nq * 4 + (long long)blockIdx.x * blockDim.x + threadIdx.x; j < P.M; j += stride) add(P.eweight[j]);
    __syncthreads();
    for (int i = threadIdx.x; i < kQBins; i += blockDim.x)
        if (h[i]) atomicAdd(P.qhist + i, (unsigned long long)h[i]);
}

template <int PASS>
__global__ void __launch_bounds__(1024) k_qselect(Params P) {
    __shared__ unsigned long long s_c[kQBins];
    __shared__ int s_bin;
    __shared__ long long s_below;
    if (!input_ok(P) || __ldcg(&P.st->filtered) == 0) return;
    const int tid = threadIdx.x;
    for (int i = tid; i < kQBins; i += blockDim.x) {
        s_c[i] = __ldcg(P.qhist + i);
        P.qhist[i] = 0;                       // ready for the next pass
    }
    __syncthreads();
    if (tid == 0) {   // 2048 bins: a serial scan is a few microseconds
        const long long r = __ldcg(&P.in->q_rank);
        long long cum = 0;
        int b = 0;
        for (; b < kQBins - 1; ++b) {
            if (cum + (long long)s_c[b] > r) break;
            cum += (long long)s_c[b];
        }
        s_bin = b;
        s_below = cum;
    }
    __syncthreads();
    if (tid == 0) {
        const int bits = PASS == 3 ? 10 : 11;
        const unsigned prefix = (__ldcg(&P.in->q_prefix) << bits) | (unsigned)s_bin;
        P.in->q_prefix = prefix;
        P.in->q_rank = __ldcg(&P.in->q_rank) - s_below;
        if (PASS == 3) P.st->threshold = (int)(prefix ^ 0x80000000u);   // phase 1: w < T
    }
}

// ---------------------------------------------------------------------------
// k_populate<PH>: one warp per 128-entry CSR chunk
// ---------------------------------------------------------------------------
template <int PH, bool SOA = false, bool BOTH = false, int DEEP = -1, bool PK2 = false>
#ifndef ECL_DEEP_PH1
#define ECL_DEEP_PH1 0
#endif
#ifndef ECL_DEEP_PH2
#define ECL_DEEP_PH2 1
#endif
#ifndef ECL_GIANT_MIN_N
#define ECL_GIANT_MIN_N (32LL << 20)   // parent[] larger than ~half the L2
#endif
#ifndef ECL_EARLY_VBITS
#define ECL_EARLY_VBITS 1
#endif
#ifndef ECL_P2_GUARD_COLD
#define ECL_P2_GUARD_COLD 0   // phase-2 populate: guard the atomicMin of slots other than the giant's
                              // (off: C4 populate2 2.60 -> 2.40 ms, C5 11.8 -> 11.4 ms)
#endif
#ifndef ECL_PACK1
#define ECL_PACK1 1   // phase 1: per-candidate work on packed candidates (C4 populate1 1.81 -> 1.48 ms)
#endif
#ifndef ECL_PACK2
#define ECL_PACK2 1   // phase 2 packs when few candidates survive per chunk (see pop_kernel)
#endif
#ifndef ECL_POP_MINB
#define ECL_POP_MINB 4
#endif
__global__ void __launch_bounds__(kPopBlock, ECL_POP_MINB) k_populate(Params P) {
    __shared__ int s_mark[kPopWarps][kChunk];
    // packed candidates (PACK)
    __shared__ int4 s_stage[(PH == 1 ? ECL_PACK1 : PK2) ? kPopWarps : 1][(PH == 1 ? ECL_PACK1 : PK2) ? kChunk : 1];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (!input_ok(P)) return;   // k_init rejected nindex: rowstart[] is not valid
    if (PH == 2 && !phase2_needed(P)) return;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        if (PH == 1) P.st->t_ns[1] = (long long)globaltimer_ns();   // init done
        else P.st->t_ns[3] = (long long)globaltimer_ns();           // flatten done
    }
    const bool filtered = __ldg(&P.st->filtered) != 0;
    const int T = __ldg(&P.st->threshold);
    const bool guard = (P.guards > 0) || (P.guards < 0 && PH == 2);
    const DS D = ds_of(P);
    // phase 2: set(x) is setid[x] after k_flatten (else a find from parent[x])
    const int* const sid = P.flatten ? P.setid : P.parent;
    // warp w takes chunks w, w + W, ... (an even sample of the whole CSR, so
    // every region -- and every k_rounds CTA -- gets the same mix even where
    // the density of u < v entries drifts along the rows) and appends its
    // tuples densely to its own region: no atomics, no CTA barrier.
    const int w = (P.pop_cta0 + (int)blockIdx.x) * kPopWarps + warp;
    if (w >= P.W) return;   // (sharded path: partial last CTA)
    int4* const out = tadd<SOA>(P.wl0, (long long)w * P.rcap);
    int cnt = 0, canon_cnt = 0, heavy_cnt = 0, cand_tot = 0;
    // PACK: per-candidate work on candidates packed one per lane (phase 1)
    constexpr bool PACK = PH == 1 ? ECL_PACK1 != 0 : PK2;
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
    // phase 2: the largest set's slot is the one almost every kept edge
    // touches; keep its minimum in a register (one atomicMin per warp at the
    // end) and give the other, cold slots a plain atomicMin
    const int kg = (PH == 2 && P.flatten) ? __ldg(&P.in->giant) : -1;
    long long gbest = kInf;
    // (no largest set: every slot may be hot -- guard them all, as in phase 1's guard rule)
    const bool guard_cold = PH == 2 ? (P.guards > 0 || (P.guards < 0 && (ECL_P2_GUARD_COLD || kg < 0))) : guard;
    auto rec = [&](int x, long long key) {
        if (PH == 2 && x == kg) gbest = min(gbest, key);
        else record_min(D.k(x), key, guard_cold);
    };
    // deep: also prefetch the next chunk's row starts (phase 2, where the
    // bitmap / parent loads already lengthen each chunk's chain)
    // (DEEP >= 0: the host's choice; phase 1 of huge graphs takes it, see pop_kernel)
    constexpr bool deep = DEEP >= 0 ? DEEP != 0 : (PH == 1 ? ECL_DEEP_PH1 : ECL_DEEP_PH2);
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
    // (only entries that can be phase-2 candidates: heavy, and v above the
    // chunk's first row -- an entry with v <= r0 <= its row is a mirror, L4)
    auto vbits = [&](const int (&vv)[kItems], const int (&ww)[kItems], int r0) {
        unsigned b = 0;
        if (PH == 2 && giant >= 0) {
#pragma unroll
            for (int k = 0; k < kItems; ++k)
                if ((unsigned)vv[k] < (unsigned)P.n && vv[k] > r0 && (!filtered || ww[k] >= T))
                    b |= ((__ldg(P.giant_bits + (vv[k] >> 5)) >> (vv[k] & 31)) & 1u) << k;
        }
        return b;
    };
    int nr0 = 0, nrl = 0, n2r0 = 0, n2rl = 0, nv[kItems], nw[kItems];
    long long nsa = LLONG_MAX, nsz = LLONG_MAX;
    unsigned nvb = 0;
    // phase 2 with the largest-set bitmap: lane i holds bitmap word
    // (r0 >> 5) + i of the next chunk's rows, so each entry takes its row's
    // bit by a shuffle instead of a dependent load
    unsigned nrw = 0;
    auto rowwords = [&](int r0, int rl) {
        unsigned x = 0;
        if (PH == 2 && giant >= 0 && (r0 >> 5) + lane <= (rl >> 5)) x = __ldg(P.giant_bits + (r0 >> 5) + lane);
        return x;
    };
    // the warp's chunks: interleaved w, w + W, ... or the contiguous slice
    // [w B, (w + 1) B) with B = P.pop_span (see P.pop_contig).  Phase 2 may
    // end with a dynamic tail (P.pop_dyn): each warp walks only its first
    // P.pop_s0 chunks, then claims batches of ECL_POP_BATCH chunks from
    // P.in->pop_ctr (ecl_mst.cu says why).  (Phase 1 keeps the static order:
    // its contiguous slices beat the balanced dynamic tail.)
    constexpr bool DYNK = PH == 2;
    const bool contig = (P.pop_contig >> (PH - 1)) & 1;
    const long long span = P.pop_span;
    const long long step = contig ? 1 : P.W;
    const long long lend = contig ? min((long long)(w + 1) * span, P.nlocal) : P.nlocal;
    auto nxt = [&](long long lc) { return lc + step; };
    // dynamic sequence (phase 2); chunk ids fit int32 (M < 2^32)
    const bool dyn = DYNK && ((P.pop_dyn >> (PH - 1)) & 1);
    const int nloc = (int)P.nlocal;
    const int ws0 = dyn ? P.pop_s0 * P.W : 0;   // first dynamic chunk
    int cur = 0, end = 0;   // the range being handed out (static: step W when interleaved)
    if (DYNK) {
        if (dyn) {
            cur = contig ? w * P.pop_s0 : w;
            end = contig ? cur + P.pop_s0 : ws0;
        } else {
            cur = contig ? (int)min((long long)w * span, P.nlocal) : w;
            end = (int)lend;
        }
    }
    // the next batch, claimed one batch ahead (lane 0's raw ticket; read only
    // when needed, so the atomic's latency hides behind a batch of chunks)
    unsigned tk_raw = 0;
    bool tk = false;
    const int tup = kChunk * (BOTH ? 2 : 1);   // tuples a chunk may add
    auto claim = [&]() {
        // room for the pipeline (up to 3 chunks), the rest of the current
        // batch and the claimed one
        tk = cnt + (2 * ECL_POP_BATCH + 3) * tup <= P.rcap;
        if (tk && lane == 0) tk_raw = atomicAdd(&P.in->pop_ctr[PH - 1], (unsigned)ECL_POP_BATCH);
    };
    auto take = [&]() -> int {
        if (cur < end) {
            const int r = cur;
            cur += (!contig && (!dyn || r < ws0)) ? P.W : 1;
            return r;
        }
        if (!dyn) return -1;
        if (!tk) claim();
        if (!tk) return -1;
        const int b = ws0 + (int)__shfl_sync(kFull, tk_raw, 0);
        if (b >= nloc) {
            tk = false;
            cur = end = nloc;
            return -1;
        }
        cur = b + 1;
        end = min(b + ECL_POP_BATCH, nloc);
        claim();
        return b;
    };
    // (chunk indices: int in the dynamic phase, where registers are tight)
    using cidx = typename std::conditional<DYNK, int, long long>::type;
    const cidx lc0 = DYNK ? (cidx)take() : (cidx)(contig ? (long long)w * span : w);
    cidx lq2 = -1;   // deep, dynamic: the chunk after the next one
    if (DYNK ? lc0 >= 0 : lc0 < lend) {
        bracket(lc0, nr0, nrl);
        load_entries(P.shard + lc0 * P.nshards, nv, nw);
        if (deep) {
            starts(nr0, nrl, nsa, nsz);
            nrw = rowwords(nr0, nrl);
            if (DYNK) {
                lq2 = take();
                if (lq2 >= 0) bracket(lq2, n2r0, n2rl);
            } else if (nxt(lc0) < lend) {
                bracket(nxt(lc0), n2r0, n2rl);
            }
        }
        nvb = vbits(nv, nw, nr0);
    }
    cidx lc_next = -1;
    for (cidx lc = lc0; DYNK ? lc >= 0 : lc < lend;) {
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
        const unsigned rw = nrw;
        int vv[kItems], ww[kItems];
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            vv[k] = nv[k];
            ww[k] = nw[k];
        }
        const cidx lcn = DYNK ? (deep ? lq2 : (cidx)take()) : (cidx)nxt(lc);
        const bool has_next = DYNK ? lcn >= 0 : lcn < lend;
        if (has_next) {
            load_entries(P.shard + lcn * P.nshards, nv, nw);
            if (deep) {
                nr0 = n2r0;
                nrl = n2rl;
                starts(nr0, nrl, nsa, nsz);
                nrw = rowwords(nr0, nrl);
                if (DYNK) {
                    lq2 = take();
                    if (lq2 >= 0) bracket(lq2, n2r0, n2rl);
                } else if (nxt(lcn) < lend) {
                    bracket(nxt(lcn), n2r0, n2rl);
                }
            } else {
                bracket(lcn, nr0, nrl);
            }
        }
        lc_next = has_next ? lcn : -1;
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
#if ECL_EARLY_VBITS
        // the next chunk's far-end bits, issued half a chunk earlier than at
        // the end of this one (its entries have arrived by now)
        if (PH == 2 && has_next) nvb = vbits(nv, nw, nr0);
#endif
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
                if (!PACK) heavy_cnt += (canon && heavy);   // (packed: |canonical| - |candidates|)
                cand[k] = canon && !heavy;
            } else {
                cand[k] = canon && heavy;
            }
        }
        int idx[kItems];   // packed position of each candidate (-1: none)
        int tot = 0;
        if constexpr (PACK) {
            // The chunk's candidates, packed one per lane through shared
            // memory: the per-candidate work below runs once per 32 of them
            // instead of once per lane item (C5: about 6 candidates per 128
            // entries in phase 1, and in phase 2 after the bitmap test).
            if (PH == 2 && giant >= 0) {   // both ends in the largest set: filtered here
#pragma unroll
                for (int k = 0; k < kItems; ++k) {
                    const int wi = (row[k] >> 5) - (r0 >> 5);
                    const unsigned wd = __shfl_sync(kFull, rw, wi & 31);
                    // (a row beyond the lanes' 32 words -- a chunk spanning
                    // over 1024 rows -- counts as outside: its edge then takes
                    // the setid path, which decides the same)
                    const bool rin = deep && wi < 32 && ((wd >> (row[k] & 31)) & 1u);
                    if (rin && ((vb >> k) & 1u)) cand[k] = false;
                }
            }
            const unsigned lt = (1u << lane) - 1u;
#pragma unroll
            for (int k = 0; k < kItems; ++k) {
                const unsigned m = __ballot_sync(kFull, cand[k]);
                idx[k] = cand[k] ? tot + __popc(m & lt) : -1;
                tot += __popc(m);
            }
            if (PH == 1) cand_tot += tot;
        }
        if constexpr (PACK) {
            const unsigned lt = (1u << lane) - 1u;
            int4* const stage = s_stage[warp];
#pragma unroll
            for (int k = 0; k < kItems; ++k)
                if (idx[k] >= 0) stage[idx[k]] = make_int4(row[k], vv[k], ww[k], p0 + k);
            __syncwarp();
            for (int base = 0; base < tot; base += 32) {
                const bool on = lane < tot - base;
                int4 e = make_int4(0, 0, 0, 0);
                bool kp = false;
                if (on) {
                    e = stage[base + lane];
                    kp = true;
                    if (PH == 2) {   // set(u), set(v): one load each after k_flatten
                        e.x = __ldca(sid + e.x);
                        e.y = __ldca(sid + e.y);
                        if (!P.flatten) {
                            e.x = find_root(D, e.x, P.halving != 0);
                            e.y = find_root(D, e.y, P.halving != 0);
                        }
                        kp = e.x != e.y;                                 // phase 2: the filter
                    }
                }
                const unsigned j = (unsigned)(c0 + e.w);
                const long long key = make_key(e.z, j);                  // L19 val <- e_w : e_id
                if (kp) {
                    rec(e.x, key);                                       // L20-21
                    rec(e.y, key);
                    if (BOTH) {   // opts.both_directions: the mirror copy records it again
                        rec(e.y, key);
                        rec(e.x, key);
                    }
                }
                // L7: append (phase 2: the kept ones, compacted)
                const unsigned km = PH == 2 ? __ballot_sync(kFull, kp) : 0u;
                const int at = PH == 2 ? __popc(km & lt) : lane;
                const int4 tt = make_int4(e.x, e.y, e.z, (int)j);
                if (kp) {
                    if (BOTH) {
                        tst_cg<SOA>(out, cnt + 2LL * at, tt, P.wlcap);
                        tst_cg<SOA>(out, cnt + 2LL * at + 1, make_int4(e.y, e.x, e.z, (int)j), P.wlcap);
                    } else {
                        tst_cg<SOA>(out, cnt + at, tt, P.wlcap);
                    }
                }
                cnt += (PH == 2 ? __popc(km) : min(32, tot - base)) * (BOTH ? 2 : 1);
            }
            __syncwarp();   // (the next chunk's stage)
        } else {
        int pk[kItems], qk[kItems];
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            pk[k] = row[k];
            qk[k] = vv[k];
        }
        if (PH == 2) {   // set(v), set(n): one load each after k_flatten
            unsigned rbit[kItems];   // the rows' bits: from the lanes' prefetched words when deep
#pragma unroll
            for (int k = 0; k < kItems; ++k) {
                const int wi = (row[k] >> 5) - (r0 >> 5);
                const unsigned wd = __shfl_sync(kFull, rw, wi & 31);
                // (a row beyond the lanes' 32 words -- a chunk spanning over
                // 1024 rows -- counts as outside the set: its edges then
                // take the setid path, which decides the same)
                rbit[k] = (deep && wi < 32) ? (wd >> (row[k] & 31)) & 1u : 0u;
            }
#pragma unroll
            for (int k = 0; k < kItems; ++k) {
                if (cand[k] && giant >= 0 && ((vb >> k) & 1u) && rbit[k]) {
                    pk[k] = qk[k] = giant;                    // both ends in the largest set: filtered
                } else if (cand[k]) {
                    pk[k] = (k > 0 && cand[k - 1] && row[k] == row[k - 1]) ? -1 : __ldca(sid + row[k]);
                    qk[k] = __ldca(sid + vv[k]);
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
                if (bp >= 0) rec(bp, best);
                bp = t[k].x;
                best = key;
            } else {
                best = min(best, key);
            }
        }
        if (bp >= 0) rec(bp, best);
#pragma unroll
        for (int k = 0; k < kItems; ++k)
            if (keep[k]) rec(t[k].y, make_key(t[k].z, (unsigned)t[k].w));
        if (BOTH) {   // opts.both_directions: the mirror copy records the same key again
#pragma unroll
            for (int k = 0; k < kItems; ++k) {
                if (keep[k]) {
                    rec(t[k].y, make_key(t[k].z, (unsigned)t[k].w));
                    rec(t[k].x, make_key(t[k].z, (unsigned)t[k].w));
                }
            }
        }
        }   // !PACK
    }
#if !ECL_EARLY_VBITS
    if (PH == 2 && lc_next >= 0) nvb = vbits(nv, nw, nr0);   // next chunk's far-end bits
#endif
    // L7: append the chunk's tuples to the warp's region (both_directions:
    // then their mirror copies <q, p, w, id>)
    if constexpr (!PACK)
    for (int copy = 0; copy < 1 + BOTH; ++copy) {
        unsigned m[kItems];
        int off[kItems];
        int tot = 0;
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
            m[i] = __ballot_sync(kFull, keep[i]);
            off[i] = tot;
            tot += __popc(m[i]);
            if (copy) t[i] = make_int4(t[i].y, t[i].x, t[i].z, t[i].w);
        }
        const unsigned lt = (1u << lane) - 1u;
#pragma unroll
        for (int i = 0; i < kItems; ++i)
            if (keep[i]) tst_cg<SOA>(out, cnt + off[i] + __popc(m[i] & lt), t[i], P.wlcap);
        cnt += tot;
    }
    lc = DYNK ? lc_next : (cidx)nxt(lc);
    }
    if (err) atomicExch(&P.st->status, ECL_MST_ERR_INPUT);
    if (PH == 2 && kg >= 0) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) gbest = min(gbest, __shfl_xor_sync(kFull, gbest, o));
        if (lane == 0 && gbest != kInf) atomicMin(D.k(kg), gbest);
    }
    if (PH == 1) {   // |E| and the deferred count of this warp's chunks
        canon_cnt = warp_sum(canon_cnt);
        heavy_cnt = PACK ? canon_cnt - cand_tot : warp_sum(heavy_cnt);
    }
    if (lane == 0) P.region[w] = make_int4(cnt, canon_cnt, heavy_cnt, 0);
    if (P.trace && lane == 0 && blockIdx.x < kMaxGrid / 2) {   // diagnostics: this CTA's last warp end, its SM
        unsigned sm;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
        atomicMax(reinterpret_cast<unsigned long long*>(P.trace + (PH == 1 ? 2 : 3) * kMaxGrid + blockIdx.x),
                  globaltimer_ns());
        P.trace[(long long)(PH == 1 ? 2 : 3) * kMaxGrid + kMaxGrid / 2 + blockIdx.x] = sm;
    }
}

// ---------------------------------------------------------------------------
// opts.populate_mode 1, "Thread-Based": one thread per vertex walks
// its whole adjacency list -- the loop on Line 3 is never spread over a warp
// -- and appends each tuple to one list with a global atomicAdd (P:154
// "Lines 7 and 18"); k_regions then cuts that list into the populate regions
// k_rounds reads.  Same tuples, keys and counts as k_populate.
// ---------------------------------------------------------------------------
template <int PH, bool SOA = false>
__global__ void __launch_bounds__(256) k_populate_thread(Params P) {
    if (!input_ok(P)) return;
    if (PH == 2 && !phase2_needed(P)) return;
    if (blockIdx.x == 0 && threadIdx.x == 0) P.st->t_ns[PH == 1 ? 1 : 3] = (long long)globaltimer_ns();
    const bool filtered = __ldg(&P.st->filtered) != 0;
    const int T = __ldg(&P.st->threshold);
    const bool guard = (P.guards > 0) || (P.guards < 0 && PH == 2);
    const bool halving = P.halving != 0;
    const DS D = ds_of(P);
    const long long stride = (long long)gridDim.x * blockDim.x;
    long long canon = 0, heavy = 0;
    bool err = false;
    for (long long u = (long long)blockIdx.x * blockDim.x + threadIdx.x; u < P.n; u += stride) {
        const long long s0 = P.nindex[u], s1 = P.nindex[u + 1];
        int pu = -1;
        for (long long j = s0; j < s1; ++j) {                      // L3: this thread, every entry
            const int v = P.nlist[j], w = P.eweight[j];
            if (PH == 1 && P.zero_mst) P.in_mst[j] = 0;
            if ((unsigned)v >= (unsigned)P.n) {
                err = true;
                continue;
            }
            if (!((int)u < v)) continue;                            // L4
            const bool hv = filtered && w >= T;                     // L6
            if (PH == 1) {
                ++canon;
                heavy += hv;
                if (hv) continue;
            } else if (!hv) {
                continue;
            }
            int p = (int)u, q = v;
            if (PH == 2) {   // set(u), set(v)
                if (pu < 0) pu = P.flatten ? __ldca(P.setid + u) : find_root(D, (int)u, halving);
                p = pu;
                q = P.flatten ? __ldca(P.setid + v) : find_root(D, v, halving);
                if (p == q) continue;
            }
            const long long key = make_key(w, (unsigned)j);
            const unsigned long long at = atomicAdd(&P.in->tcount, 1ull + P.both);   // L7
            tst_cg<SOA>(P.wl0, (long long)at, make_int4(p, q, w, (int)(unsigned)j), P.wlcap);
            if (P.both) tst_cg<SOA>(P.wl0, (long long)at + 1, make_int4(q, p, w, (int)(unsigned)j), P.wlcap);
            for (int c = 0; c < 1 + P.both; ++c) {                  // round 0's L20-21
                record_min(D.k(p), key, guard);
                record_min(D.k(q), key, guard);
            }
        }
    }
    if (err) atomicExch(&P.st->status, ECL_MST_ERR_INPUT);
    if (PH == 1) {
        canon = warp_sum(canon);
        heavy = warp_sum(heavy);
        if ((threadIdx.x & 31) == 0) {
            if (canon) atomicAdd(&P.in->tcanon, (unsigned long long)canon);
            if (heavy) atomicAdd(&P.in->theavy, (unsigned long long)heavy);
        }
    }
}

// the one list of k_populate_thread as populate regions: region w holds its
// tuples [w rcap, (w + 1) rcap), and its share of the phase-1 counts.  Resets
// the list counter for the next phase.
template <int PH>
__global__ void __launch_bounds__(256) k_regions(Params P) {
    if (!input_ok(P)) return;
    if (PH == 2 && !phase2_needed(P)) return;
    const long long K = (long long)__ldcg(&P.in->tcount);
    const long long canon = PH == 1 ? (long long)__ldcg(&P.in->tcanon) : 0;
    const long long heavy = PH == 1 ? (long long)__ldcg(&P.in->theavy) : 0;
    for (int w = threadIdx.x; w < P.W; w += blockDim.x) {
        const long long c = min(P.rcap, max(0LL, K - (long long)w * P.rcap));
        // (region counts are int: the host keeps rcap below 2^30, and the
        // phase-1 totals are spread evenly over the regions)
        const long long W = P.W;
        P.region[w] = make_int4((int)c, (int)(canon * (w + 1) / W - canon * w / W),
                                (int)(heavy * (w + 1) / W - heavy * w / W), 0);
    }
    __syncthreads();
    if (threadIdx.x == 0) P.in->tcount = 0;
}

}  // namespace eclmst
