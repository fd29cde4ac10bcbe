// dist_kernels.cuh -- device side of the edge-sharded multi-GPU path.
#pragma once

#include "rounds.cuh"

namespace eclmst {

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

// ---------------------------------------------------------------------------
// Root-compacted exchange.  Only sets that can still hold a live edge need
// their key reduced: round 0 every vertex; afterwards the roots that had a
// finite key and did not hook (the surviving end of each mutual pair) -- a set
// with key inf has no live edge anywhere (a live tuple records its key at both
// ends) and never gets one again.  The list R of those sets is built
// identically on every rank (order-preserving compaction of identical inputs),
// so the allreduce runs over |R| keys instead of n: about 1.4-1.5 n keys over
// all rounds instead of n per round.  R == nullptr: all n.
// ---------------------------------------------------------------------------
__device__ __forceinline__ long long set_of(const int* R, long long i) { return R ? (long long)__ldg(R + i) : i; }

// buf[i] = min over this rank's shards of key[R[i]] (virtual shards: the
// elementwise min NCCL would compute across ranks)
__global__ void __launch_bounds__(256) k_dist_gather(Params P, const int* R, long long nR, long long* buf) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nR; i += stride) {
        const long long x = set_of(R, i);
        long long m = kInf;
        for (int s2 = 0; s2 < P.nkeys; ++s2) m = min(m, P.keys_all[s2][x]);
        buf[i] = m;
    }
}

// after the allreduce: the reduced key back into key[R[i]] of shard 0 (the
// rep passes look up the other end's key by set id)
__global__ void __launch_bounds__(256) k_dist_scatter(Params P, const int* R, long long nR, const long long* buf) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nR; i += stride)
        P.key[set_of(R, i)] = buf[i];
}

// rep pass 1: for every set x = R[i], i in [lo, hi), with a finite (reduced)
// key, the other end's set q of its lightest edge, and whether that edge is
// q's lightest too (mutual).  Ranks split R into slices and allgather tgt[].
__global__ void __launch_bounds__(256) k_dist_reps1(Params P, const int* R, long long lo, long long hi,
                                                    const long long* buf) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    const DS D = ds_of(P);
    // four sets per thread in flight: each is a chain of dependent loads.
    // x holds one end of its edge j = (row(j), nlist[j]); when set(nlist[j])
    // is not x the other end is that set and the row search (about four
    // dependent loads) is skipped -- about half the sets
    for (long long i0 = lo + (long long)blockIdx.x * blockDim.x + threadIdx.x; i0 < hi; i0 += 4 * stride) {
        long long kx[4];
        int pv[4];
#pragma unroll
        for (int a = 0; a < 4; ++a) {
            const long long i = i0 + a * stride;
            kx[a] = i < hi ? buf[i] : kInf;
        }
#pragma unroll
        for (int a = 0; a < 4; ++a) {
            const unsigned j = (unsigned)(kx[a] & 0xffffffffll);
            pv[a] = kx[a] != kInf ? find_root(D, __ldg(P.nlist + j), false) : 0;
        }
#pragma unroll
        for (int a = 0; a < 4; ++a) {
            if (kx[a] == kInf) continue;
            const long long i = i0 + a * stride;
            const long long x = set_of(R, i);
            int q = pv[a];
            if (q == (int)x) q = find_root(D, row_of_entry(P, kx[a] & 0xffffffffll), false);
            const bool mutual = P.key[q] == kx[a];
            P.tgt[i] = q | (mutual ? (int)0x80000000 : 0);
        }
    }
}

// rep pass 2 (L30-31, L34-37): hook, mark, sum, reset -- the same rule as the
// tuple-centric pass B, so the partition after each round is the same.
// keep[i]: x stays a root with a live edge (the next round's R).
__global__ void __launch_bounds__(256) k_dist_reps2(Params P, const int* R, long long nR, const long long* buf,
                                                    unsigned char* keep, int g) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    long long wsum = 0, wcnt = 0;
    unsigned long long found = 0;   // sets with a finite key (0: the phase is done)
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nR; i += stride) {
        const long long kx = buf[i];
        const long long x = set_of(R, i);
        if (kx == kInf) {
            keep[i] = 0;
            continue;
        }
        ++found;
        const int t = P.tgt[i];
        const int q = t & 0x7fffffff;
        const bool mutual = t < 0;
        if (!mutual || (int)x > q) P.parent[x] = q;
        if (!mutual || (int)x < q) {
            P.in_mst[(unsigned)(kx & 0xffffffffll)] = 1;
            wsum += (int)(kx >> 32);
            wcnt += 1;
        }
        keep[i] = mutual && (int)x < q;
        for (int s2 = 0; s2 < P.nkeys; ++s2) P.keys_all[s2][x] = kInf;
    }
    wsum = warp_sum(wsum);
    wcnt = warp_sum(wcnt);
    found = warp_sum(found);
    if ((threadIdx.x & 31) == 0 && found) atomicAdd(reinterpret_cast<unsigned long long*>(&P.in->reps), found);
    if ((threadIdx.x & 31) == 0 && wcnt) {
        atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->total_weight), (unsigned long long)wsum);
        atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->msf_edges), (unsigned long long)wcnt);
        atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->winners[g]), (unsigned long long)wcnt);
    }
}

// keep[x] = x is a root (the sets phase 2 can record keys at)
__global__ void __launch_bounds__(256) k_dist_root_keep(Params P, unsigned char* keep) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long x = (long long)blockIdx.x * blockDim.x + threadIdx.x; x < P.n; x += stride)
        keep[x] = __ldcg(P.parent + x) == (int)x;
}

// order-preserving compaction R_next = [R[i] : keep[i]] over a fixed grid of
// contiguous slices: counts per block, then each block offsets its slice by
// the counts of the blocks before it (every rank computes the same list)
constexpr int kCompactBlock = 256;
constexpr int kCompactGridMax = 1024;
__device__ __forceinline__ void slice_of(long long nR, long long& lo, long long& hi) {
    const long long per = (nR + gridDim.x - 1) / gridDim.x;
    lo = min(nR, (long long)blockIdx.x * per);
    hi = min(nR, lo + per);
}

__global__ void __launch_bounds__(kCompactBlock) k_dist_count(long long nR, const unsigned char* keep, int* bcnt) {
    long long lo, hi;
    slice_of(nR, lo, hi);
    int c = 0;
    for (long long i = lo + threadIdx.x; i < hi; i += kCompactBlock) c += keep[i];
    c = warp_sum(c);
    __shared__ int s_c[kCompactBlock / 32];
    if ((threadIdx.x & 31) == 0) s_c[threadIdx.x >> 5] = c;
    __syncthreads();
    if (threadIdx.x == 0) {
        int t = 0;
        for (int w = 0; w < kCompactBlock / 32; ++w) t += s_c[w];
        bcnt[blockIdx.x] = t;
    }
}

// The last block also publishes {sets with a finite key, |R_next|} to a
// mapped pinned host word pair (host_out, may be null) -- the host loop reads
// them after an event on this kernel while the next pass A already runs --
// and zeroes the set counter for the next round.
__global__ void __launch_bounds__(kCompactBlock) k_dist_compact(const int* R, long long nR, const unsigned char* keep,
                                                                const int* bcnt, int* Rnext, long long* nnext,
                                                                unsigned long long* reps,
                                                                volatile long long* host_out,
                                                                const DistSplit* dsp) {
    __shared__ int s_base, s_w[kCompactBlock / 32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    {   // this block's offset: the counts of the blocks before it (block-wide sum)
        int b = 0;
        for (unsigned k = threadIdx.x; k < blockIdx.x; k += kCompactBlock) b += bcnt[k];
        b = warp_sum(b);
        if (lane == 0) s_w[warp] = b;
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        int b = 0;
        for (int w = 0; w < kCompactBlock / 32; ++w) b += s_w[w];
        s_base = b;
        if (blockIdx.x == gridDim.x - 1) {
            const long long nn = (long long)b + bcnt[blockIdx.x];
            *nnext = nn;
            if (host_out) {
                host_out[0] = (long long)*reps;
                host_out[1] = nn;
                host_out[2] = dsp ? (long long)dsp->hb : -1;
            }
            *reps = 0;
        }
    }
    __syncthreads();
    // each warp takes a contiguous piece of the block's slice: count it, then
    // emit it in order after the pieces of the warps before it
    long long lo, hi;
    slice_of(nR, lo, hi);
    constexpr int kW = kCompactBlock / 32;
    const long long per = (hi - lo + kW - 1) / kW;
    const long long wlo = min(hi, lo + warp * per), whi = min(hi, wlo + per);
    int c = 0;
    for (long long i = wlo + lane; i < whi; i += 32) c += keep[i];
    c = warp_sum(c);
    __shared__ int s_c[kW];
    if (lane == 0) s_c[warp] = c;
    __syncthreads();
    int base = s_base;
    for (int w = 0; w < warp; ++w) base += s_c[w];
    const unsigned lt = (1u << lane) - 1u;
    for (long long i0 = wlo; i0 < whi; i0 += 32) {
        const long long i = i0 + lane;
        const bool k = i < whi && keep[i];
        const unsigned m = __ballot_sync(kFull, k);
        if (k) Rnext[base + __popc(m & lt)] = (int)set_of(R, i);
        base += __popc(m);
    }
}

// Split candidates of shard P (launched once per virtual shard, k = 0..S-1,
// on live list `cur`, before that round's key exchange): from 512 samples
// spread evenly over the shard's arenas (split_threshold's rule), the weight
// of sample rank N / 2^j for j = 1..kSplitQ -- thresholds with about 2^-j of
// the live tuples below them (INT_MAX if none lies below).  The last shard's
// launch writes {-live tuples, candidates} behind the exchanged keys (ext),
// so the key allreduce(min) also yields the largest rank's live count and
// the smallest candidate of each quantile; k_dist_split_decide then picks
// the quantile nearest c x winners / live once the round's winners are known.
constexpr int kSplitQ = 8;
constexpr int kSplitExt = 1 + kSplitQ;   // slots behind the exchanged keys
__global__ void __launch_bounds__(512) k_dist_split_cand(Params P, int k, int S, int cur, long long* ext) {
    constexpr int N = kSplitSamples;
    __shared__ int s_w[N];
    __shared__ long long s_live;
    __shared__ int s_c[kSplitQ];
    const int tid = threadIdx.x;
    DistSplit* d = P.dsp;
    const int4* base = cur ? P.wl1 : P.wl0;
    if (tid == 0) s_live = 0;
    if (tid < kSplitQ) s_c[tid] = INT_MAX;
    __syncthreads();
    {
        long long l = 0;
        for (int b = tid; b < P.G; b += blockDim.x) l += P.acnt[b];
        l = warp_sum(l);
        if ((tid & 31) == 0 && l) atomicAdd(reinterpret_cast<unsigned long long*>(&s_live), (unsigned long long)l);
    }
    __syncthreads();
    const long long live = s_live;
    if (live > 0) {
        for (int i = tid; i < N; i += blockDim.x) {
            const int b = (int)((long long)i * P.G / N);                // arena of sample i
            const int i0 = (int)(((long long)b * N + P.G - 1) / P.G);   // its first sample
            const int i1 = (int)(((long long)(b + 1) * N + P.G - 1) / P.G);
            const int cnt = P.acnt[b], ks = i1 - i0, t = i - i0;
            s_w[i] = cnt > 0 ? __ldcg(&base[(long long)b * P.cap + (long long)(2 * t + 1) * cnt / (2 * ks)].z) : INT_MAX;
        }
        __syncthreads();
        for (int i = tid; i < N; i += blockDim.x) {
            const int wi = s_w[i];
            int less = 0, rank = 0;
            for (int t = 0; t < N; ++t) {
                const int wt = s_w[t];
                less += wt < wi;
                rank += (wt < wi) || (wt == wi && t < i);
            }
            for (int j = 1; j <= kSplitQ; ++j)
                if (rank == (N >> j)) s_c[j - 1] = (less > 0 && wi != INT_MAX) ? wi : INT_MAX;
        }
        __syncthreads();
    }
    if (tid == 0) {
        for (int j = 0; j < kSplitQ; ++j)
            d->cand[j] = k == 0 ? (long long)s_c[j] : min(d->cand[j], (long long)s_c[j]);
        d->live_sum = (k == 0 ? 0 : d->live_sum) + live;
        if (k == S - 1) {
            ext[0] = -d->live_sum;
            for (int j = 0; j < kSplitQ; ++j) ext[1 + j] = d->cand[j];
        }
    }
}

// After the key allreduce and the rep passes of round g: pass A g + 1's
// split threshold, the same on every rank.  The crowded rule is crowded()'s,
// with the global live count estimated as ranks x the largest rank's count;
// the threshold is the candidate quantile 2^-j closest to c x winners / live.
__global__ void k_dist_split_decide(Params P, const long long* ext, int cur, int g, int world) {
    if (threadIdx.x != 0) return;
    DistSplit* d = P.dsp;
    const long long live = -ext[0] * (long long)world;
    const long long win = __ldcg(&P.st->winners[g]);
    const int hb = d->hb;
    int T = INT_MAX;
    if ((hb < 0 || hb == (cur ^ 1)) && crowded(P, live, win, g + 1)) {
        const double f = (double)ECL_SPLIT_C * (double)win / (double)max(live, 1LL);   // target light fraction
        int j = 1;
        while (j < kSplitQ && ldexp(1.0, -(j + 1)) >= f) ++j;                         // 2^-j >= f > 2^-(j+1)
        if (f < 0.5) T = (int)min((long long)INT_MAX, ext[j]);
    }
    d->T = T;
    d->nested = T != INT_MAX && hb >= 0;
    if (T != INT_MAX) {
        d->hb = cur ^ 1;
        P.in->splits += 1;
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
    const int tid = threadIdx.x;
    const int b = blockIdx.x;
    int4* wl[2] = {P.wl0 + (long long)b * P.cap, P.wl1 + (long long)b * P.cap};
    if (tid == 0) s_out = 0;
    if (FIRST && !input_ok(P)) {   // the populate skipped a rejected CSR: no regions to read
        if (tid == 0) P.acnt[b] = 0;
        return;
    }
    if (FIRST) {
        const RegionSrc R = region_src(P, b, s_pre, s_rcnt, s_red, &P.st->live[g - 1], g - 1 == 0);
        passA(P, ds_of(P), R, wl[cur ^ 1], &s_out, P.guards != 0);
    } else {
        // a crowded-round split (decided by k_dist_split_decide): light
        // tuples to the front of the output arena, the rest deferred to its
        // back (below the tuples deferred earlier when nested)
        const int T = P.dsp ? __ldcg(&P.dsp->T) : INT_MAX;
        __shared__ int s_def;
        if (tid == 0) s_def = (T != INT_MAX && __ldcg(&P.dsp->nested)) ? P.hcnt[b] : 0;
        __syncthreads();
        const CompactSrc S = compact_src(wl[cur], P.acnt[b]);
        if (T != INT_MAX) {
            passA<true>(P, ds_of(P), S, wl[cur ^ 1], &s_out, P.guards != 0, T, wl[cur ^ 1] + P.cap, &s_def);
            __syncthreads();
            if (tid == 0) P.hcnt[b] = s_def;
        } else {
            passA(P, ds_of(P), S, wl[cur ^ 1], &s_out, P.guards != 0);
        }
    }
    __syncthreads();
    if (tid == 0) {
        P.acnt[b] = s_out;
        if (s_out) atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->live[g]), (unsigned long long)s_out);
    }
}

// The light part of a split is done everywhere: filter this shard's deferred
// tuples (back of buffer hb) into the front of buffer hb ^ 1 -- a pass A with
// guards, since every key is inf again.
__global__ void __launch_bounds__(kBlock, 2) k_dist_drain(Params P, int g, int hb) {
    __shared__ int s_out;
    const int tid = threadIdx.x;
    const int b = blockIdx.x;
    int4* wl[2] = {P.wl0 + (long long)b * P.cap, P.wl1 + (long long)b * P.cap};
    if (tid == 0) s_out = 0;
    __syncthreads();
    const int h = P.hcnt[b];
    passA(P, ds_of(P), compact_src(wl[hb] + P.cap - h, h), wl[hb ^ 1], &s_out, true);
    __syncthreads();
    if (tid == 0) {
        P.acnt[b] = s_out;
        P.hcnt[b] = 0;
        if (s_out) atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->live[g]), (unsigned long long)s_out);
    }
}

// ===========================================================================
// Device-initiated sharded round loop (opts.dist_loop 1; SURVEY §8(f)
// NEXT-4).  One cooperative kernel runs every round of a phase -- the key
// exchange, the rep passes, the root-list compaction and every shard's pass
// A -- with grid barriers between the stages and no host involvement: the
// termination test ("no set has a finite key") is a grid-wide count that
// every CTA reads.  The exchange is a device-side reduction: each reduced
// key is the min over the key arrays of all shards this GPU can address
// (Params::keys_all; with virtual shards these are local arrays, with peer
// ranks they would be their NVLink-mapped arrays).  Same data flow and same
// decisions as the host loop of ecl_mst_dist_device, so the partition, the
// round count and the MSF are identical.
// ===========================================================================
struct DistLoop {
    const Params* sps;        // device copy of every local shard's Params
    int S;                    // local shards
    int g0;                   // first global round of this phase
    const int* R0;            // first root list (nullptr: all n vertices)
    long long nR0;
    int* rl[2];               // root-list buffers
    long long* buf;           // reduced keys of the current root list
    unsigned char* keep;      // rep pass 2: the set stays in the next list
    int* bcnt;                // per CTA: kept sets of its slice
    unsigned long long* found;   // [2]: sets with a finite key, per round parity
};

// order-preserving compaction of R by keep over the cooperative grid (every
// CTA a contiguous slice); returns the new size (same in every CTA)
__device__ __forceinline__ long long dl_compact(const int* R, long long nR, const unsigned char* keep, int* bcnt,
                                                int* out, cg::grid_group& grid, int* s_w, long long (*s_red)[kWarps]) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const long long lo = nR * blockIdx.x / gridDim.x, hi = nR * (blockIdx.x + 1) / gridDim.x;
    const long long per = (hi - lo + kWarps - 1) / kWarps;
    const long long wlo = min(hi, lo + warp * per), whi = min(hi, wlo + per);
    int c = 0;
    for (long long i = wlo + lane; i < whi; i += 32) c += keep[i];
    c = warp_sum(c);
    if (lane == 0) s_w[warp] = c;
    __syncthreads();
    if (tid == 0) {
        int t = 0;
        for (int w = 0; w < kWarps; ++w) t += s_w[w];
        bcnt[blockIdx.x] = t;
    }
    grid.sync();
    long long before = 0, total = 0;   // (the CTA counts: strided over the threads, then a block sum)
    for (unsigned k = tid; k < gridDim.x; k += kBlock) {
        const long long v = __ldcg(bcnt + k);
        total += v;
        if (k < blockIdx.x) before += v;
    }
    before = warp_sum(before);
    total = warp_sum(total);
    if (lane == 0) {
        s_red[0][warp] = before;
        s_red[1][warp] = total;
    }
    __syncthreads();
    long long base = 0, tot = 0;
    for (int w = 0; w < kWarps; ++w) {
        base += s_red[0][w];
        tot += s_red[1][w];
    }
    for (int w = 0; w < warp; ++w) base += s_w[w];
    const unsigned lt = (1u << lane) - 1u;
    for (long long i0 = wlo; i0 < whi; i0 += 32) {
        const long long i = i0 + lane;
        const bool k = i < whi && keep[i];
        const unsigned m = __ballot_sync(kFull, k);
        if (k) out[base + __popc(m & lt)] = (int)set_of(R, i);
        base += __popc(m);
    }
    grid.sync();
    return tot;
}

template <int PH>
__global__ void __launch_bounds__(kBlock, 2) k_dist_loop(Params P0, DistLoop DL) {
    cg::grid_group grid = cg::this_grid();
    __shared__ int s_out, s_w[kWarps];
    __shared__ long long s_red[3][kWarps];
    __shared__ int s_pre[kMaxRegionsPerCta + 1];
    __shared__ int s_rcnt[kMaxRegionsPerCta];
    const int tid = threadIdx.x, lane = tid & 31;
    const int b = blockIdx.x;
    const bool b0 = b == 0;
    const long long gstride = (long long)gridDim.x * kBlock;
    const long long gtid = (long long)b * kBlock + tid;
    ecl_mst_stats* st = P0.st;
    if (!input_ok(P0) || (PH == 2 && !phase2_needed(P0))) return;
    int g = DL.g0;
    const int* R = DL.R0;
    long long nR = DL.nR0;
    int rb = 0;
    int cur = 0;
    bool first = true;
    // the populate output of every shard: its size (live[g0]) and, in phase
    // 1, the canonical / deferred counts -- even if no round follows
    for (int k = 0; k < DL.S; ++k)
        if (b < DL.sps[k].G) region_src(DL.sps[k], b, s_pre, s_rcnt, s_red, &st->live[g], PH == 1);
    for (;;) {
        // ---- exchange: reduced best-edge key of every set of R ----
        for (long long i = gtid; i < nR; i += gstride) {
            const long long x = set_of(R, i);
            long long m = __ldcg(P0.keys_all[0] + x);
            for (int s2 = 1; s2 < P0.nkeys; ++s2) m = min(m, __ldcg(P0.keys_all[s2] + x));
            DL.buf[i] = m;
        }
        grid.sync();
        if (P0.nkeys > 1) {   // the reduced keys by set id, in shard 0's array (one shard: already there)
            for (long long i = gtid; i < nR; i += gstride) P0.key[set_of(R, i)] = DL.buf[i];
            grid.sync();
        }
        // ---- rep pass 1: the other end of every set's lightest edge, mutual? ----
        // (four sets per thread in flight: each is a chain of dependent loads)
        const DS D = ds_of(P0);
        for (long long i0 = gtid; i0 < nR; i0 += 4 * gstride) {
            long long kx[4];
            int pv[4];
#pragma unroll
            for (int a = 0; a < 4; ++a) {
                const long long i = i0 + a * gstride;
                kx[a] = i < nR ? DL.buf[i] : kInf;
            }
#pragma unroll
            for (int a = 0; a < 4; ++a) {   // (as k_dist_reps1: the row search only when set(v) == x)
                const unsigned j = (unsigned)(kx[a] & 0xffffffffll);
                pv[a] = kx[a] != kInf ? find_root(D, __ldg(P0.nlist + j), false) : 0;
            }
#pragma unroll
            for (int a = 0; a < 4; ++a) {
                if (kx[a] == kInf) continue;
                const long long i = i0 + a * gstride;
                const long long x = set_of(R, i);
                int q = pv[a];
                if (q == (int)x) q = find_root(D, row_of_entry(P0, kx[a] & 0xffffffffll), false);
                P0.tgt[i] = q | (__ldcg(P0.key + q) == kx[a] ? (int)0x80000000 : 0);
            }
        }
        grid.sync();
        // ---- rep pass 2 (L30-31, L34-37): hook, mark, sum, reset ----
        {
            long long wsum = 0, wcnt = 0;
            unsigned long long found = 0;
            for (long long i = gtid; i < nR; i += gstride) {
                const long long kx = DL.buf[i];
                const long long x = set_of(R, i);
                if (kx == kInf) {
                    DL.keep[i] = 0;
                    continue;
                }
                ++found;
                const int t = P0.tgt[i];
                const int q = t & 0x7fffffff;
                const bool mutual = t < 0;
                if (!mutual || (int)x > q) P0.parent[x] = q;
                if (!mutual || (int)x < q) {
                    P0.in_mst[(unsigned)(kx & 0xffffffffll)] = 1;
                    wsum += (int)(kx >> 32);
                    wcnt += 1;
                }
                DL.keep[i] = mutual && (int)x < q;
                for (int s2 = 0; s2 < P0.nkeys; ++s2) P0.keys_all[s2][x] = kInf;
            }
            wsum = warp_sum(wsum);
            wcnt = warp_sum(wcnt);
            found = warp_sum(found);
            if (lane == 0 && found) atomicAdd(&DL.found[g & 1], found);
            if (lane == 0 && wcnt) {
                atomicAdd(reinterpret_cast<unsigned long long*>(&st->total_weight), (unsigned long long)wsum);
                atomicAdd(reinterpret_cast<unsigned long long*>(&st->msf_edges), (unsigned long long)wcnt);
                atomicAdd(reinterpret_cast<unsigned long long*>(&st->winners[g]), (unsigned long long)wcnt);
            }
        }
        grid.sync();
        const unsigned long long nfound = __ldcg(&DL.found[g & 1]);
        if (b0 && tid == 0) DL.found[(g + 1) & 1] = 0;   // next round's counter (its last reader was round g - 1)
        if (nfound == 0) break;                          // no set has a live edge anywhere: the phase is done
        if (g + 1 >= ECL_MST_MAX_ROUNDS) {
            if (b0 && tid == 0) atomicExch(&st->status, ECL_MST_ERR_ROUNDS);
            break;
        }
        // ---- the next root list: the roots that kept a live edge ----
        int* const Rn = DL.rl[rb];
        const long long nRn = dl_compact(R, nR, DL.keep, DL.bcnt, Rn, grid, s_w, s_red);
        // ---- pass A of round g + 1 on every local shard ----
        ++g;
        for (int k = 0; k < DL.S; ++k) {
            const Params& Pk = DL.sps[k];
            if (b >= Pk.G) continue;
            int4* wl[2] = {Pk.wl0 + (long long)b * Pk.cap, Pk.wl1 + (long long)b * Pk.cap};
            if (tid == 0) s_out = 0;
            __syncthreads();
            if (first) {
                const RegionSrc RS = region_src(Pk, b, s_pre, s_rcnt, s_red, nullptr, false);   // (counted above)
                passA(Pk, ds_of(Pk), RS, wl[cur ^ 1], &s_out, Pk.guards != 0);
            } else {
                passA(Pk, ds_of(Pk), compact_src(wl[cur], Pk.acnt[b]), wl[cur ^ 1], &s_out, Pk.guards != 0);
            }
            __syncthreads();
            if (tid == 0) {
                Pk.acnt[b] = s_out;
                if (s_out) atomicAdd(reinterpret_cast<unsigned long long*>(&st->live[g]), (unsigned long long)s_out);
            }
        }
        grid.sync();
        cur ^= 1;
        first = false;
        R = Rn;
        nR = nRn;
        rb ^= 1;
    }
    if (b0 && tid == 0) P0.in->g_end = g;
}

}  // namespace eclmst
