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

// rep pass 1: for every set x = R[i] with a finite (reduced) key, the other
// end's set q of its lightest edge, and whether that edge is q's lightest too
// (mutual)
__global__ void __launch_bounds__(256) k_dist_reps1(Params P, const int* R, long long nR, const long long* buf) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    unsigned long long found = 0;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nR; i += stride) {
        const long long kx = buf[i];
        if (kx == kInf) continue;
        const long long x = set_of(R, i);
        ++found;
        const unsigned j = (unsigned)(kx & 0xffffffffll);
        const int u = row_of_entry(P, (long long)j);
        const int v = __ldg(P.nlist + j);
        const DS D = ds_of(P);
        const int pu = find_root(D, u, false), pv = find_root(D, v, false);
        const int q = (pu == (int)x) ? pv : pu;
        const bool mutual = P.key[q] == kx;
        P.tgt[i] = q | (mutual ? (int)0x80000000 : 0);
    }
    found = warp_sum(found);
    if ((threadIdx.x & 31) == 0 && found) atomicAdd(reinterpret_cast<unsigned long long*>(&P.in->reps), found);
}

// rep pass 2 (L30-31, L34-37): hook, mark, sum, reset -- the same rule as the
// tuple-centric pass B, so the partition after each round is the same.
// keep[i]: x stays a root with a live edge (the next round's R).
__global__ void __launch_bounds__(256) k_dist_reps2(Params P, const int* R, long long nR, const long long* buf,
                                                    unsigned char* keep, int g) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    long long wsum = 0, wcnt = 0;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nR; i += stride) {
        const long long kx = buf[i];
        const long long x = set_of(R, i);
        if (kx == kInf) {
            keep[i] = 0;
            continue;
        }
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
    if ((threadIdx.x & 31) == 0 && wcnt) {
        atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->total_weight), (unsigned long long)wsum);
        atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->msf_edges), (unsigned long long)wcnt);
        atomicAdd(reinterpret_cast<unsigned long long*>(&P.st->winners[g]), (unsigned long long)wcnt);
    }
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
                                                                volatile long long* host_out) {
    __shared__ int s_base, s_w[kCompactBlock / 32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) {
        int b = 0;
        for (unsigned k = 0; k < blockIdx.x; ++k) b += bcnt[k];
        s_base = b;
        if (blockIdx.x == gridDim.x - 1) {
            const long long nn = (long long)b + bcnt[blockIdx.x];
            *nnext = nn;
            if (host_out) {
                host_out[0] = (long long)*reps;
                host_out[1] = nn;
            }
            *reps = 0;
        }
    }
    __syncthreads();
    long long lo, hi;
    slice_of(nR, lo, hi);
    for (long long i0 = lo; i0 < hi; i0 += kCompactBlock) {
        const long long i = i0 + threadIdx.x;
        const bool k = i < hi && keep[i];
        const unsigned m = __ballot_sync(kFull, k);
        if (lane == 0) s_w[warp] = __popc(m);
        __syncthreads();
        int before = 0, tot = 0;
        for (int w = 0; w < kCompactBlock / 32; ++w) {
            before += w < warp ? s_w[w] : 0;
            tot += s_w[w];
        }
        if (k) Rnext[s_base + before + __popc(m & ((1u << lane) - 1u))] = (int)set_of(R, i);
        __syncthreads();
        if (threadIdx.x == 0) s_base += tot;
        __syncthreads();
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

}  // namespace eclmst
