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
