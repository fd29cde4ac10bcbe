// common.cuh -- constants, workspace layout, kernel parameters and small
// helpers shared by the kernels of the ECL-MST hot path (ecl_mst.cu).
#pragma once

#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <climits>
#include <cstdint>

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
constexpr int kStagePieces = 8;                // host path: CSR pieces uploaded under the populate
constexpr int kSplitSamples = 512;             // crowded-round threshold: about this many samples
constexpr int kSplitSampleSlots = 1024;        // sample slots (max(1, 512 / G) per CTA, first CTAs)
constexpr int kQBins = 2048;                   // exact-quantile radix select: 11 + 11 + 10 bits
#ifndef ECL_POP_DYN
#define ECL_POP_DYN 2                          // populate: dynamic tail in phase 2 (bit 1; phase 1 keeps its
                                               // contiguous slices: C5 populate1 8.45 -> 9.83 ms with it)
#endif
#ifndef ECL_POP_BATCH
#define ECL_POP_BATCH 8                        // chunks per dynamic claim
#endif
#ifndef ECL_POP_STATIC
#define ECL_POP_STATIC 4                       // static share of each warp's chunks, in eighths
#endif
constexpr int kMaxLevels = 24;                 // relabel: contraction levels (level 0 = the vertices)
static_assert(kMaxGrid == ECL_MST_TRACE_CTAS, "trace layout");

struct Internal {
    unsigned long long reps;           // distributed path: sets with a finite key this round
    long long nroots;                  // distributed path: size of the next round's root list
    unsigned int pop_ctr[2];           // populate<PH>: dynamic batches claimed (ECL_POP_DYN)
    int g_cur;                         // first global round of the running phase
    int g_end;                         // last global round of the finished phase
    int giant;                         // root of the largest set after phase 1 (-1: none)
    int splits;                        // crowded-round splits taken so far (all phases)
    unsigned long long tcount;         // populate_mode 1: tuples appended to the one list
    unsigned long long tcanon, theavy; // populate_mode 1: canonical / deferred edges seen
    unsigned long long vc_cnt[3];      // drive 2: tuples of the last pass As (round-robin)
    unsigned q_prefix;                 // exact-quantile threshold: bits of the order key fixed so far
    long long q_rank;                  // ... and the rank still to find below that prefix
    // contraction levels (opts.relabel).  Set ids are absolute indices into
    // parent[] / key[] (2n slots each): level 0 (the vertices) is [0, n), each
    // later level the next free range of [n, 2n) (levels at least halve, so
    // they fit).  Levels below the open one are closed: every root stores
    // ~label, its id in the next level.  Written by k_rounds<1> at exit, read
    // by the flatten and by k_rounds<2>.
    int nlev;                          // closed levels
    long long lv_base;                 // first id of the open level
    long long lv_size;                 // ids in the open level
    long long lv_roots;                // roots in the open level
    long long lv_next;                 // first id of the next level
};

struct Layout {
    size_t stats, internal, trace, rowstart, region, giant, samp, qhist, lvcnt, mbits, key, parent, setid, wl0, wl1, total;
    long long wl_cap;                  // tuples per worklist buffer
};

static inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

static inline long long ceil_div(long long a, long long b) { return (a + b - 1) / b; }

// worklist tuples needed for W populate regions of ceil(nchunks/W)*kChunk
// tuples, for any W <= min(kMaxPopWarps, nchunks)
static inline long long wl_capacity(long long M) {
    const long long nchunks = ceil_div(M, kChunk);
    const long long wmax = nchunks < kMaxPopWarps ? nchunks : kMaxPopWarps;
    return (nchunks + 3 * wmax) * (long long)kChunk;   // (2 wmax: slack of the populate's dynamic tail)
}

// dup: worklist copies per canonical edge (2 for opts.both_directions)
static inline Layout layout_for(int64_t n, int64_t M, int dup = 1) {
    Layout L;
    size_t off = 0;
    const long long nchunks = ceil_div(M, kChunk);
    L.wl_cap = dup * wl_capacity(M);
    L.stats = off;    off = align_up(off + sizeof(ecl_mst_stats), 256);
    L.internal = off; off = align_up(off + sizeof(Internal), 256);
    L.trace = off;    off = align_up(off + sizeof(long long) * kTraceSlots * kMaxGrid, 256);
    L.rowstart = off; off = align_up(off + sizeof(int) * (size_t)(nchunks + 1), 256);
    L.region = off;   off = align_up(off + sizeof(int4) * (size_t)kMaxPopWarps, 256);
    L.giant = off;    off = align_up(off + sizeof(unsigned) * (size_t)((n + 31) / 32 + 1), 256);
    L.samp = off;     off = align_up(off + sizeof(int) * (size_t)kSplitSampleSlots, 256);
    L.qhist = off;    off = align_up(off + sizeof(unsigned long long) * (size_t)kQBins, 256);
    L.lvcnt = off;    off = align_up(off + sizeof(int) * (size_t)kMaxGrid, 256);
    L.mbits = off;    off = align_up(off + sizeof(unsigned) * (size_t)((M + 31) / 32 + 1), 256);
    // key / parent: 2n slots, the vertices plus the contraction levels (Internal)
    L.key = off;      off = align_up(off + sizeof(long long) * (size_t)(2 * n), 256);
    L.parent = off;   off = align_up(off + sizeof(int) * (size_t)(2 * n), 256);
    L.setid = off;    off = align_up(off + sizeof(int) * (size_t)n, 256);
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
    int pop_contig;                   // bit PH-1: populate<PH> walks contiguous slices of rcap/kChunk chunks
    int pop_cta0;                     // first populate CTA of this launch (staged host path: pieces)
    long long pop_span;               // chunks per warp of the contiguous order without a dynamic tail
    int pop_dyn;                      // bit PH-1: populate<PH> ends with dynamically claimed batches
    int pop_s0;                       // ... after this many static chunks per warp
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
    int filter_c;                     // c of P:143 (threshold targets c|V| lightest CSR entries)
    int halving;
    int guards;                       // -1 auto, 0 off, 1 on
    int flatten;
    int refilter;                     // -1 auto, 0 off, 1 forced (opts.refilter)
    int round_bound;                  // ceil(log2 n) + 1: rounds one phase or sub-phase can take
    int* samp;                        // crowded-round weight samples (kSplitSampleSlots)
    unsigned long long* qhist;        // exact-quantile histogram (kQBins)
    int relabel;                      // -1 auto, 0 off, 1 whenever the sets at least halved (opts.relabel)
    int* lvcnt;                       // per-CTA root counts of a relabel (kMaxGrid)
    int* setid;                       // set of every vertex after phase 1 (k_flatten), read by populate 2
    long long wlcap;                  // tuples per worklist buffer (plane stride of opts.tuple_layout 1)
    int both;                         // opts.both_directions: both directed copies of every edge
    int drive;                        // opts.drive: 0 data-driven, 1 topology-driven, 2 vertex-centric
    // edge sharding (distributed path; single GPU: shard 0 of 1)
    int shard;                        // global shard id
    int nshards;                      // total shards
    long long nlocal;                 // chunks of this shard: shard, shard + nshards, ...
    int zero_mst;                     // populate phase 1 zeroes its chunks of in_mst
    unsigned* mbits;                  // MSF marks as bits (k_expand writes in_mst at the end), or null: bytes
    int* acnt;                        // per arena tuple count (distributed pass A)
    int* tgt;                         // per vertex hook target (distributed rep pass)
    long long* const* keys_all;       // virtual shards: every shard's key array
    int nkeys;
    int* hcnt;                        // per arena: deferred tuples of a crowded-round split (distributed path)
    struct DistSplit* dsp;            // the split decision shared by all shards (distributed path)
};

// Crowded-round split on the distributed path (the sharded analogue of
// k_rounds' split, SURVEY §8(e) + reading Q17).  Every decision is a
// function of replicated or allreduced values, so all ranks agree.
struct DistSplit {
    long long cand[8];                // per quantile: min candidate over this rank's virtual shards (partial)
    long long live_sum;               // live tuples over this rank's virtual shards (partial)
    int T;                            // this round's split threshold (INT_MAX: no split)
    int nested;                       // the split appends below tuples already deferred in its output buffer
    int hb;                           // buffer holding deferred tuples (-1: none)
    int pad;
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

// false once a kernel has flagged the input (k_init: nindex out of range or
// not monotone, so rowstart[] may hold garbage; populate: nlist out of range).
// Set only by earlier kernels of the launch sequence, so every CTA of a
// kernel reads the same value and the cooperative kernels exit uniformly.
__device__ __forceinline__ bool input_ok(const Params& P) {
    return *reinterpret_cast<volatile const int*>(&P.st->status) == 0;
}

// phase 2 runs iff filtering is on and phase 1 deferred at least one edge
// (read-only within the kernels that ask: one L1 line per SM, not one L2
// slice hammered by every warp of the grid)
// L31: edge id joins the MSF.  With P.mbits a bit (a fire-and-forget RED.OR
// into M/8 bytes, which the L2 holds far better than a random byte store
// into the M-byte in_mst, a DRAM read-modify-write of a sector on C5);
// k_expand writes in_mst from the bits at the end.
__device__ __forceinline__ void mark_msf(const Params& P, unsigned id) {
    if (P.mbits) atomicOr(P.mbits + (id >> 5), 1u << (id & 31));
    else P.in_mst[id] = 1;
}

__device__ __forceinline__ bool phase2_needed(const Params& P) {
    return __ldg(&P.st->filtered) != 0 && __ldg(&P.st->heavy_edges) != 0 && __ldg(&P.st->status) == 0;
}

}  // namespace eclmst
