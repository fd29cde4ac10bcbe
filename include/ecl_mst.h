/*
 * ecl_mst.h -- C ABI of the B200-native ECL-MST hot path (libeclmst.so).
 *
 * Operation (§3; Alg. 2): the minimum spanning
 * forest (MSF, P:51, P:63 fn 1) of an undirected graph with 32-bit integer
 * edge weights given in CSR form with both directions of every edge (P:146,
 * P:329 fn 2), computed by the edge-centric Kruskal/Boruvka hybrid:
 * populate a worklist of edges (Alg. 2 L1-11) -> rounds of {find with implicit
 * path compression, compaction (L17-18), 64-bit
 * atomicMin of (weight:edge-id) into each representative,
 * check/join/mark (L27-31)} until the worklist is empty, with a single
 * weight-threshold filtering step.
 *
 * Edge set and ids (readings Q1/Q11): the graph's edges are exactly
 * the CSR entries j of row u with u < nlist[j] (Alg. 2 L4, "only process in
 * one direction"); the edge ID of such an edge is j.  Mirror entries and
 * self-loops are never edges; parallel entries are distinct edges.  Edges are
 * ordered by (weight as signed int32, id); under that strict order the MSF is
 * unique, and the library returns exactly it, deterministically.
 *
 * Common argument conventions
 *   n        number of vertices, 0 <= n <= 2^31 - 1.
 *   M        number of CSR entries = nindex[n], 0 <= M <= 2^32 - 1.
 *   nindex   int64[n+1], nindex[0] = 0, non-decreasing, nindex[n] = M.
 *   nlist    int32[M], 0 <= nlist[j] < n: the neighbour of entry j.
 *   eweight  int32[M]: the weight of entry j (any int32 value).
 *            (device call: nlist and eweight 16-byte aligned, in_mst 4-byte
 *            aligned -- any cudaMalloc/torch allocation is)
 *   in_mst   uint8[M] OUTPUT: 1 iff entry j is the id of an MSF edge, else 0
 *            (mirror slots are always 0).  Every byte is written.
 * Ownership: the caller owns every buffer; inputs are only read.  The library
 * keeps no state between calls except a per-thread last-error string and, for
 * the host convenience call, a cached device buffer pool (freed by
 * ecl_mst_release_host_cache).  Calls on distinct workspaces/streams are
 * independent.
 */
#ifndef ECL_MST_H
#define ECL_MST_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ECL_MST_ABI_VERSION 3

/* status codes */
#define ECL_MST_OK 0
#define ECL_MST_ERR_INVALID (-1)   /* bad argument (null pointer with M > 0, n < 0, ...) */
#define ECL_MST_ERR_TOO_LARGE (-2) /* n or M beyond the limits above */
#define ECL_MST_ERR_CUDA (-3)      /* a CUDA call failed; see ecl_mst_last_error() */
#define ECL_MST_ERR_WORKSPACE (-4) /* workspace too small or misaligned */
#define ECL_MST_ERR_INPUT (-5)     /* the device found an inconsistent CSR (stats.status) */
#define ECL_MST_ERR_ROUNDS (-6)    /* the device ran out of its ECL_MST_MAX_ROUNDS round slots
                                      (stats.status; cannot happen within the documented limits) */

#define ECL_MST_MAX_ROUNDS 128     /* global round slots (<= ceil(log2 n)+1 per phase and sub-phase) */

/* knobs; every setting returns the identical MSF (tests check this) */
typedef struct ecl_mst_options {
    int32_t filter;          /* -1 auto: filter iff M >= 4n (reading Q6); 0 off; 1 on */
    int32_t threshold_mode;  /* 0 sampled: the weight of sample rank S*c*n/M among S random entries
                                (readings Q5/Q7; S = threshold_samples); 1 fixed
                                (opts.threshold); 2 exact quantile: the weight of rank c*n among
                                all M entries, by a two-pass device radix select (SURVEY §8(f)
                                NEXT-3) */
    int32_t threshold;       /* phase 1 takes w < threshold when threshold_mode == 1 */
    int32_t path_halving;    /* 1 (default) find() halves paths it walks (P:142 reading Q15); 0 off */
    int32_t atomic_guards;   /* load-compare before each atomicMin: 1 everywhere; 0 never;
                                -1 (default) everywhere except the phase-1 populate, where the
                                slots are still mostly inf and the guard only adds latency */
    int32_t flatten;         /* 1 (default) compress every path once before the phase-2 populate; 0 off */
    int32_t max_ctas;        /* 0 = fill the GPU (SMs x resident CTAs); else cap the grid */
    int32_t trace;           /* bit 0: record every CTA's end time of every stage (ecl_mst_read_trace);
                                bit 1: CUDA events between the kernels (ecl_mst_kernel_times) */
    uint64_t seed;           /* seed of the threshold sample */
    int32_t threshold_samples; /* sample size S for threshold_mode 0 (paper: 20; default
                                  1024 -- same target, far less variance; <= 4096) */
    int32_t populate_order;  /* which CSR chunks each populate warp takes (a performance knob; the
                                result does not depend on it): 1 interleaved (chunks w, w + W, ...),
                                2 one contiguous slice per warp, 3 contiguous in phase 1 and
                                interleaved in phase 2; 0 auto (currently 3) */
    int32_t refilter;        /* crowded rounds (live edges >> sets, e.g. RMAT/uniform after the
                                giant set forms): re-apply the paper's threshold filter (P:143,
                                P:152) to the live worklist -- edges below a sampled threshold T'
                                run to completion first, the rest are deferred and filtered by
                                set(u) != set(v) afterwards.  -1 (default) auto: when >= 2^20 live
                                tuples and > 6 per MSF edge of the last round; 0 never; 1 whenever
                                live > 4 x last round's MSF edges (tests).  Same MSF either way. */
    int32_t filter_c;        /* c of P:143: the threshold targets the c|V| lightest CSR entries.
                                0 (default) auto: 3 when M >= 16n (P:394 and P:408 aim for "3
                                times"), else 4 ("we use c = 4 in our code"); "values
                                between 2 and 4 seem to work well".  Only speed depends
                                on it. */
    int32_t giant_bitmap;    /* phase 2: membership bitmap of the largest set after phase 1, so the
                                phase-2 populate filters edges inside it from n/8 bytes instead of
                                parent[]: -1 (default) auto, on iff n >= 2^25 (parent[] beyond
                                about half the L2); 0 off; 1 on at any n (tests) */
    int32_t relabel;         /* contraction: once the surviving sets of a round are few, give them
                                dense ids so the rounds' key/parent accesses stay in L2.
                                -1 (default) auto; 0 off; 1 whenever the sets at least halved
                                (tests).  Same MSF either way. */
    /* De-optimisations of the paper's Table 5, for the ablation
     * (SURVEY §8(f) NEXT-2); every setting returns the identical MSF. */
    int32_t populate_mode;   /* 0 (default) edge-centric warps over 128-entry CSR chunks;
                                1 "Thread-Based": one thread per vertex walks its row */
    int32_t both_directions; /* 0 (default) one direction per edge (Alg. 2 L4); 1 "Both Edge
                                Directions": the worklist holds both directed copies of
                                every edge (each with the edge's id) -- needs
                                ecl_mst_workspace_bytes_ex */
    int32_t tuple_layout;    /* 0 (default) 16-byte 4-tuples <p,q,w,id>; 1 "No
                                Tuples": the four items in separate arrays */
    int32_t drive;           /* 0 (default) data-driven worklist; 1 "Topology-Driven": every
                                round processes all edges of the phase again; 2 "Vertex-Centric"
                                (P:378): topology-driven with one thread per vertex and its row */
    int32_t dist_loop;       /* sharded path only: 0 (default) host-driven rounds, NCCL allreduce(min)
                                per round; 1 device-initiated: one persistent kernel per phase runs
                                every round (exchange = a device-side min over the shards' key
                                arrays, rep passes, compaction, pass A) with no host round-trip;
                                local (virtual) shards only in this build (world 1) */
} ecl_mst_options;

/* per-run statistics written by the device into the workspace */
typedef struct ecl_mst_stats {
    int32_t status;          /* 0, ECL_MST_ERR_INPUT or ECL_MST_ERR_ROUNDS */
    int32_t filtered;        /* 1 if two phases ran */
    int32_t threshold;       /* phase-1 threshold (phase 1: w < threshold) */
    int32_t rounds;          /* global rounds used (all phases; incl. final empty pass A) */
    int32_t phase2_round;    /* first global round of phase 2 (-1 if none) */
    int32_t grid;            /* CTAs of the persistent launch */
    int32_t block;           /* threads per CTA */
    int32_t refilters;       /* crowded-round splits taken (opts.refilter); each adds one sub-phase */
    int32_t relabels;        /* contraction levels opened (opts.relabel) */
    int32_t reserved;
    int64_t total_weight;
    int64_t msf_edges;
    int64_t canonical_edges; /* |E| = #{j : u < nlist[j]} */
    int64_t heavy_edges;     /* canonical edges with w >= threshold (deferred to phase 2) */
    int64_t live[ECL_MST_MAX_ROUNDS];     /* worklist size after pass A of each global round */
    int64_t winners[ECL_MST_MAX_ROUNDS];  /* MSF edges added in pass B of each global round */
    int64_t t_ns[2 * ECL_MST_MAX_ROUNDS + 4]; /* device timestamps (globaltimer) per stage */
} ecl_mst_stats;

/* Default options (filter auto, sampled threshold, seed 0x5eed, halving and
 * flatten on, guards auto). */
void ecl_mst_default_options(ecl_mst_options *opts);

/* Bytes of device workspace ecl_mst_device needs for (n, M); 0 if too large.
 * Layout: header+stats, per-arena counters, trace,
 * chunk start rows int32[M/128], key[n] int64 (best-edge slots), parent[n]
 * int32, two worklists int4[~M] (in / out of a pass). */
size_t ecl_mst_workspace_bytes(int64_t n, int64_t M);

/* Workspace bytes for (n, M) under `opts` (NULL: defaults, = the above); the
 * both_directions de-optimisation needs twice the worklist space. */
size_t ecl_mst_workspace_bytes_ex(int64_t n, int64_t M, const ecl_mst_options *opts);

/*
 * The hot path.  All pointers are DEVICE pointers (current device).  Runs
 * asynchronously on `stream` (a cudaStream_t; NULL = legacy default stream)
 * as a fixed sequence of kernels whose round loop is one persistent
 * cooperative kernel per phase: no host round-trips.
 * total_weight_out (device int64*) receives the MSF weight, or INT64_MIN if
 * the device detected an inconsistent CSR (then stats.status = ERR_INPUT and
 * in_mst is unspecified; kernels after the check exit at once, and no kernel
 * indexes memory through rejected offsets).  workspace must be >=
 * ecl_mst_workspace_bytes_ex(n, M, opts) bytes, 256-byte aligned; its contents
 * on entry are irrelevant.  opts may be NULL.  Returns ECL_MST_OK, or an
 * ECL_MST_ERR_* code: for argument errors nothing is launched; a failing CUDA
 * call inside the launch sequence (ECL_MST_ERR_CUDA) may leave the kernels
 * before it enqueued on `stream`.
 */
int ecl_mst_device(int32_t n, int64_t M, const int64_t *nindex, const int32_t *nlist,
                   const int32_t *eweight, uint8_t *in_mst_out, int64_t *total_weight_out,
                   void *workspace, size_t workspace_bytes, const ecl_mst_options *opts,
                   void *stream);

/* Synchronises `stream`, then copies the statistics of the last run that used
 * `workspace` to host memory.  Returns ECL_MST_OK or ECL_MST_ERR_CUDA. */
int ecl_mst_read_stats(const void *workspace, ecl_mst_stats *stats_out, void *stream);

/*
 * Convenience call with HOST pointers (the paper's "ECL-MST memcpy" variant,
 * P:325): copies the CSR to the device, runs ecl_mst_device, copies in_mst
 * back, synchronously.  Pinned host buffers give full PCIe bandwidth.
 * Returns the MSF weight, or INT64_MIN on any error (ecl_mst_last_error()).
 */
int64_t ecl_mst(int32_t n, const int64_t *nindex, const int32_t *nlist,
                const int32_t *eweight, uint8_t *in_mst_out);

/* Diagnostics: after a run with opts.trace = 1, synchronises `stream` and
 * copies the per-CTA stage end times (globaltimer ns) to out[slot * 4096 +
 * cta] for slot < 2*ECL_MST_MAX_ROUNDS+4 (slot numbering as stats.t_ns) and
 * cta < stats.grid; at most max_entries values.  Returns ECL_MST_OK or
 * ECL_MST_ERR_*. */
#define ECL_MST_TRACE_CTAS 4096
int ecl_mst_read_trace(const void *workspace, int64_t *out, size_t max_entries, void *stream);

/* Diagnostics: after a call with opts.trace & 2 on this thread, waits for it
 * and writes the device time (ms, CUDA events on the call's stream) of its
 * stages to ms_out: [0] memset+init, [1] populate phase 1, [2] rounds phase 1,
 * [3] flatten, [4] populate phase 2, [5] rounds phase 2, [6] finalize.
 * Returns the number of values written (<= max_stages) or ECL_MST_ERR_*. */
int ecl_mst_kernel_times(float *ms_out, int32_t max_stages);

/* ------------------------------------------------------------------------
 * Edge-sharded multi-GPU path (BASELINE.json north_star).
 * One process per GPU.  Every rank passes the SAME full CSR (replicated,
 * read-only); shard s of P = world * local_shards owns the 128-entry CSR
 * chunks s, s + P, s + 2P, ... and the worklist tuples they produce.  Per
 * round: local pass A over the rank's tuples -> ncclAllReduce(min, int64)
 * of the n best-edge keys -> a set-centric pass B that every rank applies
 * identically to its replicated union-find (a set with a finite key hooks
 * along that edge; id -> (row, nlist[id]) through the replicated CSR).
 * Output: every rank writes the full in_mst and the total weight.
 * NCCL is the process's libnccl.so.2 (dlopen; torch's when torch is loaded,
 * override with $ECLMST_NCCL_LIB).  The round loop is host-driven with one
 * 8-byte device-to-host read per round (the termination test).
 * ------------------------------------------------------------------------ */

/* 128-byte NCCL unique id for ecl_mst_dist_init (create on one rank, broadcast). */
int ecl_mst_dist_unique_id(void *uid_out);

/* Creates a handle.  world > 1 needs uid (NCCL communicator of `world` ranks,
 * this one `rank`, on the current device).  world == 1 with uid == NULL runs
 * without NCCL; world == 1 with a uid builds a one-rank communicator. */
int ecl_mst_dist_init(const void *uid, int32_t rank, int32_t world, void **handle_out);

int ecl_mst_dist_finalize(void *handle);

/* Number of CSR chunks shard `shard` of `nshards` owns (host helper). */
int64_t ecl_mst_dist_shard_chunks(int64_t M, int32_t shard, int32_t nshards);

/* Workspace bytes of ecl_mst_dist_device for one rank holding local_shards
 * shards of a world of `world` ranks; 0 if too large. */
size_t ecl_mst_dist_workspace_bytes(int64_t n, int64_t M, int32_t local_shards, int32_t world);

/* The sharded hot path; arguments as ecl_mst_device.  local_shards > 1 (only
 * with world == 1) runs that many virtual shards on this GPU with an
 * on-device min-reduction in place of the allreduce -- the same algorithm
 * and data flow, testable on one GPU.  Synchronises `stream` once per round. */
int ecl_mst_dist_device(void *handle, int32_t local_shards, int32_t n, int64_t M,
                        const int64_t *nindex, const int32_t *nlist, const int32_t *eweight,
                        uint8_t *in_mst_out, int64_t *total_weight_out, void *workspace,
                        size_t workspace_bytes, const ecl_mst_options *opts, void *stream);

/* Frees the device buffers cached by ecl_mst(). */
void ecl_mst_release_host_cache(void);

/* Message of the last failed call on this thread ("" if none). */
const char *ecl_mst_last_error(void);

int ecl_mst_abi_version(void);

#ifdef __cplusplus
}
#endif

#endif /* ECL_MST_H */
