// ecl_mst.cu -- B200 (sm_100a) implementation of the ECL-MST hot path behind
// the C ABI in include/ecl_mst.h.
//
// One MSF = one stream-ordered sequence of kernels, no host round-trip:
//
//   k_init        Alg. 1: parent[v] = v, key[v] = inf; chunk start
//                 rows (so populate needs no search); block 0 draws the filter
//                 threshold and checks nindex.
//   k_populate<1> Alg. 2 L1-11 fused with round 0 of L14-21: one warp per
//                 128-entry CSR chunk (edge-centric, high occupancy).  Emits
//                 <u,v,w,id> for u < v (L4) meeting the threshold (L6) into
//                 one of G arenas (round-robin by CTA, so every arena samples
//                 the whole CSR evenly) and atomicMins the key into both
//                 endpoints (all endpoints are roots in round 0).
//   k_rounds      persistent cooperative kernel, CTA b owns arena b:
//                 while (live > 0) { pass B ; pass A } with grid barriers.
//                 pass B  L27-31: an edge whose key won at endpoint p hooks p
//                         under the other endpoint (Boruvka hooking: each
//                         representative is written by exactly one edge, no
//                         CAS; a mutual pair keeps its smaller end as root),
//                         marks in_mst[id], adds its weight, and resets
//                         key[p] (L34-37 fused: an edge that lost at p compares
//                         unequal to the old minimum and to inf alike).
//                 pass A  L14-23: find (implicit path compression L15-18),
//                         drop p == q, compact <p,q,w,id> into the other
//                         worklist, atomicMin the key into both sets.
//   k_flatten     phase 2 only: parent[v] = find(v), so every vertex points
//                 at its root.
//   k_populate<2> P:152: heavy edges, endpoints replaced by set(u), set(v)
//                 (one load each after flattening), intra-set edges filtered.
//   k_rounds      phase 2 rounds (exits at once when there is no phase 2).
//   k_finalize    total weight / status -> caller's output.
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <dlfcn.h>

#include <algorithm>
#include <mutex>
#include <string>
#include <vector>

#include "common.cuh"
#include "populate.cuh"
#include "rounds.cuh"
#include "dist_kernels.cuh"

namespace eclmst {

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
    int occ = 0;       // resident k_rounds CTAs per SM
    int pop_occ = 0;   // resident k_populate CTAs per SM
};

static std::mutex g_dev_mu;
static DevInfo g_dev[64];

// per-thread CUDA events bracketing the kernels of the last timed call
constexpr int kTimedStages = 7;   // init, populate1, rounds1, flatten, populate2, rounds2, finalize
struct Timing {
    bool ready = false;
    bool valid = false;
    int dev = -1;                      // device the events were created on
    cudaEvent_t ev[kTimedStages + 1];
};
static thread_local Timing g_timing;

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
        if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_rounds<1>, kBlock, 0);
        int pop_occ = 0;
        if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&pop_occ, k_populate<1>, kPopBlock, 0);
        g_dev[dev].pop_occ = pop_occ > 0 ? pop_occ : 1;
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
    o->atomic_guards = -1;
    o->flatten = 1;
    o->max_ctas = 0;
    o->trace = 0;
    o->seed = 0x5eedull;
    o->threshold_samples = 1024;
    o->populate_order = 0;
    o->refilter = -1;
    o->filter_c = 0;
    o->giant_bitmap = -1;
    o->relabel = -1;
    o->populate_mode = 0;
    o->both_directions = 0;
    o->tuple_layout = 0;
    o->drive = 0;
    o->dist_loop = 0;
}

size_t ecl_mst_workspace_bytes(int64_t n, int64_t M) {
    if (n < 0 || n > INT32_MAX || M < 0 || M > (int64_t)0xFFFFFFFFLL) return 0;
    return layout_for(n, M).total;
}

size_t ecl_mst_workspace_bytes_ex(int64_t n, int64_t M, const ecl_mst_options* opts) {
    if (n < 0 || n > INT32_MAX || M < 0 || M > (int64_t)0xFFFFFFFFLL) return 0;
    return layout_for(n, M, opts && opts->both_directions ? 2 : 1).total;
}

}  // extern "C"

namespace eclmst {
// The host path's staged upload (NEXT-1, the paper's memcpy variant P:325):
// the CSR arrives on a copy stream in pieces, each piece the CSR range of one
// group of populate CTAs (contiguous slices), and each group's populate starts
// as soon as its piece has landed, so the populate hides under the PCIe copy.
struct Staging {
    cudaStream_t copy;                 // copy stream (the compute stream is the call's)
    const int64_t* h_idx;              // host CSR (pinned for overlap)
    const int32_t* h_list;
    const int32_t* h_w;
    cudaEvent_t ev[kStagePieces + 2];  // [0]: nindex (+ eweight when sampled), [1 + k]: piece k
};
}  // namespace eclmst

static int run_device(int32_t n, int64_t M, const int64_t* nindex, const int32_t* nlist, const int32_t* eweight,
                      uint8_t* in_mst_out, int64_t* total_weight_out, void* workspace, size_t workspace_bytes,
                      const ecl_mst_options* opts, void* stream, const Staging* stg);

// c of P:143 (reading Q5b): opts.filter_c if set; else the paper's target of
// "3 times" on dense graphs (M >= 16 n: C4/C5, where the light
// part then still holds most MSF edges) and its code's c = 4 below.
// ceil(log2 n) + 1: Boruvka rounds one phase (or crowded-round sub-phase)
// can take -- every round at least halves the sets that still have an edge
static inline int round_bound_for(int32_t n) {
    int b = 0;
    while ((1LL << b) < (long long)n) ++b;
    return b + 1;
}

// opts.giant_bitmap: -1 auto (parent[] beyond about half the L2), 0 off, 1 on
#ifndef ECL_MSF_BITS
#define ECL_MSF_BITS 1
#endif
static inline bool giant_bitmap_on(int32_t opt, int32_t n) {
    return opt > 0 || (opt < 0 && (long long)n >= ECL_GIANT_MIN_N);
}

// the instantiation for the de-optimisation knobs (opts.tuple_layout,
// both_directions, drive); the defaults pick <PH, false, ...0>
// (deep: phase 1 also prefetches the next chunk's row starts; measured on
// C5, M = 2e9: populate1 8.73 -> 8.31 ms, but C4 +0.26 ms, C3 +0.05: only
// from M >= 2^30 on)
// (pack: the phase-2 populate works on its surviving candidates packed one
// per lane -- it pays where few survive per chunk: graphs filtered by the
// largest-set bitmap (C5 populate2 10.43 -> 10.05 ms) or whose heavy entries
// are at most half of all (C3 0.545 -> 0.454 ms); on a dense graph without
// the bitmap about half of every chunk survives, and the per-item path, whose
// four setid loads per lane overlap, is faster (C4 2.33 vs 2.46 ms))
// (deep: the next chunk's row starts and row-bitmap words are prefetched
// too.  Phase 2 needs it for the largest-set bitmap, whose row bits come from
// the prefetched words (C5 populate2 10.0 vs 15.9 ms without); elsewhere the
// extra loads and registers cost more than they hide (C4 populate2 2.32 ->
// 2.03 ms without; phase 1 of C5 8.11 -> 7.72 ms without, with packing))
#ifndef ECL_DEEP_PH1_M
#define ECL_DEEP_PH1_M (1LL << 62)   // phase 1 deep from this M on (never)
#endif
template <int PH>
static void (*pop_kernel(bool soa, int both, bool deep = false, bool pack = false))(Params) {
    if (soa) return both ? k_populate<PH, true, true> : k_populate<PH, true, false>;
    if (both) return k_populate<PH, false, true>;
    if (PH == 2) {
        if (pack && ECL_PACK2) return deep ? k_populate<PH, false, false, 1, true> : k_populate<PH, false, false, 0, true>;
        return deep ? k_populate<PH, false, false, 1> : k_populate<PH, false, false, 0>;
    }
    return deep ? k_populate<PH, false, false, 1> : k_populate<PH, false, false, 0>;
}
// the phase-2 populate a parameter set takes (single-GPU rule, see run_device)
static void (*pop2(const Params& P))(Params) {
    const bool pack2 = P.giant_bits != nullptr || P.M <= 2LL * P.filter_c * P.n;
    return pop_kernel<2>(false, 0, P.giant_bits != nullptr, pack2);
}
template <int PH>
static const void* rounds_kernel(bool soa, int drive) {
    if (soa) {
        if (drive == 1) return reinterpret_cast<const void*>(k_rounds<PH, true, 1>);
        if (drive == 2) return reinterpret_cast<const void*>(k_rounds<PH, true, 2>);
        return reinterpret_cast<const void*>(k_rounds<PH, true, 0>);
    }
    if (drive == 1) return reinterpret_cast<const void*>(k_rounds<PH, false, 1>);
    if (drive == 2) return reinterpret_cast<const void*>(k_rounds<PH, false, 2>);
    return reinterpret_cast<const void*>(k_rounds<PH, false, 0>);
}

// threshold_mode 2: the three radix-select passes after k_init (the kernels
// return at once when the graph is not filtered)
static cudaError_t launch_quantile(const Params& P, const DevInfo& di, cudaStream_t s) {
    if (P.threshold_mode != 2 || !(P.filter_mode > 0 || (P.filter_mode < 0 && P.M >= 4LL * P.n))) return cudaSuccess;
    const unsigned hb = (unsigned)std::max<long long>(1, std::min<long long>(ceil_div(P.M / 4 + 1, 256), (long long)di.sms * 8));
    k_qhist<1><<<hb, 256, 0, s>>>(P);
    k_qselect<1><<<1, 1024, 0, s>>>(P);
    k_qhist<2><<<hb, 256, 0, s>>>(P);
    k_qselect<2><<<1, 1024, 0, s>>>(P);
    k_qhist<3><<<hb, 256, 0, s>>>(P);
    k_qselect<3><<<1, 1024, 0, s>>>(P);
    return cudaGetLastError();
}

static inline int filter_c_for(int32_t opt, int32_t n, int64_t M) {
    if (opt > 0) return opt;
    return M >= 16LL * n ? 3 : 4;
}

extern "C" {

int ecl_mst_device(int32_t n, int64_t M, const int64_t* nindex, const int32_t* nlist, const int32_t* eweight,
                   uint8_t* in_mst_out, int64_t* total_weight_out, void* workspace, size_t workspace_bytes,
                   const ecl_mst_options* opts, void* stream) {
    g_last_error.clear();
    return run_device(n, M, nindex, nlist, eweight, in_mst_out, total_weight_out, workspace, workspace_bytes, opts,
                      stream, nullptr);
}

}  // extern "C"

static int run_device(int32_t n, int64_t M, const int64_t* nindex, const int32_t* nlist, const int32_t* eweight,
                      uint8_t* in_mst_out, int64_t* total_weight_out, void* workspace, size_t workspace_bytes,
                      const ecl_mst_options* opts, void* stream, const Staging* stg) {
    if (n < 0 || M < 0) return fail(ECL_MST_ERR_INVALID, "negative n or M");
    if (M > (int64_t)0xFFFFFFFFLL) return fail(ECL_MST_ERR_TOO_LARGE, "M = %lld exceeds 2^32-1", (long long)M);
    if (!total_weight_out || !workspace) return fail(ECL_MST_ERR_INVALID, "null total_weight_out or workspace");
    if (n > 0 && !nindex) return fail(ECL_MST_ERR_INVALID, "null nindex");
    if (M > 0 && (!nlist || !eweight || !in_mst_out)) return fail(ECL_MST_ERR_INVALID, "null CSR or output array");
    if (M > 0 && n == 0) return fail(ECL_MST_ERR_INVALID, "M > 0 with n = 0");
    ecl_mst_options o;
    ecl_mst_default_options(&o);
    if (opts) o = *opts;
    if (o.threshold_mode < 0 || o.threshold_mode > 2) return fail(ECL_MST_ERR_INVALID, "threshold_mode must be 0, 1 or 2");
    if (o.populate_mode < 0 || o.populate_mode > 1 || o.both_directions < 0 || o.both_directions > 1 ||
        o.tuple_layout < 0 || o.tuple_layout > 1 || o.drive < 0 || o.drive > 2)
        return fail(ECL_MST_ERR_INVALID, "populate_mode, both_directions, tuple_layout in {0,1}; drive in {0,1,2}");
    const Layout L = layout_for(n, M, o.both_directions ? 2 : 1);
    if (workspace_bytes < L.total) return fail(ECL_MST_ERR_WORKSPACE, "workspace %zu < %zu bytes", workspace_bytes, L.total);
    if (reinterpret_cast<uintptr_t>(workspace) % 256) return fail(ECL_MST_ERR_WORKSPACE, "workspace not 256-byte aligned");
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
    const long long nchunks = ceil_div(M, kChunk);
    long long G = (long long)di.sms * di.occ;
    if (o.max_ctas > 0 && G > o.max_ctas) G = o.max_ctas;
    if (G > nchunks) G = nchunks;                 // small graphs: fewer, fuller arenas
    if (G > kMaxGrid) G = kMaxGrid;
    if (G < 1) G = 1;
    // populate: one pass of the GPU, every warp a region; W a multiple of G
    // so that every k_rounds CTA starts from the same number of regions
    long long W = (long long)di.sms * di.pop_occ * kPopWarps;
    if (W > nchunks) W = nchunks;
    if (W > kMaxPopWarps) W = kMaxPopWarps;
    if (W > G * kMaxRegionsPerCta) W = G * kMaxRegionsPerCta;
    W = std::max<long long>(1, W / G) * G;
    // chunk order of the populate warps (opts.populate_order): interleaved
    // single chunks (w, w + W, ...) balance graphs whose density of kept
    // entries drifts along the rows (RMAT phase 2: 1.4x slower populate with
    // contiguous slices); a contiguous slice of B = ceil(nchunks / W) chunks
    // per warp keeps the rounds' random accesses spatially local.
    // bit0: phase 1 contiguous, bit1: phase 2 contiguous.
    int contig = 0;
    switch (o.populate_order) {
        case 1: contig = 0; break;
        case 2: contig = 3; break;
        case 3: contig = 1; break;
        default: contig = 1; break;
    }
    // dynamic tail (ECL_POP_DYN, bit PH-1): each populate warp walks a static
    // share of ECL_POP_STATIC/8 of its chunks, then claims batches of
    // ECL_POP_BATCH chunks from one counter until none are left.  The warps
    // of an SM do not progress at one rate (the scheduler favours the oldest
    // CTAs: on C5 the populate-2 CTAs of the four residency slots ended at
    // 8.6, 9.2, 10.3 and 11.8 ms), so a fixed split leaves the GPU draining.
    // A warp claims only while its region keeps room for everything it may
    // still hold; regions get 2 B + 4 chunks of slack, which guarantees that
    // the claims never stall with chunks left.  Off for the
    // staged host path's phase 1 (a piece may not have landed yet) and the
    // thread-based populate.
    const long long span = ceil_div(nchunks, W);
    const long long dup = o.both_directions ? 2 : 1;
    int dyn = (o.populate_mode == 1 ? 0 : ECL_POP_DYN) & (stg ? 2 : 3);
    if (dyn && (span + 2 * ECL_POP_BATCH + 4) * W * kChunk * dup > L.wl_cap) dyn = 0;   // no room for the slack
    // (both_directions: every candidate edge takes two tuples)
    const long long rcap = (span + (dyn ? 2 * ECL_POP_BATCH + 4 : 0)) * kChunk * dup;
    // only warps that own a block write a region
    if (W * rcap > L.wl_cap) return fail(ECL_MST_ERR_WORKSPACE, "internal: regions exceed worklist capacity");
    // k_rounds arenas: the worklist of CTA b never exceeds its first input,
    // the W / G regions b, b + G, ...  (arenas in wl0 overlay the regions;
    // they are first written after every CTA has consumed its regions)
    const long long cap = (W / G) * rcap;
    if (cap >= (1LL << 30)) return fail(ECL_MST_ERR_TOO_LARGE, "arena of %lld tuples too large", cap);

    Params P;
    P.n = n;
    P.M = M;
    P.nchunks = nchunks;
    P.G = (int)G;
    P.cap = cap;
    P.W = (int)W;
    P.rcap = rcap;
    P.pop_contig = contig;
    P.pop_cta0 = 0;
    P.pop_span = span;
    P.pop_dyn = dyn;
    P.pop_s0 = (int)(nchunks * ECL_POP_STATIC / 8 / W);
    P.nindex = reinterpret_cast<const long long*>(nindex);
    P.nlist = nlist;
    P.eweight = eweight;
    P.in_mst = in_mst_out;
    P.total_out = reinterpret_cast<long long*>(total_weight_out);
    P.st = reinterpret_cast<ecl_mst_stats*>(ws + L.stats);
    P.in = reinterpret_cast<Internal*>(ws + L.internal);
    P.trace = o.trace ? reinterpret_cast<long long*>(ws + L.trace) : nullptr;
    P.rowstart = reinterpret_cast<int*>(ws + L.rowstart);
    P.region = reinterpret_cast<int4*>(ws + L.region);
    // the largest-set bitmap only pays when parent[] does not fit the L2
    P.giant_bits = giant_bitmap_on(o.giant_bitmap, n) ? reinterpret_cast<unsigned*>(ws + L.giant) : nullptr;
    P.key = reinterpret_cast<long long*>(ws + L.key);
    P.parent = reinterpret_cast<int*>(ws + L.parent);
    P.wl0 = reinterpret_cast<int4*>(ws + L.wl0);
    P.wl1 = reinterpret_cast<int4*>(ws + L.wl1);
    P.seed = o.seed;
    P.filter_mode = o.filter < 0 ? -1 : (o.filter ? 1 : 0);
    P.threshold_mode = o.threshold_mode;
    P.threshold_value = o.threshold;
    P.samples = o.threshold_samples > 0 ? std::min(o.threshold_samples, kMaxSamples) : 20;
    P.filter_c = filter_c_for(o.filter_c, n, M);
    P.halving = o.path_halving ? 1 : 0;
    P.guards = o.atomic_guards < 0 ? -1 : (o.atomic_guards ? 1 : 0);
    P.flatten = o.flatten ? 1 : 0;
    P.refilter = o.refilter < 0 ? -1 : (o.refilter ? 1 : 0);
    P.round_bound = round_bound_for(n);
    P.samp = reinterpret_cast<int*>(ws + L.samp);
    P.qhist = reinterpret_cast<unsigned long long*>(ws + L.qhist);
    // contraction needs the flatten (phase 2 then reads every vertex's set from setid)
    // (absolute level ids up to 2n must fit int32)
    P.relabel = (o.flatten && (long long)n <= (1LL << 30)) ? (o.relabel < 0 ? -1 : (o.relabel ? 1 : 0)) : 0;
    P.lvcnt = reinterpret_cast<int*>(ws + L.lvcnt);
    P.setid = reinterpret_cast<int*>(ws + L.setid);
    P.wlcap = L.wl_cap;
    P.both = o.both_directions ? 1 : 0;
    P.drive = o.drive;
    if (o.drive) {   // the topology-driven passes re-read the phase's edges: no splits, no contraction
        P.refilter = 0;
        P.relabel = 0;
    }
    const bool soa = o.tuple_layout == 1;
    const bool thread_pop = o.populate_mode == 1;
    P.shard = 0;
    P.nshards = 1;
    P.nlocal = nchunks;
    // MSF marks as bits, in_mst written once at the end (ECL_MSF_BITS; see mark_msf)
    P.mbits = ECL_MSF_BITS ? reinterpret_cast<unsigned*>(ws + L.mbits) : nullptr;
    P.zero_mst = P.mbits ? 0 : 1;
    P.acnt = nullptr;
    P.tgt = nullptr;
    P.hcnt = nullptr;
    P.dsp = nullptr;
    P.keys_all = nullptr;
    P.nkeys = 1;
    if ((reinterpret_cast<uintptr_t>(nlist) | reinterpret_cast<uintptr_t>(eweight)) % 16 ||
        reinterpret_cast<uintptr_t>(in_mst_out) % 4)
        return fail(ECL_MST_ERR_INVALID, "nlist/eweight must be 16-byte and in_mst 4-byte aligned");

    const long long init_blocks = std::min<long long>(ceil_div((long long)n, 256), (long long)di.sms * 8);
    const long long pop_blocks = ceil_div(W, kPopWarps);
    if (pop_blocks > INT_MAX) return fail(ECL_MST_ERR_TOO_LARGE, "too many populate CTAs");
    void* args[] = {&P};
    // opts.trace bit 1: CUDA events between the kernels (ecl_mst_kernel_times)
    const bool timing = (o.trace & 2) != 0;
    if (timing) {   // events belong to a device: recreate them when the caller switched devices
        int cur_dev = -1;
        cudaError_t e0 = cudaGetDevice(&cur_dev);
        if (e0 != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "cudaGetDevice: %s", cudaGetErrorString(e0));
        if (g_timing.ready && g_timing.dev != cur_dev) {
            int prev = -1;
            cudaGetDevice(&prev);
            cudaSetDevice(g_timing.dev);
            for (auto& ev : g_timing.ev) cudaEventDestroy(ev);
            cudaSetDevice(prev);
            g_timing.ready = false;
        }
        if (!g_timing.ready) {
            for (int i = 0; i < kTimedStages + 1; ++i) {
                e0 = cudaEventCreate(&g_timing.ev[i]);
                if (e0 != cudaSuccess) {
                    for (int k = 0; k < i; ++k) cudaEventDestroy(g_timing.ev[k]);
                    return fail(ECL_MST_ERR_CUDA, "cudaEventCreate: %s", cudaGetErrorString(e0));
                }
            }
            g_timing.ready = true;
            g_timing.dev = cur_dev;
        }
    }
    g_timing.valid = false;
    int ev_i = 0;
    auto mark = [&]() -> cudaError_t {
        return timing ? cudaEventRecord(g_timing.ev[ev_i++], s) : cudaSuccess;
    };
    const unsigned flat_blocks = (unsigned)std::max<long long>(init_blocks, 1);
    // staged upload: CTA groups of the phase-1 populate and their CSR pieces
    const bool staged = stg && (contig & 1) && !thread_pop;
    const int pieces = staged ? (int)std::min<long long>(kStagePieces, pop_blocks) : 1;
    auto group_cta = [&](int k) { return (long long)(pop_blocks * k / pieces); };
    cudaError_t e = cudaSuccess;
    if (stg) {
        // nindex first (k_init needs all of it), and eweight too when the
        // threshold samples it; then the pieces of nlist (and eweight)
        const bool sampled = (P.filter_mode > 0 || (P.filter_mode < 0 && M >= 4LL * n)) &&
                             (P.threshold_mode == 0 || P.threshold_mode == 2);
        e = cudaMemcpyAsync(const_cast<int64_t*>(nindex), stg->h_idx, sizeof(int64_t) * ((size_t)n + 1),
                            cudaMemcpyHostToDevice, stg->copy);
        if (e == cudaSuccess && sampled)
            e = cudaMemcpyAsync(const_cast<int32_t*>(eweight), stg->h_w, sizeof(int32_t) * (size_t)M,
                                cudaMemcpyHostToDevice, stg->copy);
        if (e == cudaSuccess) e = cudaEventRecord(stg->ev[0], stg->copy);
        for (int k = 0; k < pieces && e == cudaSuccess; ++k) {
            long long e0 = staged ? std::min<long long>(M, group_cta(k) * kPopWarps * span * kChunk) : 0;
            long long e1 = staged ? std::min<long long>(M, group_cta(k + 1) * kPopWarps * span * kChunk) : M;
            if (k == pieces - 1) e1 = M;
            if (e1 > e0) {
                e = cudaMemcpyAsync(const_cast<int32_t*>(nlist) + e0, stg->h_list + e0, sizeof(int32_t) * (size_t)(e1 - e0),
                                    cudaMemcpyHostToDevice, stg->copy);
                if (e == cudaSuccess && !sampled)
                    e = cudaMemcpyAsync(const_cast<int32_t*>(eweight) + e0, stg->h_w + e0,
                                        sizeof(int32_t) * (size_t)(e1 - e0), cudaMemcpyHostToDevice, stg->copy);
            }
            if (e == cudaSuccess) e = cudaEventRecord(stg->ev[1 + k], stg->copy);
        }
        if (e == cudaSuccess) e = cudaStreamWaitEvent(s, stg->ev[0], 0);
        if (e == cudaSuccess && !staged) e = cudaStreamWaitEvent(s, stg->ev[1], 0);
        if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "staged H2D: %s", cudaGetErrorString(e));
    }
    if (e == cudaSuccess) e = mark();
    if (e == cudaSuccess) e = cudaMemsetAsync(P.st, 0, sizeof(ecl_mst_stats), s);
    if (e == cudaSuccess) {
        k_init<<<flat_blocks, 256, 0, s>>>(P);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = launch_quantile(P, di, s);
    if (e == cudaSuccess) e = mark();
    if (e == cudaSuccess) {
        if (staged) {   // one launch per piece, each after its piece has landed
            for (int k = 0; k < pieces && e == cudaSuccess; ++k) {
                const long long c0 = group_cta(k), c1 = group_cta(k + 1);
                if (c1 <= c0) continue;
                e = cudaStreamWaitEvent(s, stg->ev[1 + k], 0);
                Params Pk = P;
                Pk.pop_cta0 = (int)c0;
                if (e == cudaSuccess) {
                    k_populate<1><<<(unsigned)(c1 - c0), kPopBlock, 0, s>>>(Pk);
                    e = cudaGetLastError();
                }
            }
        } else if (thread_pop) {   // opts.populate_mode 1
            if (soa) k_populate_thread<1, true><<<flat_blocks, 256, 0, s>>>(P);
            else k_populate_thread<1, false><<<flat_blocks, 256, 0, s>>>(P);
            k_regions<1><<<1, 256, 0, s>>>(P);
            e = cudaGetLastError();
        } else {
            pop_kernel<1>(soa, P.both, M >= ECL_DEEP_PH1_M)<<<(unsigned)pop_blocks, kPopBlock, 0, s>>>(P);
            e = cudaGetLastError();
        }
    }
    if (e == cudaSuccess) e = mark();
    if (e == cudaSuccess)
        e = cudaLaunchCooperativeKernel(rounds_kernel<1>(soa, P.drive), dim3((unsigned)G), dim3(kBlock), args, 0, s);
    if (e == cudaSuccess) e = mark();
    // phase 2 can only happen when filtering is on; with the automatic rule
    // (M >= 4n) the host knows that already and skips the three launches
    const bool maybe_phase2 = P.filter_mode > 0 || (P.filter_mode < 0 && M >= 4LL * n);
    if (e == cudaSuccess && maybe_phase2) {
        if (P.relabel) k_flatten<0><<<flat_blocks, 256, 0, s>>>(P);
        k_flatten<1><<<flat_blocks, 256, 0, s>>>(P);
        k_giant<<<1, 256, 0, s>>>(P);
        k_flatten<2><<<flat_blocks, 256, 0, s>>>(P);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = mark();
    if (e == cudaSuccess && maybe_phase2) {
        if (thread_pop) {
            if (soa) k_populate_thread<2, true><<<flat_blocks, 256, 0, s>>>(P);
            else k_populate_thread<2, false><<<flat_blocks, 256, 0, s>>>(P);
            k_regions<2><<<1, 256, 0, s>>>(P);
        } else {
            const bool pack2 = P.giant_bits != nullptr || M <= 2LL * P.filter_c * n;
            pop_kernel<2>(soa, P.both, P.giant_bits != nullptr, pack2)<<<(unsigned)pop_blocks, kPopBlock, 0, s>>>(P);
        }
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = mark();
    if (e == cudaSuccess && maybe_phase2)
        e = cudaLaunchCooperativeKernel(rounds_kernel<2>(soa, P.drive), dim3((unsigned)G), dim3(kBlock), args, 0, s);
    if (e == cudaSuccess) e = mark();
    if (e == cudaSuccess) {
        if (P.mbits) k_expand<<<(unsigned)std::max<long long>(1, std::min<long long>(ceil_div(M / 16, 256), (long long)di.sms * 8)), 256, 0, s>>>(P);
        k_finalize<<<1, 32, 0, s>>>(P);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = mark();
    if (e == cudaSuccess && timing) g_timing.valid = true;
    if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "launch (G=%lld): %s", G, cudaGetErrorString(e));
    return ECL_MST_OK;
}

extern "C" {

int ecl_mst_kernel_times(float* ms_out, int32_t max_stages) {
    g_last_error.clear();
    if (!ms_out) return fail(ECL_MST_ERR_INVALID, "null argument");
    if (!g_timing.valid) return fail(ECL_MST_ERR_INVALID, "no timed run on this thread (opts.trace & 2)");
    cudaError_t e = cudaEventSynchronize(g_timing.ev[kTimedStages]);
    int n = 0;
    for (; e == cudaSuccess && n < kTimedStages && n < max_stages; ++n)
        e = cudaEventElapsedTime(&ms_out[n], g_timing.ev[n], g_timing.ev[n + 1]);
    if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "kernel_times: %s", cudaGetErrorString(e));
    return n;
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
static cudaStream_t g_pool_copy = nullptr;          // staged upload (NEXT-1)
static cudaEvent_t g_pool_ev[kStagePieces + 2];
static bool g_pool_ev_ok = false;

void ecl_mst_release_host_cache(void) {
    std::lock_guard<std::mutex> lk(g_pool_mu);
    if (g_pool) cudaFree(g_pool);
    if (g_pool_stream) cudaStreamDestroy(g_pool_stream);
    if (g_pool_copy) cudaStreamDestroy(g_pool_copy);
    if (g_pool_ev_ok)
        for (auto& ev : g_pool_ev) cudaEventDestroy(ev);
    g_pool = nullptr;
    g_pool_cap = 0;
    g_pool_stream = nullptr;
    g_pool_copy = nullptr;
    g_pool_ev_ok = false;
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
            if (g_pool_copy) cudaStreamDestroy(g_pool_copy);
            g_pool_copy = nullptr;
            if (g_pool_ev_ok)
                for (auto& ev : g_pool_ev) cudaEventDestroy(ev);
            g_pool_ev_ok = false;
        }
        e = cudaMalloc(&g_pool, need);
        if (e == cudaSuccess) {
            g_pool_cap = need;
            g_pool_dev = dev;
        }
    }
    if (e == cudaSuccess && !g_pool_stream) e = cudaStreamCreateWithFlags(&g_pool_stream, cudaStreamNonBlocking);
    if (e == cudaSuccess && !g_pool_copy) e = cudaStreamCreateWithFlags(&g_pool_copy, cudaStreamNonBlocking);
    if (e == cudaSuccess && !g_pool_ev_ok) {
        int made = 0;
        for (; made < kStagePieces + 2 && e == cudaSuccess; ++made)
            e = cudaEventCreateWithFlags(&g_pool_ev[made], cudaEventDisableTiming);
        if (e == cudaSuccess) g_pool_ev_ok = true;
        else
            for (int i = 0; i + 1 < made; ++i) cudaEventDestroy(g_pool_ev[i]);
    }
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
    // H2D on the copy stream in pieces; each piece's populate starts when it lands
    Staging stg;
    stg.copy = g_pool_copy;
    stg.h_idx = nindex;
    stg.h_list = nlist;
    stg.h_w = eweight;
    for (int i = 0; i < kStagePieces + 2; ++i) stg.ev[i] = g_pool_ev[i];
    int rc = run_device(n, M, d_idx, d_list, d_w, d_mst, d_tot, d_ws, b_ws, nullptr, s, &stg);
    if (rc) {
        cudaStreamSynchronize(g_pool_copy);   // no copy may outlive the caller's buffers
        cudaStreamSynchronize(s);
        return INT64_MIN;
    }
    int64_t total = INT64_MIN;
    e = cudaMemcpyAsync(in_mst_out, d_mst, (size_t)M, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(&total, d_tot, sizeof total, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) {
        fail(ECL_MST_ERR_CUDA, "D2H/run: %s", cudaGetErrorString(e));
        return INT64_MIN;
    }
    if (total == INT64_MIN) {
        int status = ECL_MST_ERR_INPUT;   // stats.status is the first word of the workspace
        if (cudaMemcpy(&status, d_ws, sizeof status, cudaMemcpyDeviceToHost) != cudaSuccess) status = ECL_MST_ERR_INPUT;
        if (status == ECL_MST_ERR_ROUNDS) fail(ECL_MST_ERR_ROUNDS, "device ran out of round slots");
        else fail(ECL_MST_ERR_INPUT, "device found an inconsistent CSR");
    }
    return total;
}

}  // extern "C"

// ===========================================================================
// distributed (edge-sharded) path: host side
// ===========================================================================
namespace eclmst {

// NCCL is taken from the process at run time (torch's libnccl.so.2 when torch
// is loaded), so the single-GPU library has no NCCL dependency.
struct NcclUid {
    char internal[128];
};
typedef void* NcclComm;
struct NcclApi {
    bool ok = false;
    int (*getUniqueId)(NcclUid*) = nullptr;
    int (*commInitRank)(NcclComm*, int, NcclUid, int) = nullptr;
    int (*allReduce)(const void*, void*, size_t, int, int, NcclComm, cudaStream_t) = nullptr;
    int (*allGather)(const void*, void*, size_t, int, NcclComm, cudaStream_t) = nullptr;
    int (*commDestroy)(NcclComm) = nullptr;
    const char* (*getErrorString)(int) = nullptr;
};
constexpr int kNcclInt32 = 2, kNcclInt64 = 4, kNcclSum = 0, kNcclMin = 3;
static NcclApi g_nccl;
static std::mutex g_nccl_mu;

static int load_nccl() {
    std::lock_guard<std::mutex> lk(g_nccl_mu);
    if (g_nccl.ok) return ECL_MST_OK;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    const char* env = getenv("ECLMST_NCCL_LIB");
    if (!h && env) h = dlopen(env, RTLD_NOW);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW);
    if (!h) return fail(ECL_MST_ERR_CUDA, "libnccl.so.2 not found: %s", dlerror());
    g_nccl.getUniqueId = reinterpret_cast<int (*)(NcclUid*)>(dlsym(h, "ncclGetUniqueId"));
    g_nccl.commInitRank = reinterpret_cast<int (*)(NcclComm*, int, NcclUid, int)>(dlsym(h, "ncclCommInitRank"));
    g_nccl.allReduce = reinterpret_cast<int (*)(const void*, void*, size_t, int, int, NcclComm, cudaStream_t)>(
        dlsym(h, "ncclAllReduce"));
    g_nccl.allGather = reinterpret_cast<int (*)(const void*, void*, size_t, int, NcclComm, cudaStream_t)>(
        dlsym(h, "ncclAllGather"));
    g_nccl.commDestroy = reinterpret_cast<int (*)(NcclComm)>(dlsym(h, "ncclCommDestroy"));
    g_nccl.getErrorString = reinterpret_cast<const char* (*)(int)>(dlsym(h, "ncclGetErrorString"));
    if (!g_nccl.getUniqueId || !g_nccl.commInitRank || !g_nccl.allReduce || !g_nccl.allGather || !g_nccl.commDestroy)
        return fail(ECL_MST_ERR_CUDA, "libnccl.so.2 lacks the needed symbols");
    g_nccl.ok = true;
    return ECL_MST_OK;
}

struct DistHandle {
    int rank = 0, world = 1;
    NcclComm comm = nullptr;
    long long* h_pin = nullptr;   // pinned host words (phase-2 decision, stats)
    long long* h_map = nullptr;   // mapped pinned {sets with a finite key, |R_next|, deferred buffer}, written by k_dist_compact
    long long* d_map = nullptr;   // its device alias
    cudaEvent_t ev = nullptr;     // recorded after k_dist_compact each round
};

static void release(DistHandle* h) {
    if (h->ev) cudaEventDestroy(h->ev);
    if (h->h_map) cudaFreeHost(h->h_map);
    if (h->h_pin) cudaFreeHost(h->h_pin);
    delete h;
}

struct DistLayout {
    size_t stats, internal, rowstart, parent, tgt, keyptrs, rl0, rl1, rbuf, keep, bcnt, dsplit, giant, qhist, setid,
        sps, found, shard0, shard_bytes, total;
    size_t region, acnt, hcnt, key, wl0, wl1;   // offsets inside one shard block
    long long wl_cap, nlocal_max;
};

static inline DistLayout dist_layout(int64_t n, int64_t M, int S, int world) {
    DistLayout L;
    const long long nchunks = ceil_div(M, kChunk);
    const long long P = (long long)S * world;
    L.nlocal_max = ceil_div(nchunks, P);
    const long long wmax = L.nlocal_max < kMaxPopWarps ? L.nlocal_max : kMaxPopWarps;
    L.wl_cap = (L.nlocal_max + wmax) * kChunk;
    size_t off = 0;
    L.stats = off;    off = align_up(off + sizeof(ecl_mst_stats), 256);
    L.internal = off; off = align_up(off + sizeof(Internal), 256);
    L.rowstart = off; off = align_up(off + sizeof(int) * (size_t)(nchunks + 1), 256);
    L.parent = off;   off = align_up(off + sizeof(int) * (size_t)n, 256);
    L.tgt = off;      off = align_up(off + sizeof(int) * ((size_t)n + world), 256);   // (+ allgather padding)
    L.keyptrs = off;  off = align_up(off + sizeof(long long*) * (size_t)S, 256);
    L.rl0 = off;      off = align_up(off + sizeof(int) * (size_t)n, 256);     // root lists (double buffer)
    L.rl1 = off;      off = align_up(off + sizeof(int) * (size_t)n, 256);
    L.rbuf = off;     off = align_up(off + sizeof(long long) * ((size_t)n + kSplitExt), 256);   // the allreduce buffer (+ split extras)
    L.keep = off;     off = align_up(off + (size_t)n, 256);
    L.bcnt = off;     off = align_up(off + sizeof(int) * (size_t)kCompactGridMax, 256);
    L.dsplit = off;   off = align_up(off + sizeof(DistSplit), 256);
    L.giant = off;    off = align_up(off + sizeof(unsigned) * (size_t)((n + 31) / 32 + 1), 256);   // largest-set bitmap
    L.qhist = off;    off = align_up(off + sizeof(unsigned long long) * (size_t)kQBins, 256);
    L.setid = off;    off = align_up(off + sizeof(int) * (size_t)n, 256);
    L.sps = off;      off = align_up(off + sizeof(Params) * (size_t)S, 256);   // dist_loop: the shards' Params
    L.found = off;    off = align_up(off + 2 * sizeof(unsigned long long), 256);
    size_t so = 0;
    L.region = so; so = align_up(so + sizeof(int4) * (size_t)kMaxPopWarps, 256);
    L.acnt = so;   so = align_up(so + sizeof(int) * (size_t)kMaxGrid, 256);
    L.hcnt = so;   so = align_up(so + sizeof(int) * (size_t)kMaxGrid, 256);
    L.key = so;    so = align_up(so + sizeof(long long) * (size_t)n, 256);
    L.wl0 = so;    so = align_up(so + sizeof(int4) * (size_t)L.wl_cap, 256);
    L.wl1 = so;    so = align_up(so + sizeof(int4) * (size_t)L.wl_cap, 256);
    L.shard_bytes = so;
    L.shard0 = off;
    off += so * (size_t)S;
    L.total = off;
    return L;
}

}  // namespace eclmst

extern "C" {

int ecl_mst_dist_unique_id(void* uid_out) {
    g_last_error.clear();
    if (!uid_out) return fail(ECL_MST_ERR_INVALID, "null argument");
    int rc = load_nccl();
    if (rc) return rc;
    int r = g_nccl.getUniqueId(reinterpret_cast<NcclUid*>(uid_out));
    if (r) return fail(ECL_MST_ERR_CUDA, "ncclGetUniqueId: %d", r);
    return ECL_MST_OK;
}

int ecl_mst_dist_init(const void* uid, int32_t rank, int32_t world, void** handle_out) {
    g_last_error.clear();
    if (!handle_out || world < 1 || rank < 0 || rank >= world) return fail(ECL_MST_ERR_INVALID, "bad rank/world");
    DistHandle* h = new DistHandle;
    h->rank = rank;
    h->world = world;
    cudaError_t e = cudaHostAlloc(reinterpret_cast<void**>(&h->h_pin), sizeof(long long) * 4, cudaHostAllocDefault);
    if (e == cudaSuccess)
        e = cudaHostAlloc(reinterpret_cast<void**>(&h->h_map), sizeof(long long) * 4, cudaHostAllocMapped);
    if (e == cudaSuccess) e = cudaHostGetDevicePointer(reinterpret_cast<void**>(&h->d_map), h->h_map, 0);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->ev, cudaEventDisableTiming);
    if (e != cudaSuccess) {
        release(h);
        return fail(ECL_MST_ERR_CUDA, "dist_init: %s", cudaGetErrorString(e));
    }
    if (world > 1 || uid) {   // world 1 with a uid: a one-rank NCCL communicator (tests the NCCL path)
        if (!uid) {
            release(h);
            return fail(ECL_MST_ERR_INVALID, "world > 1 needs an NCCL unique id");
        }
        int rc = load_nccl();
        NcclUid id;
        if (!rc) {
            std::memcpy(id.internal, uid, sizeof id.internal);
            const int r = g_nccl.commInitRank(&h->comm, world, id, rank);
            if (r) rc = fail(ECL_MST_ERR_CUDA, "ncclCommInitRank: %s", g_nccl.getErrorString ? g_nccl.getErrorString(r) : "?");
        }
        if (rc) {
            release(h);
            return rc;
        }
    }
    *handle_out = h;
    return ECL_MST_OK;
}

int ecl_mst_dist_finalize(void* handle) {
    g_last_error.clear();
    DistHandle* h = static_cast<DistHandle*>(handle);
    if (!h) return ECL_MST_OK;
    if (h->comm && g_nccl.ok) g_nccl.commDestroy(h->comm);
    release(h);
    return ECL_MST_OK;
}

int64_t ecl_mst_dist_shard_chunks(int64_t M, int32_t shard, int32_t nshards) {
    if (M < 0 || nshards < 1 || shard < 0 || shard >= nshards) return -1;
    const long long nchunks = ceil_div(M, kChunk);
    return shard < nchunks ? (nchunks - shard + nshards - 1) / nshards : 0;
}

size_t ecl_mst_dist_workspace_bytes(int64_t n, int64_t M, int32_t local_shards, int32_t world) {
    if (n < 0 || n > INT32_MAX || M < 0 || M > (int64_t)0xFFFFFFFFLL || local_shards < 1 || world < 1) return 0;
    return dist_layout(n, M, local_shards, world).total;
}

int ecl_mst_dist_device(void* handle, int32_t local_shards, int32_t n, int64_t M, const int64_t* nindex,
                        const int32_t* nlist, const int32_t* eweight, uint8_t* in_mst_out,
                        int64_t* total_weight_out, void* workspace, size_t workspace_bytes,
                        const ecl_mst_options* opts, void* stream) {
    g_last_error.clear();
    DistHandle* h = static_cast<DistHandle*>(handle);
    if (!h) return fail(ECL_MST_ERR_INVALID, "null handle (ecl_mst_dist_init)");
    const int S = local_shards, world = h->world, rank = h->rank;
    if (S < 1 || S > 64) return fail(ECL_MST_ERR_INVALID, "local_shards must be in [1, 64]");
    if (world > 1 && S != 1) return fail(ECL_MST_ERR_INVALID, "local_shards > 1 only without NCCL (world 1)");
    if (n < 0 || M < 0) return fail(ECL_MST_ERR_INVALID, "negative n or M");
    if (M > (int64_t)0xFFFFFFFFLL) return fail(ECL_MST_ERR_TOO_LARGE, "M exceeds 2^32-1");
    if (!total_weight_out || !workspace || (n > 0 && !nindex) || (M > 0 && (!nlist || !eweight || !in_mst_out)))
        return fail(ECL_MST_ERR_INVALID, "null argument");
    if (M > 0 && n == 0) return fail(ECL_MST_ERR_INVALID, "M > 0 with n = 0");
    const DistLayout L = dist_layout(n, M, S, world);
    if (workspace_bytes < L.total) return fail(ECL_MST_ERR_WORKSPACE, "workspace %zu < %zu bytes", workspace_bytes, L.total);
    if (reinterpret_cast<uintptr_t>(workspace) % 256) return fail(ECL_MST_ERR_WORKSPACE, "workspace not 256-byte aligned");
    if ((reinterpret_cast<uintptr_t>(nlist) | reinterpret_cast<uintptr_t>(eweight)) % 16 ||
        reinterpret_cast<uintptr_t>(in_mst_out) % 4)
        return fail(ECL_MST_ERR_INVALID, "nlist/eweight must be 16-byte and in_mst 4-byte aligned");
    ecl_mst_options o;
    ecl_mst_default_options(&o);
    if (opts) o = *opts;
    if (o.populate_mode || o.both_directions || o.tuple_layout || o.drive)
        return fail(ECL_MST_ERR_INVALID, "the de-optimisation knobs are single-GPU only (ecl_mst_device)");
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    char* ws = static_cast<char*>(workspace);
    ecl_mst_stats* st = reinterpret_cast<ecl_mst_stats*>(ws + L.stats);
    Internal* in = reinterpret_cast<Internal*>(ws + L.internal);
    if (M == 0) {
        cudaError_t e = cudaMemsetAsync(st, 0, sizeof(ecl_mst_stats), s);
        if (e == cudaSuccess) e = cudaMemsetAsync(total_weight_out, 0, sizeof(int64_t), s);
        if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "memset: %s", cudaGetErrorString(e));
        return ECL_MST_OK;
    }
    DevInfo di;
    int rc = device_info(&di);
    if (rc) return rc;
    const long long nchunks = ceil_div(M, kChunk);
    const long long Pt = (long long)S * world;

    // crowded-round splits (opts.refilter, reading Q17): decided on the
    // device from allreduced values, the same on every rank
    // (auto: only where the two-phase filter is on too, M >= 4n -- the dense
    // graphs whose giant set crowds the rounds; C2 x1 4.33 vs 3.80 ms with them)
    const bool dloop = o.dist_loop != 0;
    if (dloop && (world > 1 || h->comm))
        return fail(ECL_MST_ERR_INVALID, "dist_loop 1 (device-initiated rounds) runs local shards only (world 1, no NCCL)");
    // (the device loop has no crowded-round split: every split decision of
    // the host loop rides on its allreduce)
    const bool split_on = !dloop && (o.refilter > 0 || (o.refilter < 0 && (o.filter > 0 || (o.filter < 0 && M >= 4LL * n))));
    int loop_occ = 0;
    if (dloop) {
        cudaError_t e0 = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&loop_occ, k_dist_loop<1>, kBlock, 0);
        if (e0 != cudaSuccess || loop_occ < 1) return fail(ECL_MST_ERR_CUDA, "dist_loop occupancy");
    }
    DistSplit* dsp = reinterpret_cast<DistSplit*>(ws + L.dsplit);
    // per-shard launch geometry and parameters
    std::vector<Params> sp(S);
    std::vector<long long*> keyptr(S);
    for (int k = 0; k < S; ++k) keyptr[k] = reinterpret_cast<long long*>(ws + L.shard0 + k * L.shard_bytes + L.key);
    long long** d_keyptrs = reinterpret_cast<long long**>(ws + L.keyptrs);
    cudaError_t e = cudaMemcpyAsync(d_keyptrs, keyptr.data(), sizeof(long long*) * S, cudaMemcpyHostToDevice, s);
    for (int k = 0; k < S; ++k) {
        Params& P = sp[k];
        std::memset(&P, 0, sizeof P);
        const int shard = rank * S + k;
        const long long nlocal = shard < nchunks ? (nchunks - shard + Pt - 1) / Pt : 0;
        long long G = (long long)di.sms * (dloop ? std::min(loop_occ, di.occ) : di.occ);   // (co-resident in the loop)
        if (G > std::max<long long>(nlocal, 1)) G = std::max<long long>(nlocal, 1);
        if (G > kMaxGrid) G = kMaxGrid;
        long long W = (long long)di.sms * di.pop_occ * kPopWarps;
        if (W > std::max<long long>(nlocal, 1)) W = std::max<long long>(nlocal, 1);
        if (W > kMaxPopWarps) W = kMaxPopWarps;
        if (W > G * kMaxRegionsPerCta) W = G * kMaxRegionsPerCta;
        W = std::max<long long>(1, W / G) * G;
        const long long rcap = std::max<long long>(1, ceil_div(nlocal, W)) * kChunk;
        const long long cap = (W / G) * rcap;
        if (W * rcap > L.wl_cap || cap >= (1LL << 30)) return fail(ECL_MST_ERR_TOO_LARGE, "shard worklist too large");
        char* sb = ws + L.shard0 + k * L.shard_bytes;
        P.n = n;
        P.M = M;
        P.nchunks = nchunks;
        P.G = (int)G;
        P.cap = cap;
        P.W = (int)W;
        P.rcap = rcap;
        P.pop_span = rcap / kChunk;
        P.pop_dyn = 0;
        P.pop_contig = 1;   // phase 1: each warp a contiguous slice of the shard's chunks (as on one GPU)
        P.nindex = reinterpret_cast<const long long*>(nindex);
        P.nlist = nlist;
        P.eweight = eweight;
        P.in_mst = in_mst_out;
        P.total_out = reinterpret_cast<long long*>(total_weight_out);
        P.st = st;
        P.in = in;
        P.trace = nullptr;
        P.rowstart = reinterpret_cast<int*>(ws + L.rowstart);
        P.region = reinterpret_cast<int4*>(sb + L.region);
        P.key = keyptr[k];
        P.parent = reinterpret_cast<int*>(ws + L.parent);
        P.wl0 = reinterpret_cast<int4*>(sb + L.wl0);
        P.wl1 = reinterpret_cast<int4*>(sb + L.wl1);
        P.seed = o.seed;
        P.filter_mode = o.filter < 0 ? -1 : (o.filter ? 1 : 0);
        P.threshold_mode = o.threshold_mode;
        P.threshold_value = o.threshold;
        P.samples = o.threshold_samples > 0 ? std::min(o.threshold_samples, kMaxSamples) : 20;
        P.filter_c = filter_c_for(o.filter_c, n, M);
        P.halving = o.path_halving ? 1 : 0;
        // (auto: the single-GPU rule -- no guard in the phase-1 populate, where
        // the slots are still mostly inf; the sharded pass A guards whenever
        // guards are not off.  Measured one-rank C5: populate1 12.2 -> 8.2 ms)
        P.guards = o.atomic_guards < 0 ? -1 : (o.atomic_guards ? 1 : 0);
        P.flatten = o.flatten ? 1 : 0;
        P.refilter = dloop ? 0 : (o.refilter < 0 ? -1 : (o.refilter ? 1 : 0));   // crowded-round split (Q17)
        P.round_bound = round_bound_for(n);
        P.samp = nullptr;
        P.qhist = reinterpret_cast<unsigned long long*>(ws + L.qhist);
        P.relabel = 0;   // (the replicated union-find stays on vertex ids)
        P.lvcnt = nullptr;
        P.setid = reinterpret_cast<int*>(ws + L.setid);
        P.wlcap = L.wl_cap;
        P.both = 0;
        P.drive = 0;
        P.shard = shard;
        P.nshards = (int)Pt;
        P.nlocal = nlocal;
        P.zero_mst = 0;
        P.acnt = reinterpret_cast<int*>(sb + L.acnt);
        P.tgt = reinterpret_cast<int*>(ws + L.tgt);
        P.hcnt = reinterpret_cast<int*>(sb + L.hcnt);
        // phase 2: the largest set's bitmap where parent[] exceeds the L2, as on one GPU
        P.giant_bits = giant_bitmap_on(o.giant_bitmap, n) ? reinterpret_cast<unsigned*>(ws + L.giant) : nullptr;
        P.dsp = split_on ? dsp : nullptr;
        P.keys_all = d_keyptrs;
        P.nkeys = S;
    }
    Params& P0 = sp[0];
    const unsigned vblocks = (unsigned)std::max<long long>(1, std::min<long long>(ceil_div((long long)n, 256), (long long)di.sms * 8));
    auto check = [&](const char* what) -> int {
        cudaError_t e2 = cudaGetLastError();
        if (e2 != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e2));
        return ECL_MST_OK;
    };
    auto allreduce = [&](void* buf, size_t count, int op) -> int {
        if (!h->comm) return ECL_MST_OK;
        const int r = g_nccl.allReduce(buf, buf, count, kNcclInt64, op, h->comm, s);
        if (r) return fail(ECL_MST_ERR_CUDA, "ncclAllReduce: %s", g_nccl.getErrorString ? g_nccl.getErrorString(r) : "?");
        return ECL_MST_OK;
    };
    auto read_word = [&](const void* dptr, long long* out) -> int {
        cudaError_t e2 = cudaMemcpyAsync(h->h_pin, dptr, sizeof(long long), cudaMemcpyDeviceToHost, s);
        if (e2 == cudaSuccess) e2 = cudaStreamSynchronize(s);
        if (e2 != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "sync: %s", cudaGetErrorString(e2));
        *out = *h->h_pin;
        return ECL_MST_OK;
    };

    if (e == cudaSuccess) e = cudaMemsetAsync(st, 0, sizeof(ecl_mst_stats), s);
    if (e == cudaSuccess) e = cudaMemsetAsync(in, 0, sizeof(Internal), s);   // (reps: zeroed again by each k_dist_compact)
    if (e == cudaSuccess) e = cudaMemsetAsync(&dsp->hb, 0xFF, sizeof(int), s);    // hb = -1: nothing deferred
    if (e == cudaSuccess) e = cudaMemsetAsync(in_mst_out, 0, (size_t)M, s);   // every rank returns the full mask
    if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "memset: %s", cudaGetErrorString(e));
    k_init<<<vblocks, 256, 0, s>>>(P0);
    if ((rc = check("k_init"))) return rc;
    e = launch_quantile(P0, di, s);   // every rank holds the full CSR: the same threshold everywhere
    if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "quantile: %s", cudaGetErrorString(e));
    int g = 0;
    int* const rlist[2] = {reinterpret_cast<int*>(ws + L.rl0), reinterpret_cast<int*>(ws + L.rl1)};
    unsigned char* const rkeep = reinterpret_cast<unsigned char*>(ws + L.keep);
    int* const rcnt = reinterpret_cast<int*>(ws + L.bcnt);
    long long phase2_roots = 0;
    // the current roots into `out` (count: h_map[1] after the next sync)
    auto launch_roots = [&](int* out) {
        const unsigned cb = (unsigned)std::max<long long>(1, std::min<long long>(ceil_div(n, 4096), kCompactGridMax));
        k_dist_root_keep<<<vblocks, 256, 0, s>>>(P0, rkeep);
        k_dist_count<<<cb, kCompactBlock, 0, s>>>(n, rkeep, rcnt);
        k_dist_compact<<<cb, kCompactBlock, 0, s>>>(nullptr, n, rkeep, rcnt, out, &in->nroots, &in->reps, h->d_map,
                                                    nullptr);
    };
    if (dloop) {   // ---- device-initiated rounds: one persistent kernel per phase ----
        Params* d_sps = reinterpret_cast<Params*>(ws + L.sps);
        unsigned long long* d_found = reinterpret_cast<unsigned long long*>(ws + L.found);
        e = cudaMemcpyAsync(d_sps, sp.data(), sizeof(Params) * S, cudaMemcpyHostToDevice, s);
        if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "dist_loop params: %s", cudaGetErrorString(e));
        long long Gl = 1;
        for (int k = 0; k < S; ++k) Gl = std::max<long long>(Gl, sp[k].G);
        auto run_loop = [&](int ph, int g0, const int* R0, long long nR0, int* r_a, int* r_b) -> int {
            DistLoop DL;
            DL.sps = d_sps;
            DL.S = S;
            DL.g0 = g0;
            DL.R0 = R0;
            DL.nR0 = nR0;
            DL.rl[0] = r_a;
            DL.rl[1] = r_b;
            DL.buf = reinterpret_cast<long long*>(ws + L.rbuf);
            DL.keep = rkeep;
            DL.bcnt = rcnt;
            DL.found = d_found;
            cudaError_t e2 = cudaMemsetAsync(d_found, 0, 2 * sizeof(unsigned long long), s);
            void* largs[] = {&P0, &DL};
            if (e2 == cudaSuccess)
                e2 = cudaLaunchCooperativeKernel(ph == 1 ? reinterpret_cast<const void*>(k_dist_loop<1>)
                                                         : reinterpret_cast<const void*>(k_dist_loop<2>),
                                                 dim3((unsigned)Gl), dim3(kBlock), largs, 0, s);
            long long gend = 0;
            if (e2 == cudaSuccess) e2 = cudaMemcpyAsync(h->h_pin, &in->g_end, sizeof(int), cudaMemcpyDeviceToHost, s);
            if (e2 == cudaSuccess) e2 = cudaStreamSynchronize(s);   // (once per phase)
            if (e2 != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "dist_loop: %s", cudaGetErrorString(e2));
            std::memcpy(&gend, h->h_pin, sizeof(int));
            g = (int)gend;
            return ECL_MST_OK;
        };
        for (int k = 0; k < S; ++k) k_populate<1><<<(unsigned)ceil_div(sp[k].W, kPopWarps), kPopBlock, 0, s>>>(sp[k]);
        if ((rc = check("populate"))) return rc;
        if ((rc = run_loop(1, 0, nullptr, n, rlist[0], rlist[1]))) return rc;
        long long filtered = 0, heavy = 0;
        if ((rc = read_word(&st->heavy_edges, &heavy))) return rc;
        if ((rc = read_word(&st->filtered, &filtered))) return rc;
        if ((filtered & 0xffffffffll) && heavy != 0 && g + 1 < ECL_MST_MAX_ROUNDS) {
            k_flatten<1><<<vblocks, 256, 0, s>>>(P0);
            k_giant<<<1, 256, 0, s>>>(P0);
            k_flatten<2><<<vblocks, 256, 0, s>>>(P0);
            launch_roots(rlist[0]);
            ++g;
            e = cudaMemcpyAsync(&st->phase2_round, &g, sizeof(int), cudaMemcpyHostToDevice, s);
            if (e == cudaSuccess) e = cudaStreamSynchronize(s);
            if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "phase2: %s", cudaGetErrorString(e));
            const long long nroots = reinterpret_cast<volatile long long*>(h->h_map)[1];
            for (int k = 0; k < S; ++k) pop2(sp[k])<<<(unsigned)ceil_div(sp[k].W, kPopWarps), kPopBlock, 0, s>>>(sp[k]);
            if ((rc = check("populate2"))) return rc;
            if ((rc = run_loop(2, g, rlist[0], nroots, rlist[1], rlist[0]))) return rc;
        }
    }
    for (int ph = 1; ph <= 2 && !dloop; ++ph) {
        if (ph == 2) {
            // the phase-2 decision needs the global deferred count
            if ((rc = allreduce(&st->canonical_edges, 2, kNcclSum))) return rc;
            long long filtered = 0, heavy = 0;
            if ((rc = read_word(&st->heavy_edges, &heavy))) return rc;
            if ((rc = read_word(&st->filtered, &filtered))) return rc;
            if (!(filtered & 0xffffffffll) || heavy == 0) break;
            k_flatten<1><<<vblocks, 256, 0, s>>>(P0);
            k_giant<<<1, 256, 0, s>>>(P0);   // replicated parent[]: every rank finds the same set
            k_flatten<2><<<vblocks, 256, 0, s>>>(P0);
            // phase 2 records keys at roots only (set(u), set(v) after the
            // flatten): its first exchange covers the roots, not all n
            // vertices (C5: about 1 M of 67 M after phase 1)
            launch_roots(rlist[0]);
            ++g;
            if (g >= ECL_MST_MAX_ROUNDS) return fail(ECL_MST_ERR_INPUT, "round limit");
            e = cudaMemcpyAsync(&st->phase2_round, &g, sizeof(int), cudaMemcpyHostToDevice, s);
            if (e == cudaSuccess) e = cudaStreamSynchronize(s);   // &g is a host stack value
            if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "phase2: %s", cudaGetErrorString(e));
            phase2_roots = reinterpret_cast<volatile long long*>(h->h_map)[1];
        }
        for (int k = 0; k < S; ++k) {
            if (ph == 1) k_populate<1><<<(unsigned)ceil_div(sp[k].W, kPopWarps), kPopBlock, 0, s>>>(sp[k]);
            else pop2(sp[k])<<<(unsigned)ceil_div(sp[k].W, kPopWarps), kPopBlock, 0, s>>>(sp[k]);
        }
        if ((rc = check("populate"))) return rc;
        bool first = true;
        int cur = 0;
        // the sets whose keys are exchanged: all n in the phase's first round,
        // then the roots that can still hold a live edge (root-compacted)
        int* const* rl = rlist;
        const int* R = ph == 2 ? rl[0] : nullptr;
        long long nR = ph == 2 ? phase2_roots : n;
        int rb = ph == 2 ? 1 : 0;
        long long* rbuf = reinterpret_cast<long long*>(ws + L.rbuf);
        unsigned char* keep = rkeep;
        int* bcnt = rcnt;
        // Each round is enqueued in full -- exchange, rep passes, root-list
        // compaction, and the next pass A -- before the host waits, on an
        // event behind the compaction, for the two words that decide the next
        // round (its root-list size, and whether any set still had a live
        // edge).  The pass A is speculative: when no set had a live edge every
        // worklist is already empty and it records nothing.  So the GPU runs
        // that pass A while the host reads the counts and enqueues the next
        // exchange: no stream drain per round.
        while (true) {
            const unsigned rblocks = (unsigned)std::max<long long>(1, std::min<long long>(ceil_div(nR, 256), (long long)di.sms * 8));
            const unsigned cblocks = (unsigned)std::max<long long>(1, std::min<long long>(ceil_div(nR, 4096), kCompactGridMax));
            // allreduce(min) of the live sets' best-edge keys over all shards.
            // A phase's first round exchanges all n keys: with one local shard
            // that is key[] itself, reduced in place (no gather/scatter copies;
            // reps2 resets key[x] only after reading it as buf[x]).
            // With splits on, the split candidates of the live list ride
            // behind the keys (kSplitExt slots; never in a phase's first round).
            long long* xbuf = rbuf;
            const bool split = split_on && !first;
            if (R == nullptr && S == 1 && !split) {
                xbuf = P0.key;
                if ((rc = allreduce(xbuf, (size_t)nR, kNcclMin))) return rc;
            } else {
                if (split)
                    for (int k = 0; k < S; ++k) k_dist_split_cand<<<1, 512, 0, s>>>(sp[k], k, S, cur, rbuf + nR);
                k_dist_gather<<<rblocks, 256, 0, s>>>(P0, R, nR, rbuf);
                if ((rc = allreduce(rbuf, (size_t)nR + (split ? kSplitExt : 0), kNcclMin))) return rc;
                k_dist_scatter<<<rblocks, 256, 0, s>>>(P0, R, nR, rbuf);
            }
            // rep pass 1 -- the row search and finds, the costly part -- is
            // split over the ranks (and over the virtual shards, which share
            // tgt[]), then tgt[] is allgathered; pass 2 is replicated
            if (nR > 0) {
                const long long parts = world > 1 ? world : S;
                const long long slice = ceil_div(nR, parts);
                const unsigned sblocks = (unsigned)std::max<long long>(1, std::min<long long>(ceil_div(slice, 256), (long long)di.sms * 8));
                for (long long k = (world > 1 ? rank : 0); k < (world > 1 ? rank + 1 : parts); ++k)
                    k_dist_reps1<<<sblocks, 256, 0, s>>>(P0, R, std::min(nR, k * slice), std::min(nR, (k + 1) * slice), xbuf);
                if (world > 1 && h->comm) {
                    int* tg = P0.tgt;
                    const int r = g_nccl.allGather(tg + (size_t)rank * slice, tg, (size_t)slice, kNcclInt32, h->comm, s);
                    if (r) return fail(ECL_MST_ERR_CUDA, "ncclAllGather: %s", g_nccl.getErrorString ? g_nccl.getErrorString(r) : "?");
                }
            }
            k_dist_reps2<<<rblocks, 256, 0, s>>>(P0, R, nR, xbuf, keep, g);
            k_dist_count<<<cblocks, kCompactBlock, 0, s>>>(nR, keep, bcnt);
            k_dist_compact<<<cblocks, kCompactBlock, 0, s>>>(R, nR, keep, bcnt, rl[rb], &in->nroots, &in->reps, h->d_map,
                                                             split_on ? dsp : nullptr);
            e = cudaEventRecord(h->ev, s);
            if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "event: %s", cudaGetErrorString(e));
            const bool can_continue = g + 1 < ECL_MST_MAX_ROUNDS;
            if (can_continue) {
                if (split && !first)   // is pass A g + 1 a crowded round?  (from the allreduced extras)
                    k_dist_split_decide<<<1, 32, 0, s>>>(P0, rbuf + nR, cur, g, world);
                // (first: also counts the phase's populate output -- needed even
                // when the phase turns out empty)
                for (int k = 0; k < S; ++k) {
                    if (first) k_dist_passA<true><<<sp[k].G, kBlock, 0, s>>>(sp[k], g + 1, cur);
                    else k_dist_passA<false><<<sp[k].G, kBlock, 0, s>>>(sp[k], g + 1, cur);
                }
            }
            if ((rc = check("rounds"))) return rc;
            e = cudaEventSynchronize(h->ev);
            if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "sync: %s", cudaGetErrorString(e));
            const long long reps = reinterpret_cast<volatile long long*>(h->h_map)[0];
            const long long nnext = reinterpret_cast<volatile long long*>(h->h_map)[1];
            const int hbv = (int)reinterpret_cast<volatile long long*>(h->h_map)[2];
            if (reps == 0 && hbv >= 0) {
                // the light part of a split is done on every rank: drain the
                // deferred tuples (filter + record), then continue from the
                // roots (their keys were inf in the empty round just ended)
                if (g + 2 >= ECL_MST_MAX_ROUNDS) return fail(ECL_MST_ERR_INPUT, "round limit");
                ++g;
                for (int k = 0; k < S; ++k) k_dist_drain<<<sp[k].G, kBlock, 0, s>>>(sp[k], g, hbv);
                e = cudaMemsetAsync(&dsp->hb, 0xFF, sizeof(int), s);
                if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "memset: %s", cudaGetErrorString(e));
                launch_roots(rl[0]);
                e = cudaStreamSynchronize(s);
                if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "sync: %s", cudaGetErrorString(e));
                R = rl[0];
                nR = reinterpret_cast<volatile long long*>(h->h_map)[1];
                rb = 1;
                cur = hbv ^ 1;
                first = false;
                if ((rc = check("drain"))) return rc;
                continue;
            }
            if (reps == 0) break;   // no set has a live edge anywhere: the phase is done
            if (!can_continue) return fail(ECL_MST_ERR_INPUT, "round limit");
            R = rl[rb];
            nR = nnext;
            rb ^= 1;
            ++g;
            cur ^= 1;
            first = false;
        }
    }
    const int rounds = g + 1;
    e = cudaMemcpyAsync(&st->refilters, &in->splits, sizeof(int), cudaMemcpyDeviceToDevice, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(&st->rounds, &rounds, sizeof(int), cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return fail(ECL_MST_ERR_CUDA, "stats: %s", cudaGetErrorString(e));
    k_finalize<<<1, 32, 0, s>>>(P0);
    if ((rc = check("finalize"))) return rc;
    return ECL_MST_OK;
}

}  // extern "C"
