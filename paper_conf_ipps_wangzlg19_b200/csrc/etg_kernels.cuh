// etg_kernels.cuh -- sm_100a kernels of the EtaGraph hot path.
//
// The active set (Def. 1) of the next iteration is recorded as a bitmap
// Q of n bits: a relaxation that improves label[u] sets bit u (L136: "the
// updated vertices are added to the new active set").  Per iteration
// (Proc. 1 while-loop body) two kernels run on the handle's
// stream, every size kept on the device:
//
//   expand_kernel     steps A2-A5.  A persistent CTA takes tiles of TS
//                     consecutive shadow vertices: it loads the tile's window
//                     of the compacted active set (S, B, D, F; coalesced), maps
//                     each shadow to its slice of at most K out-edges (Def. 3,
//                     reading R-2) by a binary search in shared memory, stages
//                     the tile's neighbour segments (<= TS*K words -- the bound
//                     UDC gives, L199) in shared memory with cp.async (SMP,
//                     Sec. V-B), then relaxes every staged edge, one
//                     thread per edge with kR edges in flight: a plain-load
//                     pre-filter, then a fire-and-forget red.min/red.max (BFS:
//                     a plain store -- all writers of a level write the same
//                     depth) and red.or of bit u into Q (Proc. 1 L207, readings
//                     R-4, R-5).  No thread waits on an atomic's return value.
//   udc_scan_kernel   steps A5-A6 and the UDC of the next iteration (Def. 3;
//                     Sec. IV-A).  Reads and clears Q; every set bit v
//                     gets off[v], off[v+1]; degree-0 vertices are dropped
//                     ("naturally filter active vertices with outdegree equals
//                     to 0", L142), the others get c = ceil(deg/K) shadows.  A
//                     single-pass chained (decoupled look-back) scan over the
//                     pair (kept, c) writes the compacted active set F with its
//                     start offsets B, degrees D, exclusive shadow prefix S,
//                     and tile_first[t] = the entry owning shadow t*TS.  These
//                     replace the paper's 12-byte 3-tuples (L138).  The last
//                     scan tile publishes the sizes and sets the CUDA-graph
//                     conditional ("while actSet.isNotEmpty()", L207).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace etg {

constexpr uint32_t kInf = 0xFFFFFFFFu;
constexpr uint32_t kCap = 0xFFFFFFFEu;
constexpr int kBlock = 256;                 // threads per CTA (8 warps)
constexpr int kWarps = kBlock / 32;
constexpr uint32_t kFull = 0xFFFFFFFFu;
#ifndef ETG_KR
#define ETG_KR 8
#endif
#ifndef ETG_MINB
#define ETG_MINB 3                          // expand: >= 3 CTAs (24 warps) per SM, <= 85 registers
#endif
#ifndef ETG_SGRAB
#define ETG_SGRAB 1                         // expand: first tile grab static (global warp index)
#endif
#ifndef ETG_LX_PEEK
#define ETG_LX_PEEK 1                       // shared shadow label: plain load before the compare-and-swap
#endif
#ifndef ETG_SHARED_SSSP
#define ETG_SHARED_SSSP 0                   // experiment: SSSP multi-shadow vertices share one published label too
#endif
#ifndef ETG_BAR_SLEEP
#define ETG_BAR_SLEEP 0                     // persistent loop: ns of back-off per grid-barrier poll
#endif
#ifndef ETG_PIPE
#define ETG_PIPE 1                          // software-pipelined batch loop in the warp expand
#endif
constexpr int kR = ETG_KR;                  // edges (chunks) in flight per thread in the relax loop
#ifndef ETG_KR_W
#define ETG_KR_W 6                          // ... for SSSP/SSWP (weights: two streams per chunk)
#endif

enum Alg : int { ALG_BFS = 0, ALG_SSSP = 1, ALG_CC = 2, ALG_SSWP = 3 };

// Device-resident control block (one per handle).
struct Ctl {
    uint32_t depth;       // index of the current active set (BFS: its depth)
    uint32_t epoch;       // monotone over the handle's life: chained-scan tags
    uint32_t nF;          // compacted active-set size (vertices with out-degree > 0)
    uint32_t nshadow;     // shadow vertices of the current active set
    uint32_t ntiles;      // expand tiles of the current active set
    uint32_t scan_ctr;    // dynamic tile counter of the chained scan
    uint32_t tile_ctr;    // dynamic tile counter of the expand
    uint32_t iterations;  // non-empty active sets expanded in the current call
    uint32_t error;       // ETG_VALIDATE result
    unsigned long long activations;   // set bits consumed by the scans
    unsigned long long shadows;
    unsigned long long edges;
    unsigned long long frontier;
    unsigned long long reached_v;
    unsigned long long reached_e;
    uint32_t *label;      // output label array of the current call
    uint32_t source;
    uint32_t thresh;      // near-far SSSP: marked vertices with label < thresh are expanded
    uint32_t far_min;     //   min label of the deferred (far) marked vertices of the last scan
    uint32_t far_count;   //   number of deferred marked vertices of the last scan
    uint32_t more;        // loop condition computed by the last scan
    uint32_t rd_valid;    // the last expand marked the rows it lowered labels in (RD): the scan may skip the rest
    uint32_t bar;         // persistent loop: grid-barrier arrivals in the current call
    unsigned long long t_expand_ns;   // persistent loop: %globaltimer time of the expand phases
    unsigned long long t_scan_ns;     //   ... and of the scan phases (block 0's view, barrier to barrier)
};

constexpr uint32_t kMaxPeer = 8;            // fused push exchange: ranks whose labels a kernel can reach

template <class OffT>
struct Dev {
    const OffT *off;
    const uint32_t *col;
    const uint32_t *w;
    uint32_t *Q;                // next-active-set bitmap (nwords words, zero between uses)
    uint32_t *V;                // BFS: visited bitmap as of the iteration start (label != INF)
    uint32_t *snap;             // labels at the start of the iteration (SSSP/CC/SSWP pre-filter)
    uint32_t *F;                // compacted active set (vertex ids, ascending)
    OffT *B;                    // off[F[k]]
    uint32_t *D;                // out-degree of F[k] (> 0)
    uint32_t *S;                // exclusive prefix of shadow counts (nF + 1 entries)
    uint32_t *Lx;               // snap_used: label entry k's shadows all propagate (INF = not read yet)
    uint32_t *tile_first;       // entry owning shadow t*ts
    unsigned long long *recE;   // chained scan records per scan tile: kept entries
    unsigned long long *recS;   //   and shadows (value << 32 | epoch << 2 | flag)
    Ctl *ctl;
    unsigned long long m;       // edges
    uint32_t n;
    uint32_t nwords;            // bitmap words (padded to whole scan tiles)
    uint32_t K;                 // degree limit (Def. 3); unused with NO_UDC
    uint32_t K_log2;            // log2(K) when K is a power of two, else 32
    uint32_t ts;                // shadows per expand tile (<= kBlock, power of 2)
    uint32_t ts_log2;
    uint32_t tune;              // experiment switches (ETG_TUNE env var at load); 0 = default
    uint32_t prefetch;          // warp kernel, direct mode: L2 bulk prefetch of the next tile
    uint32_t ahead;             // warp kernel: stage A of the next batch before stage B of this one
    uint32_t ahead_mid;         // ... also for SSSP/CC/SSWP in mid-size iterations (ETG_AHEAD_MID, default 1)
    uint32_t tune2;             // experiment bits (ETG_TUNE2): 1 = keep two tiles per grab in mid-size iterations
    uint32_t nf_delta;          // near-far SSSP bucket width (0: the paper's schedule)
    uint32_t snap_used;         // SSSP/CC/SSWP, single GPU: a sole shadow stores the label it expands with
    uint32_t filt_live;         // SSSP/CC/SSWP pre-filter reads the live labels, not the snapshot (label +
                                // snapshot larger than L2: one randomly gathered array instead of two)
    uint32_t scan_list;         // scan: vertex-list path 0 never, 1 sparse rows (default), 2 always
    // Dirty rows (SSSP/CC/SSWP, single GPU, 32-row scan warps): a sparse expand
    // (<= dirty_tiles tiles) marks the 32-vertex row of every label it lowers in
    // RD, and the next scan compares label and snapshot only in rows marked in
    // RD or holding deferred (near-far) vertices, FR; 0 = off.
    uint32_t dirty_tiles;
    uint32_t *RD, *FR;          // one bit per row of 32 vertices
    uint32_t split;             // expand: max warps sharing one tile in sparse iterations (1: no split)
    uint32_t scan_rows;         // scan: a warp with >= scan_rows active rows stages its offsets in shared
                                // memory with one bulk copy (0: never; needs the dynamic shared memory)
    // The vertex range this handle activates (a push-partition rank: its owned
    // range, the only vertices with local out-edges; else [0, n)): init marks
    // and the scan covers only these words, from scan tile scan_t0 on.
    uint32_t own_lo, own_hi;    // vertices
    uint32_t own_w0, own_w1;    // bitmap words [own_lo / 32, ceil(own_hi / 32))
    uint32_t scan_t0;           // first scan tile (own_w0 / (kScanV / 32))
    // Fused push exchange (NEXT-3 over peer memory): a relaxation of a vertex
    // owned by rank q != peer_rank also lands, as a red.min/max, in rank q's
    // label array (device memory of another GPU reached over NVLink, or of
    // another partition on this GPU).  npeer = 0: off.
    uint32_t npeer;
    uint32_t peer_rank;
    uint32_t peer_bounds[kMaxPeer + 1];
    uint32_t *peer_label[kMaxPeer];
};

constexpr uint32_t kTuneFilterL1 = 1u;    // pre-filter label loads cached in L1
// replay-only experiment switches (etg_debug_expand_replay; results not kept)
constexpr uint32_t kTuneNoGather = 16u;   // skip the label gather and the commit
constexpr uint32_t kTuneNoCommit = 32u;   // gather labels but never commit (counts passes)
constexpr uint32_t kTuneQMark = 64u;      // A/B: SSSP/CC/SSWP commits also set Q, the scan reads only Q
constexpr uint32_t kTuneScanDyn = 256u;   // A/B: every scan tile from the counter (no static first tile)
constexpr uint32_t kTuneNoSnapUsed = 512u; // A/B: snapshot = labels at the iteration start only
constexpr uint32_t kTunePersist = 1024u;   // experiment: the loop as one persistent kernel (loop_kernel)
constexpr uint32_t kTuneNoFilter = 4096u;  // A/B: no pre-filter gather, every relaxation commits
constexpr uint32_t kTuneNearFarClassic = 8192u;   // A/B: near-far threshold advances only when the near set empties
constexpr uint32_t kTuneNoSharedLabel = 16384u;   // A/B: multi-shadow vertices keep the scan-time snapshot
constexpr uint32_t kTuneAheadAll = 32768u;        // A/B: SMP look-ahead for SSSP/CC/SSWP too (default: BFS only)
constexpr uint32_t kTuneFiltLive = 1u << 18;      // A/B: pre-filter on the live labels at any size
constexpr uint32_t kTuneFiltSnap = 1u << 19;      // A/B: pre-filter on the snapshot at any size

// ------------------------------------------------------------------------- //
// small device helpers
// ------------------------------------------------------------------------- //
__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31; }

__device__ __forceinline__ uint32_t ld_cg(const uint32_t *p) { return __ldcg(p); }

// Control-block / cross-phase reads.  Separate kernels see each other's
// writes through L2 (L1 starts cold at every launch); inside the persistent
// loop kernel (P) a value written by another SM in an earlier phase must not
// come from a stale L1 line, so those reads bypass L1.
template <bool P, class T>
__device__ __forceinline__ T cld(const T &x) {
    if (P) return *(const volatile T *)&x;
    return x;
}
template <bool P, class T>
__device__ __forceinline__ T xld(const T *p) {
    if (P) return __ldcg(p);
    return *p;
}

// L1-cached label load (experiment switch kTuneFilterL1).  Labels move
// monotonically, so a stale copy can only let the filter pass an edge.
__device__ __forceinline__ uint32_t ld_ca(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.global.ca.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}

__device__ __forceinline__ uint32_t ld_volatile_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.volatile.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ unsigned long long ld_volatile_u64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// L2 residency policies.  The per-vertex arrays (labels, the bitmap) are
// small and hit randomly: keep them (evict_last).  The edge arrays (col, w)
// are streamed once per iteration and larger than L2: evict them first, so
// they do not push the labels out to HBM (where every random 4-byte access
// would cost a DRAM burst).
__device__ __forceinline__ uint64_t policy_keep() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t policy_stream() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

// streamed read-only edge data: no L1 allocation, evict-first in L2
__device__ __forceinline__ uint32_t ld_stream(const uint32_t *p, uint64_t pol) {
    uint32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}

// label gather for the pre-filter: L2 only, keep resident
__device__ __forceinline__ uint32_t ld_label(const uint32_t *p, uint64_t pol) {
    uint32_t v;
    asm volatile("ld.global.cg.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}

// fire-and-forget reductions (no return value: the thread never waits on them)
__device__ __forceinline__ void red_min(uint32_t *p, uint32_t v, uint64_t pol) {
    asm volatile("red.relaxed.gpu.global.L2::cache_hint.min.u32 [%0], %1, %2;" :: "l"(p), "r"(v), "l"(pol) : "memory");
}
__device__ __forceinline__ void red_max(uint32_t *p, uint32_t v, uint64_t pol) {
    asm volatile("red.relaxed.gpu.global.L2::cache_hint.max.u32 [%0], %1, %2;" :: "l"(p), "r"(v), "l"(pol) : "memory");
}
__device__ __forceinline__ void red_or(uint32_t *p, uint32_t v, uint64_t pol) {
    asm volatile("red.relaxed.gpu.global.L2::cache_hint.or.b32 [%0], %1, %2;" :: "l"(p), "r"(v), "l"(pol) : "memory");
}

// bulk L2 prefetch (TMA unit; address and size multiples of 16)
__device__ __forceinline__ void prefetch_l2(const void *p, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(p), "r"(bytes) : "memory");
}

__device__ __forceinline__ void cp_async4(void *smem, const void *gmem) {
    uint32_t s = static_cast<uint32_t>(__cvta_generic_to_shared(smem));
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" :: "r"(s), "l"(gmem) : "memory");
}

__device__ __forceinline__ void cp_async_wait_all() {
    asm volatile("cp.async.wait_all;" ::: "memory");
}

// inclusive warp scan
template <class T>
__device__ __forceinline__ T warp_incl_scan(T x) {
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        T y = __shfl_up_sync(kFull, x, d);
        if (lane_id() >= (uint32_t)d) x += y;
    }
    return x;
}

__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long x) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(kFull, x, o);
    return x;
}

// Block-wide exclusive scan of one value per thread; returns the exclusive
// prefix, writes the block total.  `wsum` is kWarps words of shared memory.
template <class T>
__device__ __forceinline__ T block_excl_scan(T x, T *wsum, T &total) {
    T incl = warp_incl_scan(x);
    const uint32_t warp = threadIdx.x >> 5;
    if (lane_id() == 31) wsum[warp] = incl;
    __syncwarp();                                   // bar.sync needs converged warps
    __syncthreads();
    if (warp == 0) {
        T s = lane_id() < (uint32_t)kWarps ? wsum[lane_id()] : T(0);
        s = warp_incl_scan(s);
        if (lane_id() < (uint32_t)kWarps) wsum[lane_id()] = s;
    }
    __syncwarp();
    __syncthreads();
    T warp_prefix = warp ? wsum[warp - 1] : T(0);
    total = wsum[kWarps - 1];
    __syncthreads();
    return warp_prefix + incl - x;
}

// Number of shadow vertices of a vertex of out-degree `deg` (Def. 3; L142:
// degree 0 gives none).
// ceil(deg / K) as a shift when K is a power of two (klog < 32): the scan
// evaluates it twice per active vertex, and a runtime integer division is a
// ~20-instruction sequence.
template <bool UDC, class D>
__device__ __forceinline__ uint32_t udc_count(D deg, uint32_t K, uint32_t klog) {
    if (!UDC) return deg > 0 ? 1u : 0u;
    if (deg == 0) return 0u;
    if (klog < 32) return (uint32_t)(((deg - 1) >> klog) + 1);
    return (uint32_t)((deg - 1) / (D)K + 1);
}

// ---- mbarrier / bulk-copy helpers (SMP stages, scan offset staging) ----
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity) {
    asm volatile("{\n .reg .pred p;\n WAIT_%=:\n"
                 " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
                 " @!p bra WAIT_%=;\n}" :: "r"(smem_u32(b)), "r"(parity) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
// TMA bulk copy global -> shared (16-byte aligned, size multiple of 16), completing on mbarrier b
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *b, uint64_t pol) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
                 :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(b)), "l"(pol) : "memory");
}
// ... without an L2 cache hint
__device__ __forceinline__ void bulk_g2s_plain(void *dst, const void *src, uint32_t bytes, uint64_t *b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(b)) : "memory");
}

// ------------------------------------------------------------------------- //
// A1: per-call control reset and label initialisation (Proc. 1 "Init label",
// "Init actSet", L207)
// ------------------------------------------------------------------------- //
__device__ __forceinline__ void ctl_begin(Ctl *ctl, uint32_t *label, uint32_t source, uint32_t thresh) {
    ctl->depth = kInf;            // the first scan makes it 0
    ctl->epoch += 1;
    ctl->nF = 0;
    ctl->nshadow = 0;
    ctl->ntiles = 0;
    ctl->scan_ctr = 0;
    ctl->iterations = 0;
    ctl->activations = 0;
    ctl->shadows = 0;
    ctl->edges = 0;
    ctl->frontier = 0;
    ctl->label = label;
    ctl->source = source;
    ctl->thresh = thresh;         // near-far SSSP: the first threshold (the source has distance 0)
    ctl->far_min = 0xFFFFFFFFu;
    ctl->far_count = 0;
    ctl->rd_valid = 0;            // the first scan compares every row
    ctl->bar = 0;
    ctl->t_expand_ns = 0;
    ctl->t_scan_ns = 0;
}

__global__ void ctl_begin_kernel(Ctl *ctl, uint32_t *label, uint32_t source) {
    ctl_begin(ctl, label, source, kInf);
}

// the scan bookkeeping an expand launch does (see expand kernels), for a scan
// that directly follows another scan (step-wise near-far: empty near set)
__global__ void ctl_rescan_kernel(Ctl *ctl) {
    ctl->scan_ctr = 0;
    ctl->epoch += 1;
    ctl->far_min = kInf;
    ctl->far_count = 0;
}

// BFS/SSSP: label = INF, label[s] = 0, Q = {s}.  SSWP: label = 0, label[s] =
// INF, Q = {s}.  CC: label[v] = v, Q = all vertices (the scan drops degree-0
// ones).  Q is all-zero on entry (every scan clears what it reads).
template <class OffT, int ALG>
__global__ __launch_bounds__(kBlock) void init_kernel(Dev<OffT> d, uint32_t *label, uint32_t source) {
    // the control block of the call (one thread; the first scan is stream-ordered after this kernel)
    if (blockIdx.x == 0 && threadIdx.x == 0) ctl_begin(d.ctl, label, source, d.nf_delta ? d.nf_delta : kInf);
    const uint32_t n = d.n;
    const uint32_t stride = gridDim.x * kBlock;
    for (uint32_t v = blockIdx.x * kBlock + threadIdx.x; v < n; v += stride) {
        uint32_t lab;
        if (ALG == ALG_CC) lab = v;
        else if (ALG == ALG_SSWP) lab = (v == source) ? kInf : 0u;
        else lab = (v == source) ? 0u : kInf;
        label[v] = lab;
        if (ALG != ALG_BFS) d.snap[v] = lab;
    }
    if (ALG == ALG_BFS) {
        for (uint32_t k = blockIdx.x * kBlock + threadIdx.x; k < d.nwords; k += stride)
            d.V[k] = 0u;                                  // the first scan moves the source from Q to V
    }
    if (ALG == ALG_CC) {
        for (uint32_t k = d.own_w0 + blockIdx.x * kBlock + threadIdx.x; k < d.own_w1; k += stride) {
            const uint32_t lo = k * 32;
            d.Q[k] = lo >= n ? 0u : (n - lo >= 32 ? kFull : ((1u << (n - lo)) - 1u));
        }
    } else if (blockIdx.x == 0 && threadIdx.x == 0 && source >= d.own_lo && source < d.own_hi) {
        d.Q[source >> 5] = 1u << (source & 31);
    }
}

// ------------------------------------------------------------------------- //
// A5/A6 + A2 of the next iteration: bitmap -> compacted active set + UDC scan.
// Scan tile = kScanV vertices; warp w of the CTA owns kWPW consecutive bitmap
// words, and lane l handles bit l of each: for word k the warp looks at the
// 32 consecutive vertices 32k .. 32k+31, so the off[] loads, the label
// writes and the compacted F/B/D/S stores are all coalesced; positions come
// from a ballot/popcount (kept entries) and a warp scan (shadow counts).
// Persistent CTAs take scan tiles in order from a counter, so the chained
// (decoupled look-back) scan always makes progress.  Values are packed
// (kept entries << 32 | shadows); neither half can carry into the other
// (entries <= n < 2^32, shadows < 2^32 checked at load time).
// ------------------------------------------------------------------------- //
#ifndef ETG_WPW
#define ETG_WPW 32
#endif
constexpr int kWPW = ETG_WPW;                             // bitmap words per warp per tile
#ifndef ETG_SCAN_G
#define ETG_SCAN_G 8
#endif
constexpr int kG = ETG_SCAN_G;                            // words whose loads are in flight together
constexpr uint32_t kScanV = (uint32_t)kWarps * kWPW * 32; // vertices per scan tile (8192)
constexpr int kLB = 4;                                    // look-back window: 32 * kLB predecessor tiles

__device__ __forceinline__ void st_volatile_u64(unsigned long long *p, unsigned long long v) {
    asm volatile("st.volatile.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}

// One look-back window (see udc_scan_kernel): records r[k] of tiles p - lane -
// 32k.  Waits (returns without progress) while a needed predecessor has not
// published; else adds the values up to and including the nearest inclusive
// prefix (done) or the whole window (moves p back by the window).
template <int N>
__device__ __forceinline__ void lookback_resolve(const unsigned long long (&r)[N], uint32_t eb, int &p,
                                                 uint32_t &excl, bool &done) {
    const uint32_t lane = lane_id();
    int firstk = N;
    uint32_t first = 32;
    bool wait = false;
#pragma unroll
    for (int k = 0; k < N; ++k) {
        const uint32_t lo = (uint32_t)r[k];
        const bool valid = (lo & ~3u) == eb && (lo & 3u) != 0;
        const uint32_t incl = __ballot_sync(kFull, valid && (lo & 3u) == 2u);
        const uint32_t inval = __ballot_sync(kFull, !valid);
        if (firstk == N) {
            if (incl) {
                firstk = k;
                first = (uint32_t)(__ffs(incl) - 1);
                const uint32_t need = first < 31 ? ((2u << first) - 1u) : kFull;
                if (inval & need) wait = true;
            } else if (inval) {
                wait = true;
            }
        }
    }
    if (wait) return;
    uint32_t v = 0;
#pragma unroll
    for (int k = 0; k < N; ++k)
        if (k < firstk || (k == firstk && lane <= first)) v += (uint32_t)(r[k] >> 32);
    excl += __reduce_add_sync(kFull, v);
    if (firstk < N) done = true;
    else p -= 32 * N;
}

// KW = bitmap words (rows of 32 vertices) per warp: a scan tile covers
// kWarps * KW * 32 vertices.  A warp walks its rows one after another, so KW is
// the length of its dependent chain: large graphs use KW = 32 (8,192-vertex
// tiles, fewest tiles and look-back steps), small ones fewer rows per warp,
// so their scans are short chains on many SMs instead of long ones on few.
template <class OffT, bool UDC, bool BFSLAB, bool P, int KW = kWPW>
__device__ __forceinline__ void scan_phase(const Dev<OffT> &d, cudaGraphConditionalHandle cond, int use_cond) {
    typedef unsigned long long u64;
    __shared__ uint32_t s_tile;
    __shared__ u64 s_prefix;
    __shared__ u64 s_wsum[kWarps];
    static_assert(KW >= 4 && KW <= 32 && (32 % KW) == 0, "rows per warp");
    __shared__ uint32_t s_acts;                           // activations of this CTA (one global atomic)
    __shared__ uint32_t s_far_cnt[kWarps], s_far_min[kWarps];   // near-far statistics per warp
    Ctl *ctl = d.ctl;
    if (threadIdx.x == 0) s_acts = 0;
    const uint32_t epoch = cld<P>(ctl->epoch) & 0x3FFFFFFFu;
    const uint32_t tile_words = (uint32_t)kWarps * KW;
    // tiles of the own range (at least one: its last tile publishes the sizes)
    const uint32_t nscan = max(1u, (d.own_w1 + tile_words - 1) / tile_words - d.scan_t0);
    const uint32_t ts = d.ts, tsl = d.ts_log2;
    const uint32_t lane = lane_id(), warp = threadIdx.x >> 5;
    const uint32_t lt = (1u << lane) - 1u;
    uint32_t *label = cld<P>(ctl->label);
    const uint32_t new_depth = cld<P>(ctl->depth) + 1;    // BFS depth of the vertices in Q
    const uint32_t th = cld<P>(ctl->thresh);              // near-far threshold (SSSP option)
    const bool qmark = !d.nf_delta && (d.tune & kTuneQMark);   // A/B switch: the expand marks Q itself
    const bool stat = !(d.tune & kTuneScanDyn);
    // Offset staging: a warp with at least d.scan_rows active rows copies its
    // KW * 32 + 1 row offsets (rounded up to 16 bytes) into shared memory with
    // ONE bulk copy (cp.async.bulk, completing on the warp's mbarrier), so both
    // passes read off[v], off[v + 1] from shared memory: one memory round trip
    // for the warp's whole range instead of one per group of kG rows and pass.
    // Sparse warps keep the direct loads (a bulk copy moves 4 KB per warp).
    constexpr uint32_t kOffPad = 16u / (uint32_t)sizeof(OffT);
    constexpr uint32_t kOffW = (uint32_t)KW * 32u + kOffPad;   // entries per warp buffer (>= KW * 32 + 1)
    extern __shared__ __align__(128) uint8_t dyn_smem[];
    OffT *soff = nullptr;
    uint16_t *slist = nullptr;                               // vertex-list path: row-local vertex indices
    uint64_t *sbar = nullptr;
    uint32_t bphase = 0;
    const bool can_stage = !P && d.scan_rows != 0;
    if (can_stage) {
        soff = reinterpret_cast<OffT *>(dyn_smem) + (size_t)warp * kOffW;
        sbar = reinterpret_cast<uint64_t *>(dyn_smem + (size_t)kWarps * kOffW * sizeof(OffT)) + warp;
        slist = reinterpret_cast<uint16_t *>(dyn_smem + (size_t)kWarps * (kOffW * sizeof(OffT) + 8u)) +
                (size_t)warp * KW * 32u;
        if (lane == 0) {
            mbar_init(sbar, 1);
            fence_mbar_init();
        }
        __syncwarp();
    }
    for (uint32_t round = 0;; ++round) {
        // first tile = blockIdx.x (CTAs are dispatched in index order, so a
        // tile's predecessors are resident); later tiles from a counter
        if (round > 0 || !stat) {
            if (stat && gridDim.x >= nscan) break;        // every tile was taken in round 0
            if (threadIdx.x == 0) s_tile = (stat ? gridDim.x : 0u) + atomicAdd(&ctl->scan_ctr, 1u);
            __syncwarp();
            __syncthreads();
        }
        const uint32_t tile = (round == 0 && stat) ? blockIdx.x : s_tile;
        __syncthreads();                                  // all have read s_tile before it is reused
        if (tile >= nscan) break;
        const uint32_t wbase = ((tile + d.scan_t0) * kWarps + warp) * KW;   // first word of this warp
        // this warp's words: lane l holds words wbase + l + 32j (read, then cleared
        // -- near-far SSSP keeps the deferred far bits); words outside the own
        // range are not looked at
        uint32_t wq[1];
        {
            const uint32_t wd = wbase + lane;
            wq[0] = (lane < (uint32_t)KW && wd >= d.own_w0 && wd < d.own_w1) ? xld<P>(&d.Q[wd]) : 0u;
        }
        uint32_t far_cnt = 0, far_min = kInf;
        const bool nf = d.nf_delta != 0;
#pragma unroll
        for (int j = 0; j < 1; ++j)
            if (wq[j]) {
                d.Q[wbase + 32 * j + lane] = 0u;
                if (BFSLAB) {
                    // visited from now on (depth written below).  Only bits not
                    // yet in V are new: an expand that read a stale V line (the
                    // persistent loop) may have marked a visited vertex again.
                    const uint32_t vw = xld<P>(&d.V[wbase + 32 * j + lane]);
                    wq[j] &= ~vw;
                    if (wq[j]) d.V[wbase + 32 * j + lane] = vw | wq[j];
                }
            }
        if (!BFSLAB && label && !qmark) {
            // SSSP/CC/SSWP: a vertex is active iff its label moved since it
            // was last expanded (label != snap; the expand marks nothing for
            // them), or init/exchange put it in Q.  Word k of the warp = the
            // ballot over vertices 32k .. 32k+31: coalesced label/snap loads.
            // Near-far SSSP: a moved vertex at distance >= thresh is deferred
            // -- its snapshot is not refreshed, so it stays "moved" and is
            // looked at again by every later scan until the threshold passes it.
            // dirty rows (KW == 32: one RD / FR word per warp): after a sparse
            // expand only the rows it marked and the rows holding deferred
            // vertices can have label != snapshot
            const bool use_rows = KW == 32 && d.dirty_tiles && !P;
            const bool dirty = use_rows && cld<P>(ctl->rd_valid);
            uint32_t far_rows = 0;
            if (dirty) {
                const uint32_t rw = wbase >> 5;
                uint32_t exm = __ldcg(&d.RD[rw]) | __ldcg(&d.FR[rw]);
                uint32_t mine = 0;
                while (exm) {                             // uniform (a word every lane read)
                    uint32_t rr[2 * kG], lv[2 * kG], sv[2 * kG];
#pragma unroll
                    for (int r = 0; r < 2 * kG; ++r) {
                        rr[r] = exm ? (uint32_t)(__ffs(exm) - 1) : 32u;
                        exm &= exm - 1u;
                        const uint32_t v = (wbase + rr[r]) * 32 + lane;
                        lv[r] = 0;
                        sv[r] = 0;
                        if (rr[r] < 32u && v < d.n) {
                            lv[r] = __ldcg(&label[v]);
                            sv[r] = __ldcg(&d.snap[v]);
                        }
                    }
#pragma unroll
                    for (int r = 0; r < 2 * kG; ++r) {
                        if (rr[r] >= 32u) continue;              // uniform
                        const bool moved = lv[r] != sv[r];
                        const bool far = nf && moved && lv[r] >= th;
                        const uint32_t b = __ballot_sync(kFull, moved && !far);
                        if (lane == rr[r]) mine = b;
                        if (moved && !far) d.snap[(wbase + rr[r]) * 32 + lane] = lv[r];   // refresh
                        if (far) {
                            ++far_cnt;
                            far_min = min(far_min, lv[r]);
                        }
                        if (__any_sync(kFull, far)) far_rows |= 1u << rr[r];
                    }
                }
                wq[0] |= mine;
                if (lane == 0) {
                    d.RD[rw] = 0u;                        // consumed
                    d.FR[rw] = far_rows;                  // rows examined now: all rows of the word that had any
                }
            }
#pragma unroll
            for (int j = 0; j < (dirty ? 0 : 1); ++j) {
                uint32_t mine = 0;
                for (uint32_t k0 = 0; k0 < (uint32_t)KW; k0 += 2 * kG) {
                    uint32_t lv[2 * kG], sv[2 * kG];
#pragma unroll
                    for (int r = 0; r < 2 * kG; ++r) {
                        const uint32_t wd = wbase + 32 * j + k0 + r;
                        const uint32_t v = wd * 32 + lane;
                        lv[r] = 0;
                        sv[r] = 0;
                        if (k0 + r < (uint32_t)KW && v < d.n && wd >= d.own_w0 && wd < d.own_w1) {
                            lv[r] = __ldcg(&label[v]);
                            sv[r] = __ldcg(&d.snap[v]);
                        }
                    }
#pragma unroll
                    for (int r = 0; r < 2 * kG; ++r) {
                        const bool moved = lv[r] != sv[r];
                        const bool far = nf && moved && lv[r] >= th;
                        const uint32_t b = __ballot_sync(kFull, moved && !far);
                        if (lane == k0 + r) mine = b;
                        if (moved && !far) d.snap[(wbase + 32 * j + k0 + r) * 32 + lane] = lv[r];   // refresh
                        if (far) {
                            ++far_cnt;
                            far_min = min(far_min, lv[r]);
                        }
                        if (use_rows && __any_sync(kFull, far)) far_rows |= 1u << (k0 + r);
                    }
                }
                wq[j] |= mine;
                if (use_rows && lane == 0) {
                    d.RD[wbase >> 5] = 0u;
                    d.FR[wbase >> 5] = far_rows;
                }
            }
            if (nf) {
                // per-warp partials; one atomic pair per tile (below): the
                // counters are two words every tile updates, so per-warp
                // atomics would serialise thousands of them on one L2 slice
                far_cnt = __reduce_add_sync(kFull, far_cnt);
                far_min = __reduce_min_sync(kFull, far_min);
                if (lane == 0) {
                    s_far_cnt[warp] = far_cnt;
                    s_far_min[warp] = far_min;
                }
            }
        }
        bool staged = false;
        // Sparse rows (mid-size active sets: most rows hold one or two active
        // vertices): the warp lists its active vertices in shared memory (in
        // vertex order) and walks the list 32 at a time, one vertex per lane,
        // instead of paying a whole warp step per row.  nlist = list length;
        // entries are indices into the warp's 32 * KW vertices.
        uint32_t nlist = 0;
        bool use_list = false;
        if (can_stage && !qmark) {
            const uint32_t pc = (uint32_t)__popc(wq[0]);
            const uint32_t rows = __ballot_sync(kFull, wq[0] != 0u);
            const uint32_t pincl = warp_incl_scan(pc);
            nlist = __shfl_sync(kFull, pincl, 31);
            use_list = nlist && (d.scan_list == 2u || (d.scan_list == 1u && (nlist + 31u) / 32u < (uint32_t)__popc(rows)));
            if (use_list) {
                __syncwarp();             // the previous tile's reads of the list are done
                uint32_t o = pincl - pc, m = wq[0];
                while (m) {
                    const uint32_t b = (uint32_t)(__ffs(m) - 1);
                    m &= m - 1u;
                    slist[o++] = (uint16_t)(lane * 32u + b);
                }
                __syncwarp();
            }
        }
        if (can_stage) {
            const uint32_t rows = __ballot_sync(kFull, wq[0] != 0u);
            if ((uint32_t)__popc(rows) >= d.scan_rows) {
                staged = true;
                // an active row holds a vertex < n, so vb < n: at least 2 entries remain
                const u64 vb = (u64)wbase * 32ull;
                const u64 avail = (u64)d.n + 1ull - vb;       // entries of off from vb on
                const uint32_t need = (uint32_t)min((u64)KW * 32ull + 1ull, avail);
                const uint32_t ncopy = (uint32_t)min((u64)kOffW, avail) & ~(kOffPad - 1u);   // whole 16 B
                __syncwarp();
                fence_proxy_async();      // this warp's earlier reads of the buffer before the async write
                if (ncopy && lane == 0) {
                    mbar_expect_tx(sbar, ncopy * (uint32_t)sizeof(OffT));
                    bulk_g2s_plain(soff, d.off + vb, ncopy * (uint32_t)sizeof(OffT), sbar);
                }
                for (uint32_t i = ncopy + lane; i < need; i += 32) soff[i] = __ldg(&d.off[vb + i]);   // array end
                if (ncopy) {
                    mbar_wait(sbar, bphase);
                    bphase ^= 1u;
                }
                __syncwarp();
            }
        }
        // pass 1: this warp's (kept, shadows); groups of kG words, all offset
        // loads of a group issued before use
        u64 wsum = 0;
        uint32_t nbits = 0;
        if (use_list) {
            nbits = nlist;
            for (uint32_t i0 = 0; i0 < nlist; i0 += 32) {
                const uint32_t i = i0 + lane;
                uint32_t c = 0;
                if (i < nlist) {
                    const uint32_t li = slist[i];
                    const uint32_t v = wbase * 32u + li;
                    const OffT b0 = staged ? soff[li] : __ldg(&d.off[v]);
                    const OffT b1 = staged ? soff[li + 1] : __ldg(&d.off[v + 1]);
                    c = udc_count<UDC>((uint32_t)(b1 - b0), d.K, d.K_log2);
                }
                const uint32_t kept = __ballot_sync(kFull, c > 0);
                wsum += ((u64)__popc(kept) << 32) | __reduce_add_sync(kFull, c);
            }
        }
#pragma unroll
        for (int j = 0; j < (use_list ? 0 : 1); ++j) {
            for (uint32_t k0 = 0; k0 < (uint32_t)KW; k0 += kG) {
                uint32_t word[kG], any = 0;
#pragma unroll
                for (int r = 0; r < kG; ++r) {
                    word[r] = __shfl_sync(kFull, wq[j], k0 + r);
                    any |= word[r];
                }
                if (!any) continue;
                OffT ob[kG], oe[kG];
#pragma unroll
                for (int r = 0; r < kG; ++r) {
                    ob[r] = 0;
                    oe[r] = 0;
                    if ((word[r] >> lane) & 1u) {
                        const uint32_t v = (wbase + 32 * j + k0 + r) * 32 + lane;
                        const uint32_t li = (k0 + r) * 32 + lane;
                        ob[r] = staged ? soff[li] : __ldg(&d.off[v]);
                        oe[r] = staged ? soff[li + 1] : __ldg(&d.off[v + 1]);
                    }
                }
#pragma unroll
                for (int r = 0; r < kG; ++r) {
                    if (!word[r]) continue;
                    nbits += __popc(word[r]);
                    const uint32_t c = ((word[r] >> lane) & 1u) ? udc_count<UDC>((uint32_t)(oe[r] - ob[r]), d.K, d.K_log2) : 0u;
                    const uint32_t kept = __ballot_sync(kFull, c > 0);
                    wsum += ((u64)__popc(kept) << 32) | __reduce_add_sync(kFull, c);
                }
            }
        }
        // block scan over the warps (warp order = vertex order)
        if (lane == 0) s_wsum[warp] = wsum;
        __syncwarp();
        __syncthreads();
        u64 wprefix = 0, btotal = 0;
        for (int k = 0; k < kWarps; ++k) {
            const u64 x = s_wsum[k];
            if (k < (int)warp) wprefix += x;
            btotal += x;
        }
        if (threadIdx.x < 32) {
            // Single-pass chained scan, one 64-bit record per tile and per
            // quantity (E = kept entries, S = shadows): value << 32 | epoch << 2
            // | flag (1 aggregate, 2 inclusive prefix).  A record is one aligned
            // 64-bit store, so value and flag are seen together (no fences).
            // Look-back: a window of 32 * kLB predecessors, all loads in flight
            // at once; aggregates are summed up to the nearest inclusive prefix.
            const uint32_t eb = epoch << 2;
            const uint32_t aggE = (uint32_t)(btotal >> 32), aggS = (uint32_t)btotal;
            uint32_t exclE = 0, exclS = 0;
            if (lane == 0) {
                if (d.nf_delta && label && !BFSLAB && !qmark) {
                    // near-far statistics of the tile, visible before its record
                    uint32_t fc = 0, fm = kInf;
                    for (int k = 0; k < kWarps; ++k) {
                        fc += s_far_cnt[k];
                        fm = min(fm, s_far_min[k]);
                    }
                    if (fc) {
                        atomicAdd(&ctl->far_count, fc);
                        atomicMin(&ctl->far_min, fm);
                        __threadfence();
                    }
                }
                const uint32_t fl = tile == 0 ? 2u : 1u;
                st_volatile_u64(&d.recE[tile], ((u64)aggE << 32) | eb | fl);
                st_volatile_u64(&d.recS[tile], ((u64)aggS << 32) | eb | fl);
            }
            // A tile with nothing to write needs no prefix: its aggregate (0)
            // lets successors look past it.  Only the last tile, which
            // publishes the totals, always resolves its prefix.
            if (tile > 0 && (btotal != 0 || tile == nscan - 1)) {
                bool doneE = false, doneS = false;
                int pE = (int)tile - 1, pS = (int)tile - 1;   // nearest predecessor at window position 0
                const u64 none = (u64)(eb | 1u);               // beyond tile 0: an empty aggregate
                while (!(doneE && doneS)) {
                    u64 re[kLB], rs[kLB];
#pragma unroll
                    for (int k = 0; k < kLB; ++k) {
                        const int qE = pE - (int)lane - 32 * k, qS = pS - (int)lane - 32 * k;
                        re[k] = (doneE || qE < 0) ? none : ld_volatile_u64(&d.recE[qE]);
                        rs[k] = (doneS || qS < 0) ? none : ld_volatile_u64(&d.recS[qS]);
                    }
                    if (!doneE) lookback_resolve(re, eb, pE, exclE, doneE);
                    if (!doneS) lookback_resolve(rs, eb, pS, exclS, doneS);
                }
                if (lane == 0) {
                    st_volatile_u64(&d.recE[tile], ((u64)(exclE + aggE) << 32) | eb | 2u);
                    st_volatile_u64(&d.recS[tile], ((u64)(exclS + aggS) << 32) | eb | 2u);
                }
            }
            if (lane == 0) s_prefix = ((u64)exclE << 32) | exclS;
            __syncwarp();
        }
        __syncthreads();
        // pass 2: write the compacted entries, in vertex order, coalesced
        u64 run = s_prefix + wprefix;
        if (use_list) {
            for (uint32_t i0 = 0; i0 < nlist; i0 += 32) {
                const uint32_t i = i0 + lane;
                uint32_t v = 0, c = 0, dg = 0;
                OffT ob = 0;
                if (i < nlist) {
                    const uint32_t li = slist[i];
                    v = wbase * 32u + li;
                    ob = staged ? soff[li] : __ldg(&d.off[v]);
                    dg = (uint32_t)((staged ? soff[li + 1] : __ldg(&d.off[v + 1])) - ob);
                    if (BFSLAB) label[v] = new_depth;         // BFS: depth written once, on compaction
                    c = udc_count<UDC>(dg, d.K, d.K_log2);
                }
                const uint32_t kept = __ballot_sync(kFull, c > 0);
                const uint32_t cincl = __all_sync(kFull, c <= 1u) ? __popc(kept & ((2u << lane) - 1u))
                                                                  : warp_incl_scan(c);
                if (c) {
                    const uint32_t pos = (uint32_t)(run >> 32) + __popc(kept & lt);
                    const uint32_t sh = (uint32_t)run + cincl - c;
                    d.F[pos] = v;
                    d.B[pos] = ob;
                    d.D[pos] = dg;
                    d.S[pos] = sh;
                    if (!BFSLAB && c > 1 && d.snap_used == 2u) d.Lx[pos] = kInf;   // CC: not read yet
                    for (uint32_t t = (sh + ts - 1) >> tsl; (t << tsl) < sh + c; ++t) d.tile_first[t] = pos;
                }
                run += ((u64)__popc(kept) << 32) | __shfl_sync(kFull, cincl, 31);
            }
        }
#pragma unroll
        for (int j = 0; j < (use_list ? 0 : 1); ++j) {
            for (uint32_t k0 = 0; k0 < (uint32_t)KW; k0 += kG) {
                uint32_t word[kG], any = 0;
#pragma unroll
                for (int r = 0; r < kG; ++r) {
                    word[r] = __shfl_sync(kFull, wq[j], k0 + r);
                    any |= word[r];
                }
                if (!any) continue;
                OffT ob[kG], oe[kG];
                uint32_t lv[kG];
#pragma unroll
                for (int r = 0; r < kG; ++r) {
                    ob[r] = 0;
                    oe[r] = 0;
                    lv[r] = 0;
                    if ((word[r] >> lane) & 1u) {
                        const uint32_t v = (wbase + 32 * j + k0 + r) * 32 + lane;
                        const uint32_t li = (k0 + r) * 32 + lane;
                        ob[r] = staged ? soff[li] : __ldg(&d.off[v]);
                        oe[r] = staged ? soff[li + 1] : __ldg(&d.off[v + 1]);
                        if (!BFSLAB && label && qmark) lv[r] = __ldcg(&label[v]);
                    }
                }
#pragma unroll
                for (int r = 0; r < kG; ++r) {
                    if (!word[r]) continue;
                    const bool bit = (word[r] >> lane) & 1u;
                    const uint32_t v = (wbase + 32 * j + k0 + r) * 32 + lane;
                    if (bit) {
                        if (BFSLAB) label[v] = new_depth;         // BFS: depth written once, on compaction
                        else if (label && qmark) d.snap[v] = lv[r];   // refresh the snapshot (Q-mark mode)
                    }
                    const uint32_t dg = (uint32_t)(oe[r] - ob[r]);
                    const uint32_t c = bit ? udc_count<UDC>(dg, d.K, d.K_log2) : 0u;
                    const uint32_t kept = __ballot_sync(kFull, c > 0);
                    // every vertex of the row <= K edges (the common case): the
                    // inclusive prefix of c is a popcount
                    const uint32_t cincl = __all_sync(kFull, c <= 1u) ? __popc(kept & ((2u << lane) - 1u))
                                                                      : warp_incl_scan(c);
                    if (c) {
                        const uint32_t pos = (uint32_t)(run >> 32) + __popc(kept & lt);
                        const uint32_t sh = (uint32_t)run + cincl - c;
                        d.F[pos] = v;
                        d.B[pos] = ob[r];
                        d.D[pos] = dg;
                        d.S[pos] = sh;
                        if (!BFSLAB && c > 1 && d.snap_used == 2u) d.Lx[pos] = kInf;   // CC: not read yet
                        // tiles whose first shadow t*ts lies in [sh, sh + c)
                        for (uint32_t t = (sh + ts - 1) >> tsl; (t << tsl) < sh + c; ++t) d.tile_first[t] = pos;
                    }
                    run += ((u64)__popc(kept) << 32) | __shfl_sync(kFull, cincl, 31);
                }
            }
        }
        if (lane == 0 && nbits) atomicAdd(&s_acts, nbits);
        if (tile == nscan - 1 && threadIdx.x == 0) {
            const u64 total = s_prefix + btotal;
            const uint32_t nF = (uint32_t)(total >> 32), N = (uint32_t)total;
            d.S[nF] = N;
            ctl->nF = nF;
            ctl->nshadow = N;
            ctl->ntiles = (N + ts - 1) >> tsl;
            ctl->tile_ctr = 0;
            ctl->depth = cld<P>(ctl->depth) + 1;
            bool more = nF > 0;
            // (the statistics of other tiles: volatile reads -- this SM's L1 may
            // hold the control block's line from the kernel start)
            if (d.nf_delta && cld<true>(ctl->far_count)) {
                more = true;
                if (nF == 0) {                        // near set empty: next bucket
                    const unsigned long long thn = (unsigned long long)cld<true>(ctl->far_min) + d.nf_delta;
                    ctl->thresh = thn > kInf ? kInf : (uint32_t)thn;
                } else if (!(d.tune & kTuneNearFarClassic)) {   // wave: the threshold advances every iteration
                    const unsigned long long thn = (unsigned long long)th + d.nf_delta;
                    ctl->thresh = thn > kInf ? kInf : (uint32_t)thn;
                }
            }
            ctl->more = more ? 1u : 0u;
            if (use_cond) cudaGraphSetConditional(cond, more ? 1u : 0u);
        }
        __syncwarp();
        __syncthreads();
    }
    if (threadIdx.x == 0 && s_acts) atomicAdd(&ctl->activations, (u64)s_acts);   // result unused: RED
}

// Programmatic dependent launch (the loop's CUDA graph links expand -> scan
// with a programmatic edge): a kernel lets its dependent grid launch at once
// -- the dependent's CTAs take SM slots as this grid's CTAs exit, so there is
// no launch gap -- and waits for its own primary grid (completion and memory
// visibility) before touching anything the primary writes.  Without a
// programmatic edge both instructions are no-ops.
__device__ __forceinline__ void pdl_begin() {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

template <class OffT, bool UDC, bool BFSLAB, int KW = kWPW>
__global__ __launch_bounds__(kBlock, 4) void udc_scan_kernel(Dev<OffT> d, cudaGraphConditionalHandle cond,
                                                          int use_cond) {
    pdl_begin();
    scan_phase<OffT, UDC, BFSLAB, false, KW>(d, cond, use_cond);
}

// ------------------------------------------------------------------------- //
// Tile mapping shared by expand_kernel and udc_dump_kernel.  Every compacted
// entry owns >= 1 shadow, so the entries of tile t lie in [j0, j0 + ts) with
// j0 = tile_first[t] and the window has at most ts + 1 entries of S.
// ------------------------------------------------------------------------- //
template <class OffT>
struct Window {
    uint32_t S[kBlock + 1];
    OffT B[kBlock];
    uint32_t D[kBlock];
    uint32_t F[kBlock];
};

template <class OffT, bool LAB>
__device__ __forceinline__ uint32_t load_window(const Dev<OffT> &d, uint32_t t, uint32_t nF,
                                                Window<OffT> &win) {
    const uint32_t j0 = d.tile_first[t];
    const uint32_t W = min(d.ts + 1, nF + 1 - j0);
    for (uint32_t k = threadIdx.x; k < W; k += kBlock) {
        win.S[k] = d.S[j0 + k];
        if (k < d.ts && j0 + k < nF) {          // entry ts is only the upper fence
            win.B[k] = d.B[j0 + k];
            win.D[k] = d.D[j0 + k];
            if (LAB) win.F[k] = d.F[j0 + k];
        }
    }
    return W;
}

// shadow i -> (entry jj in the window, start, len) per Def. 3 / reading R-2
template <class OffT, bool UDC>
__device__ __forceinline__ uint32_t map_shadow(const Dev<OffT> &d, uint32_t i, uint32_t W,
                                               const Window<OffT> &win, OffT &start, uint32_t &len) {
    uint32_t lo = 0, hi = W;                      // largest jj with S[jj] <= i
    while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (win.S[mid] <= i) lo = mid; else hi = mid;
    }
    if (UDC) {
        const uint32_t qk = (i - win.S[lo]) * d.K;  // < deg, so no overflow
        start = win.B[lo] + (OffT)qk;
        const uint32_t rem = win.D[lo] - qk;
        len = rem < d.K ? rem : d.K;
    } else {
        start = win.B[lo];
        len = win.D[lo];
    }
    return lo;
}

// ------------------------------------------------------------------------- //
// A4: relaxation (Proc. 1 L207 "if label[v'] > label[v] + 1 then label[v'] =
// label[v] + 1").  BFS passes the candidate level + 1 as `lab`.
// ------------------------------------------------------------------------- //
template <int ALG>
__device__ __forceinline__ uint32_t candidate(uint32_t lab, uint32_t w) {
    if (ALG == ALG_SSSP) {
        const unsigned long long s = (unsigned long long)lab + w;
        return s > kCap ? kCap : (uint32_t)s;                 // saturating add (R-9)
    }
    if (ALG == ALG_SSWP) return lab < w ? lab : w;             // max-min (L62)
    return lab;                                                // BFS: level + 1; CC: label[v]
}

template <int ALG>
__device__ __forceinline__ bool improves(uint32_t cand, uint32_t cur) {
    if (ALG == ALG_BFS) return cur == kInf;                    // all writers of a level agree
    if (ALG == ALG_SSWP) return cand > cur;
    return cand < cur;
}

// Commit an improving relaxation.  The plain load saw label[u] worse than
// cand, so after this label[u] is strictly better than its value at some
// moment of this iteration: u changed and is active next iteration, whichever
// thread's value wins (reading R-5: the bitmap de-duplicates).  BFS only sets
// the bit: every discoverer of u in this iteration would write the same depth,
// and the scan that compacts u writes it once.
// SSSP/CC/SSWP set no bit: the scan finds the moved labels by comparing them
// with the iteration-start snapshot (one random access per commit instead of
// two); only the near-far schedule, which defers marks in Q, still sets it.
template <int ALG>
__device__ __forceinline__ void commit(uint32_t *label, uint32_t *Q, uint32_t u, uint32_t cand,
                                       uint64_t pol, bool markQ) {
    if (ALG == ALG_SSWP) red_max(&label[u], cand, pol);
    else if (ALG != ALG_BFS) red_min(&label[u], cand, pol);
    if (ALG == ALG_BFS || markQ) red_or(&Q[u >> 5], 1u << (u & 31), pol);
}

// Fused push exchange: the local label is the proposal cache (and the
// pre-filter's snapshot after the next scan), the owner's copy gets the same
// reduction over peer memory.  System-scope reductions: the owner's next scan
// runs after this kernel has completed on every rank and a host barrier.
__device__ __forceinline__ void red_min_sys(uint32_t *p, uint32_t v) {
    asm volatile("red.relaxed.sys.global.min.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void red_max_sys(uint32_t *p, uint32_t v) {
    asm volatile("red.relaxed.sys.global.max.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}

template <class OffT, int ALG>
__device__ __forceinline__ void commit_peer(const Dev<OffT> &d, uint32_t *label, uint32_t u, uint32_t cand,
                                            uint64_t pol) {
    if (ALG == ALG_SSWP) red_max(&label[u], cand, pol);
    else red_min(&label[u], cand, pol);
    uint32_t q = 0;
#pragma unroll
    for (uint32_t k = 1; k < kMaxPeer; ++k)
        q += (k < d.npeer && u >= d.peer_bounds[k]) ? 1u : 0u;
    if (q != d.peer_rank) {
        if (ALG == ALG_SSWP) red_max_sys(d.peer_label[q] + u, cand);
        else red_min_sys(d.peer_label[q] + u, cand);
    }
}

// ------------------------------------------------------------------------- //
// A2-A5: expand.  Persistent grid; tile t covers shadows [t*ts, t*ts + ts).
// Template switches: UDC (shadows of <= K edges, else one item per vertex),
// IDX (a per-element owner index sidx in shared memory -- needs the UDC bound
// ts*K <= cap_e), SMP (stage the segments in shared memory, Sec. V-B).
// Dynamic shared memory: col_s[cap_e] and w_s[cap_e] (SMP), sidx[cap_e] (IDX).
// ------------------------------------------------------------------------- //
template <class OffT, int ALG, bool UDC, bool IDX, bool SMP>
__global__ __launch_bounds__(kBlock) void expand_kernel(Dev<OffT> d, uint32_t cap_e) {
    extern __shared__ __align__(128) uint8_t dyn_smem[];
    constexpr bool kW = (ALG == ALG_SSSP || ALG == ALG_SSWP);
    constexpr bool kLab = (ALG != ALG_BFS);
    __shared__ Window<OffT> win;
    __shared__ OffT sb[kBlock];          // slice start in col
    __shared__ uint32_t so[kBlock + 1];  // flat offset of the slice in the tile
    __shared__ uint32_t slab[kBlock];    // source label of each shadow
    __shared__ uint32_t s_wsum[kWarps];

    uint32_t *col_s = reinterpret_cast<uint32_t *>(dyn_smem);
    uint32_t *w_s = col_s + cap_e;
    uint8_t *sidx = SMP ? reinterpret_cast<uint8_t *>(kW ? (w_s + cap_e) : w_s) : dyn_smem;

    Ctl *ctl = d.ctl;
    const uint32_t nF = ctl->nF, N = ctl->nshadow, ntiles = ctl->ntiles;
    const uint32_t level = ctl->depth + 1;
    uint32_t *label = ctl->label;
    uint32_t *Q = d.Q;
    const uint32_t tid = threadIdx.x;
    const bool l1 = (d.tune & kTuneFilterL1) != 0;
    const uint64_t keep = policy_keep();
    unsigned long long my_edges = 0;
    if (blockIdx.x == 0 && tid == 0) {
        // bookkeeping for the scan that follows this kernel (stream-ordered)
        ctl->scan_ctr = 0;
        ctl->far_min = kInf;
        ctl->far_count = 0;
        ctl->epoch += 1;
        if (nF) ctl->iterations += 1;
        ctl->frontier += nF;
        ctl->shadows += N;
    }

    for (uint32_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const uint32_t W = load_window<OffT, kLab>(d, t, nF, win);
        const uint32_t cnt = min(d.ts, N - (t << d.ts_log2));
        __syncthreads();
        uint32_t len = 0;
        OffT start = 0;
        uint32_t lab = level;
        if (tid < cnt) {
            const uint32_t jj = map_shadow<OffT, UDC>(d, (t << d.ts_log2) + tid, W, win, start, len);
            if (kLab) lab = ld_cg(&label[win.F[jj]]);      // fresh source label (R-6)
        }
        uint32_t E;
        const uint32_t excl = block_excl_scan<uint32_t>(len, s_wsum, E);
        sb[tid] = start;
        so[tid] = excl;
        slab[tid] = lab;
        if (tid == 0) so[kBlock] = E;
        if (IDX) {
            // owner index of every element of this shadow's slice (len <= K)
            uint32_t a = excl;
            const uint32_t e = excl + len;
            const uint32_t pat = tid * 0x01010101u;
            while (a < e && (a & 3u)) sidx[a++] = (uint8_t)tid;
            for (; a + 4 <= e; a += 4) *reinterpret_cast<uint32_t *>(&sidx[a]) = pat;
            while (a < e) sidx[a++] = (uint8_t)tid;
        }
        __syncthreads();
        if (SMP) {
            // SMP (Sec. V-B): stage the tile's segments into shared memory, one
            // element per thread (consecutive threads -> consecutive words).
            for (uint32_t x = tid; x < E; x += kBlock) {
                const uint32_t s = sidx[x];
                const OffT e = sb[s] + (OffT)(x - so[s]);
                cp_async4(&col_s[x], &d.col[e]);
                if (kW) cp_async4(&w_s[x], &d.w[e]);
            }
            cp_async_wait_all();
            __syncthreads();
        }
        // A4 + A5 in batches of kR edges per thread: the batch's label loads
        // are all issued before any is consumed; commits never wait.
        for (uint32_t x0 = 0; x0 < E; x0 += kBlock * kR) {
            uint32_t u[kR], c[kR], cur[kR];
            bool act[kR];
#pragma unroll
            for (int r = 0; r < kR; ++r) {
                const uint32_t x = x0 + r * kBlock + tid;
                act[r] = x < E;
                u[r] = 0;
                c[r] = 0;
                if (act[r]) {
                    uint32_t s, w = 0;
                    if (IDX) {
                        s = sidx[x];
                    } else {
                        uint32_t lo = 0, hi = cnt;            // largest s with so[s] <= x
                        while (hi - lo > 1) {
                            const uint32_t mid = (lo + hi) >> 1;
                            if (so[mid] <= x) lo = mid; else hi = mid;
                        }
                        s = lo;
                    }
                    if (SMP) {
                        u[r] = col_s[x];
                        if (kW) w = w_s[x];
                    } else {
                        const OffT e = sb[s] + (OffT)(x - so[s]);
                        u[r] = __ldg(&d.col[e]);
                        if (kW) w = __ldg(&d.w[e]);
                    }
                    c[r] = candidate<ALG>(slab[s], w);
                }
            }
#pragma unroll
            for (int r = 0; r < kR; ++r)
                cur[r] = act[r] ? (l1 ? ld_ca(&label[u[r]]) : ld_cg(&label[u[r]])) : 0u;
#pragma unroll
            for (int r = 0; r < kR; ++r)
                if (act[r] && improves<ALG>(c[r], cur[r])) commit<ALG>(label, Q, u[r], c[r], keep, (d.tune & kTuneQMark) != 0);
        }
        my_edges += E;
        __syncthreads();
    }
    if (tid == 0 && my_edges) atomicAdd(&ctl->edges, my_edges);
}

// ------------------------------------------------------------------------- //
// Warp-centric expand (the default).  One warp owns a tile of 32 consecutive
// shadow vertices (ts = 32) and processes it with registers and warp
// intrinsics only -- no shared memory, no block barrier -- so the random label
// gathers are the only traffic in the SM's memory pipe.
//
// warp_map: lane i gets shadow t*32 + i.  The tile's entries j0 .. j0+31
// (j0 = tile_first[t]) are loaded one per lane; entry j > j0 starts a shadow
// inside the tile at position p_j = S[j] - 32t, so OR-reducing 1 << p_j gives
// the mask of entry starts, and the entry owning position i is j0 plus the
// number of starts at positions <= i (entry j0 covers position 0).
// ------------------------------------------------------------------------- //
template <class OffT, bool UDC>
struct WarpShadow {
    OffT start;
    uint32_t len;
    uint32_t v;
    uint32_t j;        // its entry in the compacted active set
    bool sole;         // the vertex's only shadow (its whole row)
};

template <class OffT, bool UDC, bool P = false>
__device__ __forceinline__ WarpShadow<OffT, UDC> warp_map(const Dev<OffT> &d, uint32_t t, uint32_t nF,
                                                          uint32_t N) {
    const uint32_t lane = lane_id();
    const uint32_t j0 = xld<P>(&d.tile_first[t]);
    const uint32_t j = j0 + lane;
    uint32_t Sj = kInf, Dj = 0, Fj = 0;
    OffT Bj = 0;
    if (j < nF) {
        Sj = xld<P>(&d.S[j]);
        Bj = xld<P>(&d.B[j]);
        Dj = xld<P>(&d.D[j]);
        Fj = xld<P>(&d.F[j]);
    }
    const uint32_t base = t << 5;
    const uint32_t p = Sj - base;                              // wraps to huge if Sj < base
    const uint32_t startmask = __reduce_or_sync(kFull, (lane > 0 && p < 32u) ? (1u << p) : 0u);
    const uint32_t jj = __popc(startmask & ((2u << lane) - 1u));
    const uint32_t sS = __shfl_sync(kFull, Sj, jj);
    const OffT sB = __shfl_sync(kFull, Bj, jj);
    const uint32_t sD = __shfl_sync(kFull, Dj, jj);
    WarpShadow<OffT, UDC> r;
    r.v = __shfl_sync(kFull, Fj, jj);
    r.j = j0 + jj;
    r.len = 0;
    r.start = 0;
    r.sole = !UDC || sD <= d.K;
    const uint32_t i = base + lane;
    if (i < N) {
        if (UDC) {
            const uint32_t qk = (i - sS) * d.K;              // < deg
            r.start = sB + (OffT)qk;
            const uint32_t rem = sD - qk;
            r.len = rem < d.K ? rem : d.K;
        } else {
            r.start = sB;
            r.len = sD;
        }
    }
    return r;
}

// Per-tile state of a warp: its 32 shadows and where their edges live.
template <class OffT, bool UDC>
struct WarpTile {
    WarpShadow<OffT, UDC> sh;
    uint32_t o;        // flat offset of this lane's slice in the tile
    uint32_t E;        // edges in the tile
    OffT delta;        // element x of this lane's slice is col[delta + x]      (direct)
    uint32_t sdelta;   // ... and stage[sdelta + x] in shared memory            (SMP)
    uint32_t x0;       // first batch of this warp-unit (tile split: unit / ntiles batches in)
};

template <class OffT, int ALG, bool UDC, bool SMP, bool P, bool PEER = false>
__device__ __forceinline__ void expand_phase(const Dev<OffT> &d, uint32_t capw) {
    constexpr bool kW = (ALG == ALG_SSSP || ALG == ALG_SSWP);
    constexpr uint32_t kArrays = kW ? 2u : 1u;
    constexpr int kRB = kW ? ETG_KR_W : kR;                // chunks per batch (weighted: fewer, no spills)
    extern __shared__ __align__(128) uint8_t dyn_smem[];
    Ctl *ctl = d.ctl;
    const uint32_t nF = cld<P>(ctl->nF), N = cld<P>(ctl->nshadow), ntiles = cld<P>(ctl->ntiles);
    const uint32_t level = cld<P>(ctl->depth) + 1;
    uint32_t *label = cld<P>(ctl->label);
    uint32_t *Q = d.Q;
    const uint32_t lane = lane_id();
    const uint32_t lt_eq = (2u << lane) - 1u;
    const uint32_t wib = threadIdx.x >> 5;                 // warp in block
    const uint64_t keep = policy_keep(), stream = policy_stream();
    unsigned long long my_edges = 0;
    uint32_t my_passes = 0;                               // replay experiment counter
    // dirty rows: a sparse launch marks the rows of the labels it lowers
    const bool mark_rows = !P && ALG != ALG_BFS && d.dirty_tiles && ntiles <= d.dirty_tiles;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        // bookkeeping for the scan that follows this kernel (stream-ordered)
        ctl->rd_valid = mark_rows ? 1u : 0u;
        ctl->scan_ctr = 0;
        ctl->epoch = cld<P>(ctl->epoch) + 1;
        ctl->far_min = kInf;
        ctl->far_count = 0;
        if (nF) ctl->iterations = cld<P>(ctl->iterations) + 1;
        ctl->frontier = cld<P>(ctl->frontier) + nF;
        ctl->shadows = cld<P>(ctl->shadows) + N;
    }
    // SMP: two shared-memory stages per warp, each kArrays x capw words, and
    // one mbarrier per stage (the TMA bulk copies complete on it).
    uint32_t *wbuf = nullptr;
    uint64_t *bars = nullptr;
    if (SMP) {
        wbuf = reinterpret_cast<uint32_t *>(dyn_smem) + (size_t)wib * 2u * kArrays * capw;
        bars = reinterpret_cast<uint64_t *>(dyn_smem + (size_t)kWarps * 2u * kArrays * capw * 4u) + 2u * wib;
        if (lane == 0) {
            mbar_init(&bars[0], 1);
            mbar_init(&bars[1], 1);
            fence_mbar_init();
        }
        __syncwarp();
    }
    const OffT m_floor4 = (OffT)(d.m & ~3ull);            // whole 16-byte groups inside col/w

    // Dynamic schedule: a warp grabs kGrab consecutive tiles at a time, so the
    // slowest warp ends within one grab of the rest (tiles carry 32..32K edges).
    // The first grab is static (global warp index), later ones come from the
    // counter: a small active set costs no atomic at all, and a large one
    // one atomic per grab after the first.
    // Tile split (sparse iterations): with fewer tiles than warps, G warps share
    // each tile, warp-unit u taking tile u % ntiles and its batches u / ntiles,
    // u / ntiles + G, ... -- a hub's edges are not walked by one warp alone.
    uint32_t G = 1;
#if ETG_PIPE
    if (!SMP && !P && d.split && ntiles) {
        const uint32_t per = (gridDim.x * kWarps) / ntiles;
        G = per >= 8 ? 8u : per >= 4 ? 4u : per >= 2 ? 2u : 1u;
        if (G > d.split) G = d.split;
    }
#endif
    const uint32_t nunits = ntiles * G;
    // two tiles per grab only when there are plenty (>= 4 per warp): with fewer,
    // a static grab of two would leave half of the warps without a tile
    const uint32_t mid = (nunits < 4u * gridDim.x * kWarps) ? 1u : 0u;
    const uint32_t kGrab = (G > 1 || (mid && (d.tune2 & 1u) == 0)) ? 1u : 2u;
    const uint32_t n_static = gridDim.x * kWarps * kGrab;
    uint32_t g_next = 0, g_end = 0;
    bool first_grab = true;
    auto next_tile = [&]() -> uint32_t {
        if (g_next == g_end) {
            uint32_t g = 0;
            if (first_grab && ETG_SGRAB) {
                g = (blockIdx.x * kWarps + wib) * kGrab;
                first_grab = false;
            } else {
                const uint32_t base = ETG_SGRAB ? n_static : 0u;
                if (lane == 0 && base < nunits) g = base + atomicAdd(&ctl->tile_ctr, kGrab);
                g = base < nunits ? __shfl_sync(kFull, g, 0) : nunits;
            }
            g_next = g;
            g_end = g_next >= nunits ? g_next : min(g_next + kGrab, nunits);
            if (g_next >= nunits) return nunits;
        }
        return g_next++;
    };
    // Map tile t and start fetching its neighbour segments: SMP -> TMA bulk
    // copies into stage `st` (Sec. V-B: fetch the shadow's neighbours to
    // shared memory before processing them); direct -> L2 bulk prefetch.
    auto prepare = [&](uint32_t u, uint32_t st) -> WarpTile<OffT, UDC> {
        WarpTile<OffT, UDC> w;
        const uint32_t t = G > 1 ? u % ntiles : u;
        w.x0 = G > 1 ? (u / ntiles) * 32u * (uint32_t)kRB : 0u;
        w.sh = warp_map<OffT, UDC, P>(d, t, nF, N);
        const uint32_t incl = warp_incl_scan(w.sh.len);
        w.o = incl - w.sh.len;
        w.E = __shfl_sync(kFull, incl, 31);
        w.delta = w.sh.start - (OffT)w.o;
        w.sdelta = 0;
        if (SMP) {
            // 16-byte-aligned superset of the slice (reading R-3: the over-fetched
            // words are never relaxed); the tail past the last whole 16-byte
            // group of col is loaded by the lane itself.
            const OffT a_lo = w.sh.start & ~(OffT)3;
            OffT a_hi = (w.sh.start + w.sh.len + 3) & ~(OffT)3;
            const uint32_t pw = w.sh.len ? (uint32_t)(a_hi - a_lo) : 0u;
            const uint32_t pincl = warp_incl_scan(pw);
            const uint32_t slot = pincl - pw;
            const uint32_t T = __shfl_sync(kFull, pincl, 31);
            w.sdelta = slot + (uint32_t)(w.sh.start - a_lo) - w.o;
            uint32_t *buf = wbuf + (size_t)st * kArrays * capw;
            if (a_hi > m_floor4) a_hi = a_lo > m_floor4 ? a_lo : m_floor4;
            const uint32_t tma_words = w.sh.len ? (uint32_t)(a_hi - a_lo) : 0u;
            const uint32_t tma_total = __reduce_add_sync(kFull, tma_words);
            if (lane == 0) mbar_expect_tx(&bars[st], tma_total * 4u * kArrays);
            __syncwarp();
            fence_proxy_async();
            if (tma_words) {
                bulk_g2s(buf + slot, d.col + a_lo, tma_words * 4u, &bars[st], stream);
                if (kW) bulk_g2s(buf + capw + slot, d.w + a_lo, tma_words * 4u, &bars[st], stream);
            }
            // tail words [a_hi, start + len) (only the slice that ends the edge array)
            for (OffT e = a_hi > w.sh.start ? a_hi : w.sh.start; e < w.sh.start + w.sh.len; ++e) {
                buf[slot + (uint32_t)(e - a_lo)] = d.col[e];
                if (kW) buf[capw + slot + (uint32_t)(e - a_lo)] = d.w[e];
            }
            (void)T;
        } else if (w.sh.len && d.prefetch) {
            // whole 16-byte groups inside col only (never past the array's end)
            const uintptr_t lo = reinterpret_cast<uintptr_t>(d.col + w.sh.start) & ~(uintptr_t)15;
            uintptr_t hi = (reinterpret_cast<uintptr_t>(d.col + w.sh.start + w.sh.len) + 15) & ~(uintptr_t)15;
            const uintptr_t end = reinterpret_cast<uintptr_t>(d.col + m_floor4);
            if (hi > end) hi = end;
            if (hi > lo) prefetch_l2(reinterpret_cast<const void *>(lo), (uint32_t)(hi - lo));
            if (kW && hi > lo)
                prefetch_l2(reinterpret_cast<const void *>(lo - reinterpret_cast<uintptr_t>(d.col) +
                                                           reinterpret_cast<uintptr_t>(d.w)),
                            (uint32_t)(hi - lo));
        }
        return w;
    };

#if ETG_PIPE
    // Software pipeline over the warp's stream of batches (kRB chunks of 32
    // elements; a tile is one or more batches).  Stage A of batch b+1 (owner
    // masks, column/weight loads, candidates) is issued before stage B of batch
    // b (label gathers, commits), so the column loads of the next batch are in
    // flight while the gathers of this one are: one memory latency per batch
    // instead of two.  Stage B needs only registers, so a tile's shared-memory
    // stage (SMP) can be refilled once stage A has left the tile.
    const bool markQ = (d.tune & kTuneQMark) != 0;   // near-far defers through the snapshot, not Q
    // BFS: live labels; else the snapshot (R-4, R-6), or the live labels when
    // label + snapshot do not fit in L2 (one random stream instead of two)
    const uint32_t *filt = (ALG == ALG_BFS || d.filt_live) ? label : d.snap;
    const uint32_t xstep = 32u * (uint32_t)kRB * G;       // batch stride of a warp-unit
    uint32_t t = next_tile();
    if (t < nunits) {
        WarpTile<OffT, UDC> nxt = prepare(t, 0);
        // stage-A cursor: tile A_t (sequence number kt), batch start A_x0
        WarpTile<OffT, UDC> A_t = nxt;
        uint32_t kt = 0;
        uint32_t tn = next_tile();
        if (tn < nunits) nxt = prepare(tn, 1);
        // fresh source label (R-6).  Single GPU: a vertex expanded by a sole
        // shadow records the label it propagates in the snapshot, so the scan
        // re-activates it only if its label moves after this read (R-5).
        const bool snap_used = ALG != ALG_BFS && d.snap_used;
        // A vertex cut into several shadows (Def. 3): the first of its shadows
        // to start publishes the label it read in Lx (compare-and-swap on
        // the "not read" INF), and every shadow propagates that one value, so
        // it can be recorded in the snapshot too (snap_used == 2).
        auto src_label = [&](const WarpShadow<OffT, UDC> &sh) -> uint32_t {
            if (!sh.len) return 0u;
            uint32_t l = ld_cg(&label[sh.v]);
            if (snap_used) {
                if (sh.sole) {
                    // (tile split: the slice may straddle two warps' batches, read
                    // at different times -- the snapshot keeps the scan-time value)
                    if (G == 1) d.snap[sh.v] = l;
                } else if ((ALG == ALG_CC || (ETG_SHARED_SSSP && ALG == ALG_SSSP)) && d.snap_used == 2u) {
#if ETG_LX_PEEK
                    // published already? (a plain load: hubs of many shadows do not
                    // serialise on one compare-and-swap)
                    uint32_t o = ld_cg(&d.Lx[sh.j]);
                    if (o == kInf) o = atomicCAS(&d.Lx[sh.j], kInf, l);
#else
                    const uint32_t o = atomicCAS(&d.Lx[sh.j], kInf, l);
#endif
                    if (o != kInf) l = o;
                    d.snap[sh.v] = l;
                }
            }
            return l;
        };
        uint32_t A_lab = (ALG == ALG_BFS) ? level : src_label(A_t.sh);
        uint32_t A_x0 = A_t.x0, A_owner = 0xFFFFFFFFu;
        const uint32_t *A_sbuf = nullptr;
        if (SMP) {
            mbar_wait(&bars[0], 0);
            __syncwarp();
            A_sbuf = wbuf;
        }
        if (A_t.x0 == 0) my_edges += A_t.E;
        bool A_valid = true;
        uint32_t u0[kRB], c0[kRB], w0[kRB], u1[kRB], c1[kRB], w1[kRB];
        uint32_t am0 = 0, am1 = 0;
        // stage A: the batch at (A_t, A_x0) into (u, c, am); then advance the cursor
        auto stage_a = [&](uint32_t (&u)[kRB], uint32_t (&c)[kRB], uint32_t (&wv)[kRB], uint32_t &am) {
            // owner of the element before the batch (tile split: batches are skipped)
            if (G > 1) A_owner = (uint32_t)__popc(__ballot_sync(kFull, A_t.sh.len && A_t.o < A_x0)) - 1u;
            const uint32_t pos = A_t.o - A_x0;                 // this lane's slice start in the batch
            const bool in_win = A_t.sh.len && pos < 32u * kRB;
            uint32_t wm[kRB];
#pragma unroll
            for (int r = 0; r < kRB; ++r)
                wm[r] = __reduce_or_sync(kFull, (in_win && (pos >> 5) == (uint32_t)r) ? (1u << (pos & 31)) : 0u);
            am = 0;
#pragma unroll
            for (int r = 0; r < kRB; ++r) {
                const uint32_t own = A_owner + __popc(wm[r] & lt_eq);
                A_owner += __popc(wm[r]);
                const uint32_t src = own & 31u;
                const uint32_t ll = (ALG == ALG_BFS) ? level : __shfl_sync(kFull, A_lab, src);
                const uint32_t x = A_x0 + 32u * r + lane;
                const bool act = x < A_t.E;
                am |= act ? (1u << r) : 0u;
                u[r] = 0;
                c[r] = ll;
                wv[r] = 0;
                if (SMP) {
                    const uint32_t sd = __shfl_sync(kFull, A_t.sdelta, src);
                    if (act) {
                        u[r] = A_sbuf[sd + x];
                        if (kW) wv[r] = A_sbuf[capw + sd + x];
                    }
                } else {
                    const OffT dl = __shfl_sync(kFull, A_t.delta, src);
                    if (act) {
                        const OffT e = dl + (OffT)x;
                        u[r] = ld_stream(&d.col[e], stream);
                        if (kW) wv[r] = ld_stream(&d.w[e], stream);
                    }
                }
            }
            // (the candidates need the weights: computed in stage B, so the
            // column and weight loads of this batch stay in flight until then)
            // advance: next batch of this tile, or the next tile
            A_x0 += xstep;
            if (A_x0 >= A_t.E) {
                if (tn >= nunits) {
                    A_valid = false;
                } else {
                    A_t = nxt;
                    ++kt;
                    tn = next_tile();
                    if (tn < nunits) nxt = prepare(tn, (kt + 1) & 1);   // refills the stage of tile kt-1
                    A_lab = (ALG == ALG_BFS) ? level : src_label(A_t.sh);
                    A_x0 = A_t.x0;                             // (>= E: an empty unit, one empty batch)
                    A_owner = 0xFFFFFFFFu;
                    if (A_t.x0 == 0) my_edges += A_t.E;
                    if (SMP) {
                        mbar_wait(&bars[kt & 1], (kt >> 1) & 1);
                        __syncwarp();
                        A_sbuf = wbuf + (size_t)(kt & 1) * kArrays * capw;
                    }
                }
            }
        };
        // stage B: pre-filter gathers, then fire-and-forget commits
        auto stage_b = [&](const uint32_t (&u)[kRB], uint32_t (&c)[kRB], const uint32_t (&wv)[kRB], uint32_t am) {
            if (kW) {
#pragma unroll
                for (int r = 0; r < kRB; ++r) c[r] = candidate<ALG>(c[r], wv[r]);
            }
            if (d.tune & kTuneNoGather) {                     // replay experiment
                uint32_t x = 0;
#pragma unroll
                for (int r = 0; r < kRB; ++r) x += ((am >> r) & 1u) ? u[r] + c[r] : 0u;
                if (x == 0x9E3779B9u) Q[0] = x;
                return;
            }
            uint32_t cur[kRB];
            if (d.tune & kTuneNoFilter) {                     // A/B: every edge commits
#pragma unroll
                for (int r = 0; r < kRB; ++r) cur[r] = (ALG == ALG_SSWP) ? 0u : kInf;
            } else if (ALG == ALG_BFS) {
                // visited test on the bitmap V (n/8 bytes, read-only in this
                // kernel, cached in L1: hits never reach the L2 request path)
#pragma unroll
                for (int r = 0; r < kRB; ++r)
                    cur[r] = ((am >> r) & 1u) ? ((((P ? ld_ca(&d.V[u[r] >> 5]) : __ldg(&d.V[u[r] >> 5])) >> (u[r] & 31)) & 1u) ? 0u : kInf) : 0u;
            } else if (ALG == ALG_CC && level == 1) {
                // CC's first expand: the snapshot is still the initial labelling
                // label[u] = u (A1), so the pre-filter needs no gather at all
#pragma unroll
                for (int r = 0; r < kRB; ++r) cur[r] = u[r];
            } else {
#pragma unroll
                for (int r = 0; r < kRB; ++r) cur[r] = ((am >> r) & 1u) ? ld_label(&filt[u[r]], keep) : 0u;
            }
            if (d.tune & kTuneNoCommit) {                     // replay experiment: count passes
                uint32_t x = 0;
#pragma unroll
                for (int r = 0; r < kRB; ++r) x += (((am >> r) & 1u) && improves<ALG>(c[r], cur[r])) ? 1u : 0u;
                my_passes += x;
                return;
            }
            if constexpr (PEER && ALG != ALG_BFS) {
#pragma unroll
                for (int r = 0; r < kRB; ++r)
                    if (((am >> r) & 1u) && improves<ALG>(c[r], cur[r])) commit_peer<OffT, ALG>(d, label, u[r], c[r], keep);
            } else {
#pragma unroll
                for (int r = 0; r < kRB; ++r)
                    if (((am >> r) & 1u) && improves<ALG>(c[r], cur[r])) {
                        commit<ALG>(label, Q, u[r], c[r], keep, markQ);
                        if (ALG != ALG_BFS && mark_rows) red_or(&d.RD[u[r] >> 10], 1u << ((u[r] >> 5) & 31u), keep);
                    }
            }
        };
        stage_a(u0, c0, w0, am0);
        // look-ahead: d.ahead (BFS), and every algorithm in mid-size
        // iterations (fewer than 4 tiles per warp: latency-bound, each warp
        // walks a few batches back to back)
        if (!(d.ahead || (mid && d.ahead_mid))) {
            // ETG_NO_SMP ("w/o SMP" ablation): each batch's segments are loaded
            // and relaxed back to back, nothing is fetched ahead of its use
            for (;;) {
                stage_b(u0, c0, w0, am0);
                if (!A_valid) break;
                stage_a(u0, c0, w0, am0);
            }
        } else for (;;) {
            // two named register sets alternate, so no copies between iterations
            const bool more1 = A_valid;
            if (more1) stage_a(u1, c1, w1, am1);
            stage_b(u0, c0, w0, am0);
            if (!more1) break;
            const bool more0 = A_valid;
            if (more0) stage_a(u0, c0, w0, am0);
            stage_b(u1, c1, w1, am1);
            if (!more0) break;
        }
    }
#else
    uint32_t t = next_tile();
    if (t < ntiles) {
        WarpTile<OffT, UDC> nxt = prepare(t, 0);
        for (uint32_t k = 0;; ++k) {
            const WarpTile<OffT, UDC> cur_t = nxt;
            const uint32_t tn = next_tile();
            if (tn < ntiles) nxt = prepare(tn, (k + 1) & 1);   // one tile ahead
            const WarpShadow<OffT, UDC> &sh = cur_t.sh;
            const uint32_t o = cur_t.o, E = cur_t.E;
            const uint32_t lab = (ALG == ALG_BFS) ? level
                                 : (sh.len ? ld_cg(&label[sh.v]) : 0u);   // fresh source label (R-6)
            my_edges += E;
            const uint32_t *sbuf = nullptr;
            if (SMP) {
                mbar_wait(&bars[k & 1], (k >> 1) & 1);
                __syncwarp();
                sbuf = wbuf + (size_t)(k & 1) * kArrays * capw;
            }
            uint32_t owner = 0xFFFFFFFFu;                     // owner of the element before x0
            // Batches of kRB chunks of 32 elements.  The owner of element x is
            // the number of slice starts <= x, minus one: the batch's kRB words of
            // the start mask come from kRB independent OR-reductions, then a
            // popcount prefix -- no serial dependency between chunks.
            for (uint32_t x0 = 0; x0 < E; x0 += 32u * kRB) {
                uint32_t u[kRB], c[kRB], cur[kRB], wv[kRB];
                bool act[kRB];
                const uint32_t pos = o - x0;                  // this lane's slice start in the batch
                const bool in_win = sh.len && pos < 32u * kRB;
                uint32_t wm[kRB];
#pragma unroll
                for (int r = 0; r < kRB; ++r)
                    wm[r] = __reduce_or_sync(kFull, (in_win && (pos >> 5) == (uint32_t)r) ? (1u << (pos & 31)) : 0u);
#pragma unroll
                for (int r = 0; r < kRB; ++r) {
                    const uint32_t own = owner + __popc(wm[r] & lt_eq);
                    owner += __popc(wm[r]);
                    const uint32_t src = own & 31u;
                    const uint32_t ll = (ALG == ALG_BFS) ? level : __shfl_sync(kFull, lab, src);
                    const uint32_t x = x0 + 32u * r + lane;
                    act[r] = x < E;
                    u[r] = 0;
                    c[r] = ll;
                    wv[r] = 0;
                    if (SMP) {
                        const uint32_t sd = __shfl_sync(kFull, cur_t.sdelta, src);
                        if (act[r]) {
                            u[r] = sbuf[sd + x];
                            if (kW) wv[r] = sbuf[capw + sd + x];
                        }
                    } else {
                        const OffT dl = __shfl_sync(kFull, cur_t.delta, src);
                        if (act[r]) {
                            const OffT e = dl + (OffT)x;
                            u[r] = ld_stream(&d.col[e], stream);
                            if (kW) wv[r] = ld_stream(&d.w[e], stream);
                        }
                    }
                }
                if (kW) {
#pragma unroll
                    for (int r = 0; r < kRB; ++r) c[r] = candidate<ALG>(c[r], wv[r]);
                }
                if (d.tune & kTuneNoGather) {                 // replay experiment
                    uint32_t x = 0;
#pragma unroll
                    for (int r = 0; r < kRB; ++r) x += act[r] ? u[r] + c[r] : 0u;
                    if (x == 0x9E3779B9u) Q[0] = x;
                    continue;
                }
                // pre-filter: BFS reads the labels (written only by the scan);
                // the others read the iteration-start snapshot, so the gathers
                // and the red.min/max commits never touch the same lines (R-4, R-6)
                const uint32_t *filt = (ALG == ALG_BFS) ? label : d.snap;
#pragma unroll
                for (int r = 0; r < kRB; ++r) cur[r] = act[r] ? ld_label(&filt[u[r]], keep) : 0u;
                if (d.tune & kTuneNoCommit) {                 // replay experiment: count passes
                    uint32_t x = 0;
#pragma unroll
                    for (int r = 0; r < kRB; ++r) x += (act[r] && improves<ALG>(c[r], cur[r])) ? 1u : 0u;
                    my_passes += x;
                    continue;
                }
#pragma unroll
                for (int r = 0; r < kRB; ++r)
                    if (act[r] && improves<ALG>(c[r], cur[r])) commit<ALG>(label, Q, u[r], c[r], keep, (d.tune & kTuneQMark) != 0);
            }
            if (tn >= ntiles) break;
        }
    }
#endif
    // statistics: one global atomic per CTA (per-warp partials in shared memory)
    __shared__ unsigned long long s_edges;
    __syncwarp();                                         // reconverge before the block barrier
    if (threadIdx.x == 0) s_edges = 0;
    __syncthreads();
    if (lane == 0 && my_edges) atomicAdd(&s_edges, my_edges);
    __syncthreads();
    if (threadIdx.x == 0 && s_edges) atomicAdd(&ctl->edges, s_edges);
    if (d.tune & kTuneNoCommit) {
        my_passes = __reduce_add_sync(kFull, my_passes);
        if (lane == 0 && my_passes) atomicAdd(&ctl->reached_v, (unsigned long long)my_passes);
    }
}

template <class OffT, int ALG, bool UDC, bool SMP, bool PEER = false>
__global__ __launch_bounds__(kBlock, ETG_MINB) void expand_warp_kernel(Dev<OffT> d, uint32_t capw) {
    pdl_begin();
    expand_phase<OffT, ALG, UDC, SMP, false, PEER>(d, capw);
}

// ------------------------------------------------------------------------- //
// A6 as one persistent kernel: the whole "while actSet.isNotEmpty()" loop of
// Proc. 1 (L207) -- expand (A2-A5), grid barrier, scan (A5 + A2 of the next
// iteration), grid barrier -- in one cooperative launch, so an iteration pays
// two barriers instead of two kernel launches.  Same phase code as the
// separate kernels; cross-phase reads bypass L1 (P = true).
// ------------------------------------------------------------------------- //
__device__ __forceinline__ unsigned long long globaltimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

// Grid barrier over a monotone arrival counter (zeroed by ctl_begin_kernel):
// barrier k of the call completes when the counter reaches k * gridDim.x.
// Release on arrival, acquire on exit.  All CTAs are co-resident (cooperative
// launch), so it cannot deadlock; a spin longer than ~10 s traps instead of
// hanging the device.
__device__ __forceinline__ void grid_barrier(uint32_t *bar, uint32_t &k) {
    __syncthreads();
    ++k;
    if (threadIdx.x == 0) {
        const uint32_t target = k * gridDim.x;
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" :: "l"(bar) : "memory");
        const long long t0 = clock64();
        for (;;) {
            uint32_t v;
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(bar) : "memory");
            if ((int)(v - target) >= 0) break;
            if (clock64() - t0 > 20000000000ll) __trap();
#if ETG_BAR_SLEEP
            __nanosleep(ETG_BAR_SLEEP);
#endif
        }
    }
    __syncthreads();
}

template <class OffT, int ALG, bool UDC>
__global__ __launch_bounds__(kBlock, ETG_MINB) void loop_kernel(Dev<OffT> d, uint32_t capw) {
    Ctl *ctl = d.ctl;
    uint32_t k = 0;
    const bool timer = blockIdx.x == 0 && threadIdx.x == 0;
    while (cld<true>(ctl->more)) {
        const unsigned long long t0 = timer ? globaltimer() : 0ull;
        expand_phase<OffT, ALG, UDC, false, true>(d, capw);
        grid_barrier(&ctl->bar, k);
        const unsigned long long t1 = timer ? globaltimer() : 0ull;
        scan_phase<OffT, UDC, ALG == ALG_BFS, true>(d, 0, 0);
        grid_barrier(&ctl->bar, k);
        if (timer) {
            const unsigned long long t2 = globaltimer();
            ctl->t_expand_ns = cld<true>(ctl->t_expand_ns) + (t1 - t0);
            ctl->t_scan_ns = cld<true>(ctl->t_scan_ns) + (t2 - t1);
        }
    }
}

// ------------------------------------------------------------------------- //
// A2 debug dump: the (v, start, end) of every shadow, via the same mapping.
// ------------------------------------------------------------------------- //
template <class OffT, bool UDC>
__global__ __launch_bounds__(kBlock) void udc_dump_kernel(Dev<OffT> d, uint32_t *out_id,
                                                           uint64_t *out_start, uint64_t *out_end) {
    __shared__ Window<OffT> win;
    Ctl *ctl = d.ctl;
    const uint32_t nF = ctl->nF, N = ctl->nshadow, ntiles = ctl->ntiles;
    for (uint32_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const uint32_t W = load_window<OffT, true>(d, t, nF, win);
        const uint32_t cnt = min(d.ts, N - (t << d.ts_log2));
        __syncthreads();
        if (threadIdx.x < cnt) {
            const uint32_t i = (t << d.ts_log2) + threadIdx.x;
            OffT start;
            uint32_t len;
            const uint32_t jj = map_shadow<OffT, UDC>(d, i, W, win, start, len);
            out_id[i] = win.F[jj];
            out_start[i] = (uint64_t)start;
            out_end[i] = (uint64_t)start + len;
        }
        __syncthreads();
    }
}

// Mark the vertices of an explicit active set in Q (debug entry etg_udc_slices).
__global__ void mark_kernel(uint32_t *Q, const uint32_t *act, uint32_t n_act) {
    for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < n_act; k += gridDim.x * blockDim.x)
        atomicOr(&Q[act[k] >> 5], 1u << (act[k] & 31));
}

// Fused destination-partition exchange (replaces the all-gather of owned
// slices): the owner of [lo, hi) stores what changed in its range straight
// into every peer's copy -- BFS: the non-zero words of its bitmap Q (no other
// rank marks those vertices, so a plain store is the union); SSSP/CC/SSWP:
// the labels that moved this iteration (label != snapshot).
struct PeerSet {
    uint32_t P, rank;
    uint32_t *ptr[kMaxPeer];    // peer q's Q (BFS) or label array, mapped into this process
};

template <bool BFS>
__global__ __launch_bounds__(kBlock) void publish_kernel(const uint32_t *Q, const uint32_t *label,
                                                         const uint32_t *snap, uint32_t lo, uint32_t hi,
                                                         PeerSet ps) {
    const uint32_t stride = gridDim.x * blockDim.x;
    const uint32_t a = BFS ? lo >> 5 : lo, b = BFS ? (hi + 31) >> 5 : hi;
    for (uint32_t i = a + blockIdx.x * blockDim.x + threadIdx.x; i < b; i += stride) {
        uint32_t x;
        if (BFS) {
            x = Q[i];
            if (!x) continue;
        } else {
            x = __ldcg(&label[i]);
            if (x == __ldcg(&snap[i])) continue;
        }
        for (uint32_t q = 0; q < ps.P; ++q)
            if (q != ps.rank) ps.ptr[q][i] = x;
    }
}

// ------------------------------------------------------------------------- //
// statistics and validation
// ------------------------------------------------------------------------- //
// Sum of the edge weights (ETG_SSSP_DELTA_AUTO) into ctl->reached_e.
__global__ __launch_bounds__(kBlock) void weight_sum_kernel(const uint32_t *w, unsigned long long m, Ctl *ctl) {
    unsigned long long acc = 0;
    for (unsigned long long e = blockIdx.x * (unsigned long long)kBlock + threadIdx.x; e < m;
         e += (unsigned long long)gridDim.x * kBlock)
        acc += __ldcs(&w[e]);
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(kFull, acc, o);
    if (lane_id() == 0 && acc) atomicAdd(&ctl->reached_e, acc);
}

template <class OffT>
__global__ __launch_bounds__(kBlock) void reach_kernel(Dev<OffT> d, const uint32_t *label,
                                                        uint32_t unreached) {
    unsigned long long rv = 0, re = 0;
    for (uint32_t v = blockIdx.x * kBlock + threadIdx.x; v < d.n; v += gridDim.x * kBlock) {
        if (label[v] != unreached) {
            rv += 1;
            re += (unsigned long long)(d.off[v + 1] - d.off[v]);
        }
    }
    for (int o = 16; o > 0; o >>= 1) {
        rv += __shfl_xor_sync(kFull, rv, o);
        re += __shfl_xor_sync(kFull, re, o);
    }
    if (lane_id() == 0 && (rv || re)) {
        atomicAdd(&d.ctl->reached_v, rv);
        atomicAdd(&d.ctl->reached_e, re);
    }
}

template <class OffT>
__global__ __launch_bounds__(kBlock) void validate_kernel(Dev<OffT> d, unsigned long long m) {
    const uint64_t gsz = (uint64_t)gridDim.x * kBlock;
    const uint64_t t0 = (uint64_t)blockIdx.x * kBlock + threadIdx.x;
    if (t0 == 0 && (d.off[0] != 0 || (unsigned long long)d.off[d.n] != m)) atomicOr(&d.ctl->error, 1u);
    for (uint64_t v = t0; v < d.n; v += gsz) {
        if (d.off[v + 1] < d.off[v]) atomicOr(&d.ctl->error, 2u);
        else if ((unsigned long long)(d.off[v + 1] - d.off[v]) > 0xFFFFFFFFull) atomicOr(&d.ctl->error, 8u);
    }
    for (uint64_t e = t0; e < m; e += gsz)
        if (d.col[e] >= d.n) atomicOr(&d.ctl->error, 4u);
}

}  // namespace etg
