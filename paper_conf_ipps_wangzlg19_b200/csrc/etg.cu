// etg.cu -- host engine and C ABI of libetg.so (see include/etg.h).
//
// The engine owns nothing on the device: the CSR and a caller-provided
// workspace are borrowed (etg_load_csr).  Per traversal call it enqueues, on the
// handle's stream: ctl_begin + init (A1) and the first udc_scan, then the
// Proc. 1 while-loop as a CUDA graph with a conditional WHILE
// node whose body is expand -> udc_scan (A2-A6); the scan's last tile sets the
// loop condition on the device, so the host synchronises once per call, not
// once per iteration.  ETG_HOST_LOOP replaces the graph by a host loop that
// reads the active-set size back every iteration (the paper's own control flow).
#include <cuda.h>
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nvtx3/nvToolsExt.h>   // header-only: ranges cost nothing unless a tool is attached

#include <algorithm>
#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>

#include "../../include/etg.h"
#include "etg_comm.h"
#include "etg_kernels.cuh"

using namespace etg;

namespace {

thread_local std::string g_err;

uint32_t env_tune() {
    const char *t = getenv("ETG_TUNE");
    return t ? (uint32_t)strtoul(t, nullptr, 0) : 0u;
}
std::atomic<uint64_t> g_launches{0};

etg_status fail(etg_status s, const std::string &msg) {
    g_err = msg;
    return s;
}

#define ETG_CU(call)                                                                          \
    do {                                                                                      \
        cudaError_t e_ = (call);                                                              \
        if (e_ != cudaSuccess) {                                                              \
            return fail(ETG_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_));     \
        }                                                                                     \
    } while (0)

constexpr size_t kAlign = 256;
size_t align_up(size_t x) { return (x + kAlign - 1) & ~(kAlign - 1); }

struct Params {
    uint32_t K;
    uint32_t ts;
    uint32_t ts_log2;
    bool udc;
    bool warp;  // warp-centric expand (ts = 32, registers only); else the CTA-tile kernel
    bool idx;   // per-element owner index in shared memory (needs ts*K <= kCapE)
    bool smp;
    bool prefetch;  // warp kernel: L2 bulk prefetch of the next tile's segments (ETG_TUNE 128)
    bool ahead;     // warp kernel: next batch's segments loaded one batch ahead (SMP; off: ETG_NO_SMP)
    bool u64;
    bool persist;   // the iteration loop as one persistent cooperative kernel (loop_kernel)
    uint32_t nf_delta;  // near-far SSSP bucket width (0 = paper schedule)
};

Params derive(const etg_options *opt, uint32_t tune) {
    Params p;
    p.warp = !(tune & 2u);
    p.nf_delta = opt ? opt->sssp_delta : 0u;
    const uint32_t flags = opt ? opt->flags : 0u;
    p.K = (opt && opt->degree_limit_k) ? opt->degree_limit_k : 32u;
    p.udc = !(flags & ETG_NO_UDC);
    p.u64 = (flags & ETG_OFFSETS_U64) != 0;
    // tile of ts shadows; SMP stages at most ts*K words (the UDC bound, L199)
    constexpr uint32_t kCapE = 8192;
    p.ts = kBlock;
    if (p.udc && p.K > kCapE / kBlock) {
        uint32_t ts = kBlock;
        while (ts > 32 && ts * (uint64_t)p.K > kCapE) ts >>= 1;
        p.ts = ts;
    }
    p.idx = p.udc && (uint64_t)p.ts * p.K <= kCapE;
    p.smp = p.idx && !(flags & ETG_NO_SMP);
    p.prefetch = false;
    p.ahead = !(flags & ETG_NO_SMP);
    if (p.warp) {
        // warp kernel: tiles of 32 shadows; SMP = per-warp TMA stages of
        // 32 * (K + 6) words, affordable in shared memory for K <= 32
        p.ts = 32;
        p.idx = false;
        const bool host_edges = (flags & ETG_HOST_EDGES) != 0;   // no TMA on host-mapped memory
        p.smp = p.udc && (flags & ETG_SMP_SHARED) && !(flags & ETG_NO_SMP) && p.K <= 32 && !host_edges;
        // the bulk prefetch is issued per lane through the uniform datapath (a
        // 32-way serialised loop in SASS): measured slower than the register
        // look-ahead alone, so it is an experiment switch only
        p.prefetch = p.udc && (tune & 128u) && !(flags & ETG_NO_SMP) && !p.smp && !host_edges;
    }
    p.persist = p.warp && !p.smp && (tune & kTunePersist);
    p.ts_log2 = 0;
    while ((1u << p.ts_log2) < p.ts) ++p.ts_log2;
    return p;
}

struct Layout {
    size_t Q, Lfull, V, snap, F, B, D, S, Lx, tile_first, recE, recS, RD, FR, ctl, total;
    uint32_t nwords;
};

Layout layout(uint64_t n, uint64_t m, const Params &p) {
    Layout L;
    size_t o = 0;
    auto take = [&](size_t bytes) {
        size_t at = o;
        o = align_up(o + bytes);
        return at;
    };
    const uint64_t max_shadows = p.udc ? (m + p.K - 1) / p.K + n : n;   // sum ceil(d/K) <= m/K + |F|
    const uint64_t max_tiles = (max_shadows + 31) / 32 + 2;      // sized for the smallest tile (32)
    const uint64_t max_scan_tiles = (n + 1023) / 1024 + 2;      // sized for the smallest scan tile (4 rows per warp)
    const uint64_t words = (n + 31) / 32;
    const uint64_t tile_words = kScanV / 32;
    L.nwords = (uint32_t)((words + tile_words - 1) / tile_words * tile_words);
    L.Q = take(4ull * L.nwords);
    L.Lfull = take(4 * (n + 1));   // communicator handles: the full-size label array (peers write into it)
    L.V = take(4ull * L.nwords);
    L.snap = take(4 * (n + 1));
    L.F = take(4 * (n + 1));
    L.B = take((p.u64 ? 8 : 4) * (n + 1));
    L.D = take(4 * (n + 1));
    L.S = take(4 * (n + 2));
    L.Lx = take(4 * (n + 1));
    L.tile_first = take(4 * max_tiles);
    L.recE = take(8 * max_scan_tiles);
    L.recS = take(8 * max_scan_tiles);
    L.RD = take(4ull * ((L.nwords + 31) / 32));      // dirty rows (one bit per 32 vertices)
    L.FR = take(4ull * ((L.nwords + 31) / 32));      // rows holding deferred (near-far) vertices
    L.ctl = take(sizeof(Ctl));
    L.total = o;
    return L;
}

}  // namespace

struct etg_comm {
    etg::Comm c;
};

struct etg_graph {
    uint64_t n = 0, m = 0;
    uint32_t flags = 0;
    Params p{};
    const void *off = nullptr;
    const uint32_t *col = nullptr;
    const uint32_t *w = nullptr;
    cudaStream_t stream = nullptr;
    uint8_t *ws = nullptr;
    Layout L{};
    Ctl *ctl = nullptr;
    int num_sms = 0;
    int l2_bytes = 0;
    uint32_t tune = 0;                    // ETG_TUNE (experiments only)
    int grid_scan = 0;
    int scan_kw = kWPW;                   // bitmap words per scan warp (tile = 8 x scan_kw x 32 vertices)
    uint32_t scan_smem = 0;               // scan: dynamic shared memory (offset staging buffers + mbarriers)
    uint32_t scan_rows = 0;               // scan: active rows from which a warp stages its offsets (0: never)
    uint32_t split = 8;                   // expand: max warps sharing one tile in sparse iterations (ETG_SPLIT)
    uint32_t ahead_mid = 1;               // expand: look-ahead in mid-size iterations for every algorithm (ETG_AHEAD_MID)
    uint32_t tune2 = 0;                   // experiment bits (ETG_TUNE2)
    bool dirty = true;                    // dirty-row scans after sparse expands (ETG_DIRTY=0: off)
    uint32_t scan_list = 1;               // scan: vertex-list path 0 never, 1 for sparse rows, 2 always (ETG_SCAN_LIST)
    bool pdl = false;                     // loop graph: programmatic expand -> scan edges (ETG_PDL=1; measured
                                          // 1 % slower on C2, per-iteration floor unchanged: off by default)
    int grid_init = 0;
    Ctl *h_ctl = nullptr;                 // pinned host mirror for readback
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    cudaEvent_t pev[3] = {nullptr, nullptr, nullptr};   // ETG_PROFILE: scan / expand brackets
    int step_alg = -1;                    // algorithm of the step-wise (distributed) run
    uint32_t *step_label = nullptr;       // its label array
    uint32_t npeer = 0, peer_rank = 0;    // ETG_PUSH communicator handles: the fused push exchange
    uint32_t peer_bounds[kMaxPeer + 1] = {};
    uint32_t *peer_label[kMaxPeer] = {};
    uint32_t dpeer = 0, dpeer_rank = 0;   // destination-partition communicator handles: publish targets
    uint32_t dpeer_lo = 0, dpeer_hi = 0;
    uint32_t *dpeer_Q[kMaxPeer] = {};
    uint32_t *dpeer_label[kMaxPeer] = {};
    uint64_t step_launches = 0;
    uint64_t step_acts = 0;               // activations counted so far (cumulative)
    bool delta_auto = false;              // sssp_delta was ETG_SSSP_DELTA_AUTO at load (sticky)
    bool has_w = false;                   // weights given (or no edges)
    etg::Comm *comm = nullptr;            // communicator (borrowed), NULL = single partition
    bool push = false;                    // ETG_PUSH: source partition + fused push exchange
    uint32_t v_lo = 0, v_hi = 0;          // owned vertex range
    void *ipc_base[kMaxPeer] = {};        // peer workspaces mapped with cudaIpcOpenMemHandle
    cudaGraphExec_t exec[4] = {nullptr, nullptr, nullptr, nullptr};
    int grid_loop[4] = {0, 0, 0, 0};      // loop_kernel grid per algorithm (resident CTAs x SMs)
    cudaGraph_t graph[4] = {nullptr, nullptr, nullptr, nullptr};
};

namespace {

template <class OffT>
Dev<OffT> make_dev(const etg_graph *g, int alg = -1) {
    Dev<OffT> d;
    d.nf_delta = (alg == ALG_SSSP) ? g->p.nf_delta : 0u;
    d.off = static_cast<const OffT *>(g->off);
    d.col = g->col;
    d.w = g->w;
    d.Q = reinterpret_cast<uint32_t *>(g->ws + g->L.Q);
    d.V = reinterpret_cast<uint32_t *>(g->ws + g->L.V);
    d.nwords = g->L.nwords;
    d.snap = reinterpret_cast<uint32_t *>(g->ws + g->L.snap);
    d.F = reinterpret_cast<uint32_t *>(g->ws + g->L.F);
    d.B = reinterpret_cast<OffT *>(g->ws + g->L.B);
    d.D = reinterpret_cast<uint32_t *>(g->ws + g->L.D);
    d.S = reinterpret_cast<uint32_t *>(g->ws + g->L.S);
    d.Lx = reinterpret_cast<uint32_t *>(g->ws + g->L.Lx);
    d.tile_first = reinterpret_cast<uint32_t *>(g->ws + g->L.tile_first);
    d.recE = reinterpret_cast<unsigned long long *>(g->ws + g->L.recE);
    d.recS = reinterpret_cast<unsigned long long *>(g->ws + g->L.recS);
    d.ctl = g->ctl;
    d.n = (uint32_t)g->n;
    d.m = g->m;
    d.prefetch = g->p.prefetch ? 1u : 0u;
    // SMP look-ahead (the next batch's segments loaded while this one relaxes):
    // BFS, SSSP and SSWP -- the weighted ones since their candidates are formed
    // in stage B (SSSP C2 1.835 -> 1.79 ms, C3 2.24 -> 2.15 ms); not CC, whose
    // plain batch loop measured faster (1.232 vs 1.26 ms on C2)
    d.ahead = (g->p.ahead && (alg != ALG_CC || (g->tune & kTuneAheadAll))) ? 1u : 0u;
    d.K = g->p.K;
    d.K_log2 = 32;
    if (d.K && !(d.K & (d.K - 1))) {
        d.K_log2 = 0;
        while ((1u << d.K_log2) < d.K) ++d.K_log2;
    }
    d.ts = g->p.ts;
    d.ts_log2 = g->p.ts_log2;
    d.tune = g->tune;
    d.snap_used = 0;
    // the pre-filter's gather array: the snapshot keeps the gathers and the
    // red.min commits on different lines while both fit in L2 (C2: 2 x 16.8 MB);
    // beyond L2 (C4: 2 x 166 MB vs 126 MB) every random access is a DRAM sector,
    // and gathering the live labels halves the randomly accessed bytes
    d.filt_live = (g->tune & kTuneFiltLive) ? 1u
                  : (g->tune & kTuneFiltSnap) ? 0u
                  : (8ull * g->n > (uint64_t)g->l2_bytes ? 1u : 0u);
    // own range: a push-partition rank activates only the vertices it owns (the
    // only ones with local out-edges), so its init and scans cover [v_lo, v_hi)
    // -- scan cost falls with P; the foreign labels it lowers (its proposal
    // cache) are never re-scanned, so its pre-filter reads the live labels
    const bool own = g->push && g->comm;
    d.own_lo = own ? g->v_lo : 0u;
    d.own_hi = own ? g->v_hi : (uint32_t)g->n;
    d.own_w0 = d.own_lo >> 5;
    d.own_w1 = own ? (uint32_t)((g->v_hi + 31ull) >> 5) : g->L.nwords;
    if (d.own_w1 < d.own_w0) d.own_w1 = d.own_w0;
    d.scan_t0 = d.own_w0 / ((uint32_t)kWarps * (uint32_t)g->scan_kw);
    if (own) d.filt_live = 1u;
    d.scan_rows = g->scan_smem ? g->scan_rows : 0u;
    d.split = g->split;
    d.scan_list = g->scan_list;
    d.RD = reinterpret_cast<uint32_t *>(g->ws + g->L.RD);
    d.FR = reinterpret_cast<uint32_t *>(g->ws + g->L.FR);
    d.dirty_tiles = 0;                        // the fused single-GPU loop only (make_dev_fused)
    d.ahead_mid = g->p.ahead ? g->ahead_mid : 0u;
    d.tune2 = g->tune2;
    d.npeer = g->npeer;
    d.peer_rank = g->peer_rank;
    for (uint32_t k = 0; k <= kMaxPeer; ++k) d.peer_bounds[k] = g->peer_bounds[k];
    for (uint32_t k = 0; k < kMaxPeer; ++k) d.peer_label[k] = g->peer_label[k];
    return d;
}

// Dev of the fused single-GPU loop: the snapshot also records the label each
// sole shadow expanded with (not in the step-wise path, whose ranks must
// agree on the activated set).
template <class OffT>
Dev<OffT> make_dev_fused(const etg_graph *g, int alg) {
    Dev<OffT> d = make_dev<OffT>(g, alg);
    d.npeer = 0;                              // the fused loop is single-partition
    // dirty rows: SSSP/CC/SSWP with 32-row scan warps; an expand with at most
    // one tile per warp marks the rows it lowers labels in (ETG_DIRTY=0: off)
    if (alg != ALG_BFS && g->scan_kw == 32 && g->dirty && !g->comm)
        d.dirty_tiles = (uint32_t)g->num_sms * 3u * (uint32_t)kWarps;
    // 2 = multi-shadow vertices share one published label too -- CC only:
    // measured 1.48 -> 1.28 ms on C2; SSSP 1.96 -> 2.03 and SSWP 2.13 ->
    // 2.17 (the compare-and-swap round trip per tile costs more than the
    // re-expansions it saves), so they record sole shadows only
    d.snap_used = (alg != ALG_BFS && !(g->tune & (kTuneQMark | kTuneNoSnapUsed)))
                      ? (((alg != ALG_CC && !(ETG_SHARED_SSSP && alg == ALG_SSSP)) || (g->tune & kTuneNoSharedLabel))
                             ? 1u : 2u) : 0u;
    return d;
}

// --- kernel selection ------------------------------------------------------ //
template <class OffT, int ALG>
const void *expand_fn(bool udc, bool idx, bool smp) {
    if (!udc) return (const void *)expand_kernel<OffT, ALG, false, false, false>;
    if (smp) return (const void *)expand_kernel<OffT, ALG, true, true, true>;
    if (idx) return (const void *)expand_kernel<OffT, ALG, true, true, false>;
    return (const void *)expand_kernel<OffT, ALG, true, false, false>;
}

template <class OffT, int ALG>
const void *expand_warp_fn(bool udc, bool smp, bool peer = false) {
    if (peer && ALG != ALG_BFS)     // fused push exchange (step-wise runs only)
        return udc ? (const void *)expand_warp_kernel<OffT, ALG, true, false, true>
                   : (const void *)expand_warp_kernel<OffT, ALG, false, false, true>;
    if (!udc) return (const void *)expand_warp_kernel<OffT, ALG, false, false>;
    return smp ? (const void *)expand_warp_kernel<OffT, ALG, true, true>
               : (const void *)expand_warp_kernel<OffT, ALG, true, false>;
}

template <class OffT>
const void *expand_fn_alg(int alg, bool udc, bool idx, bool smp, bool warp, bool peer = false) {
    if (warp) {
        switch (alg) {
            case ALG_BFS: return expand_warp_fn<OffT, ALG_BFS>(udc, smp);
            case ALG_SSSP: return expand_warp_fn<OffT, ALG_SSSP>(udc, smp, peer);
            case ALG_CC: return expand_warp_fn<OffT, ALG_CC>(udc, smp, peer);
            default: return expand_warp_fn<OffT, ALG_SSWP>(udc, smp, peer);
        }
    }
    switch (alg) {
        case ALG_BFS: return expand_fn<OffT, ALG_BFS>(udc, idx, smp);
        case ALG_SSSP: return expand_fn<OffT, ALG_SSSP>(udc, idx, smp);
        case ALG_CC: return expand_fn<OffT, ALG_CC>(udc, idx, smp);
        default: return expand_fn<OffT, ALG_SSWP>(udc, idx, smp);
    }
}

template <class OffT, int ALG>
const void *loop_fn_udc(bool udc) {
    return udc ? (const void *)loop_kernel<OffT, ALG, true> : (const void *)loop_kernel<OffT, ALG, false>;
}

template <class OffT>
const void *loop_fn(int alg, bool udc) {
    switch (alg) {
        case ALG_BFS: return loop_fn_udc<OffT, ALG_BFS>(udc);
        case ALG_SSSP: return loop_fn_udc<OffT, ALG_SSSP>(udc);
        case ALG_CC: return loop_fn_udc<OffT, ALG_CC>(udc);
        default: return loop_fn_udc<OffT, ALG_SSWP>(udc);
    }
}

template <class OffT>
const void *init_fn(int alg) {
    switch (alg) {
        case ALG_BFS: return (const void *)init_kernel<OffT, ALG_BFS>;
        case ALG_SSSP: return (const void *)init_kernel<OffT, ALG_SSSP>;
        case ALG_CC: return (const void *)init_kernel<OffT, ALG_CC>;
        default: return (const void *)init_kernel<OffT, ALG_SSWP>;
    }
}

template <class OffT, int KW>
const void *scan_fn_kw(bool udc, int alg) {
    if (alg == ALG_BFS)
        return udc ? (const void *)udc_scan_kernel<OffT, true, true, KW> : (const void *)udc_scan_kernel<OffT, false, true, KW>;
    return udc ? (const void *)udc_scan_kernel<OffT, true, false, KW> : (const void *)udc_scan_kernel<OffT, false, false, KW>;
}

// the scan kernel of a handle: KW = g->scan_kw bitmap words (rows) per warp
template <class OffT>
const void *scan_fn(const etg_graph *g, int alg) {
    switch (g->scan_kw) {
        case 4: return scan_fn_kw<OffT, 4>(g->p.udc, alg);
        case 8: return scan_fn_kw<OffT, 8>(g->p.udc, alg);
        case 16: return scan_fn_kw<OffT, 16>(g->p.udc, alg);
        default: return scan_fn_kw<OffT, kWPW>(g->p.udc, alg);
    }
}

// one scan launch on stream s (the handle's grid and shared memory)
template <class OffT>
cudaError_t launch_scan(const etg_graph *g, int alg, void **args, cudaStream_t s) {
    return cudaLaunchKernel(scan_fn<OffT>(g, alg), dim3(g->grid_scan), dim3(kBlock), args, g->scan_smem, s);
}

// shared memory of the scan kernels with KW rows per warp: per warp KW * 32 + 1
// offsets rounded up to 16 bytes, one mbarrier, and the vertex list (KW * 32
// 16-bit indices)
template <class OffT>
uint32_t scan_smem_bytes(int kw) {
    return (uint32_t)(kWarps * ((uint32_t)kw * 32u + 16u / (uint32_t)sizeof(OffT)) * sizeof(OffT) + kWarps * 8 +
                      kWarps * (uint32_t)kw * 32u * 2u);
}

// second argument of the expand kernels: CTA kernel -> staging capacity in
// edges; warp kernel -> words per SMP stage array
uint32_t expand_arg(const Params &p) { return p.warp ? 32u * (p.K + 6u) : p.ts * p.K; }

size_t expand_smem(const Params &p, int alg) {
    const bool kw = (alg == ALG_SSSP || alg == ALG_SSWP);
    if (p.warp) return p.smp ? (size_t)kWarps * 2 * (kw ? 2 : 1) * expand_arg(p) * 4 + kWarps * 16 : 0;
    if (!p.idx) return 0;
    const size_t cap = (size_t)p.ts * p.K;
    return (p.smp ? cap * 4 * (kw ? 2 : 1) : 0) + cap;
}

struct Launch {
    const void *fn;
    dim3 grid;
    size_t smem;
};

template <class OffT>
etg_status expand_launch(etg_graph *g, int alg, Launch &out, bool peer = false) {
    out.fn = expand_fn_alg<OffT>(alg, g->p.udc, g->p.idx, peer ? false : g->p.smp, g->p.warp, peer);
    out.smem = peer ? 0 : expand_smem(g->p, alg);
    ETG_CU(cudaFuncSetAttribute(out.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)out.smem));
    // no dynamic shared memory: leave the unified L1/shared array to L1 (the
    // BFS visited bitmap is read through it); SMP stages: maximum shared memory
    ETG_CU(cudaFuncSetAttribute(out.fn, cudaFuncAttributePreferredSharedMemoryCarveout,
                                out.smem ? 100 : 0));
    int nb = 0;
    ETG_CU(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, out.fn, kBlock, out.smem));
    if (nb < 1) nb = 1;
    out.grid = dim3((unsigned)(nb * g->num_sms));
    return ETG_OK;
}

// Build the while-loop graph for one algorithm (lazily, cached per handle).
template <class OffT>
etg_status build_graph(etg_graph *g, int alg) {
    if (g->exec[alg]) return ETG_OK;
    Dev<OffT> d = make_dev_fused<OffT>(g, alg);
    Launch ex;
    etg_status s = expand_launch<OffT>(g, alg, ex);
    if (s != ETG_OK) return s;
    uint32_t cap_e = expand_arg(g->p);
    cudaGraph_t graph;
    ETG_CU(cudaGraphCreate(&graph, 0));
    cudaGraphConditionalHandle cond;
    ETG_CU(cudaGraphConditionalHandleCreate(&cond, graph, 1, cudaGraphCondAssignDefault));
    cudaGraphNodeParams cp = {};
    cp.type = cudaGraphNodeTypeConditional;
    cp.conditional.handle = cond;
    cp.conditional.type = cudaGraphCondTypeWhile;
    cp.conditional.size = 1;
    cudaGraphNode_t cnode;
    ETG_CU(cudaGraphAddNode(&cnode, graph, nullptr, 0, &cp));
    cudaGraph_t body = cp.conditional.phGraph_out[0];

    cudaKernelNodeParams kp;
    cudaGraphNode_t n_scan, n_exp;
    void *exp_args[] = {&d, &cap_e};
    memset(&kp, 0, sizeof(kp));
    kp.func = const_cast<void *>(ex.fn);
    kp.gridDim = ex.grid;
    kp.blockDim = dim3(kBlock);
    kp.sharedMemBytes = (unsigned)ex.smem;
    kp.kernelParams = exp_args;
    ETG_CU(cudaGraphAddKernelNode(&n_exp, body, nullptr, 0, &kp));

    int use_cond = 1;
    void *scan_args[] = {&d, &cond, &use_cond};
    // expand -> scan: a programmatic edge (PDL, ETG_PDL=0 disables) -- the
    // scan grid launches while the expand drains and waits on the device
    cudaGraphNodeParams np = {};
    np.type = cudaGraphNodeTypeKernel;
    np.kernel.func = const_cast<void *>(scan_fn<OffT>(g, alg));
    np.kernel.gridDim = dim3(g->grid_scan);
    np.kernel.blockDim = dim3(kBlock);
    np.kernel.sharedMemBytes = g->scan_smem;
    np.kernel.kernelParams = scan_args;
    cudaGraphEdgeData ed = {};
    if (g->pdl) {
        ed.from_port = cudaGraphKernelNodePortProgrammatic;
        ed.type = cudaGraphDependencyTypeProgrammatic;
    }
    ETG_CU(cudaGraphAddNode_v2(&n_scan, body, &n_exp, &ed, 1, &np));

    cudaError_t ie = cudaGraphInstantiate(&g->exec[alg], graph, 0);
    if (ie != cudaSuccess && g->pdl) {
        // programmatic edges not accepted here: plain edges
        (void)cudaGetLastError();
        cudaGraphDestroy(graph);
        g->pdl = false;
        return build_graph<OffT>(g, alg);
    }
    ETG_CU(ie);
    g->graph[alg] = graph;
    return ETG_OK;
}

template <class OffT>
etg_status run_impl(etg_graph *g, int alg, uint32_t source, uint32_t *label, etg_stats *st) {
    Dev<OffT> d = make_dev_fused<OffT>(g, alg);
    cudaStream_t s = g->stream;
    const bool profile = (g->flags & ETG_PROFILE) != 0;
    const bool host_loop = profile || (g->flags & ETG_HOST_LOOP) != 0;
    float scan_ms = 0.f, expand_ms = 0.f;
    uint32_t expand_launches = 0;
    const bool persist = !host_loop && g->p.persist;
    if (persist && !g->grid_loop[alg]) {
        const void *fn = loop_fn<OffT>(alg, g->p.udc);
        ETG_CU(cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, 0));
        int nb = 0;
        ETG_CU(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, kBlock, 0));
        if (nb < 1) return fail(ETG_ECUDA, "loop_kernel: no resident CTA");
        g->grid_loop[alg] = nb * g->num_sms;
    }
    if (!host_loop && !persist) {
        etg_status rc = build_graph<OffT>(g, alg);
        if (rc != ETG_OK) return rc;
    }
    ETG_CU(cudaEventRecord(g->ev0, s));
    {
        void *args[] = {&d, &label, &source};
        ETG_CU(cudaLaunchKernel(init_fn<OffT>(alg), dim3(g->grid_init), dim3(kBlock), args, 0, s));
    }
    cudaGraphConditionalHandle none = 0;
    int zero = 0;
    void *scan_args[] = {&d, &none, &zero};
    // A2 of the initial active set (Proc. 1 "Init actSet")
    ETG_CU(launch_scan<OffT>(g, alg, scan_args, s));
    uint64_t launches = 2;                       // init (+ control block), first scan
    if (persist) {
        // the whole loop in one cooperative launch (all CTAs co-resident)
        const void *fn = loop_fn<OffT>(alg, g->p.udc);
        uint32_t cap_e = expand_arg(g->p);
        void *largs[] = {&d, &cap_e};
        ETG_CU(cudaLaunchCooperativeKernel(fn, dim3((unsigned)g->grid_loop[alg]), dim3(kBlock), largs, 0, s));
        launches += 1;
    } else if (host_loop) {
        Launch ex;
        etg_status rc = expand_launch<OffT>(g, alg, ex);
        if (rc != ETG_OK) return rc;
        uint32_t cap_e = expand_arg(g->p);
        void *exp_args[] = {&d, &cap_e};
            for (;;) {
            // "while actSet.isNotEmpty()" (L207): read the compacted size back
            ETG_CU(cudaMemcpyAsync(&g->h_ctl->more, &g->ctl->more, 4, cudaMemcpyDeviceToHost, s));
            ETG_CU(cudaStreamSynchronize(s));
            if (g->h_ctl->more == 0) break;
            nvtxRangePushA("etg_iteration");
            if (profile) ETG_CU(cudaEventRecord(g->pev[0], s));
            ETG_CU(cudaLaunchKernel(ex.fn, ex.grid, dim3(kBlock), exp_args, ex.smem, s));
            if (profile) ETG_CU(cudaEventRecord(g->pev[1], s));
            ETG_CU(launch_scan<OffT>(g, alg, scan_args, s));
            if (profile) ETG_CU(cudaEventRecord(g->pev[2], s));
            nvtxRangePop();
            launches += 2;
            if (profile) {
                ETG_CU(cudaEventSynchronize(g->pev[2]));
                float a = 0.f, b = 0.f;
                ETG_CU(cudaEventElapsedTime(&a, g->pev[0], g->pev[1]));
                ETG_CU(cudaEventElapsedTime(&b, g->pev[1], g->pev[2]));
                expand_ms += a;
                scan_ms += b;
                ++expand_launches;
            }
        }
    } else {
        ETG_CU(cudaGraphLaunch(g->exec[alg], s));
    }
    ETG_CU(cudaEventRecord(g->ev1, s));
    ETG_CU(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    ETG_CU(cudaStreamSynchronize(s));
    ETG_CU(cudaGetLastError());
    if (!host_loop && !persist) launches += 2ull * g->h_ctl->depth;   // body runs = scans after the first
    g_launches += launches;
    if (st) {
        float ms = 0.f;
        ETG_CU(cudaEventElapsedTime(&ms, g->ev0, g->ev1));
        st->iterations = g->h_ctl->iterations;
        st->expand_launches = expand_launches;
        st->activations = g->h_ctl->activations;
        st->frontier_total = g->h_ctl->frontier;
        if (persist) {
            // phase times of the persistent loop (%globaltimer, barrier to barrier)
            scan_ms = (float)(g->h_ctl->t_scan_ns * 1e-6);
            expand_ms = (float)(g->h_ctl->t_expand_ns * 1e-6);
            expand_launches = g->h_ctl->depth;
        }
        st->scan_ms = scan_ms;
        st->expand_ms = expand_ms;
        st->reserved = 0.f;
        st->shadows = g->h_ctl->shadows;
        st->edges_processed = g->h_ctl->edges;
        st->vertices_reached = 0;
        st->edges_reached = 0;
        st->ms = ms;
    }
    return ETG_OK;
}


// --------------------------------------------------------------------------- //
// Step-wise driving (multi-GPU partitions, A6 exchanged between steps): the
// caller runs begin, then { expand; exchange Q (and labels); scan } while the
// active set is non-empty, then end.  Same kernels as the fused loop.
// --------------------------------------------------------------------------- //
template <class OffT>
etg_status step_scan_impl(etg_graph *g, uint32_t *n_active);

template <class OffT>
etg_status step_begin_impl(etg_graph *g, int alg, uint32_t source, uint32_t *label, uint32_t *n_active,
                           int skip_scan) {
    Dev<OffT> d = make_dev<OffT>(g, alg);
    cudaStream_t s = g->stream;
    void *iargs[] = {&d, &label, &source};
    ETG_CU(cudaLaunchKernel(init_fn<OffT>(alg), dim3(g->grid_init), dim3(kBlock), iargs, 0, s));
    g->step_launches = 1;
    g->step_alg = alg;
    g->step_label = label;
    g->step_acts = 0;
    if (!skip_scan) return step_scan_impl<OffT>(g, n_active);
    ETG_CU(cudaStreamSynchronize(s));
    *n_active = 0;
    return ETG_OK;
}

template <class OffT>
etg_status step_scan_impl(etg_graph *g, uint32_t *n_active) {
    Dev<OffT> d = make_dev<OffT>(g, g->step_alg);
    cudaStream_t s = g->stream;
    cudaGraphConditionalHandle none = 0;
    int zero = 0;
    void *scan_args[] = {&d, &none, &zero};
    for (int rescan = 0;; ++rescan) {
        if (rescan) {
            ctl_rescan_kernel<<<1, 1, 0, s>>>(g->ctl);
            g->step_launches += 1;
        }
        ETG_CU(launch_scan<OffT>(g, g->step_alg, scan_args, s));
        g->step_launches += 1;
        ETG_CU(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
        ETG_CU(cudaStreamSynchronize(s));
        ETG_CU(cudaGetLastError());
        // near-far: an empty near set with deferred vertices advanced the
        // threshold; scan again (nothing changed in between) until some
        // vertices are activated or none remain
        if (!d.nf_delta || g->h_ctl->activations != g->step_acts || !g->h_ctl->more) break;
    }
    // vertices activated (bits consumed) by this scan: the same on every rank
    *n_active = (uint32_t)(g->h_ctl->activations - g->step_acts);
    g->step_acts = g->h_ctl->activations;
    return ETG_OK;
}

template <class OffT>
etg_status step_expand_impl(etg_graph *g) {
    Dev<OffT> d = make_dev<OffT>(g, g->step_alg);
    Launch ex;
    const bool peer = g->npeer > 0 && g->step_alg != ALG_BFS;
    etg_status rc = expand_launch<OffT>(g, g->step_alg, ex, peer);
    if (rc != ETG_OK) return rc;
    uint32_t cap_e = expand_arg(g->p);
    void *exp_args[] = {&d, &cap_e};
    ETG_CU(cudaLaunchKernel(ex.fn, ex.grid, dim3(kBlock), exp_args, ex.smem, g->stream));
    g->step_launches += 1;
    return ETG_OK;
}

// ---- communicator plumbing (etg_comm_*; host control plane in etg_comm.h) ----
etg_status comm_fail(int rc, const char *what) {
    return fail(ETG_ENCCL, std::string(what) + (rc == -2 ? ": a peer process died" : ": timed out waiting for the peers"));
}

#define ETG_BAR(c, what)                                   \
    do {                                                   \
        const int brc_ = etg::comm_barrier(c);             \
        if (brc_) return comm_fail(brc_, what);            \
    } while (0)

// All-gather of k <= kCommVals 64-bit values at slot positions [at, at + k):
// write, barrier, read.  No trailing barrier: every caller uses positions that
// are rewritten only after at least one more barrier.
etg_status comm_gather(const etg::Comm &c, int at, const uint64_t *mine, int k,
                       uint64_t (*out)[etg::kCommVals]) {
    for (int i = 0; i < k; ++i) c.sh->slot[c.rank].val[at + i] = mine[i];
    ETG_BAR(c, "all-gather");
    for (int q = 0; q < c.world; ++q)
        for (int i = 0; i < k; ++i) out[q][at + i] = c.sh->slot[q].val[at + i];
    return ETG_OK;
}

// ETG_SSSP_DELTA_AUTO: Delta = 6 x mean edge weight / mean out-degree (>= 1),
// resolved once per handle; on a communicator handle from the GLOBAL sums (all
// ranks then run the same schedule as the single-GPU call).
etg_status resolve_delta(etg_graph *g) {
    if (g->p.nf_delta != ETG_SSSP_DELTA_AUTO) return ETG_OK;
    uint32_t delta = 1;
    unsigned long long wsum = 0;
    if (g->m && g->w) {
        ETG_CU(cudaMemsetAsync(&g->ctl->reached_e, 0, sizeof(unsigned long long), g->stream));
        weight_sum_kernel<<<g->num_sms * 8, kBlock, 0, g->stream>>>(g->w, g->m, g->ctl);
        ETG_CU(cudaGetLastError());
        ETG_CU(cudaMemcpyAsync(&g->h_ctl->reached_e, &g->ctl->reached_e, sizeof(unsigned long long),
                               cudaMemcpyDeviceToHost, g->stream));
        ETG_CU(cudaStreamSynchronize(g->stream));
        wsum = g->h_ctl->reached_e;
    }
    uint64_t m = g->m;
    if (g->comm && g->comm->world > 1) {
        uint64_t mine[2] = {wsum, g->m}, all[etg::kCommMaxRanks][etg::kCommVals];
        etg_status rc = comm_gather(*g->comm, 8, mine, 2, all);   // positions 8, 9: only used here
        if (rc != ETG_OK) return rc;
        wsum = 0;
        m = 0;
        for (int q = 0; q < g->comm->world; ++q) {
            wsum += all[q][8];
            m += all[q][9];
        }
    }
    if (m && wsum) {
        // 6 x mean weight / mean out-degree: C2 (deg 16) 12, C3 (14.4) 13,
        // C4 (35.3) 6 -- each within a few % of its measured best Delta
        const double mean_w = (double)wsum / (double)m;
        const double mean_deg = (double)m / (double)(g->n ? g->n : 1);
        const double d = 6.0 * mean_w / mean_deg + 0.5;
        delta = d < 1.0 ? 1u : (d > 2147483647.0 ? 0x7FFFFFFFu : (uint32_t)d);
    }
    g->p.nf_delta = delta;
    return ETG_OK;
}

etg_status publish_impl(etg_graph *g);

// The whole partitioned traversal of one rank (Proc. 1 L207 on a
// 1-D vertex partition).  Destination partition (default): every rank expands
// the replicated active set over its sub-CSR (edges INTO its range), relaxes
// owned vertices only, then publishes what changed in its range straight into
// every peer's copy (publish_kernel over peer memory); push partition
// (ETG_PUSH): every rank expands its own vertices and the expand kernel itself
// reduces each relaxation of a foreign vertex into the owner's labels.
// Per iteration: expand [-> publish] -> stream sync -> barrier -> scan ->
// barrier with the termination count.  The count is identical on every rank
// in the destination partition (checked); the push partition stops when no
// rank has work left.
template <class OffT>
etg_status comm_run_impl(etg_graph *g, int alg, uint32_t source, uint32_t *out, etg_stats *st) {
    const etg::Comm &c = *g->comm;
    cudaStream_t s = g->stream;
    uint32_t *lab = reinterpret_cast<uint32_t *>(g->ws + g->L.Lfull);
    const bool multi = c.world > 1;
    uint64_t all[etg::kCommMaxRanks][etg::kCommVals];
    ETG_CU(cudaEventRecord(g->ev0, s));
    uint32_t nact = 0;
    etg_status rc = step_begin_impl<OffT>(g, alg, source, lab, &nact, 0);
    if (rc != ETG_OK) return rc;
    ETG_BAR(c, "init");                  // every copy initialised before anyone writes into it
    uint64_t nf_all = 0;                 // compacted frontier summed over the ranks (statistics)
    auto live_count = [&](uint64_t &live) -> etg_status {
        // push: any rank with work (compacted vertices or deferred far ones);
        // destination: the activation count, identical on every rank
        uint64_t mine[2] = {g->push ? (uint64_t)g->h_ctl->more : (uint64_t)nact, (uint64_t)g->h_ctl->nF};
        if (!multi) {
            live = mine[0];
            nf_all = mine[1];
            return ETG_OK;
        }
        etg_status r = comm_gather(c, 6, mine, 2, all);   // positions 6, 7
        if (r != ETG_OK) return r;
        live = 0;
        nf_all = 0;
        for (int q = 0; q < c.world; ++q) {
            if (!g->push && all[q][6] != mine[0])
                return fail(ETG_ENCCL, "ranks disagree on the active-set size (not the same graph or arguments?)");
            live += all[q][6];
            nf_all += all[q][7];
        }
        return ETG_OK;
    };
    uint64_t live = 0;
    rc = live_count(live);
    if (rc != ETG_OK) return rc;
    uint32_t trips = 0;                  // Proc. 1 iterations: trips that expand a non-empty frontier
    while (live) {
        if (nf_all) ++trips;             // (on some rank: the same count on every rank)
        nvtxRangePushA("etg_iteration");
        rc = step_expand_impl<OffT>(g);
        if (rc != ETG_OK) return rc;
        if (!g->push && multi) {
            rc = publish_impl(g);
            if (rc != ETG_OK) return rc;
        }
        if (multi) {
            ETG_CU(cudaStreamSynchronize(s));
            ETG_BAR(c, "exchange");      // every rank's writes into this rank's copy have landed
        }
        rc = step_scan_impl<OffT>(g, &nact);
        if (rc != ETG_OK) return rc;
        rc = live_count(live);           // also: nobody writes iteration k+1 into a copy still being scanned
        nvtxRangePop();
        if (rc != ETG_OK) return rc;
    }
    ETG_CU(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    if (g->v_hi > g->v_lo)
        ETG_CU(cudaMemcpyAsync(out, lab + g->v_lo, 4ull * (g->v_hi - g->v_lo), cudaMemcpyDeviceToDevice, s));
    ETG_CU(cudaEventRecord(g->ev1, s));
    ETG_CU(cudaStreamSynchronize(s));
    ETG_CU(cudaGetLastError());
    g_launches += g->step_launches + 1;
    g->step_alg = -1;
    float ms = 0.f;
    ETG_CU(cudaEventElapsedTime(&ms, g->ev0, g->ev1));
    const Ctl &h = *g->h_ctl;
    uint64_t mine[5] = {h.edges, h.shadows, h.frontier, h.activations, 0};
    memcpy(&mine[4], &ms, sizeof(float));
    uint64_t tot[5] = {mine[0], mine[1], mine[2], mine[3], 0};
    float ms_max = ms;
    if (multi) {
        rc = comm_gather(c, 1, mine, 5, all);
        if (rc != ETG_OK) return rc;
        for (int i = 0; i < 4; ++i) tot[i] = 0;
        for (int q = 0; q < c.world; ++q) {
            for (int i = 0; i < 4; ++i) tot[i] += all[q][1 + i];
            float mq = 0.f;
            memcpy(&mq, &all[q][5], sizeof(float));
            ms_max = std::max(ms_max, mq);
        }
        if (!g->push) tot[3] = h.activations;   // replicated active set: the same on every rank
    }
    if (st) {
        memset(st, 0, sizeof(*st));
        st->iterations = trips;          // global (a rank's own non-empty frontiers can be fewer)
        st->edges_processed = tot[0];
        st->shadows = tot[1];
        st->frontier_total = tot[2];
        st->activations = tot[3];
        st->ms = ms_max;                 // max over ranks
        st->reserved = ms;               // this rank's own device time
    }
    return ETG_OK;
}

etg_status run_checked(etg_graph *g, int alg, uint32_t source, uint32_t *label, etg_stats *st);

// One traversal call, bracketed by an NVTX range named after the algorithm
// (and "/comm" for a communicator handle) for timeline tools.
etg_status run(etg_graph *g, int alg, uint32_t source, uint32_t *label, etg_stats *st) {
    static const char *names[2][4] = {{"etg_bfs", "etg_sssp", "etg_cc", "etg_sswp"},
                                      {"etg_bfs/comm", "etg_sssp/comm", "etg_cc/comm", "etg_sswp/comm"}};
    nvtxRangePushA(names[g && g->comm ? 1 : 0][alg & 3]);
    const etg_status rc = run_checked(g, alg, source, label, st);
    nvtxRangePop();
    return rc;
}

etg_status run_checked(etg_graph *g, int alg, uint32_t source, uint32_t *label, etg_stats *st) {
    if (!g || !label) return fail(ETG_EINVAL, "null handle or label pointer");
    if (alg != ALG_CC && source >= g->n) return fail(ETG_EINVAL, "source >= n");
    if ((alg == ALG_SSSP || alg == ALG_SSWP) && !g->has_w) return fail(ETG_ENOWEIGHTS, "graph loaded without weights");
    if (alg == ALG_SSSP) {
        etg_status rc = resolve_delta(g);
        if (rc != ETG_OK) return rc;
    }
    if (alg == ALG_CC && !(g->flags & ETG_SYMMETRIC)) return fail(ETG_ENOTSYM, "etg_cc needs ETG_SYMMETRIC");
    if (g->n == 0) return ETG_OK;
    if (g->comm) {
        if (g->push && alg == ALG_BFS) return fail(ETG_EINVAL, "ETG_PUSH handles serve SSSP/CC/SSWP (BFS: destination partition)");
        if (g->comm->device >= 0) ETG_CU(cudaSetDevice(g->comm->device));
        return g->p.u64 ? comm_run_impl<uint64_t>(g, alg, source, label, st)
                        : comm_run_impl<uint32_t>(g, alg, source, label, st);
    }
    return g->p.u64 ? run_impl<uint64_t>(g, alg, source, label, st)
                    : run_impl<uint32_t>(g, alg, source, label, st);
}

template <class OffT>
etg_status validate_impl(etg_graph *g) {
    Dev<OffT> d = make_dev<OffT>(g);
    validate_kernel<OffT><<<g->num_sms * 4, kBlock, 0, g->stream>>>(d, (unsigned long long)g->m);
    g_launches += 1;
    ETG_CU(cudaMemcpyAsync(&g->h_ctl->error, &g->ctl->error, 4, cudaMemcpyDeviceToHost, g->stream));
    ETG_CU(cudaStreamSynchronize(g->stream));
    if (g->h_ctl->error) return fail(ETG_EINVALID_CSR, "CSR validation failed, code " + std::to_string(g->h_ctl->error));
    return ETG_OK;
}

template <class OffT>
etg_status reach_impl(etg_graph *g, const uint32_t *label, uint32_t unreached, etg_stats *st) {
    Dev<OffT> d = make_dev<OffT>(g);
    ETG_CU(cudaMemsetAsync(&g->ctl->reached_v, 0, 16, g->stream));
    reach_kernel<OffT><<<g->num_sms * 4, kBlock, 0, g->stream>>>(d, label, unreached);
    g_launches += 1;
    ETG_CU(cudaMemcpyAsync(&g->h_ctl->reached_v, &g->ctl->reached_v, 16, cudaMemcpyDeviceToHost, g->stream));
    ETG_CU(cudaStreamSynchronize(g->stream));
    ETG_CU(cudaGetLastError());
    st->vertices_reached = g->h_ctl->reached_v;
    st->edges_reached = g->h_ctl->reached_e;
    return ETG_OK;
}

template <class OffT>
etg_status udc_impl(etg_graph *g, const uint32_t *act, uint32_t n_act, uint32_t *id, uint64_t *start,
                    uint64_t *end, uint64_t cap, uint64_t *n_out) {
    Dev<OffT> d = make_dev<OffT>(g);
    cudaStream_t s = g->stream;
    ctl_begin_kernel<<<1, 1, 0, s>>>(g->ctl, nullptr, 0);
    if (n_act) mark_kernel<<<g->num_sms, kBlock, 0, s>>>(d.Q, act, n_act);
    {
        cudaGraphConditionalHandle none = 0;
        int zero = 0;
        void *args[] = {&d, &none, &zero};
        ETG_CU(launch_scan<OffT>(g, ALG_SSSP, args, s));
    }
    ETG_CU(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    ETG_CU(cudaStreamSynchronize(s));
    *n_out = g->h_ctl->nshadow;
    if (g->h_ctl->nshadow > cap) return fail(ETG_ENOMEM, "cap too small for the shadow list");
    udc_dump_kernel<OffT, true><<<g->num_sms * 4, kBlock, 0, s>>>(d, id, start, end);
    g_launches += 3;
    ETG_CU(cudaStreamSynchronize(s));
    ETG_CU(cudaGetLastError());
    return ETG_OK;
}

// Debug/tuning: advance a traversal to the active set of `depth`, snapshot the
// state, then time `reps` launches of the expand kernel on that same state with
// the given tune bits (labels and the bitmap restored before every launch).
template <class OffT>
etg_status replay_impl(etg_graph *g, int alg, uint32_t source, uint32_t depth, uint32_t tune, int reps,
                       uint32_t *label, uint32_t *saved, float *ms_out, uint64_t *edges_out,
                       uint32_t *nF_out) {
    Dev<OffT> d = make_dev<OffT>(g);
    cudaStream_t s = g->stream;
    Launch ex;
    etg_status rc = expand_launch<OffT>(g, alg, ex);
    if (rc != ETG_OK) return rc;
    uint32_t cap_e = expand_arg(g->p);
    void *exp_args[] = {&d, &cap_e};
    cudaGraphConditionalHandle none = 0;
    int zero = 0;
    void *scan_args[] = {&d, &none, &zero};
    ctl_begin_kernel<<<1, 1, 0, s>>>(g->ctl, label, source);
    void *iargs[] = {&d, &label, &source};
    ETG_CU(cudaLaunchKernel(init_fn<OffT>(alg), dim3(g->grid_init), dim3(kBlock), iargs, 0, s));
    ETG_CU(launch_scan<OffT>(g, alg, scan_args, s));
    for (;;) {
        ETG_CU(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
        ETG_CU(cudaStreamSynchronize(s));
        if (g->h_ctl->depth >= depth || g->h_ctl->nF == 0) break;
        ETG_CU(cudaLaunchKernel(ex.fn, ex.grid, dim3(kBlock), exp_args, ex.smem, s));
        ETG_CU(launch_scan<OffT>(g, alg, scan_args, s));
    }
    ETG_CU(cudaMemsetAsync(&g->ctl->reached_v, 0, 8, s));
    ETG_CU(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    ETG_CU(cudaStreamSynchronize(s));
    const Ctl snap = *g->h_ctl;
    *nF_out = snap.nF;
    ETG_CU(cudaMemcpyAsync(saved, label, 4ull * g->n, cudaMemcpyDeviceToDevice, s));
    Dev<OffT> dt = d;
    dt.tune = tune;
    void *targs[] = {&dt, &cap_e};
    float total = 0.f;
    for (int r = 0; r < reps; ++r) {
        ETG_CU(cudaMemcpyAsync(label, saved, 4ull * g->n, cudaMemcpyDeviceToDevice, s));
        if (alg != ALG_BFS)   // the pre-filter snapshot equals the labels at an iteration start
            ETG_CU(cudaMemcpyAsync(d.snap, saved, 4ull * g->n, cudaMemcpyDeviceToDevice, s));
        ETG_CU(cudaMemsetAsync(d.Q, 0, 4ull * g->L.nwords, s));
        *g->h_ctl = snap;
        ETG_CU(cudaMemcpyAsync(g->ctl, g->h_ctl, sizeof(Ctl), cudaMemcpyHostToDevice, s));
        ETG_CU(cudaEventRecord(g->pev[0], s));
        ETG_CU(cudaLaunchKernel(ex.fn, ex.grid, dim3(kBlock), targs, ex.smem, s));
        ETG_CU(cudaEventRecord(g->pev[1], s));
        ETG_CU(cudaEventSynchronize(g->pev[1]));
        float ms = 0.f;
        ETG_CU(cudaEventElapsedTime(&ms, g->pev[0], g->pev[1]));
        total += ms;
    }
    ETG_CU(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    ETG_CU(cudaStreamSynchronize(s));
    *edges_out = g->h_ctl->edges - snap.edges;
    if (tune & 32u) *nF_out = (uint32_t)(g->h_ctl->reached_v / (reps ? reps : 1));   // passes
    *ms_out = reps ? total / reps : 0.f;
    // leave the handle consistent: labels restored, bitmap clear
    ETG_CU(cudaMemcpyAsync(label, saved, 4ull * g->n, cudaMemcpyDeviceToDevice, s));
    ETG_CU(cudaMemsetAsync(d.Q, 0, 4ull * g->L.nwords, s));
    ETG_CU(cudaStreamSynchronize(s));
    ETG_CU(cudaGetLastError());
    return ETG_OK;
}

// Destination partition: store what changed in the owned range into every
// peer's copy (BFS: non-zero bitmap words; SSSP/CC/SSWP: moved labels).
etg_status publish_impl(etg_graph *g) {
    if (g->dpeer < 2 || g->dpeer_hi <= g->dpeer_lo) return ETG_OK;
    PeerSet ps;
    ps.P = g->dpeer;
    ps.rank = g->dpeer_rank;
    const bool bfs = g->step_alg == ALG_BFS;
    for (uint32_t k = 0; k < kMaxPeer; ++k) ps.ptr[k] = bfs ? g->dpeer_Q[k] : g->dpeer_label[k];
    const uint32_t *Q = reinterpret_cast<const uint32_t *>(g->ws + g->L.Q);
    const uint32_t *snap = reinterpret_cast<const uint32_t *>(g->ws + g->L.snap);
    if (bfs)
        publish_kernel<true><<<g->grid_init, kBlock, 0, g->stream>>>(Q, g->step_label, snap, g->dpeer_lo,
                                                                     g->dpeer_hi, ps);
    else
        publish_kernel<false><<<g->grid_init, kBlock, 0, g->stream>>>(Q, g->step_label, snap, g->dpeer_lo,
                                                                      g->dpeer_hi, ps);
    ETG_CU(cudaGetLastError());
    g->step_launches += 1;
    return ETG_OK;
}

// Base of the allocation holding d_ptr (driver API, resolved at run time: the
// library does not link libcuda), its CUDA-IPC handle and d_ptr's offset.
etg_status ipc_handle_of(const void *d_ptr, uint8_t *out_handle, uint64_t *out_offset) {
    typedef CUresult (*get_attr_t)(void *, CUpointer_attribute, CUdeviceptr);
    static get_attr_t get_attr = nullptr;
    if (!get_attr) {
        void *h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_GLOBAL);
        if (h) get_attr = (get_attr_t)dlsym(h, "cuPointerGetAttribute");
        if (!get_attr) return fail(ETG_ECUDA, "cuPointerGetAttribute unavailable (no libcuda.so.1)");
    }
    CUdeviceptr base = 0;
    if (get_attr(&base, CU_POINTER_ATTRIBUTE_RANGE_START_ADDR, (CUdeviceptr)d_ptr) != CUDA_SUCCESS)
        return fail(ETG_ECUDA, "cuPointerGetAttribute(RANGE_START_ADDR) failed");
    cudaIpcMemHandle_t hd;
    ETG_CU(cudaIpcGetMemHandle(&hd, (void *)base));
    memcpy(out_handle, &hd, sizeof(hd));
    *out_offset = (uint64_t)((CUdeviceptr)d_ptr - base);
    return ETG_OK;
}

// Collective part of etg_load_csr on a communicator: exchange owned ranges and
// workspace handles, check that the ranges tile [0, n), map every peer's
// workspace (CUDA IPC; peers in this process: their pointer as is) and wire
// the exchange of the chosen partition.  Uses slot positions 10..15 and ends
// with a barrier.
etg_status comm_setup(etg_graph *g, uint32_t v_lo, uint32_t v_hi) {
    const etg::Comm &c = *g->comm;
    etg::CommSlot &me = c.sh->slot[c.rank];
    if (c.world > 1) {
        etg_status rc = ipc_handle_of(g->ws, me.ipc, &me.ipc_off);
        if (rc != ETG_OK) return rc;
    }
    me.ws_ptr = reinterpret_cast<uint64_t>(g->ws);
    const uint64_t mine[6] = {g->n, v_lo, v_hi, g->L.Q, g->L.Lfull, g->push ? 1u : 0u};
    uint64_t all[etg::kCommMaxRanks][etg::kCommVals];
    etg_status rc = comm_gather(c, 10, mine, 6, all);
    if (rc != ETG_OK) return rc;
    std::string err;
    uint32_t bounds[kMaxPeer + 1] = {};
    for (int q = 0; q < c.world && err.empty(); ++q) {
        if (all[q][10] != g->n) err = "ranks disagree on n";
        else if (all[q][15] != mine[5]) err = "ranks disagree on ETG_PUSH";
        else if (all[q][11] != (q ? all[q - 1][12] : 0ull)) err = "owned ranges must tile [0, n) in rank order";
        else if (q && (all[q][11] & 31u)) err = "inner range bounds must be multiples of 32";
        bounds[q] = (uint32_t)all[q][11];
    }
    if (err.empty() && all[c.world - 1][12] != g->n) err = "owned ranges must tile [0, n) in rank order";
    bounds[c.world] = (uint32_t)g->n;
    uint32_t *peer_ws[kMaxPeer] = {};
    for (int q = 0; q < c.world && err.empty(); ++q) {
        if (q == c.rank) {
            peer_ws[q] = reinterpret_cast<uint32_t *>(g->ws);
            continue;
        }
        const etg::CommSlot &o = c.sh->slot[q];
        if (o.pid == getpid()) {
            peer_ws[q] = reinterpret_cast<uint32_t *>(o.ws_ptr);    // same address space
            continue;
        }
        cudaIpcMemHandle_t hd;
        memcpy(&hd, o.ipc, sizeof(hd));
        void *base = nullptr;
        cudaError_t e = cudaIpcOpenMemHandle(&base, hd, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) {
            err = std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e);
            break;
        }
        g->ipc_base[q] = base;
        peer_ws[q] = reinterpret_cast<uint32_t *>(static_cast<uint8_t *>(base) + o.ipc_off);
    }
    ETG_BAR(c, "load");                  // slots 10..15 read by everyone; peers mapped
    if (!err.empty()) return fail(ETG_ENCCL, err);
    const uint32_t P = (uint32_t)c.world;
    for (uint32_t q = 0; q < P; ++q) {
        uint8_t *base = reinterpret_cast<uint8_t *>(peer_ws[q]);
        g->dpeer_Q[q] = reinterpret_cast<uint32_t *>(base + all[q][13]);
        g->dpeer_label[q] = reinterpret_cast<uint32_t *>(base + all[q][14]);
    }
    if (g->push) {
        for (uint32_t k = 0; k <= kMaxPeer; ++k) g->peer_bounds[k] = k <= P ? bounds[k] : (uint32_t)g->n;
        for (uint32_t k = 0; k < kMaxPeer; ++k) g->peer_label[k] = k < P ? g->dpeer_label[k] : nullptr;
        g->peer_rank = (uint32_t)c.rank;
        g->npeer = P > 1 ? P : 0;
    } else {
        g->dpeer_lo = v_lo;
        g->dpeer_hi = v_hi;
        g->dpeer_rank = (uint32_t)c.rank;
        g->dpeer = P;
    }
    return ETG_OK;
}

}  // namespace

// =========================================================================== //
// C ABI
// =========================================================================== //
extern "C" {

size_t etg_workspace_bytes(uint64_t n, uint64_t m, const etg_options *opt) {
    return layout(n, m, derive(opt, env_tune())).total;
}

etg_status etg_load_csr(etg_graph **out, uint64_t n, uint64_t m, const void *d_row_offsets,
                        const uint32_t *d_col_idx, const uint32_t *d_weights, void *d_workspace,
                        size_t workspace_bytes, void *stream, const etg_options *opt, const etg_comm *comm,
                        uint32_t v_lo, uint32_t v_hi) {
    if (!out) return fail(ETG_EINVAL, "out is NULL");
    *out = nullptr;
    if (comm && (v_lo > v_hi || v_hi > n)) return fail(ETG_EINVAL, "owned range [v_lo, v_hi) must lie in [0, n]");
    if (!comm && opt && (opt->flags & ETG_PUSH)) return fail(ETG_EINVAL, "ETG_PUSH needs a communicator");
    if (!d_row_offsets || (m && !d_col_idx) || !d_workspace) return fail(ETG_EINVAL, "NULL device pointer");
    const uint32_t tune = env_tune();
    const Params p = derive(opt, tune);
    const uint32_t flags = opt ? opt->flags : 0u;
    if (n > 0xFFFFFFFEull) return fail(ETG_ERANGE, "n > 2^32 - 2");
    if (!p.u64 && m > 0xFFFFFFFFull) return fail(ETG_ERANGE, "m >= 2^32 needs ETG_OFFSETS_U64");
    if (p.udc && p.K == 0) return fail(ETG_EINVAL, "K = 0");
    const uint64_t max_shadows = p.udc ? (m + p.K - 1) / p.K + n : n;
    if (max_shadows >= 0xFFFFFFFFull) return fail(ETG_ERANGE, "shadow count may exceed 2^32 (raise K)");
    const Layout L = layout(n, m, p);
    if (workspace_bytes < L.total) return fail(ETG_ENOMEM, "workspace too small: need " + std::to_string(L.total));
    if (reinterpret_cast<uintptr_t>(d_workspace) % kAlign) return fail(ETG_EINVAL, "workspace must be 256-byte aligned");

    etg_graph *g = new (std::nothrow) etg_graph();
    if (!g) return fail(ETG_ENOMEM, "host allocation failed");
    g->n = n;
    g->m = m;
    g->flags = flags;
    g->p = p;
    g->off = d_row_offsets;
    g->col = d_col_idx;
    g->w = d_weights;
    g->has_w = d_weights != nullptr || m == 0;   // no edge needs a weight (e.g. a partition that owns nothing)
    g->stream = static_cast<cudaStream_t>(stream);
    g->ws = static_cast<uint8_t *>(d_workspace);
    g->L = L;
    g->delta_auto = p.nf_delta == ETG_SSSP_DELTA_AUTO;
    if (comm) {
        g->comm = const_cast<etg::Comm *>(&comm->c);
        g->push = (flags & ETG_PUSH) != 0;
        g->v_lo = (uint32_t)v_lo;
        g->v_hi = (uint32_t)v_hi;
    } else {
        g->v_lo = 0;
        g->v_hi = (uint32_t)n;
    }
    g->ctl = reinterpret_cast<Ctl *>(g->ws + L.ctl);
    auto bail = [&](etg_status s) {
        etg_free(g);
        return s;
    };
    int dev = 0;
    cudaError_t e;
    if (comm && comm->c.device >= 0 && (e = cudaSetDevice(comm->c.device)) != cudaSuccess)
        return bail(fail(ETG_ECUDA, std::string("load: ") + cudaGetErrorString(e)));
    if ((e = cudaGetDevice(&dev)) != cudaSuccess ||
        (e = cudaDeviceGetAttribute(&g->num_sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess ||
        (e = cudaDeviceGetAttribute(&g->l2_bytes, cudaDevAttrL2CacheSize, dev)) != cudaSuccess ||
        (e = cudaMallocHost(&g->h_ctl, sizeof(Ctl))) != cudaSuccess ||
        (e = cudaEventCreate(&g->ev0)) != cudaSuccess || (e = cudaEventCreate(&g->ev1)) != cudaSuccess ||
        (e = cudaEventCreate(&g->pev[0])) != cudaSuccess || (e = cudaEventCreate(&g->pev[1])) != cudaSuccess ||
        (e = cudaEventCreate(&g->pev[2])) != cudaSuccess ||
        (e = cudaMemsetAsync(g->ctl, 0, sizeof(Ctl), g->stream)) != cudaSuccess ||
        (e = cudaMemsetAsync(g->ws + L.Q, 0, 4ull * L.nwords, g->stream)) != cudaSuccess ||
        (e = cudaMemsetAsync(g->ws + L.recE, 0, L.ctl - L.recE, g->stream)) != cudaSuccess) {   // (records, RD, FR)
        return bail(fail(ETG_ECUDA, std::string("load: ") + cudaGetErrorString(e)));
    }
    g->tune = tune;
    // no more scan CTAs than scan tiles, no more init CTAs than 256-vertex
    // blocks: a small graph does not launch hundreds of CTAs that exit at once
    // scan tiles: 32 rows per warp (8,192-vertex tiles) when that still gives
    // >= 2 tiles per SM, else fewer rows per warp -- a small graph's scan is
    // then short dependent chains on many SMs; ETG_SCAN_KW (4, 8, 16, 32)
    // overrides for experiments
    int kw = kWPW;
    while (kw > 4 && (n + 256ull * kw - 1) / (256ull * kw) < 2ull * (uint64_t)g->num_sms) kw >>= 1;
    if (const char *e_kw = getenv("ETG_SCAN_KW")) {
        const int v = atoi(e_kw);
        if (v == 4 || v == 8 || v == 16 || v == 32) kw = v;
    }
    if (p.persist) kw = kWPW;             // the persistent loop's scan phase uses 32 rows
    g->scan_kw = kw;
    const uint64_t nscan = (n + 256ull * kw - 1) / (256ull * kw);
    const uint64_t ninit = (std::max<uint64_t>(n, L.nwords) + kBlock - 1) / kBlock;
    // scan offset staging (a 16-byte-aligned offset array; not in the persistent
    // loop): a warp with >= ETG_SCAN_ROWS active rows (default 4; 0 disables)
    // bulk-copies its offsets into shared memory
    if (const char *e_s = getenv("ETG_SPLIT")) g->split = (uint32_t)std::max(1, atoi(e_s));
    if (const char *e_p = getenv("ETG_PDL")) g->pdl = atoi(e_p) != 0;
    if (const char *e_l = getenv("ETG_SCAN_LIST")) g->scan_list = (uint32_t)atoi(e_l);
    if (const char *e_d = getenv("ETG_DIRTY")) g->dirty = atoi(e_d) != 0;
    if (const char *e_a = getenv("ETG_AHEAD_MID")) g->ahead_mid = (uint32_t)atoi(e_a);
    if (const char *e_t = getenv("ETG_TUNE2")) g->tune2 = (uint32_t)atoi(e_t);
    g->scan_rows = 4;
    if (const char *e_r = getenv("ETG_SCAN_ROWS")) g->scan_rows = (uint32_t)atoi(e_r);
    g->scan_smem = 0;
    int scan_occ = 4;
    if (g->scan_rows && (reinterpret_cast<uintptr_t>(d_row_offsets) & 15u) == 0 && !p.persist) {
        g->scan_smem = p.u64 ? scan_smem_bytes<uint64_t>(kw) : scan_smem_bytes<uint32_t>(kw);
        for (int a = 0; a < 2; ++a) {
            const int alg = a ? ALG_SSSP : ALG_BFS;
            const void *fn = p.u64 ? scan_fn<uint64_t>(g, alg) : scan_fn<uint32_t>(g, alg);
            int nb = 0;
            if ((e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g->scan_smem)) != cudaSuccess ||
                (e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, kBlock, g->scan_smem)) != cudaSuccess)
                return bail(fail(ETG_ECUDA, std::string("load (scan): ") + cudaGetErrorString(e)));
            scan_occ = std::max(1, std::min(scan_occ, nb));
        }
    }
    g->grid_scan = (int)std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)g->num_sms * scan_occ, nscan));
    g->grid_init = (int)std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)g->num_sms * 8, ninit));
    if (flags & ETG_VALIDATE) {
        etg_status s = p.u64 ? validate_impl<uint64_t>(g) : validate_impl<uint32_t>(g);
        if (s != ETG_OK) return bail(s);
    }
    if ((e = cudaStreamSynchronize(g->stream)) != cudaSuccess)
        return bail(fail(ETG_ECUDA, std::string("load sync: ") + cudaGetErrorString(e)));
    if (g->comm) {
        etg_status s = comm_setup(g, (uint32_t)v_lo, (uint32_t)v_hi);
        if (s != ETG_OK) return bail(s);
    }
    *out = g;
    return ETG_OK;
}

etg_status etg_bfs(etg_graph *g, uint32_t source, uint32_t *d_depth, etg_stats *st) {
    return run(g, ALG_BFS, source, d_depth, st);
}

etg_status etg_sssp(etg_graph *g, uint32_t source, uint32_t *d_dist, etg_stats *st) {
    return run(g, ALG_SSSP, source, d_dist, st);
}

etg_status etg_cc(etg_graph *g, uint32_t *d_label, etg_stats *st) {
    return run(g, ALG_CC, 0, d_label, st);
}

etg_status etg_sswp(etg_graph *g, uint32_t source, uint32_t *d_width, etg_stats *st) {
    return run(g, ALG_SSWP, source, d_width, st);
}

etg_status etg_reach_stats(etg_graph *g, const uint32_t *d_label, uint32_t unreached, etg_stats *st) {
    if (!g || !d_label || !st) return fail(ETG_EINVAL, "NULL argument");
    if (g->n == 0) {
        st->vertices_reached = st->edges_reached = 0;
        return ETG_OK;
    }
    return g->p.u64 ? reach_impl<uint64_t>(g, d_label, unreached, st)
                    : reach_impl<uint32_t>(g, d_label, unreached, st);
}

etg_status etg_udc_slices(etg_graph *g, const uint32_t *d_active, uint32_t n_active, uint32_t *d_id,
                          uint64_t *d_start, uint64_t *d_end, uint64_t cap, uint64_t *n_out) {
    if (!g || !n_out || (n_active && !d_active)) return fail(ETG_EINVAL, "NULL argument");
    if (!g->p.udc) return fail(ETG_EINVAL, "etg_udc_slices needs a UDC handle");
    if (n_active > g->n) return fail(ETG_EINVAL, "active set larger than n");
    return g->p.u64 ? udc_impl<uint64_t>(g, d_active, n_active, d_id, d_start, d_end, cap, n_out)
                    : udc_impl<uint32_t>(g, d_active, n_active, d_id, d_start, d_end, cap, n_out);
}

etg_status etg_debug_expand_replay(etg_graph *g, int alg, uint32_t source, uint32_t depth, uint32_t tune,
                                   int reps, uint32_t *d_label, uint32_t *d_saved, float *ms,
                                   uint64_t *edges, uint32_t *n_active) {
    if (!g || !d_label || !d_saved || !ms || !edges || !n_active) return fail(ETG_EINVAL, "NULL argument");
    if (alg < 0 || alg > 3) return fail(ETG_EINVAL, "alg must be 0..3");
    if ((alg == ALG_SSSP || alg == ALG_SSWP) && !g->has_w) return fail(ETG_ENOWEIGHTS, "no weights");
    return g->p.u64 ? replay_impl<uint64_t>(g, alg, source, depth, tune, reps, d_label, d_saved, ms, edges, n_active)
                    : replay_impl<uint32_t>(g, alg, source, depth, tune, reps, d_label, d_saved, ms, edges, n_active);
}

etg_status etg_step_begin(etg_graph *g, int alg, uint32_t source, uint32_t *d_label, uint32_t *n_active) {
    if (!g || !d_label || !n_active) return fail(ETG_EINVAL, "NULL argument");
    if (alg < 0 || alg > 3) return fail(ETG_EINVAL, "alg must be 0..3");
    if (alg != ALG_CC && source >= g->n) return fail(ETG_EINVAL, "source >= n");
    if ((alg == ALG_SSSP || alg == ALG_SSWP) && !g->has_w) return fail(ETG_ENOWEIGHTS, "graph loaded without weights");
    if (alg == ALG_CC && !(g->flags & ETG_SYMMETRIC)) return fail(ETG_ENOTSYM, "etg_cc needs ETG_SYMMETRIC");
    if (alg == ALG_SSSP && g->delta_auto)   // each rank would derive its own Delta from its own edges
        return fail(ETG_EINVAL, "step-wise runs need an explicit sssp_delta (every rank the same); "
                                "communicator handles resolve auto from the global sums");
    if (g->n == 0) { *n_active = 0; return ETG_OK; }
    return g->p.u64 ? step_begin_impl<uint64_t>(g, alg, source, d_label, n_active, 0)
                    : step_begin_impl<uint32_t>(g, alg, source, d_label, n_active, 0);
}

etg_status etg_step_expand(etg_graph *g) {
    if (!g || g->step_alg < 0) return fail(ETG_EINVAL, "no step-wise run in progress");
    return g->p.u64 ? step_expand_impl<uint64_t>(g) : step_expand_impl<uint32_t>(g);
}

etg_status etg_step_scan(etg_graph *g, uint32_t *n_active) {
    if (!g || !n_active || g->step_alg < 0) return fail(ETG_EINVAL, "no step-wise run in progress");
    return g->p.u64 ? step_scan_impl<uint64_t>(g, n_active) : step_scan_impl<uint32_t>(g, n_active);
}

etg_status etg_step_end(etg_graph *g, etg_stats *st) {
    if (!g || g->step_alg < 0) return fail(ETG_EINVAL, "no step-wise run in progress");
    ETG_CU(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, g->stream));
    ETG_CU(cudaStreamSynchronize(g->stream));
    g_launches += g->step_launches;
    g->step_alg = -1;
    if (st) {
        memset(st, 0, sizeof(*st));
        st->iterations = g->h_ctl->iterations;
        st->activations = g->h_ctl->activations;
        st->frontier_total = g->h_ctl->frontier;
        st->shadows = g->h_ctl->shadows;
        st->edges_processed = g->h_ctl->edges;
    }
    return ETG_OK;
}

etg_status etg_bitmap_layout(etg_graph *g, size_t *offset_bytes, uint32_t *nwords) {
    if (!g || !offset_bytes || !nwords) return fail(ETG_EINVAL, "NULL argument");
    *offset_bytes = g->L.Q;
    *nwords = g->L.nwords;
    return ETG_OK;
}

void etg_free(etg_graph *g) {
    if (!g) return;
    for (uint32_t q = 0; q < kMaxPeer; ++q)
        if (g->ipc_base[q]) cudaIpcCloseMemHandle(g->ipc_base[q]);
    for (int a = 0; a < 4; ++a) {
        if (g->exec[a]) cudaGraphExecDestroy(g->exec[a]);
        if (g->graph[a]) cudaGraphDestroy(g->graph[a]);
    }
    if (g->ev0) cudaEventDestroy(g->ev0);
    if (g->ev1) cudaEventDestroy(g->ev1);
    for (int k = 0; k < 3; ++k)
        if (g->pev[k]) cudaEventDestroy(g->pev[k]);
    if (g->h_ctl) cudaFreeHost(g->h_ctl);
    delete g;
}

size_t etg_host_scratch_bytes(uint64_t n, uint64_t m, int has_weights, const etg_options *opt) {
    const Params p = derive(opt, env_tune());
    size_t o = 0;
    o = align_up(o + (p.u64 ? 8 : 4) * (n + 1));
    o = align_up(o + 4 * m);
    if (has_weights) o = align_up(o + 4 * m);
    o = align_up(o + 4 * n);                 // two label buffers: the D2H of one query
    o = align_up(o + 4 * n);                 // overlaps the traversal of the next
    return o + layout(n, m, p).total;
}

namespace {

// Host-buffer entry (etg_run_host / etg_run_host_batch): H2D of the CSR into
// the scratch, the queries on a handle over it, D2H of each query's labels.
// Overlap: off and col go first on the call's stream; w follows on a copy
// stream, so queries that need no weights (BFS, CC) run while it is in
// flight; each query's labels go back on the copy stream while the next query
// runs (two device label buffers).
etg_status run_host_impl(uint64_t n, uint64_t m, const void *h_off, const uint32_t *h_col, const uint32_t *h_w,
                         uint32_t nq, const int *algs, const uint32_t *sources, uint32_t *h_labels,
                         void *d_scratch, size_t scratch_bytes, void *stream, const etg_options *opt,
                         etg_stats *st) {
    if (!h_off || (m && !h_col) || !h_labels || !d_scratch || !algs || (nq && !sources)) return fail(ETG_EINVAL, "NULL argument");
    bool has_w = false;
    for (uint32_t q = 0; q < nq; ++q) {
        if (algs[q] < 0 || algs[q] > 3) return fail(ETG_EINVAL, "alg must be 0..3");
        has_w |= (algs[q] == ALG_SSSP || algs[q] == ALG_SSWP);
    }
    const Params p = derive(opt, env_tune());
    if (has_w && !h_w) return fail(ETG_ENOWEIGHTS, "weights required");
    if (scratch_bytes < etg_host_scratch_bytes(n, m, has_w, opt)) return fail(ETG_ENOMEM, "scratch too small");
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    uint8_t *base = static_cast<uint8_t *>(d_scratch);
    size_t o = 0;
    const size_t offsz = (p.u64 ? 8 : 4) * (n + 1);
    uint8_t *d_off = base + o;
    o = align_up(o + offsz);
    uint32_t *d_col = reinterpret_cast<uint32_t *>(base + o);
    o = align_up(o + 4 * m);
    uint32_t *d_w = nullptr;
    if (has_w) {
        d_w = reinterpret_cast<uint32_t *>(base + o);
        o = align_up(o + 4 * m);
    }
    uint32_t *d_lab[2];
    d_lab[0] = reinterpret_cast<uint32_t *>(base + o);
    o = align_up(o + 4 * n);
    d_lab[1] = reinterpret_cast<uint32_t *>(base + o);
    o = align_up(o + 4 * n);
    // A handle over this scratch layout is kept per thread and reused by the
    // next call with the same sizes, scratch, stream and options: the handle
    // holds only pointers into the scratch, so reuse just re-zeroes its
    // device control state; the host-side setup (pinned control block,
    // events, the instantiated CUDA graph of the loop, the copy stream) is
    // paid once.
    struct Cached {
        uint64_t n, m;
        int has_w;
        void *scratch;
        size_t bytes;
        cudaStream_t s;
        uint32_t K, flags, delta, tune;
        etg_graph *g;
        cudaStream_t cs;         // copy stream (w in, labels out)
        cudaEvent_t ev[5];       // w arrived; query done x 2; labels copied x 2
    };
    thread_local Cached cache[4] = {};
    thread_local unsigned next_slot = 0;
    const uint32_t K = opt ? opt->degree_limit_k : 0u, fl = opt ? opt->flags : 0u, dl = opt ? opt->sssp_delta : 0u;
    const uint32_t tune = env_tune();
    Cached *cc = nullptr;
    for (Cached &c : cache)
        if (c.g && c.n == n && c.m == m && c.has_w == (int)has_w && c.scratch == d_scratch && c.bytes == scratch_bytes &&
            c.s == s && c.K == K && c.flags == fl && c.delta == dl && c.tune == tune) {
            cc = &c;
            break;
        }
    etg_status rc = ETG_OK;
    if (!cc) {
        Cached &c = cache[next_slot++ % 4];
        if (c.g) {
            etg_free(c.g);
            cudaStreamDestroy(c.cs);
            for (cudaEvent_t e : c.ev) cudaEventDestroy(e);
            c.g = nullptr;
        }
        ETG_CU(cudaStreamCreateWithFlags(&c.cs, cudaStreamNonBlocking));
        for (cudaEvent_t &e : c.ev) ETG_CU(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        c.n = n; c.m = m; c.has_w = (int)has_w; c.scratch = d_scratch; c.bytes = scratch_bytes; c.s = s;
        c.K = K; c.flags = fl; c.delta = dl; c.tune = tune;
        cc = &c;
    }
    cudaStream_t cs = cc->cs;
    // H2D: offsets and columns on the call's stream; weights on the copy stream
    ETG_CU(cudaMemcpyAsync(d_off, h_off, offsz, cudaMemcpyHostToDevice, s));
    if (m) ETG_CU(cudaMemcpyAsync(d_col, h_col, 4 * m, cudaMemcpyHostToDevice, s));
    if (has_w && m) ETG_CU(cudaMemcpyAsync(d_w, h_w, 4 * m, cudaMemcpyHostToDevice, cs));
    ETG_CU(cudaEventRecord(cc->ev[0], cs));
    etg_graph *g = cc->g;
    if (g) {
        ETG_CU(cudaMemsetAsync(g->ctl, 0, sizeof(Ctl), s));
        ETG_CU(cudaMemsetAsync(g->ws + g->L.Q, 0, 4ull * g->L.nwords, s));
        ETG_CU(cudaMemsetAsync(g->ws + g->L.recE, 0, g->L.ctl - g->L.recE, s));
        // the reused handle sees this call's CSR: validate it like a fresh load would
        if (g->flags & ETG_VALIDATE) {
            rc = p.u64 ? validate_impl<uint64_t>(g) : validate_impl<uint32_t>(g);
            if (rc != ETG_OK) return rc;
        }
    } else {
        rc = etg_load_csr(&g, n, m, d_off, d_col, d_w, base + o, scratch_bytes - o, stream, opt, nullptr, 0, 0);
        if (rc != ETG_OK) return rc;
        cc->g = g;
    }
    bool w_ready = !has_w;
    for (uint32_t q = 0; q < nq && rc == ETG_OK; ++q) {
        const int b = q & 1;
        if (q >= 2) ETG_CU(cudaStreamWaitEvent(s, cc->ev[3 + b], 0));   // buffer b copied out
        if (!w_ready && (algs[q] == ALG_SSSP || algs[q] == ALG_SSWP)) {
            ETG_CU(cudaStreamWaitEvent(s, cc->ev[0], 0));
            w_ready = true;
        }
        rc = run(g, algs[q], sources[q], d_lab[b], st ? st + q : nullptr);
        if (rc != ETG_OK) break;
        ETG_CU(cudaEventRecord(cc->ev[1 + b], s));
        ETG_CU(cudaStreamWaitEvent(cs, cc->ev[1 + b], 0));
        ETG_CU(cudaMemcpyAsync(h_labels + (size_t)q * n, d_lab[b], 4 * n, cudaMemcpyDeviceToHost, cs));
        ETG_CU(cudaEventRecord(cc->ev[3 + b], cs));
    }
    cudaError_t e = cudaStreamSynchronize(cs);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess && rc == ETG_OK) rc = fail(ETG_ECUDA, std::string("run_host D2H: ") + cudaGetErrorString(e));
    return rc;
}

}  // namespace

etg_status etg_run_host(int alg, uint64_t n, uint64_t m, const void *h_off, const uint32_t *h_col,
                        const uint32_t *h_w, uint32_t source, uint32_t *h_labels, void *d_scratch,
                        size_t scratch_bytes, void *stream, const etg_options *opt, etg_stats *st) {
    return run_host_impl(n, m, h_off, h_col, h_w, 1, &alg, &source, h_labels, d_scratch, scratch_bytes, stream,
                         opt, st);
}

etg_status etg_run_host_batch(uint64_t n, uint64_t m, const void *h_off, const uint32_t *h_col,
                              const uint32_t *h_w, uint32_t n_queries, const int *algs, const uint32_t *sources,
                              uint32_t *h_labels, void *d_scratch, size_t scratch_bytes, void *stream,
                              const etg_options *opt, etg_stats *st) {
    return run_host_impl(n, m, h_off, h_col, h_w, n_queries, algs, sources, h_labels, d_scratch, scratch_bytes,
                         stream, opt, st);
}

// ---- communicator ---------------------------------------------------------
etg_status etg_comm_unique_id(uint8_t *id) {
    if (!id) return fail(ETG_EINVAL, "NULL id");
    memset(id, 0, etg::kCommIdBytes);
    memcpy(id, &etg::kCommMagic, 8);
    FILE *f = fopen("/dev/urandom", "rb");
    const size_t got = f ? fread(id + 8, 1, 24, f) : 0;
    if (f) fclose(f);
    if (got != 24) return fail(ETG_ENCCL, "could not read /dev/urandom");
    return ETG_OK;
}

etg_status etg_comm_init(etg_comm **out, int rank, int world, const uint8_t *id, int device) {
    if (!out || !id) return fail(ETG_EINVAL, "NULL argument");
    *out = nullptr;
    etg_comm *c = new (std::nothrow) etg_comm();
    if (!c) return fail(ETG_ENOMEM, "host allocation failed");
    bool bad_arg = false;
    const std::string err = etg::comm_open(c->c, id, rank, world, device, &bad_arg);
    if (!err.empty()) {
        etg::comm_close(c->c);
        delete c;
        return fail(bad_arg ? ETG_EINVAL : ETG_ENCCL, "etg_comm_init: " + err);
    }
    *out = c;
    return ETG_OK;
}

etg_status etg_comm_barrier(const etg_comm *c) {
    if (!c) return fail(ETG_EINVAL, "NULL communicator");
    ETG_BAR(c->c, "etg_comm_barrier");
    return ETG_OK;
}

void etg_comm_free(etg_comm *c) {
    if (!c) return;
    etg::comm_close(c->c);
    delete c;
}

const char *etg_status_str(etg_status s) {
    switch (s) {
        case ETG_OK: return "ETG_OK";
        case ETG_EINVAL: return "ETG_EINVAL";
        case ETG_ENOMEM: return "ETG_ENOMEM";
        case ETG_ECUDA: return "ETG_ECUDA";
        case ETG_ENCCL: return "ETG_ENCCL";
        case ETG_ENOTSYM: return "ETG_ENOTSYM";
        case ETG_ERANGE: return "ETG_ERANGE";
        case ETG_ENOWEIGHTS: return "ETG_ENOWEIGHTS";
        case ETG_EINVALID_CSR: return "ETG_EINVALID_CSR";
    }
    return "unknown";
}

const char *etg_last_error(void) { return g_err.c_str(); }

uint64_t etg_kernel_launches(void) { return g_launches.load(); }

etg_status etg_sssp_delta(etg_graph *g, uint32_t *delta) {
    if (!g || !delta) return fail(ETG_EINVAL, "NULL argument");
    if (g->has_w) {
        etg_status rc = resolve_delta(g);
        if (rc != ETG_OK) return rc;
    }
    *delta = g->p.nf_delta;
    return ETG_OK;
}

etg_status etg_debug_counters(etg_graph *g, uint64_t *out) {
    if (!g || !out) return fail(ETG_EINVAL, "null handle or output");
    const Ctl &c = *g->h_ctl;
    out[0] = c.depth;
    out[1] = c.nF;
    out[2] = c.nshadow;
    out[3] = c.edges;
    out[4] = c.activations;
    out[5] = c.iterations;
    return ETG_OK;
}

}  // extern "C"
