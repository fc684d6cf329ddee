// etg_kernels.cuh -- sm_100a kernels of the EtaGraph hot path.
//
// Per iteration (Proc. 1 while-loop body), three kernels run on
// the handle's stream with every size kept on the device (no host readback):
//
//   udc_scan_kernel   step A2 (Def. 3; Sec. IV-A).  Reads the
//                     raw active set R (vertices activated last iteration), and
//                     for each v gathers off[v], off[v+1] once: degree-0 vertices
//                     are dropped ("naturally filter active vertices with
//                     outdegree equals to 0", L142); the others get
//                     c = ceil(deg/K) shadow vertices.  A single-pass chained
//                     (decoupled look-back) scan over the pair (kept, c) writes
//                     the compacted active set F with, per entry, the start
//                     offset B, the degree D, the exclusive shadow prefix S,
//                     and tile_first[t] = the
//                     entry owning shadow t*TS.  These arrays replace the
//                     paper's 12-byte 3-tuples (L138): a shadow is recomputed
//                     from (S, B, D) in O(1) once its entry is known.
//   expand_kernel     steps A2-A5.  A persistent CTA takes tiles of TS
//                     consecutive shadows: it loads the tile's window of
//                     (S, B, D, F) (coalesced), maps each shadow to its slice
//                     by a binary search in shared memory, stages the tile's
//                     neighbour segments (<= TS*K words -- the bound UDC gives,
//                     L199) in shared memory with cp.async (SMP, Sec. V-B
//                     L197-209), then relaxes every staged edge, one thread per
//                     edge and kR edges in flight per thread: plain-load
//                     pre-filter, atomicMin/Max (Proc. 1 L207, reading R-4),
//                     and a warp-aggregated append of the winners to R (L217).
//   advance_kernel    step A6: iteration bookkeeping; sets the CUDA-graph
//                     conditional ("while actSet.isNotEmpty()", L207).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace etg {

constexpr uint32_t kInf = 0xFFFFFFFFu;
constexpr uint32_t kCap = 0xFFFFFFFEu;
constexpr int kBlock = 256;                 // threads per CTA (8 warps)
constexpr int kWarps = kBlock / 32;
constexpr int kScanItems = 8;               // active-set entries per thread in the scan
constexpr int kScanTile = kBlock * kScanItems;
constexpr uint32_t kFull = 0xFFFFFFFFu;
constexpr int kR = 8;                       // edges in flight per thread in the relax loop
constexpr uint32_t kQCap = 256;             // per-warp append queue (>= 32 * kR)

enum Alg : int { ALG_BFS = 0, ALG_SSSP = 1, ALG_CC = 2, ALG_SSWP = 3 };

// Device-resident control block (one per handle).
struct Ctl {
    uint32_t iter;        // iteration index within the current call
    uint32_t epoch;       // monotone over the handle's life: scan tags and stamps
    uint32_t count[2];    // raw active-set sizes; count[iter & 1] is the current one
    uint32_t nF;          // compacted active-set size (entries with out-degree > 0)
    uint32_t nshadow;     // shadow vertices in the current iteration
    uint32_t ntiles;      // expand tiles in the current iteration
    uint32_t scan_ctr;    // dynamic tile counter of the chained scan
    uint32_t iterations;  // non-empty iterations of the current call
    uint32_t error;       // ETG_VALIDATE result
    unsigned long long activations;
    unsigned long long shadows;
    unsigned long long edges;
    unsigned long long frontier;
    unsigned long long reached_v;
    unsigned long long reached_e;
    uint32_t *label;      // output label array of the current call
    uint32_t source;
    uint32_t pad;
};

template <class OffT>
struct Dev {
    const OffT *off;
    const uint32_t *col;
    const uint32_t *w;
    uint32_t *R;                // raw active set (appended by expand, read by scan)
    uint32_t *F;                // compacted active set (vertex ids)
    OffT *B;                    // off[F[k]]
    uint32_t *D;                // out-degree of F[k] (> 0)
    uint32_t *S;                // exclusive prefix of shadow counts (nF + 1 entries)
    uint32_t *tile_first;       // entry owning shadow t*ts
    uint32_t *stamp;            // per-vertex iteration stamp (SSSP/CC/SSWP de-dup)
    uint32_t *st_flag;          // chained scan: per scan tile (epoch << 2 | flag)
    unsigned long long *st_agg; //   aggregate  (entries << 32 | shadows)
    unsigned long long *st_inc; //   inclusive prefix, same packing
    Ctl *ctl;
    uint32_t n;
    uint32_t K;                 // degree limit (Def. 3); unused with NO_UDC
    uint32_t ts;                // shadows per expand tile (<= kBlock, power of 2)
    uint32_t ts_log2;
    uint32_t tune;              // experiment switches (ETG_TUNE env var at load); 0 = default
};

// tune bits
constexpr uint32_t kTuneFilterL1 = 1u;    // pre-filter label loads cached in L1
constexpr uint32_t kTuneMatchAny = 2u;    // suppress same-vertex atomics within a warp
constexpr uint32_t kTuneBfsStore = 4u;    // EXPERIMENT ONLY: BFS plain store, duplicates kept

// ------------------------------------------------------------------------- //
// small device helpers
// ------------------------------------------------------------------------- //
__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31; }

__device__ __forceinline__ uint32_t ld_cg(const uint32_t *p) { return __ldcg(p); }

// Pre-filter load of a label (reading R-4): cached in L1, so a hub's label is
// fetched once per SM instead of once per in-edge.  Labels move monotonically
// (down for BFS/SSSP/CC, up for SSWP), so a stale L1 copy can only make the
// filter pass an edge the atomic then rejects -- never drop an improvement.
__device__ __forceinline__ uint32_t ld_filter(const uint32_t *p) {
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

// Block-wide exclusive scan of one value per thread; returns the exclusive
// prefix, writes the block total.  `wsum` is kWarps words of shared memory.
template <class T>
__device__ __forceinline__ T block_excl_scan(T x, T *wsum, T &total) {
    T incl = warp_incl_scan(x);
    const uint32_t warp = threadIdx.x >> 5;
    if (lane_id() == 31) wsum[warp] = incl;
    __syncthreads();
    if (warp == 0) {
        T s = lane_id() < (uint32_t)kWarps ? wsum[lane_id()] : T(0);
        s = warp_incl_scan(s);
        if (lane_id() < (uint32_t)kWarps) wsum[lane_id()] = s;
    }
    __syncthreads();
    T warp_prefix = warp ? wsum[warp - 1] : T(0);
    total = wsum[kWarps - 1];
    __syncthreads();
    return warp_prefix + incl - x;
}

// Number of shadow vertices of a vertex of out-degree `deg` (Def. 3; L142:
// degree 0 gives none).
template <bool UDC, class D>
__device__ __forceinline__ uint32_t udc_count(D deg, uint32_t K) {
    if (UDC) return (uint32_t)((deg + (D)K - 1) / (D)K);
    return deg > 0 ? 1u : 0u;
}

// ------------------------------------------------------------------------- //
// A1: per-call control reset and label initialisation (Proc. 1 "Init label",
// "Init actSet", L207)
// ------------------------------------------------------------------------- //
__global__ void ctl_begin_kernel(Ctl *ctl, uint32_t *label, uint32_t source) {
    ctl->iter = 0;
    ctl->epoch += 1;
    ctl->count[0] = 0;
    ctl->count[1] = 0;
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
}

// BFS/SSSP: label = INF, label[s] = 0, R = {s}.  SSWP: label = 0, label[s] =
// INF.  CC: label[v] = v, R = all vertices (the scan drops degree-0 ones).
template <class OffT, int ALG>
__global__ __launch_bounds__(kBlock) void init_kernel(Dev<OffT> d, uint32_t *label, uint32_t source) {
    const uint32_t n = d.n;
    const uint32_t stride = gridDim.x * kBlock;
    for (uint32_t v = blockIdx.x * kBlock + threadIdx.x; v < n; v += stride) {
        uint32_t lab;
        if (ALG == ALG_CC) {
            lab = v;
            d.R[v] = v;
        } else if (ALG == ALG_SSWP) {
            lab = (v == source) ? kInf : 0u;
        } else {
            lab = (v == source) ? 0u : kInf;
        }
        label[v] = lab;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        if (ALG == ALG_CC) {
            d.ctl->count[0] = n;
        } else {
            d.R[0] = source;
            d.ctl->count[0] = 1;
        }
    }
}

// ------------------------------------------------------------------------- //
// A2: UDC count + compaction + chained exclusive scan (+ tile_first).
// Persistent CTAs take scan tiles in order from a counter, so the look-back
// always makes progress.  Values are packed (kept entries << 32 | shadows);
// neither half can carry into the other (entries <= n < 2^32, shadows < 2^32
// checked at load time).  The look-back is warp-parallel: warp 0 inspects 32
// predecessors per step.
// ------------------------------------------------------------------------- //
__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long x) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(kFull, x, o);
    return x;
}

template <class OffT, bool UDC>
__global__ __launch_bounds__(kBlock) void udc_scan_kernel(Dev<OffT> d) {
    typedef unsigned long long u64;
    __shared__ uint32_t s_tile;
    __shared__ u64 s_prefix;
    __shared__ u64 s_wsum[kWarps];
    Ctl *ctl = d.ctl;
    const uint32_t cur = ctl->iter & 1;
    const uint32_t nR = ctl->count[cur];
    const uint32_t epoch = ctl->epoch & 0x3FFFFFFFu;
    const uint32_t nscan = (nR + kScanTile - 1) / kScanTile;
    const uint32_t ts = d.ts, tsl = d.ts_log2;
    const uint32_t lane = lane_id();
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        ctl->count[cur ^ 1] = 0;              // the next raw active set starts empty (L140)
        if (nR == 0) {
            ctl->nF = 0;
            ctl->nshadow = 0;
            ctl->ntiles = 0;
            d.S[0] = 0;
        }
    }
    for (;;) {
        if (threadIdx.x == 0) s_tile = atomicAdd(&ctl->scan_ctr, 1u);
        __syncthreads();
        const uint32_t tile = s_tile;
        if (tile >= nscan) break;
        const uint32_t base = tile * kScanTile + threadIdx.x * kScanItems;
        uint32_t v[kScanItems], c[kScanItems];
        OffT ob[kScanItems], deg[kScanItems];
        u64 tsum = 0;
#pragma unroll
        for (int k = 0; k < kScanItems; ++k) v[k] = (base + k < nR) ? d.R[base + k] : kInf;
#pragma unroll
        for (int k = 0; k < kScanItems; ++k) {
            ob[k] = 0;
            deg[k] = 0;
            if (v[k] != kInf) {
                ob[k] = d.off[v[k]];
                deg[k] = d.off[v[k] + 1] - ob[k];
            }
        }
#pragma unroll
        for (int k = 0; k < kScanItems; ++k) {
            c[k] = udc_count<UDC>(deg[k], d.K);
            tsum += ((u64)(c[k] > 0) << 32) | c[k];
        }
        u64 btotal;
        const u64 tprefix = block_excl_scan<u64>(tsum, s_wsum, btotal);
        if (threadIdx.x < 32) {
            u64 excl = 0;
            if (tile == 0) {
                if (lane == 0) {
                    d.st_inc[0] = btotal;
                    __threadfence();
                    atomicExch(&d.st_flag[0], (epoch << 2) | 2u);
                }
            } else {
                if (lane == 0) {
                    d.st_agg[tile] = btotal;
                    __threadfence();
                    atomicExch(&d.st_flag[tile], (epoch << 2) | 1u);
                }
                int p = (int)tile - 1;                  // nearest predecessor in lane 0
                for (;;) {
                    const int q = p - (int)lane;
                    uint32_t f = (epoch << 2) | 1u;     // q < 0: beyond tile 0, never used
                    if (q >= 0) f = ld_volatile_u32(&d.st_flag[q]);
                    const bool valid = (f >> 2) == epoch && (f & 3u) != 0;
                    const uint32_t incl = __ballot_sync(kFull, valid && (f & 3u) == 2u && q >= 0);
                    const uint32_t inval = __ballot_sync(kFull, !valid);
                    const uint32_t first = incl ? (uint32_t)(__ffs(incl) - 1) : 32u;
                    const uint32_t need = first < 31 ? ((2u << first) - 1u) : kFull;
                    if (inval & need) continue;         // a needed predecessor is not published yet
                    __threadfence();
                    u64 val = 0;
                    if (lane < first && q >= 0) val = ld_volatile_u64(&d.st_agg[q]);
                    else if (lane == first) val = ld_volatile_u64(&d.st_inc[q]);
                    excl += warp_sum_u64(val);
                    if (first < 32) break;
                    p -= 32;
                }
                if (lane == 0) {
                    d.st_inc[tile] = excl + btotal;
                    __threadfence();
                    atomicExch(&d.st_flag[tile], (epoch << 2) | 2u);
                }
            }
            if (lane == 0) s_prefix = excl;
        }
        __syncthreads();
        u64 run = s_prefix + tprefix;
#pragma unroll
        for (int k = 0; k < kScanItems; ++k) {
            if (c[k]) {
                const uint32_t pos = (uint32_t)(run >> 32);
                const uint32_t sh = (uint32_t)run;
                d.F[pos] = v[k];
                d.B[pos] = ob[k];
                d.D[pos] = (uint32_t)deg[k];
                d.S[pos] = sh;
                // tiles whose first shadow t*ts lies in [sh, sh + c)
                for (uint32_t t = (sh + ts - 1) >> tsl; (t << tsl) < sh + c[k]; ++t) d.tile_first[t] = pos;
            }
            run += ((u64)(c[k] > 0) << 32) | c[k];
        }
        if (tile == nscan - 1 && threadIdx.x == 0) {
            const u64 total = s_prefix + btotal;
            const uint32_t nF = (uint32_t)(total >> 32), N = (uint32_t)total;
            d.S[nF] = N;
            ctl->nF = nF;
            ctl->nshadow = N;
            ctl->ntiles = (N + ts - 1) >> tsl;
        }
        __syncthreads();
    }
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
// label[v] + 1"), split in three so a thread keeps kR independent edges in
// flight: candidate -> plain-load pre-filter -> atomic (R-4).  BFS passes the
// candidate level + 1 as `lab`.
// ------------------------------------------------------------------------- //
// Copy a warp's queue of qn activated vertices to the raw active set R.
__device__ __forceinline__ void warp_flush(const uint32_t *wq, uint32_t qn, uint32_t *R,
                                           uint32_t *cnt) {
    uint32_t base = 0;
    if (lane_id() == 0) base = atomicAdd(cnt, qn);
    base = __shfl_sync(kFull, base, 0);
    for (uint32_t k = lane_id(); k < qn; k += 32) R[base + k] = wq[k];
    __syncwarp();
}

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

// true iff this thread's atomic lowered (raised, SSWP) the label
template <int ALG>
__device__ __forceinline__ bool atomic_improve(uint32_t *p, uint32_t cand) {
    if (ALG == ALG_SSWP) return atomicMax(p, cand) < cand;
    return atomicMin(p, cand) > cand;
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
    extern __shared__ __align__(16) uint8_t dyn_smem[];
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
    const uint32_t it = ctl->iter, nxt = (it & 1) ^ 1;
    const uint32_t nF = ctl->nF, N = ctl->nshadow, ntiles = ctl->ntiles;
    const uint32_t tag = ctl->epoch;
    uint32_t *label = ctl->label;
    uint32_t *Rn = d.R;
    uint32_t *cnt_n = &ctl->count[nxt];
    const uint32_t level = it + 1;
    const uint32_t lane = lane_id();
    const uint32_t tid = threadIdx.x;
    unsigned long long my_edges = 0;
    uint32_t my_acts = 0;
    __shared__ uint32_t s_queue[kWarps][kQCap];    // per-warp queue of activated vertices
    uint32_t *wq = s_queue[tid >> 5];
    uint32_t qn = 0;                                // warp-uniform queue length

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
        // A4 + A5 in batches of kR edges per thread: all loads of a batch are
        // issued before any is consumed (memory-level parallelism).
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
                cur[r] = act[r] ? ((d.tune & kTuneFilterL1) ? ld_filter(&label[u[r]]) : ld_cg(&label[u[r]])) : 0u;
#pragma unroll
            for (int r = 0; r < kR; ++r) act[r] = act[r] && improves<ALG>(c[r], cur[r]);
            if (d.tune & kTuneMatchAny) {
#pragma unroll
                for (int r = 0; r < kR; ++r) {
                    const uint32_t peers = __match_any_sync(kFull, act[r] ? u[r] : kInf);
                    // among lanes proposing the same vertex keep the best candidate
                    // (BFS: all equal, so the lowest lane)
                    uint32_t best = act[r] ? c[r] : (ALG == ALG_SSWP ? 0u : kInf);
                    for (uint32_t m = peers; m; m &= m - 1) {
                        const uint32_t o = __shfl_sync(peers, best, __ffs(m) - 1);
                        (void)o;
                    }
                    if (act[r] && (peers & ((1u << lane) - 1)) && ALG == ALG_BFS) act[r] = false;
                }
            }
            if (ALG == ALG_BFS && (d.tune & kTuneBfsStore)) {
#pragma unroll
                for (int r = 0; r < kR; ++r)
                    if (act[r]) label[u[r]] = c[r];
            } else {
#pragma unroll
                for (int r = 0; r < kR; ++r)
                    if (act[r]) act[r] = atomic_improve<ALG>(&label[u[r]], c[r]);
            }
            if (ALG != ALG_BFS) {                              // once per iteration (R-5)
#pragma unroll
                for (int r = 0; r < kR; ++r)
                    if (act[r]) act[r] = atomicExch(&d.stamp[u[r]], tag) != tag;
            }
            // A5: append the winners to the warp's shared-memory queue; the
            // queue is flushed to R with ONE atomicAdd per kQCap entries
            // (L217's atomic append, aggregated: a single global counter would
            // otherwise serialise every warp of the grid).
            uint32_t masks[kR], total = 0;
#pragma unroll
            for (int r = 0; r < kR; ++r) {
                masks[r] = __ballot_sync(kFull, act[r]);
                total += __popc(masks[r]);
            }
            if (total) {
                if (qn + total > kQCap) {
                    warp_flush(wq, qn, Rn, cnt_n);
                    qn = 0;
                }
                uint32_t base = qn;
                const uint32_t lt = (1u << lane) - 1;
#pragma unroll
                for (int r = 0; r < kR; ++r) {
                    if (act[r]) wq[base + __popc(masks[r] & lt)] = u[r];
                    base += __popc(masks[r]);
                }
                qn += total;
                my_acts += (lane == 0) ? total : 0u;
                __syncwarp();
            }
        }
        my_edges += E;
        __syncthreads();
    }
    if (qn) warp_flush(wq, qn, Rn, cnt_n);
    // statistics: one atomic per CTA
    __shared__ uint32_t s_acts[kWarps];
    if (lane == 0) s_acts[tid >> 5] = my_acts;
    __syncthreads();
    if (tid == 0) {
        uint32_t a = 0;
        for (int k = 0; k < kWarps; ++k) a += s_acts[k];
        if (a) atomicAdd(&ctl->activations, (unsigned long long)a);
        if (my_edges) atomicAdd(&ctl->edges, my_edges);
    }
}

// ------------------------------------------------------------------------- //
// A6: iteration control (Proc. 1 "while actSet.isNotEmpty()", L207; reset of
// the consumed active set, L140).
// ------------------------------------------------------------------------- //
__global__ void advance_kernel(Ctl *ctl, cudaGraphConditionalHandle cond, int use_cond) {
    const uint32_t cur = ctl->iter & 1;
    if (ctl->nF > 0) ctl->iterations += 1;
    ctl->frontier += ctl->nF;
    ctl->shadows += ctl->nshadow;
    ctl->iter += 1;
    ctl->epoch += 1;
    ctl->scan_ctr = 0;
    if (use_cond) cudaGraphSetConditional(cond, ctl->count[cur ^ 1] > 0 ? 1u : 0u);
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
        const uint32_t W = load_window<OffT, false>(d, t, nF, win);
        const uint32_t cnt = min(d.ts, N - (t << d.ts_log2));
        __syncthreads();
        if (threadIdx.x < cnt) {
            const uint32_t i = (t << d.ts_log2) + threadIdx.x;
            OffT start;
            uint32_t len;
            const uint32_t jj = map_shadow<OffT, UDC>(d, i, W, win, start, len);
            out_id[i] = d.F[d.tile_first[t] + jj];
            out_start[i] = (uint64_t)start;
            out_end[i] = (uint64_t)start + len;
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------------------- //
// statistics and validation
// ------------------------------------------------------------------------- //
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
    for (uint64_t v = t0; v < d.n; v += gsz)
        if (d.off[v + 1] < d.off[v]) atomicOr(&d.ctl->error, 2u);
    for (uint64_t e = t0; e < m; e += gsz)
        if (d.col[e] >= d.n) atomicOr(&d.ctl->error, 4u);
}

}  // namespace etg
