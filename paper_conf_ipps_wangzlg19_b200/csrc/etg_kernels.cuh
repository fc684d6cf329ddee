// etg_kernels.cuh -- sm_100a kernels of the EtaGraph hot path.
//
// Per iteration (Proc. 1 while-loop body), three kernels run on
// the handle's stream with every size kept on the device (no host readback):
//
//   udc_scan_kernel   step A2 (Def. 3; Sec. IV-A): for each
//                     active vertex v_j, c_j = ceil(deg(v_j)/K) shadow vertices;
//                     single-pass chained (decoupled look-back) exclusive scan
//                     S = scan(c), plus tile_first[t] = the active index owning
//                     shadow t*TS.  The scan replaces the paper's 12-byte
//                     3-tuples (L138): shadows are recomputed from (S, off).
//   expand_kernel     steps A2-A5: a persistent CTA maps a tile of TS shadows to
//                     (v, start, end) by a binary search in a shared-memory window
//                     of S; stages the tile's neighbour segments (<= TS*K words,
//                     the bound UDC gives, L199) in shared memory with cp.async
//                     (SMP, Sec. V-B); relaxes every staged edge with one
//                     thread per edge, a plain-load pre-filter and atomicMin/Max
//                     (Proc. 1 L207, reading R-4); appends activated vertices of
//                     out-degree >= 1 with one atomicAdd per warp (L217, R-5).
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

enum Alg : int { ALG_BFS = 0, ALG_SSSP = 1, ALG_CC = 2, ALG_SSWP = 3 };

// Device-resident control block (one per handle).
struct Ctl {
    uint32_t iter;        // iteration index within the current call
    uint32_t epoch;       // monotone over the handle's life: scan tags and stamps
    uint32_t count[2];    // active-set sizes; count[iter & 1] is the current one
    uint32_t nshadow;     // shadow vertices in the current iteration
    uint32_t ntiles;      // expand tiles in the current iteration
    uint32_t scan_ctr;    // dynamic tile counter of the chained scan
    uint32_t iterations;  // non-empty iterations of the current call
    unsigned long long activations;
    unsigned long long shadows;
    unsigned long long edges;
    unsigned long long frontier;
    uint32_t *label;      // output label array of the current call
    uint32_t source;
    uint32_t error;       // ETG_VALIDATE result
    unsigned long long reached_v;
    unsigned long long reached_e;
};

template <class OffT>
struct Dev {
    const OffT *off;
    const uint32_t *col;
    const uint32_t *w;
    uint32_t *F[2];             // active set ping-pong (capacity n)
    uint32_t *S;                // exclusive scan of shadow counts (capacity n+1)
    uint32_t *tile_first;       // active index owning shadow t*ts
    uint32_t *stamp;            // per-vertex iteration stamp (SSSP/CC/SSWP de-dup)
    unsigned long long *scan_status;  // chained-scan tile descriptors
    Ctl *ctl;
    uint32_t n;
    uint32_t K;                 // degree limit (Def. 3); unused with NO_UDC
    uint32_t ts;                // shadows per expand tile (<= kBlock, power of 2)
    uint32_t ts_log2;
};

// ------------------------------------------------------------------------- //
// small device helpers
// ------------------------------------------------------------------------- //
__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31; }

__device__ __forceinline__ uint32_t ld_cg(const uint32_t *p) { return __ldcg(p); }

__device__ __forceinline__ unsigned long long ld_volatile_u64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_volatile_u64(unsigned long long *p, unsigned long long v) {
    asm volatile("st.volatile.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void cp_async4(void *smem, const void *gmem) {
    uint32_t s = static_cast<uint32_t>(__cvta_generic_to_shared(smem));
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" :: "r"(s), "l"(gmem) : "memory");
}

__device__ __forceinline__ void cp_async_wait_all() {
    asm volatile("cp.async.wait_all;" ::: "memory");
}

// Active-set buffer k (0/1) without dynamic indexing of the kernel parameter
// (which would copy the parameter struct to local memory).
template <class OffT>
__device__ __forceinline__ uint32_t *fbuf(const Dev<OffT> &d, uint32_t k) { return k ? d.F[1] : d.F[0]; }

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

template <class OffT, int ALG>
__global__ __launch_bounds__(kBlock) void init_kernel(Dev<OffT> d, uint32_t *label, uint32_t source) {
    const uint32_t n = d.n;
    uint32_t *F0 = d.F[0];
    for (uint32_t v = blockIdx.x * kBlock + threadIdx.x; v - threadIdx.x < n; v += gridDim.x * kBlock) {
        const bool valid = v < n;
        bool act = false;
        if (valid) {
            uint32_t lab;
            if (ALG == ALG_CC) {
                lab = v;
                act = d.off[v + 1] > d.off[v];          // CC: every vertex with out-edges is active
            } else if (ALG == ALG_SSWP) {
                lab = (v == source) ? kInf : 0u;
            } else {
                lab = (v == source) ? 0u : kInf;
            }
            if (ALG != ALG_CC && v == source) act = d.off[v + 1] > d.off[v];
            label[v] = lab;
        }
        const uint32_t mask = __ballot_sync(kFull, act);
        if (mask) {
            const uint32_t leader = __ffs(mask) - 1;
            uint32_t pos = 0;
            if (lane_id() == leader) pos = atomicAdd(&d.ctl->count[0], __popc(mask));
            pos = __shfl_sync(kFull, pos, leader);
            if (act) F0[pos + __popc(mask & ((1u << lane_id()) - 1))] = v;
        }
    }
}

// ------------------------------------------------------------------------- //
// A2: UDC count + chained exclusive scan (+ tile_first), persistent CTAs with
// dynamically assigned scan tiles (in-order, so look-back always progresses).
// Tile descriptor: high 32 bits = (epoch << 2) | flag, low 32 bits = value;
// flag 1 = aggregate, 2 = inclusive prefix.
// ------------------------------------------------------------------------- //
template <class OffT, bool UDC>
__global__ __launch_bounds__(kBlock) void udc_scan_kernel(Dev<OffT> d) {
    __shared__ uint32_t s_tile;
    __shared__ uint32_t s_prefix;
    __shared__ uint32_t s_wsum[kWarps];
    Ctl *ctl = d.ctl;
    const uint32_t cur = ctl->iter & 1;
    const uint32_t nF = ctl->count[cur];
    const uint32_t epoch = ctl->epoch & 0x3FFFFFFFu;
    const uint32_t *F = fbuf(d, cur);
    const uint32_t nscan = (nF + kScanTile - 1) / kScanTile;
    const uint32_t ts = d.ts, tsl = d.ts_log2;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        ctl->count[cur ^ 1] = 0;              // the next active set starts empty (L140)
        if (nF == 0) {
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
        uint32_t c[kScanItems];
        uint32_t tsum = 0;
#pragma unroll
        for (int k = 0; k < kScanItems; ++k) {
            c[k] = 0;
            if (base + k < nF) {
                const uint32_t v = F[base + k];
                c[k] = udc_count<UDC>(d.off[v + 1] - d.off[v], d.K);
            }
            tsum += c[k];
        }
        uint32_t btotal;
        uint32_t tprefix = block_excl_scan(tsum, s_wsum, btotal);
        if (threadIdx.x == 0) {
            unsigned long long *st = d.scan_status;
            uint32_t excl = 0;
            if (tile == 0) {
                st_volatile_u64(&st[0], ((unsigned long long)((epoch << 2) | 2u) << 32) | btotal);
            } else {
                st_volatile_u64(&st[tile], ((unsigned long long)((epoch << 2) | 1u) << 32) | btotal);
                int p = (int)tile - 1;
                for (;;) {
                    const unsigned long long x = ld_volatile_u64(&st[p]);
                    const uint32_t hi = (uint32_t)(x >> 32);
                    if ((hi >> 2) != epoch || (hi & 3u) == 0) continue;   // not yet published
                    excl += (uint32_t)x;
                    if ((hi & 3u) == 2u) break;
                    --p;
                }
                st_volatile_u64(&st[tile], ((unsigned long long)((epoch << 2) | 2u) << 32) | (excl + btotal));
            }
            s_prefix = excl;
        }
        __syncthreads();
        uint32_t run = s_prefix + tprefix;
#pragma unroll
        for (int k = 0; k < kScanItems; ++k) {
            const uint32_t j = base + k;
            if (j < nF) {
                d.S[j] = run;
                // tiles whose first shadow t*ts lies in [run, run + c)
                for (uint32_t t = (run + ts - 1) >> tsl; (t << tsl) < run + c[k]; ++t) d.tile_first[t] = j;
            }
            run += c[k];
        }
        if (tile == nscan - 1 && threadIdx.x == kBlock - 1) {
            const uint32_t total = s_prefix + btotal;
            d.S[nF] = total;
            ctl->nshadow = total;
            ctl->ntiles = (total + ts - 1) >> tsl;
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------------------- //
// Tile mapping shared by expand_kernel and udc_dump_kernel: thread tid < cnt
// gets shadow i = t*ts + tid as (v, start, len).  The window sS/sF holds
// S[j0 ..] and F[j0 ..] with j0 = tile_first[t]; every active entry owns >= 1
// shadow, so the tile's entries lie in [j0, j0 + ts) and the window has at
// most ts + 1 entries.
// ------------------------------------------------------------------------- //
template <class OffT, bool UDC>
struct TileMap {
    uint32_t cnt;       // shadows in this tile
    uint32_t W;         // window entries
};

template <class OffT, bool UDC>
__device__ __forceinline__ TileMap<OffT, UDC> tile_load_window(const Dev<OffT> &d, uint32_t t,
                                                               uint32_t N, uint32_t nF,
                                                               const uint32_t *F,
                                                               uint32_t *sS, uint32_t *sF) {
    TileMap<OffT, UDC> tm;
    const uint32_t base = t << d.ts_log2;
    tm.cnt = min(d.ts, N - base);
    const uint32_t j0 = d.tile_first[t];
    tm.W = min(d.ts + 1, nF + 1 - j0);
    for (uint32_t k = threadIdx.x; k < tm.W; k += kBlock) {
        sS[k] = d.S[j0 + k];
        if (j0 + k < nF) sF[k] = F[j0 + k];
    }
    return tm;
}

// shadow i -> (v, start, len); sS window as loaded above.
template <class OffT, bool UDC>
__device__ __forceinline__ void map_shadow(const Dev<OffT> &d, uint32_t i, uint32_t W,
                                           const uint32_t *sS, const uint32_t *sF,
                                           uint32_t &v, OffT &start, OffT &len) {
    // largest jj with sS[jj] <= i (upper_bound - 1)
    uint32_t lo = 0, hi = W;
    while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (sS[mid] <= i) lo = mid; else hi = mid;
    }
    v = sF[lo];
    const OffT ob = d.off[v], oe = d.off[v + 1];
    if (UDC) {
        const OffT q = (OffT)(i - sS[lo]);
        start = ob + q * (OffT)d.K;
        const OffT rem = oe - start;
        len = rem < (OffT)d.K ? rem : (OffT)d.K;
    } else {
        start = ob;
        len = oe - ob;
    }
}

// ------------------------------------------------------------------------- //
// A4: relaxation of one edge (v -> u) with the source label `lab`
// (BFS: lab = level + 1 is the candidate itself).  Returns true iff u is
// activated (R-4, R-5).
// ------------------------------------------------------------------------- //
template <int ALG>
__device__ __forceinline__ bool relax(uint32_t *label, uint32_t *stamp, uint32_t tag,
                                      uint32_t u, uint32_t lab, uint32_t w) {
    if (ALG == ALG_BFS) {
        if (ld_cg(&label[u]) != kInf) return false;            // plain-load pre-filter
        return atomicMin(&label[u], lab) > lab;                // exactly one winner per vertex
    } else if (ALG == ALG_SSWP) {
        const uint32_t cand = lab < w ? lab : w;               // max-min (L62)
        if (cand <= ld_cg(&label[u])) return false;
        if (atomicMax(&label[u], cand) >= cand) return false;
        return atomicExch(&stamp[u], tag) != tag;
    } else {
        uint32_t cand;
        if (ALG == ALG_SSSP) {
            const unsigned long long s = (unsigned long long)lab + w;
            cand = s > kCap ? kCap : (uint32_t)s;              // saturating add (R-9)
        } else {
            cand = lab;                                        // CC: min-label propagation
        }
        if (cand >= ld_cg(&label[u])) return false;
        if (atomicMin(&label[u], cand) <= cand) return false;
        return atomicExch(&stamp[u], tag) != tag;              // once per iteration (R-5)
    }
}

// ------------------------------------------------------------------------- //
// A2-A5: expand.  Persistent grid; tile t covers shadows [t*ts, t*ts + ts).
// Dynamic shared memory (SMP only): col_s[cap_e], (w_s[cap_e]), sidx[cap_e].
// ------------------------------------------------------------------------- //
template <class OffT, int ALG, bool UDC, bool SMP>
__global__ __launch_bounds__(kBlock) void expand_kernel(Dev<OffT> d, uint32_t cap_e) {
    extern __shared__ __align__(16) uint8_t dyn_smem[];
    __shared__ uint32_t sS[kBlock + 1];
    __shared__ uint32_t sF[kBlock];
    __shared__ OffT sb[kBlock];          // segment start in col
    __shared__ OffT so[kBlock + 1];      // flat offset of the segment in the tile
    __shared__ uint32_t slab[kBlock];    // source label of each shadow
    __shared__ OffT s_wsum[kWarps];
    constexpr bool kW = (ALG == ALG_SSSP || ALG == ALG_SSWP);

    uint32_t *col_s = reinterpret_cast<uint32_t *>(dyn_smem);
    uint32_t *w_s = col_s + cap_e;
    uint8_t *sidx = reinterpret_cast<uint8_t *>(kW ? (w_s + cap_e) : w_s);

    Ctl *ctl = d.ctl;
    const uint32_t it = ctl->iter, cur = it & 1, nxt = cur ^ 1;
    const uint32_t nF = ctl->count[cur], N = ctl->nshadow, ntiles = ctl->ntiles;
    const uint32_t tag = ctl->epoch;
    uint32_t *label = ctl->label;
    const uint32_t *F = fbuf(d, cur);
    uint32_t *Fn = fbuf(d, nxt);
    uint32_t *cnt_n = &ctl->count[nxt];
    const uint32_t level = it + 1;
    const uint32_t lane = lane_id();
    const uint32_t tid = threadIdx.x;
    unsigned long long my_edges = 0;
    uint32_t my_acts = 0;

    for (uint32_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const TileMap<OffT, UDC> tm = tile_load_window<OffT, UDC>(d, t, N, nF, F, sS, sF);
        __syncthreads();
        OffT len = 0, start = 0;
        uint32_t lab = level;
        if (tid < tm.cnt) {
            uint32_t v;
            map_shadow<OffT, UDC>(d, (t << d.ts_log2) + tid, tm.W, sS, sF, v, start, len);
            if (ALG != ALG_BFS) lab = ld_cg(&label[v]);       // fresh source label (R-6)
        }
        OffT E;
        const OffT excl = block_excl_scan<OffT>(len, s_wsum, E);
        sb[tid] = start;
        so[tid] = excl;
        slab[tid] = lab;
        if (tid == 0) so[kBlock] = E;
        __syncthreads();
        if (SMP) {
            // SMP (Sec. V-B): stage every shadow's segment into shared memory;
            // warp w copies shadows w, w+8, ... with its lanes over the segment.
            for (uint32_t s = tid >> 5; s < tm.cnt; s += kWarps) {
                const OffT b = sb[s];
                const uint32_t o = (uint32_t)so[s];
                const uint32_t l = (uint32_t)(so[s + 1] - so[s]);
                for (uint32_t k = lane; k < l; k += 32) {
                    cp_async4(&col_s[o + k], &d.col[b + k]);
                    if (kW) cp_async4(&w_s[o + k], &d.w[b + k]);
                    sidx[o + k] = (uint8_t)s;
                }
            }
            cp_async_wait_all();
            __syncthreads();
        }
        for (OffT x0 = 0; x0 < E; x0 += kBlock) {
            const OffT x = x0 + tid;
            bool act = false;
            uint32_t u = 0;
            if (x < E) {
                uint32_t s, w = 0;
                if (SMP) {
                    s = sidx[x];
                    u = col_s[x];
                    if (kW) w = w_s[x];
                } else {
                    uint32_t lo = 0, hi = tm.cnt;             // largest s with so[s] <= x
                    while (hi - lo > 1) {
                        const uint32_t mid = (lo + hi) >> 1;
                        if (so[mid] <= x) lo = mid; else hi = mid;
                    }
                    s = lo;
                    const OffT e = sb[s] + (x - so[s]);
                    u = __ldg(&d.col[e]);
                    if (kW) w = __ldg(&d.w[e]);
                }
                if (relax<ALG>(label, d.stamp, tag, u, slab[s], w)) {
                    ++my_acts;
                    act = d.off[u + 1] > d.off[u];            // degree-0 vertices make no shadow (L142)
                }
            }
            // A5: warp-aggregated append to the next active set (L217)
            const uint32_t mask = __ballot_sync(kFull, act);
            if (mask) {
                const uint32_t leader = __ffs(mask) - 1;
                uint32_t pos = 0;
                if (lane == leader) pos = atomicAdd(cnt_n, __popc(mask));
                pos = __shfl_sync(kFull, pos, leader);
                if (act) Fn[pos + __popc(mask & ((1u << lane) - 1))] = u;
            }
        }
        my_edges += E;
        __syncthreads();
    }
    // statistics: one atomic per CTA
    for (int o = 16; o > 0; o >>= 1) my_acts += __shfl_xor_sync(kFull, my_acts, o);
    __shared__ uint32_t s_acts[kWarps];
    if (lane == 0) s_acts[tid >> 5] = my_acts;
    __syncthreads();
    if (tid == 0) {
        uint32_t a = 0;
        for (int k = 0; k < kWarps; ++k) a += s_acts[k];
        if (a) atomicAdd(&ctl->activations, (unsigned long long)a);
        if (my_edges) atomicAdd(&ctl->edges, (unsigned long long)my_edges);
    }
}

// ------------------------------------------------------------------------- //
// A6: iteration control (Proc. 1 "while actSet.isNotEmpty()", L207; reset of
// the consumed active set, L140).
// ------------------------------------------------------------------------- //
__global__ void advance_kernel(Ctl *ctl, cudaGraphConditionalHandle cond, int use_cond) {
    const uint32_t cur = ctl->iter & 1;
    if (ctl->count[cur] > 0) ctl->iterations += 1;
    ctl->frontier += ctl->count[cur];
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
    __shared__ uint32_t sS[kBlock + 1];
    __shared__ uint32_t sF[kBlock];
    Ctl *ctl = d.ctl;
    const uint32_t cur = ctl->iter & 1;
    const uint32_t nF = ctl->count[cur], N = ctl->nshadow, ntiles = ctl->ntiles;
    for (uint32_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const TileMap<OffT, UDC> tm = tile_load_window<OffT, UDC>(d, t, N, nF, fbuf(d, cur), sS, sF);
        __syncthreads();
        if (threadIdx.x < tm.cnt) {
            const uint32_t i = (t << d.ts_log2) + threadIdx.x;
            uint32_t v;
            OffT start, len;
            map_shadow<OffT, UDC>(d, i, tm.W, sS, sF, v, start, len);
            out_id[i] = v;
            out_start[i] = (uint64_t)start;
            out_end[i] = (uint64_t)(start + len);
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
