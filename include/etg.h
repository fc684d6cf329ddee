/*
 * etg.h -- C ABI of the B200-native EtaGraph frontier-expansion library (libetg.so).
 *
 * What it computes (Sec. II-C): "Graph traversal is to calculate
 * labels of all nodes reachable from a given root node."  Procedure 1 (L205-207):
 * Data = graph in CSR format, Result = vertex labels, computed by push expansion
 * of an active set (Def. 1), each active vertex cut into shadow vertices of
 * at most K out-edges (Unified Degree Cut, Def. 3), neighbour segments
 * staged in shared memory (SMP, Sec. V-B), labels relaxed with an
 * atomic min and the next active set compacted (L136-140, L217).
 *
 * Conventions (DESIGN.md readings):
 *   - vertex ids, labels, depths, distances and weights are uint32;
 *   - INF = 0xFFFFFFFF marks "unreached" (BFS, SSSP); SSSP distances saturate at
 *     CAP = 0xFFFFFFFE (R-9); n must be <= 0xFFFFFFFE;
 *   - CSR: row offsets off[n+1] (uint32, or uint64 with ETG_OFFSETS_U64),
 *     column ids col[m], weights w[m] (structure of arrays, L55).
 *
 * Ownership: every d_* pointer is caller-owned DEVICE memory that the library
 * borrows; the CSR arrays and the workspace must outlive the handle.  Output
 * arrays are fully overwritten (n entries).  Apart from the handle itself (host
 * memory) and one small pinned host word, the library allocates nothing, except
 * in etg_run_host, which works on host buffers.
 *
 * Streams: all work is enqueued on the handle's stream (a cudaStream_t passed as
 * void*, NULL = legacy default stream).  Traversal calls return after the work
 * has completed (they read back the iteration statistics).  A handle is not
 * thread-safe; separate handles are independent.
 *
 * Errors: functions return a negative etg_status on failure; nothing partial is
 * guaranteed then.  etg_last_error() returns a thread-local detail string.
 *
 * Results never depend on K, ETG_NO_UDC, ETG_NO_SMP or ETG_HOST_LOOP
 * (Theorems 1-2, L119-127): the labels are unique fixpoints.
 */
#ifndef ETG_H
#define ETG_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct etg_graph etg_graph; /* opaque handle */
typedef struct etg_comm etg_comm;   /* opaque communicator (multi-GPU partitions on one node); NULL = one GPU */

typedef enum {
    ETG_OK = 0,
    ETG_EINVAL = -1,      /* bad argument (NULL pointer, source >= n, K = 0 with UDC, ...) */
    ETG_ENOMEM = -2,      /* workspace too small, or host allocation failed */
    ETG_ECUDA = -3,       /* a CUDA runtime error (detail in etg_last_error) */
    ETG_ENCCL = -4,       /* communicator failure: rendezvous, peer mapping, a peer that died or timed out
                             (ETG_COMM_TIMEOUT_S, default 600 s), ranks that disagree on the graph */
    ETG_ENOTSYM = -5,     /* etg_cc on a handle loaded without ETG_SYMMETRIC */
    ETG_ERANGE = -6,      /* sizes exceed the index types (n > 2^32-2, m >= 2^32 with u32 offsets, ...) */
    ETG_ENOWEIGHTS = -7,  /* etg_sssp / etg_sswp on a handle loaded without weights */
    ETG_EINVALID_CSR = -8 /* ETG_VALIDATE found a malformed CSR */
} etg_status;

enum {
    ETG_SYMMETRIC = 1u << 0,   /* caller asserts the CSR is symmetric (required by etg_cc) */
    ETG_NO_UDC = 1u << 1,      /* ablation: one work item per active vertex (K = infinity) */
    ETG_NO_SMP = 1u << 2,      /* ablation ("w/o SMP", Sec. VI-C): no look-ahead fetch of the
                                  next batch's neighbour segments (default: register look-ahead,
                                  BFS) */
    ETG_OFFSETS_U64 = 1u << 3, /* d_row_offsets holds uint64 (needed when m >= 2^32) */
    ETG_VALIDATE = 1u << 4,    /* etg_load_csr runs an O(n+m) device check of the CSR */
    ETG_HOST_LOOP = 1u << 5,   /* drive iterations from the host (count read back each
                                  iteration) instead of a CUDA-graph conditional while node */
    ETG_PROFILE = 1u << 6,     /* implies ETG_HOST_LOOP; CUDA events around every scan and
                                  expand launch on the handle's stream fill scan_ms/expand_ms */
    ETG_SMP_SHARED = 1u << 7,  /* SMP as literally described (L199): TMA bulk copies of the next
                                  tile's segments into per-warp shared-memory stages (K <= 32) */
    ETG_HOST_EDGES = 1u << 8,  /* host-resident edge mode (NEXT-2; Sec. IV-B): d_col_idx
                                  and d_weights point to pinned, device-mapped HOST memory (UVA
                                  zero-copy); each iteration reads only the active vertices' edges
                                  over the host link.  Offsets and workspace stay in HBM. */
    ETG_PUSH = 1u << 9         /* communicator handles only: the CSR is the rank's SOURCE partition
                                  (rows v_lo..v_hi-1 keep their out-edges, the others are empty;
                                  global ids) and the expand kernel reduces every relaxation of a
                                  foreign vertex into its owner's labels over peer memory (SURVEY
                                  8(f) NEXT-3).  SSSP/CC/SSWP; etg_bfs returns ETG_EINVAL. */
};

typedef struct {
    uint32_t degree_limit_k; /* K of Def. 3; 0 -> default 32 */
    uint32_t flags;          /* ETG_* bits above */
    uint32_t sssp_delta;     /* 0: the paper's schedule (every improved vertex is active in the
                                next iteration, L64/L78).  > 0: wave schedule for SSSP --
                                improved vertices at distance >= a threshold stay active but are
                                deferred; the threshold advances by sssp_delta after every
                                iteration (and jumps past an empty gap).  Same distances (unique
                                fixpoint), fewer redundant relaxations.  ETG_SSSP_DELTA_AUTO:
                                6 x mean edge weight / mean out-degree, at least 1 (one O(m)
                                reduction at the first SSSP call of the handle; 12 / 13 / 6 for
                                the C2 / C3 / C4 configs).
                                The step-wise (multi-GPU) API honours it too: the deferred
                                vertices keep a stale snapshot, identical on every rank. */
} etg_options;
#define ETG_SSSP_DELTA_AUTO 0xFFFFFFFFu

typedef struct {
    uint32_t iterations;       /* non-empty active sets processed (Proc. 1 while-loop trips) */
    uint32_t expand_launches;  /* expand kernel launches (ETG_PROFILE) */
    uint64_t activations;      /* vertex activations: (vertex, iteration) pairs marked active,
                                  the initial active set included (degree-0 vertices too) */
    uint64_t frontier_total;   /* sum over iterations of the active-set size */
    uint64_t shadows;          /* shadow vertices processed, summed over iterations (|N|, L152) */
    uint64_t edges_processed;  /* edges relaxed, summed over iterations */
    uint64_t vertices_reached; /* filled by etg_reach_stats */
    uint64_t edges_reached;    /* filled by etg_reach_stats: sum of out-degrees of reached vertices */
    float ms;                  /* device time of the traversal call (CUDA events) */
    float scan_ms;             /* ETG_PROFILE: summed CUDA-event time of the udc_scan launches */
    float expand_ms;           /* ETG_PROFILE: summed CUDA-event time of the expand launches */
    float reserved;
} etg_stats;

/* Bytes of device workspace etg_load_csr needs for n vertices and m edges. */
size_t etg_workspace_bytes(uint64_t n, uint64_t m, const etg_options *opt);

/* Create a handle over a caller-owned device CSR (Proc. 1 "Load data", L207;
 * the CSR is used unmodified, L113).  d_weights may be NULL (then SSSP/SSWP
 * return ETG_ENOWEIGHTS).  stream is a cudaStream_t (void* here).
 *
 * comm == NULL: one GPU; v_lo / v_hi are ignored (the handle owns [0, n)).
 * comm != NULL (collective: every rank of the communicator calls it, in any
 * order, each with its own partition): the 1-D vertex partition of SURVEY
 * 8(e) -- rank r owns [v_lo, v_hi); the ranges must tile [0, n) in rank order
 * with inner bounds multiples of 32 (one bitmap word, one owner).  n is the
 * GLOBAL vertex count and m the number of edges of this rank's sub-CSR:
 *   default (destination partition): rows = all n sources, only the edges
 *     whose destination lies in [v_lo, v_hi), global ids;
 *   ETG_PUSH (source partition): rows v_lo..v_hi-1 keep all their out-edges,
 *     every other row is empty.
 * The call exchanges the workspaces' CUDA-IPC handles through the
 * communicator and maps every peer's workspace into this process, so each
 * traversal's per-iteration exchange is done by the library's kernels writing
 * into the peers' device memory (NVLink / NVSwitch between GPUs).  Errors:
 * ETG_EINVAL (range outside [0, n], ETG_PUSH without comm), ETG_ENCCL (ranges
 * that do not tile [0, n), ranks that disagree on n or ETG_PUSH, a peer that
 * cannot be mapped or does not arrive). */
etg_status etg_load_csr(etg_graph **out, uint64_t n, uint64_t m,
                        const void *d_row_offsets, const uint32_t *d_col_idx,
                        const uint32_t *d_weights, void *d_workspace,
                        size_t workspace_bytes, void *stream, const etg_options *opt,
                        const etg_comm *comm, uint32_t v_lo, uint32_t v_hi);

/* BFS (Proc. 1 Kernel BFS, L207): d_depth[v] = hop distance from source, INF if
 * unreachable.
 * On a communicator handle (all four traversals): collective -- every rank
 * calls it with the same source; the whole partitioned Proc. 1 loop runs
 * inside the call (per iteration: expand, exchange over peer memory, host
 * barrier, scan, barrier with the termination count) and the output array
 * receives the OWNED slice only: v_hi - v_lo entries, d_out[i] = label of
 * vertex v_lo + i.  Statistics are summed over the ranks; st->ms is the
 * maximum over the ranks of the call's device time (st->reserved: this
 * rank's own). */
etg_status etg_bfs(etg_graph *g, uint32_t source, uint32_t *d_depth, etg_stats *st_or_null);

/* SSSP (L62, L78): d_dist[v] = saturating shortest-path distance (CAP), INF if
 * unreachable. */
etg_status etg_sssp(etg_graph *g, uint32_t source, uint32_t *d_dist, etg_stats *st_or_null);

/* CC (BASELINE.json north_star; R-12): d_label[v] = minimum vertex id of v's
 * connected component.  Requires a handle loaded with ETG_SYMMETRIC. */
etg_status etg_cc(etg_graph *g, uint32_t *d_label, etg_stats *st_or_null);

/* SSWP (L62, L249; NEXT-1): d_width[v] = max over paths of the minimum edge
 * weight; width[source] = INF, unreachable = 0. */
etg_status etg_sswp(etg_graph *g, uint32_t source, uint32_t *d_width, etg_stats *st_or_null);

/* Reach statistics of a label array: vertices with label != unreached and the
 * sum of their out-degrees (m of the activatable subgraph, Def. 2). */
etg_status etg_reach_stats(etg_graph *g, const uint32_t *d_label, uint32_t unreached,
                           etg_stats *st);

/* Step A2 exposed for testing: the Unified Degree Cut of an active set, computed
 * by the same device code the traversal uses (Def. 3; Sec. IV-A).
 * d_active[n_active] (device) is the active set (a set: duplicates are merged);
 * degree-0 vertices produce no shadow (L142).  Active vertices are taken in
 * increasing id order (the library keeps the active set as a bitmap); shadow q
 * of vertex v is written as (d_id, d_start, d_end) = (v, off[v]+qK,
 * min(off[v]+(q+1)K, off[v+1])), uint32/uint64/uint64 device arrays of `cap`
 * entries; *n_out receives the number of shadows (ETG_ENOMEM if > cap). */
etg_status etg_udc_slices(etg_graph *g, const uint32_t *d_active, uint32_t n_active,
                          uint32_t *d_id, uint64_t *d_start, uint64_t *d_end,
                          uint64_t cap, uint64_t *n_out);

/* Tuning/debug: run `alg` from `source` until the active set of iteration
 * `depth` is ready, snapshot it, then time `reps` launches of the expand kernel
 * on that same state (labels restored from d_saved, n words of device scratch,
 * before each launch).  tune = experiment bits (0 = the production kernel).
 * Outputs the mean launch time, the edges one launch relaxes and the active-set
 * size.  Not part of the traversal path; d_label is left as the snapshot. */
etg_status etg_debug_expand_replay(etg_graph *g, int alg, uint32_t source, uint32_t depth,
                                   uint32_t tune, int reps, uint32_t *d_label, uint32_t *d_saved,
                                   float *ms, uint64_t *edges, uint32_t *n_active);

/* ---- Step-wise driving of one handle (per-iteration tracing and tuning;
 * the communicator loop is built from the same steps).  Protocol:
 *   etg_step_begin -> while (n_active) { etg_step_expand; etg_step_scan } ->
 *   etg_step_end.
 * etg_step_begin runs A1 and the first scan (the initial active set);
 * n_active is the number of vertices the scan activated (bitmap bits
 * consumed).  The Proc. 1 loop is identical to etg_bfs/... except that the
 * host reads n_active back every iteration.  etg_bitmap_layout: the active-set
 * bitmap Q is nwords uint32 words at offset_bytes into the workspace.
 * ETG_EINVAL: NULL arguments, alg outside 0..3, source >= n, a step without
 * etg_step_begin, SSSP on a handle loaded with ETG_SSSP_DELTA_AUTO. */
etg_status etg_step_begin(etg_graph *g, int alg, uint32_t source, uint32_t *d_label,
                          uint32_t *n_active);
etg_status etg_step_expand(etg_graph *g);
etg_status etg_step_scan(etg_graph *g, uint32_t *n_active);
etg_status etg_step_end(etg_graph *g, etg_stats *st_or_null);
etg_status etg_bitmap_layout(etg_graph *g, size_t *offset_bytes, uint32_t *nwords);

/* The SSSP wave width Delta the handle uses (etg_options.sssp_delta; auto is
 * resolved here if no SSSP ran yet -- collective on a communicator handle). */
etg_status etg_sssp_delta(etg_graph *g, uint32_t *delta);

/* Tracing (step-wise runs): the device counters as of the last etg_step_* call
 * that synchronised (begin/scan/end): out[0] depth, [1] compacted active-set
 * size |F| (Proc. 1 actSet, L207), [2] shadow vertices of F (Def. 3),
 * [3] cumulative edges expanded, [4] cumulative activations, [5] iterations.
 * `out` is host memory of 6 entries.  ETG_EINVAL on NULL arguments. */
etg_status etg_debug_counters(etg_graph *g, uint64_t *out);

/* Release a handle (does not free the borrowed device memory). */
void etg_free(etg_graph *g);

/* End-to-end entry on HOST buffers (the paper's "total time", L247: transfer +
 * execution).  alg: 0 = BFS, 1 = SSSP, 2 = CC, 3 = SSWP.  Copies the CSR
 * host->device into d_scratch (caller-owned device memory of at least
 * etg_host_scratch_bytes), runs the traversal and copies the n labels back into
 * h_labels.  Host buffers should be pinned for full PCIe bandwidth.  The
 * internal handle over d_scratch is kept per calling thread (up to 4) and
 * reused by a later call with the same n, m, weights, scratch, stream and
 * options (its device state is re-zeroed; nothing is read from the previous
 * call), so only the first call pays the host-side setup.  Not re-entrant
 * across threads sharing one scratch buffer. */
size_t etg_host_scratch_bytes(uint64_t n, uint64_t m, int has_weights, const etg_options *opt);
/* Several traversals of ONE host graph (Proc. 1 per query; the paper times
 * each with its own transfer, L247 -- here the CSR crosses the host link once
 * for all of them): algs[q] / sources[q] for q < n_queries (sources ignored
 * for CC), h_labels receives n_queries x n labels (query q at h_labels + q*n),
 * st_or_null n_queries entries.  The weights are copied on an internal copy
 * stream while the queries that need none run; each query's labels are
 * copied back while the next one runs.  Same scratch, caching and error
 * rules as etg_run_host (ETG_ENOWEIGHTS if a query needs weights and h_w is
 * NULL). */
etg_status etg_run_host_batch(uint64_t n, uint64_t m, const void *h_row_offsets, const uint32_t *h_col_idx,
                              const uint32_t *h_weights, uint32_t n_queries, const int *algs,
                              const uint32_t *sources, uint32_t *h_labels, void *d_scratch,
                              size_t scratch_bytes, void *stream, const etg_options *opt,
                              etg_stats *st_or_null);
etg_status etg_run_host(int alg, uint64_t n, uint64_t m, const void *h_row_offsets,
                        const uint32_t *h_col_idx, const uint32_t *h_weights,
                        uint32_t source, uint32_t *h_labels, void *d_scratch,
                        size_t scratch_bytes, void *stream, const etg_options *opt,
                        etg_stats *st_or_null);

/* ---- Communicator (one process -- or thread -- per partition on
 * ONE node).  Rank 0 calls etg_comm_unique_id and hands the 128 bytes to the
 * other ranks by any means (the binding uses torch.distributed); every rank
 * then calls etg_comm_init with its rank, the world size (1..8) and the CUDA
 * device it drives (-1: the calling thread's current device).  The
 * communicator is the control plane only -- a POSIX shared-memory segment
 * with one slot per rank (workspace IPC handles, owned ranges, termination
 * counts) and a host barrier; the data plane is the library's kernels.
 * etg_comm_init blocks until all `world` ranks have joined.  Errors:
 * ETG_EINVAL (rank >= world, world outside 1..8, not a unique id, rank
 * taken twice), ETG_ENCCL (shared memory unavailable, timeout, a peer died).
 * etg_comm_barrier: a host barrier over the ranks (plumbing and tests).
 * etg_comm_free after every handle loaded with it has been freed. */
etg_status etg_comm_unique_id(uint8_t *id /* 128 bytes */);
etg_status etg_comm_init(etg_comm **out, int rank, int world, const uint8_t *id, int device);
etg_status etg_comm_barrier(const etg_comm *comm);
void etg_comm_free(etg_comm *comm);

const char *etg_status_str(etg_status s);
const char *etg_last_error(void);
/* Number of CUDA kernels this library launched since load (for bench claims). */
uint64_t etg_kernel_launches(void);

#ifdef __cplusplus
}
#endif
#endif /* ETG_H */
