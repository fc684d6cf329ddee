/*
 * oracle.c -- plain, slow, obviously-correct CPU oracle for the EtaGraph hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing in the product path (the CUDA library under
 * paper_conf_ipps_wangzlg19_b200/) may include, link or call this file.  Only
 * tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs use it.  It shares no code, header, table or helper with the CUDA path.
 *
 * Citations are to /root/reference/PAPER.md ("L<n>" = line n) of
 * Wang, Zhang, Li, Guo, "Excavating the Potential of GPU for Accelerating Graph
 * Traversal" (IPDPS 2019), and to the readings recorded in DESIGN.md ("R-n").
 *
 * What the method computes (L62, Sec. II-C "Notion of Graph Traversal"):
 *   "Graph traversal is to calculate labels of all nodes reachable from a given
 *    root node."  Proc. 1 (L207): Data = CSR graph, Result = vertex labels.
 * EtaGraph reaches, by Theorems 1-2 (L119-127, Sec. III-B), exactly the labels of
 * the plain definitions below, so each oracle is that definition written out as
 * the textbook algorithm (FIFO BFS, binary-heap Dijkstra, union-find), not the
 * paper's GPU procedure.
 *
 * Conventions (readings R-9, R-21): labels are uint32; INF = 0xFFFFFFFF
 * marks "unreached"; SSSP distances saturate at CAP = 0xFFFFFFFE.
 * CSR: row offsets off[n+1] (uint64 here, for generality), column ids col[m]
 * (uint32), weights w[m] (uint32), structure of arrays (L55, Sec. II-B).
 *
 * Every function returns 0 on success and a negative value on bad input.
 *
 * Parity status: every function here is pinned by tests/test_oracle_*.py against
 * closed forms, brute force, scipy/networkx and certificates.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORC_INF 0xFFFFFFFFu
#define ORC_CAP 0xFFFFFFFEu

/* ------------------------------------------------------------------------- */
/* O-BFS.  L62 (Sec. II-C), L66 (Def. 1), Proc. 1 L207 ("label[v'] > label[v]+1"). */
/* depth[s] = 0; depth[v] = fewest edges on a directed s->v path; INF if none.  */
/* Textbook FIFO-queue breadth-first search over the CSR out-edges: a vertex's  */
/* depth is set when it is first discovered, which is its hop distance.         */
/* ------------------------------------------------------------------------- */
int oracle_bfs(uint64_t n, const uint64_t *off, const uint32_t *col,
               uint32_t source, uint32_t *depth)
{
    if (source >= n) return -1;
    uint32_t *queue = (uint32_t *)malloc((n ? n : 1) * sizeof(uint32_t));
    if (!queue) return -2;
    for (uint64_t v = 0; v < n; ++v) depth[v] = ORC_INF;
    uint64_t head = 0, tail = 0;
    depth[source] = 0;
    queue[tail++] = source;
    while (head < tail) {
        uint32_t v = queue[head++];
        for (uint64_t e = off[v]; e < off[v + 1]; ++e) {
            uint32_t u = col[e];
            if (depth[u] == ORC_INF) {
                depth[u] = depth[v] + 1;
                queue[tail++] = u;
            }
        }
    }
    free(queue);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* O-SSSP.  L62 (SSSP named as a traversal problem), L66/L78 (re-activation     */
/* when edges are not uniformly weighted).  dist[s] = 0; dist[v] = min over     */
/* s->v paths of the weight sum, saturated at CAP (reading R-9); INF if no path.*/
/* Textbook Dijkstra with a binary min-heap and lazy deletion.  Weights are     */
/* unsigned, hence non-negative, so Dijkstra is exact.                          */
/* ------------------------------------------------------------------------- */
typedef struct { uint32_t d; uint32_t v; } heap_item;

static void heap_push(heap_item *h, uint64_t *sz, heap_item x)
{
    uint64_t i = (*sz)++;
    h[i] = x;
    while (i > 0) {
        uint64_t p = (i - 1) / 2;
        if (h[p].d <= h[i].d) break;
        heap_item t = h[p]; h[p] = h[i]; h[i] = t;
        i = p;
    }
}

static heap_item heap_pop(heap_item *h, uint64_t *sz)
{
    heap_item top = h[0];
    h[0] = h[--(*sz)];
    uint64_t i = 0;
    for (;;) {
        uint64_t l = 2 * i + 1, r = l + 1, s = i;
        if (l < *sz && h[l].d < h[s].d) s = l;
        if (r < *sz && h[r].d < h[s].d) s = r;
        if (s == i) break;
        heap_item t = h[s]; h[s] = h[i]; h[i] = t;
        i = s;
    }
    return top;
}

int oracle_sssp(uint64_t n, const uint64_t *off, const uint32_t *col,
                const uint32_t *w, uint32_t source, uint32_t *dist)
{
    if (source >= n) return -1;
    uint64_t m = off[n];
    /* lazy deletion: at most one push per successful relaxation, <= m + 1 */
    heap_item *heap = (heap_item *)malloc((m + 1) * sizeof(heap_item));
    if (!heap) return -2;
    uint64_t sz = 0;
    for (uint64_t v = 0; v < n; ++v) dist[v] = ORC_INF;
    dist[source] = 0;
    heap_item s0 = {0u, source};
    heap_push(heap, &sz, s0);
    while (sz > 0) {
        heap_item it = heap_pop(heap, &sz);
        if (it.d != dist[it.v]) continue;           /* stale entry */
        for (uint64_t e = off[it.v]; e < off[it.v + 1]; ++e) {
            uint32_t u = col[e];
            uint64_t nd = (uint64_t)it.d + (uint64_t)w[e];
            if (nd > ORC_CAP) nd = ORC_CAP;          /* saturating add, R-9 */
            if (nd < dist[u]) {
                dist[u] = (uint32_t)nd;
                heap_item x = {(uint32_t)nd, u};
                heap_push(heap, &sz, x);
            }
        }
    }
    free(heap);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* O-CC.  Not in the paper (BASELINE.json north_star adds it; reading R-12).    */
/* label[v] = min{ u : u and v are weakly connected } -- edge direction ignored.*/
/* Textbook union-find (path halving, union by size) over every CSR edge, then  */
/* one ascending pass that names each set by its smallest member.              */
/* ------------------------------------------------------------------------- */
static uint32_t uf_find(uint32_t *parent, uint32_t x)
{
    while (parent[x] != x) {
        parent[x] = parent[parent[x]];               /* path halving */
        x = parent[x];
    }
    return x;
}

int oracle_cc(uint64_t n, const uint64_t *off, const uint32_t *col, uint32_t *label)
{
    uint32_t *parent = (uint32_t *)malloc((n ? n : 1) * sizeof(uint32_t));
    uint32_t *size = (uint32_t *)malloc((n ? n : 1) * sizeof(uint32_t));
    uint32_t *minid = (uint32_t *)malloc((n ? n : 1) * sizeof(uint32_t));
    if (!parent || !size || !minid) { free(parent); free(size); free(minid); return -2; }
    for (uint64_t v = 0; v < n; ++v) { parent[v] = (uint32_t)v; size[v] = 1; minid[v] = ORC_INF; }
    for (uint64_t v = 0; v < n; ++v) {
        for (uint64_t e = off[v]; e < off[v + 1]; ++e) {
            uint32_t a = uf_find(parent, (uint32_t)v), b = uf_find(parent, col[e]);
            if (a == b) continue;
            if (size[a] < size[b]) { uint32_t t = a; a = b; b = t; }
            parent[b] = a;
            size[a] += size[b];
        }
    }
    for (uint64_t v = 0; v < n; ++v) {           /* ascending: first member seen is the min */
        uint32_t r = uf_find(parent, (uint32_t)v);
        if (minid[r] == ORC_INF) minid[r] = (uint32_t)v;
        label[v] = minid[r];
    }
    free(parent); free(size); free(minid);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* O-UDC: the Unified Degree Cut of an active set (test oracle for step A2).    */
/* Def. 3 (L101-107, Sec. III-A): vertex v with edge set E_v maps to shadow     */
/* vertices with the same ID whose edge sets are disjoint, cover E_v, and have  */
/* size <= K.  Sec. IV-A (L136-140) and Fig. 3 (L138-148): each active vertex is*/
/* turned into 3-tuples (ID, Start Index, End Index) appended to the virtual    */
/* active set; a vertex with out-degree 0 produces none; a vertex with degree   */
/* <= K is one shadow.  Slices are cut contiguously from Start Index (reading   */
/* R-2): shadow q of v covers [off[v] + qK, min(off[v] + (q+1)K, off[v+1])).    */
/* Output in active-set order, shadows of one vertex in increasing q.           */
/* Returns the number of shadows written (<= cap), or -1 on bad input, or       */
/* -(needed) - 2 if cap is too small.                                            */
/* ------------------------------------------------------------------------- */
int64_t oracle_udc_slices(uint64_t n, const uint64_t *off,
                          const uint32_t *act, uint64_t n_act, uint64_t K,
                          uint32_t *out_id, uint64_t *out_start, uint64_t *out_end,
                          uint64_t cap)
{
    if (K == 0) return -1;
    uint64_t cnt = 0;
    for (uint64_t j = 0; j < n_act; ++j) {
        uint32_t v = act[j];
        if (v >= n) return -1;
        uint64_t start = off[v];
        while (start < off[v + 1]) {               /* degree 0 -> no shadow */
            uint64_t end = start + K;
            if (end > off[v + 1]) end = off[v + 1];
            if (cnt < cap) { out_id[cnt] = v; out_start[cnt] = start; out_end[cnt] = end; }
            ++cnt;
            start = end;
        }
    }
    if (cnt > cap) return -(int64_t)cnt - 2;
    return (int64_t)cnt;
}

/* ------------------------------------------------------------------------- */
/* O-SSWP (NEXT-1, Sec. II-C; Table III): single-source widest     */
/* path.  width[s] = INF (0xFFFFFFFF); width[v] = max over s->v paths of the    */
/* minimum edge weight on the path; 0 if v is unreachable (reading R-24).       */
/* Textbook max-bottleneck Dijkstra (max-heap on width).                        */
/* ------------------------------------------------------------------------- */
static void maxheap_push(heap_item *h, uint64_t *sz, heap_item x)
{
    uint64_t i = (*sz)++;
    h[i] = x;
    while (i > 0) {
        uint64_t p = (i - 1) / 2;
        if (h[p].d >= h[i].d) break;
        heap_item t = h[p]; h[p] = h[i]; h[i] = t;
        i = p;
    }
}

static heap_item maxheap_pop(heap_item *h, uint64_t *sz)
{
    heap_item top = h[0];
    h[0] = h[--(*sz)];
    uint64_t i = 0;
    for (;;) {
        uint64_t l = 2 * i + 1, r = l + 1, s = i;
        if (l < *sz && h[l].d > h[s].d) s = l;
        if (r < *sz && h[r].d > h[s].d) s = r;
        if (s == i) break;
        heap_item t = h[s]; h[s] = h[i]; h[i] = t;
        i = s;
    }
    return top;
}

int oracle_sswp(uint64_t n, const uint64_t *off, const uint32_t *col,
                const uint32_t *w, uint32_t source, uint32_t *width)
{
    if (source >= n) return -1;
    uint64_t m = off[n];
    heap_item *heap = (heap_item *)malloc((m + 1) * sizeof(heap_item));
    if (!heap) return -2;
    uint64_t sz = 0;
    for (uint64_t v = 0; v < n; ++v) width[v] = 0;
    width[source] = ORC_INF;
    heap_item s0 = {ORC_INF, source};
    maxheap_push(heap, &sz, s0);
    while (sz > 0) {
        heap_item it = maxheap_pop(heap, &sz);
        if (it.d != width[it.v]) continue;          /* stale entry */
        for (uint64_t e = off[it.v]; e < off[it.v + 1]; ++e) {
            uint32_t u = col[e];
            uint32_t nw = it.d < w[e] ? it.d : w[e];
            if (nw > width[u]) {
                width[u] = nw;
                heap_item x = {nw, u};
                maxheap_push(heap, &sz, x);
            }
        }
    }
    free(heap);
    return 0;
}
