/*
 * oracle/oracle.c -- TEST INFRASTRUCTURE, NOT PRODUCT CODE.
 *
 * The plain, slow, obviously-correct CPU oracle for the hot path of
 * Troendle, Ta & Jang, "A Specialized Concurrent Queue for Scheduling
 * Irregular Workloads on GPUs", ICPP 2019 (/root/reference/PAPER.md, cited
 * P:<line>).  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no
 * code, header, table or constant with the CUDA path (include/, the package
 * csrc/), and it never includes or links them.
 *
 * Contents
 *   1. oracle_bfs_levels        classic sequential top-down BFS (§5.1,
 *                               "classic top-down BFS [4, 15]" = Cormen /
 *                               Sedgewick): FIFO array queue over the CSR.
 *   2. oracle_min_id_parents    parent[v] = the smallest-id neighbour u with
 *                               level[u] = level[v]-1 (SURVEY §8(c)(i) and
 *                               DESIGN.md reading R5: the paper outputs only
 *                               Costs[]; a unique parent needs a rule).
 *   3. oracle_traversed_edges   TEPS edge count (reading R16).
 *   4. oracle_validate_tree     Graph500-style BFS-tree validation (the
 *                               north star's "parent tree that validates
 *                               Graph500-style").
 *   5. oq_*                     the sequential ticket model of the queue
 *                               (§4, §4.1, Listings 1-3
 *                               P:177-273, queue-full P:71 fn2 / P:281 §4.4).
 *
 * Pins (tests/test_oracle_*.py): Floyd-Warshall brute force, exhaustive
 * 5-vertex graphs, closed forms (path, star, complete, grid r+c, 4-ary heap
 * tree), scipy.sparse.csgraph cross-check, the paper's worked dequeue
 * example (tests/golden/p167_dequeue_example.json), and mutation
 * tests of the validator.  No function here is "parity unpinned".
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>

/* ------------------------------------------------------------------ */
/* 1. Sequential BFS levels: level[v] = hop distance from root, */
/*    -1 if unreachable.  Returns the number of reached vertices, or -1 */
/*    on bad arguments.                                                 */
/* ------------------------------------------------------------------ */
int64_t oracle_bfs_levels(int64_t n, const int64_t *row_ptr, const int32_t *col,
                          int32_t root, int32_t *level)
{
    if (n <= 0 || root < 0 || root >= n) return -1;
    int32_t *fifo = (int32_t *)malloc((size_t)n * sizeof(int32_t));
    if (!fifo) return -1;
    for (int64_t v = 0; v < n; ++v) level[v] = -1;
    int64_t head = 0, tail = 0;
    level[root] = 0;
    fifo[tail++] = root;
    while (head < tail) {
        int32_t v = fifo[head++];
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
            int32_t u = col[e];
            if (level[u] < 0) {
                level[u] = level[v] + 1;
                fifo[tail++] = u;
            }
        }
    }
    free(fifo);
    return tail;
}

/* ------------------------------------------------------------------ */
/* 2. Min-id parent rule, a separate pass over each reached row so the  */
/*    result follows the definition, not the queue order.              */
/* ------------------------------------------------------------------ */
int oracle_min_id_parents(int64_t n, const int64_t *row_ptr, const int32_t *col,
                          const int32_t *level, int32_t root, int32_t *parent)
{
    if (n <= 0 || root < 0 || root >= n) return -1;
    for (int64_t v = 0; v < n; ++v) {
        parent[v] = -1;
        if (level[v] < 0) continue;
        if (v == root) { parent[v] = root; continue; }
        int32_t best = -1;
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
            int32_t u = col[e];
            if (level[u] == level[v] - 1 && (best < 0 || u < best)) best = u;
        }
        parent[v] = best;
    }
    return 0;
}

/* Convenience: levels + min-id parents, wall time of the BFS proper (the */
/* level pass; CSR preloaded) returned in *seconds_levels, total in      */
/* *seconds_total.                                                        */
int64_t oracle_bfs(int64_t n, const int64_t *row_ptr, const int32_t *col, int32_t root,
                   int32_t *level, int32_t *parent, double *seconds_levels,
                   double *seconds_total)
{
    struct timespec t0, t1, t2;
    clock_gettime(CLOCK_MONOTONIC, &t0);
    int64_t reached = oracle_bfs_levels(n, row_ptr, col, root, level);
    clock_gettime(CLOCK_MONOTONIC, &t1);
    if (reached >= 0 && parent)
        if (oracle_min_id_parents(n, row_ptr, col, level, root, parent) != 0) reached = -1;
    clock_gettime(CLOCK_MONOTONIC, &t2);
    if (seconds_levels)
        *seconds_levels = (t1.tv_sec - t0.tv_sec) + 1e-9 * (t1.tv_nsec - t0.tv_nsec);
    if (seconds_total)
        *seconds_total = (t2.tv_sec - t0.tv_sec) + 1e-9 * (t2.tv_nsec - t0.tv_nsec);
    return reached;
}

/* ------------------------------------------------------------------ */
/* 3. Traversed edges: undirected, deduplicated, loop-free edges with a */
/*    reached endpoint = (sum of degrees of reached vertices) / 2 on a  */
/*    symmetric CSR (reading R16).                            */
/* ------------------------------------------------------------------ */
int64_t oracle_traversed_edges(int64_t n, const int64_t *row_ptr, const int32_t *level)
{
    int64_t s = 0;
    for (int64_t v = 0; v < n; ++v)
        if (level[v] >= 0) s += row_ptr[v + 1] - row_ptr[v];
    return s / 2;
}

/* ------------------------------------------------------------------ */
/* 4. Graph500-style validation of (level, parent).  Returns 0 if valid, */
/*    else the number of the first failed rule:                          */
/*      1 root: parent[root] != root or level[root] != 0                 */
/*      2 reached-ness: level[v] >= 0 iff parent[v] >= 0; ids in range;  */
/*        level 0 only at the root                                        */
/*      3 tree edge (parent[v], v) is not a graph edge                    */
/*      4 level[v] != level[parent[v]] + 1                                */
/*      5 a graph edge joins a reached and an unreached vertex, or spans  */
/*        more than one level                                            */
/*    Rule 4 makes every parent chain strictly decrease in level down to  */
/*    the unique level-0 vertex (the root), so the tree has no cycles and */
/*    spans exactly the reached set; rule 5 makes the reached set the     */
/*    root's connected component and levels shortest-path consistent.     */
/* ------------------------------------------------------------------ */
static int row_has(const int64_t *row_ptr, const int32_t *col, int32_t v, int32_t u)
{
    int64_t lo = row_ptr[v], hi = row_ptr[v + 1];
    for (int64_t e = lo; e < hi; ++e)   /* linear: obviously correct, rows are short */
        if (col[e] == u) return 1;
    return 0;
}

int oracle_validate_tree(int64_t n, const int64_t *row_ptr, const int32_t *col, int32_t root,
                         const int32_t *level, const int32_t *parent, int64_t *bad_vertex)
{
    if (bad_vertex) *bad_vertex = -1;
    if (root < 0 || root >= n) return 1;
    if (parent[root] != root || level[root] != 0) { if (bad_vertex) *bad_vertex = root; return 1; }
    for (int64_t v = 0; v < n; ++v) {
        int reached_l = level[v] >= 0, reached_p = parent[v] >= 0;
        if (reached_l != reached_p || parent[v] >= n || level[v] < -1 ||
            (level[v] == 0 && v != root)) {
            if (bad_vertex) *bad_vertex = v;
            return 2;
        }
    }
    for (int64_t v = 0; v < n; ++v) {
        if (level[v] < 0 || v == root) continue;
        int32_t p = parent[v];
        if (!row_has(row_ptr, col, (int32_t)v, p)) { if (bad_vertex) *bad_vertex = v; return 3; }
        if (level[v] != level[p] + 1) { if (bad_vertex) *bad_vertex = v; return 4; }
    }
    for (int64_t v = 0; v < n; ++v) {
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
            int32_t u = col[e];
            int rv = level[v] >= 0, ru = level[u] >= 0;
            if (rv != ru) { if (bad_vertex) *bad_vertex = v; return 5; }
            if (rv) {
                int32_t d = level[v] - level[u];
                if (d > 1 || d < -1) { if (bad_vertex) *bad_vertex = v; return 5; }
            }
        }
    }
    return 0;
}

/* ------------------------------------------------------------------ */
/* 4b. Single-source shortest paths (NEXT row 4: the queue reused as a */
/*     generic scheduler, "it can be used for other purposes with */
/*     little change").  Textbook Dijkstra with a binary heap (Cormen   */
/*     et al., the paper's ref. [4], ch. 24) over positive integer      */
/*     weights w[e] >= 1 of each CSR entry; dist[v] = 0xFFFFFFFF if     */
/*     unreachable; paths must sum below 2^32 - 1.  parent[v] = the     */
/*     smallest-id u with dist[u] + w(u->v) == dist[v], parent[src] =   */
/*     src, -1 unreached (the same tie rule as the BFS min-id parent).  */
/* ------------------------------------------------------------------ */
typedef struct { uint64_t key; int32_t v; } oheap_item;

static void oheap_push(oheap_item *h, int64_t *n, uint64_t key, int32_t v)
{
    int64_t i = (*n)++;
    h[i].key = key;
    h[i].v = v;
    while (i > 0) {
        int64_t p = (i - 1) / 2;
        if (h[p].key <= h[i].key) break;
        oheap_item t = h[p]; h[p] = h[i]; h[i] = t;
        i = p;
    }
}

static oheap_item oheap_pop(oheap_item *h, int64_t *n)
{
    oheap_item top = h[0];
    h[0] = h[--(*n)];
    int64_t i = 0;
    for (;;) {
        int64_t l = 2 * i + 1, r = l + 1, m = i;
        if (l < *n && h[l].key < h[m].key) m = l;
        if (r < *n && h[r].key < h[m].key) m = r;
        if (m == i) break;
        oheap_item t = h[m]; h[m] = h[i]; h[i] = t;
        i = m;
    }
    return top;
}

int64_t oracle_sssp(int64_t n, const int64_t *row_ptr, const int32_t *col, const int32_t *w,
                    int32_t src, uint32_t *dist, int32_t *parent)
{
    if (n <= 0 || src < 0 || src >= n) return -1;
    const int64_t nnz = row_ptr[n];
    oheap_item *heap = (oheap_item *)malloc((size_t)(nnz + 1) * sizeof(oheap_item));
    uint8_t *settled = (uint8_t *)calloc((size_t)n, 1);
    if (!heap || !settled) { free(heap); free(settled); return -1; }
    for (int64_t v = 0; v < n; ++v) dist[v] = 0xFFFFFFFFu;
    int64_t hn = 0, reached = 0;
    dist[src] = 0;
    oheap_push(heap, &hn, 0, src);
    while (hn > 0) {
        oheap_item it = oheap_pop(heap, &hn);
        int32_t v = it.v;
        if (settled[v]) continue;
        settled[v] = 1;
        ++reached;
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
            int32_t u = col[e];
            uint64_t nd = (uint64_t)dist[v] + (uint64_t)(uint32_t)w[e];
            if (nd < 0xFFFFFFFFull && nd < dist[u]) {
                dist[u] = (uint32_t)nd;
                oheap_push(heap, &hn, nd, u);
            }
        }
    }
    free(heap);
    free(settled);
    if (parent) {
        for (int64_t v = 0; v < n; ++v) parent[v] = -1;
        parent[src] = src;
        /* min-id predecessor: scan every edge u->v once */
        for (int64_t u = 0; u < n; ++u) {
            if (dist[u] == 0xFFFFFFFFu) continue;
            for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
                int32_t v = col[e];
                if (v == src) continue;
                if ((uint64_t)dist[u] + (uint32_t)w[e] == dist[v] &&
                    (parent[v] < 0 || u < parent[v]))
                    parent[v] = (int32_t)u;
            }
        }
    }
    return reached;
}

/* ------------------------------------------------------------------ */
/* 5. Sequential ticket model of the RF/AN queue.   */
/*                                                                     */
/* State: Front, Rear, capacity C (bounded array) */
/* and, per ticket t, the item stored there and whether it was taken.   */
/* A dequeue "returns the slot index where the task tokens will be ...  */
/* dequeued": dequeue_n(k) hands out tickets Front..Front+k-1   */
/* (P:169-171).  take(t) returns the item once it has arrived, else the */
/* data-not-arrived sentinel (Listing 2).  enqueue_n      */
/* reserves Rear..Rear+n-1 and writes each item; the write to   */
/* ticket t finds its slot (t mod C) still holding the entry of ticket  */
/* t-C when t >= C and t-C has not been taken -> queue-full abort, no   */
/* retry (Listing 3 line 25, P:71 fn2).                    */
/* ------------------------------------------------------------------ */
typedef struct {
    uint64_t cap;         /* C */
    uint64_t max_tickets; /* size of the per-ticket arrays */
    uint64_t front, rear;
    uint64_t n_taken;
    uint32_t *item;       /* item[t] */
    uint8_t *state;       /* 0 = not written, 1 = written (arrived), 2 = taken */
    int aborted;
} oq_model;

#define OQ_DNA 0xFFFFFFFFFFFFFFFFull /* take(): data not arrived */

oq_model *oq_create(uint64_t cap, uint64_t max_tickets)
{
    if (cap == 0 || max_tickets == 0) return NULL;
    oq_model *q = (oq_model *)calloc(1, sizeof(oq_model));
    if (!q) return NULL;
    q->cap = cap;
    q->max_tickets = max_tickets;
    q->item = (uint32_t *)calloc(max_tickets, sizeof(uint32_t));
    q->state = (uint8_t *)calloc(max_tickets, 1);
    if (!q->item || !q->state) { free(q->item); free(q->state); free(q); return NULL; }
    return q;
}

void oq_destroy(oq_model *q)
{
    if (!q) return;
    free(q->item);
    free(q->state);
    free(q);
}

/* Start counters at a given ticket (e.g. the paper's example, Front = 2). */
/* Tickets below `t0` are treated as already enqueued and taken.           */
int oq_start_at(oq_model *q, uint64_t t0)
{
    if (t0 > q->max_tickets) return -1;
    for (uint64_t t = 0; t < t0; ++t) q->state[t] = 2;
    q->front = q->rear = t0;
    q->n_taken = t0;
    return 0;
}

uint64_t oq_front(const oq_model *q) { return q->front; }
uint64_t oq_rear(const oq_model *q) { return q->rear; }
int oq_aborted(const oq_model *q) { return q->aborted; }

/* Listing 1: one reservation of k slots; returns the base ticket. */
uint64_t oq_dequeue_n(oq_model *q, uint64_t k)
{
    uint64_t base = q->front;
    q->front += k;
    return base;
}

/* Listing 3: reserve n tickets at Rear, then write items in ticket order. */
/* Returns the base ticket, or OQ_DNA if the model ran out of ticket space,  */
/* and sets aborted (returning the base) on queue-full.                     */
uint64_t oq_enqueue_n(oq_model *q, const uint32_t *items, uint64_t n)
{
    uint64_t base = q->rear;
    if (base + n > q->max_tickets) return OQ_DNA;
    q->rear += n;
    for (uint64_t i = 0; i < n; ++i) {
        uint64_t t = base + i;
        if (t >= q->cap && q->state[t - q->cap] != 2) { q->aborted = 1; return base; }
        q->item[t] = items[i];
        q->state[t] = 1;
    }
    return base;
}

/* Listing 2: non-atomic arrival check of one ticket.  Returns the item, or */
/* OQ_DNA when no data has arrived for that ticket yet.                     */
uint64_t oq_take(oq_model *q, uint64_t t)
{
    if (t >= q->max_tickets || t >= q->rear || q->state[t] != 1) return OQ_DNA;
    q->state[t] = 2;
    q->n_taken++;
    return q->item[t];
}

/* Replay: enqueue-all then dequeue-all of n items through a queue of      */
/* capacity C in batches of b (the sequential analogue of one bench warp); */
/* returns elapsed seconds, writes (count, sum, xor) of splitmix64(item)   */
/* over dequeued items.  Used as the queue-bench CPU baseline.             */
static uint64_t mix64(uint64_t x)
{
    x ^= x >> 30; x *= 0xBF58476D1CE4E5B9ull;
    x ^= x >> 27; x *= 0x94D049BB133111EBull;
    x ^= x >> 31;
    return x;
}

double oq_replay(uint64_t cap, const uint32_t *items, uint64_t n, uint64_t b,
                 uint64_t out_fp[3])
{
    struct timespec t0, t1;
    oq_model *q = oq_create(cap, n);
    if (!q || b == 0) { oq_destroy(q); return -1.0; }
    uint64_t cnt = 0, sum = 0, x = 0;
    clock_gettime(CLOCK_MONOTONIC, &t0);
    for (uint64_t i = 0; i < n; i += b) {
        uint64_t k = (n - i < b) ? n - i : b;
        oq_enqueue_n(q, items + i, k);
        if (q->aborted) break;
        uint64_t base = oq_dequeue_n(q, k);
        for (uint64_t j = 0; j < k; ++j) {
            uint64_t it = oq_take(q, base + j);
            if (it == OQ_DNA) continue;
            uint64_t f = mix64(it);
            cnt++; sum += f; x ^= f;
        }
    }
    clock_gettime(CLOCK_MONOTONIC, &t1);
    int ab = q->aborted;
    oq_destroy(q);
    out_fp[0] = cnt; out_fp[1] = sum; out_fp[2] = x;
    if (ab) return -2.0;
    return (t1.tv_sec - t0.tv_sec) + 1e-9 * (t1.tv_nsec - t0.tv_nsec);
}
