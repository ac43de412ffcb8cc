/*
 * oracle.c — CPU ORACLE for exact kNN. TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference leg may load this library. It shares no code, header, table or
 * helper with the CUDA path (paper_conf_icpp_namkn16_b200/csrc); neither side
 * includes or links the other.
 *
 * What it computes: PSB is an EXACT kNN method
 * ("there exist many application domains that cannot accept approximate nearest
 * neighbors", §I; "ours is a tree traversal algorithm for exact
 * kNN queries", L1129-1130 §VI). So the oracle is the plain definition:
 *
 *   dist(q,p) = s_d,  s_0 = +0.0f,  s_{j+1} = fl(s_j + fl(fl(p_j - q_j) * fl(p_j - q_j)))
 *
 * in IEEE binary32, round-to-nearest-even, no FMA contraction (compiled with
 * -ffp-contract=off -fno-fast-math), dimensions in order 0..d-1; the result is
 * the k smallest (dist, id) pairs in lexicographic order, ascending, padded
 * with (+inf, -1) when k > n.
 *
 * Two independent routes to that result:
 *   oracle_knn_bruteforce — all n distances, keep the k best (dist, id);
 *   oracle_knn_bnb        — the textbook recursive branch-and-bound kNN of
 *                           Roussopoulos et al. [17] (§III,
 *                           ref [17] L1198-1199) over the oracle's OWN tree: a
 *                           top-down binary median-split box tree (oracle_tree_build),
 *                           deliberately unlike the GPU's bottom-up packed F-ary
 *                           R-tree.
 * Pins: tests/test_oracle_pins.py (hand-worked cases, lattice closed forms,
 * FMA-sensitive case, exact-integer distances, 1-D two-pointer, brute == B&B).
 */
#include <float.h>
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#if defined(FLT_EVAL_METHOD) && FLT_EVAL_METHOD != 0
#error "oracle requires FLT_EVAL_METHOD == 0 (binary32 evaluated in binary32)"
#endif

/* ---- distance and box bounds ---------------- */

/* Squared Euclidean distance, fixed dimension order, each op rounded once. */
float oracle_dist(const float *q, const float *p, int d)
{
    float s = 0.0f;
    for (int j = 0; j < d; ++j) {
        float t = p[j] - q[j];
        float t2 = t * t;
        s = s + t2;
    }
    return s;
}

/* MINDIST(q, box) (Roussopoulos [17] Def. of MINDIST, §III,
 * for an MBR): per dimension the gap to the nearer face, 0 inside. */
float oracle_mindist(const float *q, const float *lo, const float *hi, int d)
{
    float s = 0.0f;
    for (int j = 0; j < d; ++j) {
        float t = 0.0f;
        if (q[j] < lo[j]) t = lo[j] - q[j];
        else if (q[j] > hi[j]) t = q[j] - hi[j];
        float t2 = t * t;
        s = s + t2;
    }
    return s;
}

/* MAXDIST(q, box): distance to the farthest corner (§III
 * "getMaxDistance"; SURVEY.md §8(c) reading 2). */
float oracle_maxdist(const float *q, const float *lo, const float *hi, int d)
{
    float s = 0.0f;
    for (int j = 0; j < d; ++j) {
        float a = fabsf(q[j] - lo[j]);
        float b = fabsf(q[j] - hi[j]);
        float t = a > b ? a : b;
        float t2 = t * t;
        s = s + t2;
    }
    return s;
}

/* ---- (dist, id) order and the bounded "best k" list ------------------------- */

/* lexicographic (dist, id); ids compared as signed ints, all real ids >= 0 */
static int pair_less(float da, int32_t ia, float db, int32_t ib)
{
    return da < db || (da == db && ia < ib);
}

/* best[0..cnt) ascending; offer one pair, keep at most k. */
static void best_offer(float *bd, int32_t *bi, int *cnt, int k, float d, int32_t id)
{
    int c = *cnt;
    if (c == k && !pair_less(d, id, bd[k - 1], bi[k - 1])) return;
    int pos = c == k ? k - 1 : c;              /* slot freed for the new pair */
    while (pos > 0 && pair_less(d, id, bd[pos - 1], bi[pos - 1])) {
        bd[pos] = bd[pos - 1];
        bi[pos] = bi[pos - 1];
        --pos;
    }
    bd[pos] = d;
    bi[pos] = id;
    if (c < k) *cnt = c + 1;
}

static void best_emit(const float *bd, const int32_t *bi, int cnt, int k,
                      int32_t *out_ids, float *out_dists)
{
    for (int r = 0; r < k; ++r) {
        out_ids[r] = r < cnt ? bi[r] : -1;
        out_dists[r] = r < cnt ? bd[r] : INFINITY;
    }
}

static void set_threads(int threads)
{
#ifdef _OPENMP
    if (threads > 0) omp_set_num_threads(threads);
#else
    (void)threads;
#endif
}

int oracle_max_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* ---- brute force ------------------------------------------------------------ */

int oracle_knn_bruteforce(const float *pts, int64_t n, int d, const float *qs, int64_t nq,
                          int k, int32_t *out_ids, float *out_dists, int threads)
{
    if (n < 0 || nq < 0 || d < 1 || k < 1) return -1;
    set_threads(threads);
    int bad = 0;
#pragma omp parallel
    {
        float *bd = (float *)malloc(sizeof(float) * (size_t)k);
        int32_t *bi = (int32_t *)malloc(sizeof(int32_t) * (size_t)k);
        if (!bd || !bi) {
#pragma omp atomic write
            bad = 1;
        } else {
#pragma omp for schedule(dynamic, 1)
            for (int64_t i = 0; i < nq; ++i) {
                const float *q = qs + i * d;
                int cnt = 0;
                for (int64_t p = 0; p < n; ++p)
                    best_offer(bd, bi, &cnt, k, oracle_dist(q, pts + p * d, d), (int32_t)p);
                best_emit(bd, bi, cnt, k, out_ids + i * k, out_dists + i * k);
            }
        }
        free(bd);
        free(bi);
    }
    return bad ? -2 : 0;
}

/* ---- the oracle's own tree: top-down binary median split --------------------- */

typedef struct {
    int64_t a, b;         /* point range [a, b) of perm                 */
    int64_t left, right;  /* child node indices, -1 for a leaf          */
} onode;

typedef struct {
    const float *pts;     /* caller's points (not copied: caller keeps them alive) */
    int64_t n;
    int d;
    int leaf_size;
    int32_t *perm;        /* point ids in tree order                    */
    onode *nodes;
    float *lo, *hi;       /* node boxes, [node][d]                      */
    int64_t nnodes, cap;
} otree;

static int coord_less(const otree *t, int dim, int32_t a, int32_t b)
{
    float ca = t->pts[(int64_t)a * t->d + dim], cb = t->pts[(int64_t)b * t->d + dim];
    return ca < cb || (ca == cb && a < b);
}

/* Quickselect: after it, perm[m] is the element of rank m-a within [a,b) under
 * (coord, id), everything left of m is <=, everything right is >=. */
static void select_kth(otree *t, int dim, int64_t a, int64_t b, int64_t m)
{
    int32_t *v = t->perm;
    while (b - a > 1) {
        int32_t pivot = v[a + (b - a) / 2];
        int64_t i = a, j = b - 1;
        while (i <= j) {
            while (coord_less(t, dim, v[i], pivot)) ++i;
            while (coord_less(t, dim, pivot, v[j])) --j;
            if (i <= j) {
                int32_t s = v[i]; v[i] = v[j]; v[j] = s;
                ++i; --j;
            }
        }
        if (m <= j) b = j + 1;
        else if (m >= i) a = i;
        else return;
    }
}

static int64_t tree_new_node(otree *t, int64_t a, int64_t b)
{
    if (t->nnodes == t->cap) {
        int64_t cap = t->cap ? 2 * t->cap : 1024;
        onode *nn = (onode *)realloc(t->nodes, sizeof(onode) * (size_t)cap);
        float *nl = (float *)realloc(t->lo, sizeof(float) * (size_t)(cap * t->d));
        float *nh = (float *)realloc(t->hi, sizeof(float) * (size_t)(cap * t->d));
        if (nn) t->nodes = nn;
        if (nl) t->lo = nl;
        if (nh) t->hi = nh;
        if (!nn || !nl || !nh) return -1;
        t->cap = cap;
    }
    int64_t id = t->nnodes++;
    t->nodes[id].a = a;
    t->nodes[id].b = b;
    t->nodes[id].left = t->nodes[id].right = -1;
    float *lo = t->lo + id * t->d, *hi = t->hi + id * t->d;
    for (int j = 0; j < t->d; ++j) { lo[j] = INFINITY; hi[j] = -INFINITY; }
    for (int64_t i = a; i < b; ++i) {
        const float *p = t->pts + (int64_t)t->perm[i] * t->d;
        for (int j = 0; j < t->d; ++j) {
            if (p[j] < lo[j]) lo[j] = p[j];
            if (p[j] > hi[j]) hi[j] = p[j];
        }
    }
    return id;
}

/* Split [a,b) at the median of the widest dimension (ties -> lowest dim). */
static int tree_split(otree *t, int64_t node)
{
    int64_t a = t->nodes[node].a, b = t->nodes[node].b;
    if (b - a <= t->leaf_size) return 0;
    const float *lo = t->lo + node * t->d, *hi = t->hi + node * t->d;
    int dim = 0;
    float best = -1.0f;
    for (int j = 0; j < t->d; ++j) {
        float ext = hi[j] - lo[j];
        if (ext > best) { best = ext; dim = j; }
    }
    int64_t m = a + (b - a) / 2;
    select_kth(t, dim, a, b, m);
    int64_t l = tree_new_node(t, a, m);
    if (l < 0) return -1;
    int64_t r = tree_new_node(t, m, b);
    if (r < 0) return -1;
    t->nodes[node].left = l;
    t->nodes[node].right = r;
    if (tree_split(t, l) < 0) return -1;
    return tree_split(t, r);
}

void oracle_tree_free(void *h)
{
    otree *t = (otree *)h;
    if (!t) return;
    free(t->perm);
    free(t->nodes);
    free(t->lo);
    free(t->hi);
    free(t);
}

/* Build over pts[n][d]; the caller keeps `pts` alive while the tree is used. */
void *oracle_tree_build(const float *pts, int64_t n, int d, int leaf_size)
{
    if (n < 0 || d < 1 || leaf_size < 1 || n > INT32_MAX) return NULL;
    otree *t = (otree *)calloc(1, sizeof(otree));
    if (!t) return NULL;
    t->pts = pts; t->n = n; t->d = d; t->leaf_size = leaf_size;
    t->perm = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    if (!t->perm) { oracle_tree_free(t); return NULL; }
    for (int64_t i = 0; i < n; ++i) t->perm[i] = (int32_t)i;
    if (tree_new_node(t, 0, n) < 0 || tree_split(t, 0) < 0) { oracle_tree_free(t); return NULL; }
    return t;
}

int64_t oracle_tree_nodes(const void *h) { return h ? ((const otree *)h)->nnodes : -1; }

/* Node box and point range, for the invariant tests. */
int oracle_tree_node(const void *h, int64_t node, float *lo, float *hi, int64_t *a, int64_t *b,
                     int64_t *left, int64_t *right)
{
    const otree *t = (const otree *)h;
    if (!t || node < 0 || node >= t->nnodes) return -1;
    memcpy(lo, t->lo + node * t->d, sizeof(float) * (size_t)t->d);
    memcpy(hi, t->hi + node * t->d, sizeof(float) * (size_t)t->d);
    *a = t->nodes[node].a; *b = t->nodes[node].b;
    *left = t->nodes[node].left; *right = t->nodes[node].right;
    return 0;
}

int oracle_tree_perm(const void *h, int32_t *out)
{
    const otree *t = (const otree *)h;
    if (!t) return -1;
    memcpy(out, t->perm, sizeof(int32_t) * (size_t)t->n);
    return 0;
}

/* ---- recursive branch-and-bound (Roussopoulos [17]) ------------------------ */

typedef struct {
    float *bd;
    int32_t *bi;
    int cnt, k;
} okstate;

/* visit(node): leaf -> offer every point; internal -> active-branch list sorted by
 * (MINDIST, child index), visited in order, stop at the first branch whose
 * MINDIST exceeds the current k-th distance (strict '>' keeps equal-distance
 * subtrees, which may hold smaller ids). k-th distance is +inf until k found. */
static void bnb_visit(const otree *t, int64_t node, const float *q, okstate *s)
{
    const onode *nd = &t->nodes[node];
    if (nd->left < 0) {
        for (int64_t i = nd->a; i < nd->b; ++i) {
            int32_t id = t->perm[i];
            best_offer(s->bd, s->bi, &s->cnt, s->k,
                       oracle_dist(q, t->pts + (int64_t)id * t->d, t->d), id);
        }
        return;
    }
    int64_t ch[2] = {nd->left, nd->right};
    float md[2];
    for (int c = 0; c < 2; ++c)
        md[c] = oracle_mindist(q, t->lo + ch[c] * t->d, t->hi + ch[c] * t->d, t->d);
    int order[2] = {0, 1};
    if (md[1] < md[0]) { order[0] = 1; order[1] = 0; }   /* ties keep child index order */
    for (int r = 0; r < 2; ++r) {
        int c = order[r];
        float kth = s->cnt == s->k ? s->bd[s->k - 1] : INFINITY;
        if (md[c] > kth) break;
        bnb_visit(t, ch[c], q, s);
    }
}

int oracle_knn_bnb(const void *h, const float *qs, int64_t nq, int k,
                   int32_t *out_ids, float *out_dists, int threads)
{
    const otree *t = (const otree *)h;
    if (!t || nq < 0 || k < 1) return -1;
    set_threads(threads);
    int bad = 0;
#pragma omp parallel
    {
        okstate s;
        s.k = k;
        s.bd = (float *)malloc(sizeof(float) * (size_t)k);
        s.bi = (int32_t *)malloc(sizeof(int32_t) * (size_t)k);
        if (!s.bd || !s.bi) {
#pragma omp atomic write
            bad = 1;
        } else {
#pragma omp for schedule(dynamic, 16)
            for (int64_t i = 0; i < nq; ++i) {
                s.cnt = 0;
                const float *q = qs + i * t->d;
                if (t->n > 0) bnb_visit(t, 0, q, &s);
                best_emit(s.bd, s.bi, s.cnt, k, out_ids + i * k, out_dists + i * k);
            }
        }
        free(s.bd);
        free(s.bi);
    }
    return bad ? -2 : 0;
}
