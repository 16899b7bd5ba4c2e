/*
 * ORACLE — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, single-threaded C99 implementation of the two-pass min-wise
 * Shingling of Gibson et al. exactly as Wu & Kalyanaraman describe it
 * (gpClust, IPDPSW 2013).  Citations "P:Lx-y" point into the paper text
 * (PAPER.md lines x-y); "AMB-n" / "R-n" are the readings fixed in DESIGN.md §3
 * where the paper is silent or garbled.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  It shares no code, header,
 * table or constant generator with the CUDA path (paper_conf_ipps_wuk13_b200/
 * csrc); every constant below is restated from the paper or DESIGN.md.
 *
 * Pins (tests/test_oracle_*.py, -m "not gpu"): splitmix64 published
 * known-answer vector; big-integer hash incl. adversarial zero / max residues;
 * brute-force full sort == insertion top-s for every (row, trial); twins;
 * planted cliques; min-wise collision rate == closed form (binomial tail);
 * exact-tuple grouping == id grouping; id round trip through A^-1;
 * CC-locality; union-find == BFS components; N-version equality with the
 * pure-Python twin (oracle/twin.py).  Nothing here is "parity unpinned"
 * except the absolute outputs against the paper, which prints none.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* P = 2^31 - 1, "a big prime number" (reading AMB-1). */
#define OR_P 2147483647ULL

/* ---------------------------------------------------------------------- */
/* Random pairs {<A_j, B_j> | j in [1, c]}.       */
/* Drawn from a splitmix64 stream (reading AMB-2).                          */
/* ---------------------------------------------------------------------- */

/* splitmix64 finaliser (Steele, Lea & Flood 2014; Vigna's splitmix64.c). */
uint64_t or_mix64(uint64_t z)
{
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}

/* next(): state += golden gamma; return mix64(state). */
uint64_t or_splitmix_next(uint64_t *state)
{
    *state += 0x9E3779B97F4A7C15ULL;
    return or_mix64(*state);
}

/* A_j = 1 + next() % (P-1)  (A_j != 0 so h_j is a bijection);
 * B_j = next() % P; drawn in the order A_0, B_0, A_1, B_1, ... */
void or_hash_params(uint64_t seed, int32_t c, uint32_t *A, uint32_t *B)
{
    uint64_t state = seed;
    for (int32_t j = 0; j < c; j++) {
        A[j] = (uint32_t)(1 + or_splitmix_next(&state) % (OR_P - 1));
        B[j] = (uint32_t)(or_splitmix_next(&state) % OR_P);
    }
}

/* v^j = (A_j * v + B_j) % P. */
uint32_t or_hash(uint32_t A, uint32_t B, uint32_t v)
{
    return (uint32_t)(((uint64_t)A * (uint64_t)v + (uint64_t)B) % OR_P);
}

/* ---------------------------------------------------------------------- */
/* Input validation (reading AMB-8): 0 <= n < P, row_ptr monotone from 0   */
/* to nnz, each row strictly increasing, 0 <= col < n.                      */
/* ---------------------------------------------------------------------- */
int32_t or_validate(int64_t n, int64_t nnz, const int64_t *row_ptr, const int32_t *col)
{
    if (n < 0 || (uint64_t)n >= OR_P || nnz < 0) return 1;
    if (row_ptr[0] != 0 || row_ptr[n] != nnz) return 1;
    for (int64_t u = 0; u < n; u++) {
        if (row_ptr[u + 1] < row_ptr[u]) return 1;
        for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) {
            if (col[e] < 0 || (int64_t)col[e] >= n) return 1;
            if (e > row_ptr[u] && col[e] <= col[e - 1]) return 1;
        }
    }
    return 0;
}

/* ---------------------------------------------------------------------- */
/* One shingle: the s minimum elements of Gamma_j(u), kept in an s-sized  */
/* array by insertion sort during an on-the-fly enumeration. */
/* mins[] receives the hashed values ascending, argv[] the vertices.      */
/* ---------------------------------------------------------------------- */
static uint64_t g_hash_evals = 0;

static void top_s_insertion(const uint32_t *row, int64_t deg, int32_t s,
                            uint32_t A, uint32_t B, uint32_t *mins, uint32_t *argv)
{
    int32_t filled = 0;
    for (int64_t e = 0; e < deg; e++) {
        uint32_t v = row[e];
        uint32_t h = or_hash(A, B, v);
        g_hash_evals++;
        if (filled == s && h >= mins[s - 1]) continue;
        int32_t i = (filled < s) ? filled++ : s - 1;   /* drop the largest */
        while (i > 0 && mins[i - 1] > h) {
            mins[i] = mins[i - 1];
            argv[i] = argv[i - 1];
            i--;
        }
        mins[i] = h;
        argv[i] = v;
    }
}

/* Integer representation of a shingle (reading AMB-4):
 *   s = 1 : id = h_1
 *   s = 2 : id = h_1 * 2^31 + h_2            (exact, collision free)
 *   s >= 3: z = mix64(seed ^ mix64(j + 1)); z = mix64(z + h_i) for i = 1..s */
uint64_t or_shingle_id(int32_t s, uint64_t seed, int32_t j, const uint32_t *mins)
{
    if (s == 1) return (uint64_t)mins[0];
    if (s == 2) return (uint64_t)mins[0] * 2147483648ULL + (uint64_t)mins[1];
    uint64_t z = or_mix64(seed ^ or_mix64((uint64_t)j + 1));
    for (int32_t i = 0; i < s; i++) z = or_mix64(z + (uint64_t)mins[i]);
    return z;
}

/* The c shingle ids of one row (all trials), plus optional constituents. */
void or_row_shingles(const uint32_t *row, int64_t deg, int32_t s, int32_t c, uint64_t seed,
                     const uint32_t *A, const uint32_t *B, uint64_t *ids_out)
{
    uint32_t mins[16], argv[16];
    for (int32_t j = 0; j < c; j++) {
        top_s_insertion(row, deg, s, A[j], B[j], mins, argv);
        ids_out[j] = or_shingle_id(s, seed, j, mins);
    }
}

/* The s vertices constituting the trial-j shingle of a row, ascending by hash. */
void or_row_constituents(const uint32_t *row, int64_t deg, int32_t s, uint32_t A, uint32_t B,
                         uint32_t *verts_out)
{
    uint32_t mins[16];
    top_s_insertion(row, deg, s, A, B, mins, verts_out);
}

uint64_t or_hash_evals(void) { return g_hash_evals; }
void or_reset_hash_evals(void) { g_hash_evals = 0; }

/* ---------------------------------------------------------------------- */
/* Grouping: "a sorting is done to gather all vertices that generated each */
/* shingle ... once for each random trial" (reading AMB-5),    */
/* tuples <s_j, L(s_j)>.  Canonical order (reading AMB-19):   */
/* per trial, groups by key = mix64(id) ascending, members ascending.      */
/* ---------------------------------------------------------------------- */
typedef struct {
    uint64_t key;
    uint64_t id;
    uint32_t member;
} or_pair;

/* Plain top-down stable merge sort by key. */
static void merge_sort_by_key(or_pair *a, or_pair *tmp, int64_t lo, int64_t hi)
{
    if (hi - lo < 2) return;
    int64_t mid = lo + (hi - lo) / 2;
    merge_sort_by_key(a, tmp, lo, mid);
    merge_sort_by_key(a, tmp, mid, hi);
    int64_t i = lo, k = mid, o = lo;
    while (i < mid && k < hi) {
        if (a[k].key < a[i].key) tmp[o++] = a[k++];
        else tmp[o++] = a[i++];           /* ties keep the left (earlier) one */
    }
    while (i < mid) tmp[o++] = a[i++];
    while (k < hi) tmp[o++] = a[k++];
    memcpy(a + lo, tmp + lo, (size_t)(hi - lo) * sizeof(or_pair));
}

typedef struct {
    int32_t c;
    int64_t ngroups;
    int64_t npairs;
    int64_t *trial_goffs;  /* [c+1]: groups of trial j are [trial_goffs[j], trial_goffs[j+1]) */
    uint64_t *ids;         /* [ngroups] shingle id */
    int64_t *offs;         /* [ngroups+1] into members */
    uint32_t *members;     /* [npairs] L(s), ascending within a group */
} or_groups;

/* ids is the shingle matrix [nrows x c] row-major; member[r] is the value
 * emitted by row r (pass 1: the vertex id; pass 2: the S1' index). */
static int group_pass(int64_t nrows, int32_t c, const uint64_t *ids, const uint32_t *member,
                      or_groups *G)
{
    G->c = c;
    G->npairs = nrows * (int64_t)c;
    G->trial_goffs = (int64_t *)calloc((size_t)c + 1, sizeof(int64_t));
    G->members = (uint32_t *)malloc((size_t)(G->npairs > 0 ? G->npairs : 1) * sizeof(uint32_t));
    /* worst case: every pair its own group */
    G->ids = (uint64_t *)malloc((size_t)(G->npairs > 0 ? G->npairs : 1) * sizeof(uint64_t));
    G->offs = (int64_t *)malloc((size_t)(G->npairs + 1) * sizeof(int64_t));
    or_pair *pairs = (or_pair *)malloc((size_t)(nrows > 0 ? nrows : 1) * sizeof(or_pair));
    or_pair *tmp = (or_pair *)malloc((size_t)(nrows > 0 ? nrows : 1) * sizeof(or_pair));
    if (!G->trial_goffs || !G->members || !G->ids || !G->offs || !pairs || !tmp) return 1;
    int64_t ng = 0, np = 0;
    for (int32_t j = 0; j < c; j++) {
        G->trial_goffs[j] = ng;
        for (int64_t r = 0; r < nrows; r++) {        /* emission order */
            pairs[r].id = ids[r * c + j];
            pairs[r].key = or_mix64(pairs[r].id);
            pairs[r].member = member[r];
        }
        merge_sort_by_key(pairs, tmp, 0, nrows);
        for (int64_t r = 0; r < nrows; r++) {
            if (r == 0 || pairs[r].key != pairs[r - 1].key) {
                G->ids[ng] = pairs[r].id;
                G->offs[ng] = np;
                ng++;
            }
            G->members[np++] = pairs[r].member;
        }
    }
    G->trial_goffs[c] = ng;
    G->offs[ng] = np;
    G->ngroups = ng;
    free(pairs);
    free(tmp);
    return 0;
}

static void free_groups(or_groups *G)
{
    free(G->trial_goffs);
    free(G->ids);
    free(G->offs);
    free(G->members);
    memset(G, 0, sizeof(*G));
}

/* ---------------------------------------------------------------------- */
/* The whole two-pass method (Fig. 2).             */
/* ---------------------------------------------------------------------- */
typedef struct {
    int32_t s1, c1, s2, c2;
    uint64_t seed1, seed2;
    uint32_t *A1, *B1, *A2, *B2;
    int64_t n;
    const int64_t *row_ptr;   /* borrowed CSR of G (needed by the report) */
    const int32_t *col;
    /* Pass I */
    int64_t n_e;              /* vertices with >= s1 links */
    uint32_t *rows1;          /* [n_e] those vertices, ascending */
    uint64_t *M1;             /* [n_e x c1] row-major shingle ids */
    or_groups G1;
    /* S1' = first-level shingles with |L| >= s2: the pass-II rows */
    int64_t n_s1p;
    int64_t *s1p_group;       /* [n_s1p] index into G1 of S1' node k */
    uint64_t *M2;             /* [n_s1p x c2] */
    or_groups G2;
    uint64_t hash_evals;
    int32_t status;
} or_result;

void or_free(or_result *R);

or_result *or_shingling(int64_t n, int64_t nnz, const int64_t *row_ptr, const int32_t *col,
                        int32_t s1, int32_t c1, uint64_t seed1,
                        int32_t s2, int32_t c2, uint64_t seed2)
{
    or_result *R = (or_result *)calloc(1, sizeof(or_result));
    if (!R) return NULL;
    R->s1 = s1; R->c1 = c1; R->s2 = s2; R->c2 = c2;
    R->seed1 = seed1; R->seed2 = seed2;
    R->n = n; R->row_ptr = row_ptr; R->col = col;
    if (s1 < 1 || s1 > 16 || s2 < 1 || s2 > 16 || c1 < 1 || c2 < 1 ||
        or_validate(n, nnz, row_ptr, col)) {
        R->status = 1;
        return R;
    }
    or_reset_hash_evals();

    /* H = {<A_j, B_j>} for each pass, independent seeds (reading AMB-3). */
    R->A1 = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)c1);
    R->B1 = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)c1);
    R->A2 = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)c2);
    R->B2 = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)c2);
    or_hash_params(seed1, c1, R->A1, R->B1);
    or_hash_params(seed2, c2, R->A2, R->B2);

    /* Pass I: every u in V_l with at least s1 links, c1 shingles. */
    int64_t n_e = 0;
    for (int64_t u = 0; u < n; u++)
        if (row_ptr[u + 1] - row_ptr[u] >= s1) n_e++;
    R->n_e = n_e;
    R->rows1 = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)(n_e > 0 ? n_e : 1));
    R->M1 = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(n_e > 0 ? n_e * c1 : 1));
    int64_t r = 0;
    for (int64_t u = 0; u < n; u++) {
        int64_t deg = row_ptr[u + 1] - row_ptr[u];
        if (deg < s1) continue;
        R->rows1[r] = (uint32_t)u;
        or_row_shingles((const uint32_t *)(col + row_ptr[u]), deg, s1, c1, seed1,
                        R->A1, R->B1, R->M1 + r * c1);
        r++;
    }
    if (group_pass(n_e, c1, R->M1, R->rows1, &R->G1)) { R->status = 2; return R; }

    /* S1' and the pass-II input G_I: rows are L(s) of groups with |L| >= s2. */
    int64_t n_s1p = 0;
    for (int64_t g = 0; g < R->G1.ngroups; g++)
        if (R->G1.offs[g + 1] - R->G1.offs[g] >= s2) n_s1p++;
    R->n_s1p = n_s1p;
    R->s1p_group = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n_s1p > 0 ? n_s1p : 1));
    R->M2 = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(n_s1p > 0 ? n_s1p * c2 : 1));
    uint32_t *member2 = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)(n_s1p > 0 ? n_s1p : 1));
    int64_t k = 0;
    for (int64_t g = 0; g < R->G1.ngroups; g++) {
        int64_t len = R->G1.offs[g + 1] - R->G1.offs[g];
        if (len < s2) continue;
        R->s1p_group[k] = g;
        member2[k] = (uint32_t)k;
        /* Pass II: "the same series of steps as in Phase I". */
        or_row_shingles(R->G1.members + R->G1.offs[g], len, s2, c2, seed2,
                        R->A2, R->B2, R->M2 + k * c2);
        k++;
    }
    if (group_pass(n_s1p, c2, R->M2, member2, &R->G2)) { R->status = 2; free(member2); return R; }
    free(member2);
    R->hash_evals = or_hash_evals();
    R->status = 0;
    return R;
}

void or_free(or_result *R)
{
    if (!R) return;
    free(R->A1); free(R->B1); free(R->A2); free(R->B2);
    free(R->rows1); free(R->M1); free(R->s1p_group); free(R->M2);
    free_groups(&R->G1);
    free_groups(&R->G2);
    free(R);
}

/* Plain accessors for the ctypes wrapper (oracle/__init__.py). */
int32_t or_status(const or_result *R) { return R->status; }
int64_t or_n_e(const or_result *R) { return R->n_e; }
int64_t or_n_s1p(const or_result *R) { return R->n_s1p; }
uint64_t or_result_hash_evals(const or_result *R) { return R->hash_evals; }
const uint32_t *or_rows1(const or_result *R) { return R->rows1; }
const uint64_t *or_M1(const or_result *R) { return R->M1; }
const uint64_t *or_M2(const or_result *R) { return R->M2; }
const int64_t *or_s1p_group(const or_result *R) { return R->s1p_group; }
const uint32_t *or_params(const or_result *R, int32_t which)
{
    switch (which) {
    case 0: return R->A1;
    case 1: return R->B1;
    case 2: return R->A2;
    default: return R->B2;
    }
}
static const or_groups *pick(const or_result *R, int32_t level) { return level == 1 ? &R->G1 : &R->G2; }
int64_t or_g_ngroups(const or_result *R, int32_t level) { return pick(R, level)->ngroups; }
int64_t or_g_npairs(const or_result *R, int32_t level) { return pick(R, level)->npairs; }
const int64_t *or_g_trial_goffs(const or_result *R, int32_t level) { return pick(R, level)->trial_goffs; }
const uint64_t *or_g_ids(const or_result *R, int32_t level) { return pick(R, level)->ids; }
const int64_t *or_g_offs(const or_result *R, int32_t level) { return pick(R, level)->offs; }
const uint32_t *or_g_members(const or_result *R, int32_t level) { return pick(R, level)->members; }

/* ---------------------------------------------------------------------- */
/* Phase III, approach 2: union-find of size n;   */
/* for each connected component of G_II, union the vertices of G that      */
/* constitute its first- and second-level shingles (mode 0, reading AMB-9) */
/* or that generated its first-level shingles (mode 1).  label(v) = the    */
/* smallest vertex of its set (AMB-10); sets smaller than min_size are     */
/* reported as singletons.                                                 */
/* ---------------------------------------------------------------------- */
static int64_t uf_find(int64_t *p, int64_t x)
{
    while (p[x] != x) {
        p[x] = p[p[x]];
        x = p[x];
    }
    return x;
}

static void uf_union(int64_t *p, int64_t a, int64_t b)
{
    a = uf_find(p, a);
    b = uf_find(p, b);
    if (a == b) return;
    if (a < b) p[b] = a; else p[a] = b;   /* root = smaller index */
}

/* The s1 vertices that constitute first-level shingle node k (its trial-j
 * shingle, recomputed from the smallest generator; reading AMB-18). */
static void constituents1(const or_result *R, int64_t g, uint32_t *out)
{
    int32_t j = 0;
    while (R->G1.trial_goffs[j + 1] <= g) j++;
    uint32_t u = R->G1.members[R->G1.offs[g]];       /* min L (members ascending) */
    or_row_constituents((const uint32_t *)(R->col + R->row_ptr[u]),
                        R->row_ptr[u + 1] - R->row_ptr[u], R->s1, R->A1[j], R->B1[j], out);
}

/* The s2 vertices that constitute second-level shingle h (G2 group). */
static void constituents2(const or_result *R, int64_t h, uint32_t *out)
{
    int32_t t = 0;
    while (R->G2.trial_goffs[t + 1] <= h) t++;
    uint32_t kmin = R->G2.members[R->G2.offs[h]];
    int64_t g = R->s1p_group[kmin];
    or_row_constituents(R->G1.members + R->G1.offs[g], R->G1.offs[g + 1] - R->G1.offs[g],
                        R->s2, R->A2[t], R->B2[t], out);
}

int32_t or_report(const or_result *R, int32_t mode, int32_t min_size, int32_t *labels,
                  int64_t *n_clusters)
{
    if (R->status != 0) return 1;
    int64_t n = R->n;
    /* 1. connected components of G_II over its S1' nodes */
    int64_t *pc = (int64_t *)malloc(sizeof(int64_t) * (size_t)(R->n_s1p > 0 ? R->n_s1p : 1));
    for (int64_t k = 0; k < R->n_s1p; k++) pc[k] = k;
    for (int64_t h = 0; h < R->G2.ngroups; h++)
        for (int64_t e = R->G2.offs[h] + 1; e < R->G2.offs[h + 1]; e++)
            uf_union(pc, R->G2.members[R->G2.offs[h]], R->G2.members[e]);
    /* 2. per component, the vertex set to union: list (component, vertex) */
    int64_t cap = 16, cnt = 0;
    int64_t *cv = (int64_t *)malloc(sizeof(int64_t) * 2 * (size_t)cap);
    uint32_t buf[16];
#define PUSH(C, V) do { if (cnt == cap) { cap *= 2; cv = (int64_t *)realloc(cv, sizeof(int64_t) * 2 * (size_t)cap); } \
                        cv[2 * cnt] = (C); cv[2 * cnt + 1] = (V); cnt++; } while (0)
    for (int64_t k = 0; k < R->n_s1p; k++) {
        int64_t comp = uf_find(pc, k);
        int64_t g = R->s1p_group[k];
        if (mode == 0) {
            constituents1(R, g, buf);
            for (int32_t i = 0; i < R->s1; i++) PUSH(comp, buf[i]);
        } else {
            for (int64_t e = R->G1.offs[g]; e < R->G1.offs[g + 1]; e++) PUSH(comp, R->G1.members[e]);
        }
    }
    if (mode == 0) {
        for (int64_t h = 0; h < R->G2.ngroups; h++) {
            int64_t comp = uf_find(pc, R->G2.members[R->G2.offs[h]]);
            constituents2(R, h, buf);
            for (int32_t i = 0; i < R->s2; i++) PUSH(comp, buf[i]);
        }
    }
#undef PUSH
    /* 3. union-find of size n; union every vertex of a component's set with
     *    the first vertex recorded for that component */
    int64_t *pv = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int64_t *first = (int64_t *)malloc(sizeof(int64_t) * (size_t)(R->n_s1p > 0 ? R->n_s1p : 1));
    for (int64_t v = 0; v < n; v++) pv[v] = v;
    for (int64_t k = 0; k < R->n_s1p; k++) first[k] = -1;
    for (int64_t i = 0; i < cnt; i++) {
        int64_t comp = cv[2 * i], v = cv[2 * i + 1];
        if (first[comp] < 0) first[comp] = v;
        else uf_union(pv, first[comp], v);
    }
    /* 4. labels: root = smallest vertex of the set; small sets -> singletons */
    int64_t *size = (int64_t *)calloc((size_t)(n > 0 ? n : 1), sizeof(int64_t));
    for (int64_t v = 0; v < n; v++) size[uf_find(pv, v)]++;
    int64_t nc = 0;
    int64_t thr = min_size > 2 ? min_size : 2;
    for (int64_t v = 0; v < n; v++) {
        int64_t root = uf_find(pv, v);
        if (size[root] >= min_size) labels[v] = (int32_t)root;
        else labels[v] = (int32_t)v;
        if (root == v && size[root] >= thr) nc++;
    }
    *n_clusters = nc;
    free(pc); free(cv); free(pv); free(first); free(size);
    return 0;
}

/* ---------------------------------------------------------------------- */
/* Trial-outer streaming run of the same method, for graphs whose full     */
/* outputs do not fit in host memory (the 2M and 640M configurations).     */
/* The loop order of P:L445-460 (vertex-outer) versus trial-outer does not  */
/* change any output, and grouping is per trial (AMB-5), so    */
/* trial j of G_I depends only on column j of the pass-I matrix.  Pass I   */
/* and G_I are computed one trial at a time for all c1 trials; the S1'     */
/* nodes of trial j (groups with |L| >= s2) get their dense    */
/* index k in canonical (trial, key) order and their pass-II shingles for  */
/* the requested pass-II trials only (pass II "the same series of steps",  */
/* P:L461-462); G_II is formed for those trials.  Kept: the pass-I columns */
/* and G_I trials listed in keep1, the pass-II columns and G_II trials     */
/* listed in keep2, the S1' map, counts, and per-trial digests of every    */
/* pass-I column and G_I trial.                                            */
/*                                                                          */
/* Digest (test infrastructure, order- and position-sensitive): a column   */
/* x_0..x_{N-1} digests to sum_i mix64(x_i + mix64(i)) mod 2^64; a grouped */
/* trial with group ids id_g and members m_p (head bit h_p = 1 at the first */
/* member of a group) to sum_g mix64(id_g + mix64(2g))                     */
/*                     + sum_p mix64((m_p | h_p << 32) + mix64(2p + 1)).   */
/* ---------------------------------------------------------------------- */
static uint64_t dig_col_term(uint64_t x, uint64_t i) { return or_mix64(x + or_mix64(i)); }
static uint64_t dig_gid_term(uint64_t id, uint64_t g) { return or_mix64(id + or_mix64(2 * g)); }
static uint64_t dig_mem_term(uint32_t m, int head, uint64_t p)
{
    return or_mix64(((uint64_t)m | ((uint64_t)(head ? 1 : 0) << 32)) + or_mix64(2 * p + 1));
}

/* The within-trial id of one row for trial j: insertion top-s + id. */
static uint64_t row_trial_id(const uint32_t *row, int64_t deg, int32_t s, uint64_t seed, int32_t j,
                             uint32_t A, uint32_t B)
{
    uint32_t mins[16], argv[16];
    top_s_insertion(row, deg, s, A, B, mins, argv);
    return or_shingle_id(s, seed, j, mins);
}

typedef struct {
    int64_t n, cap;
    void *p;
    size_t esz;
} or_vec;

static int vec_push(or_vec *v, const void *x)
{
    if (v->n == v->cap) {
        int64_t nc = v->cap ? v->cap * 2 : 1024;
        void *q = realloc(v->p, (size_t)nc * v->esz);
        if (!q) return 1;
        v->p = q;
        v->cap = nc;
    }
    memcpy((char *)v->p + (size_t)v->n * v->esz, x, v->esz);
    v->n++;
    return 0;
}

typedef struct {
    int32_t status;
    int32_t c1, c2, nkeep1, nkeep2;
    int64_t n_e, groups1, pairs1, n_s1p, e2;
    uint32_t *rows1;          /* [n_e] */
    uint64_t *dig_M1;         /* [c1] */
    uint64_t *dig_G1;         /* [c1] */
    uint64_t *M1k;            /* [n_e x nkeep1] columns keep1[] of the pass-I matrix */
    or_groups G1k;            /* G_I restricted to trials keep1[] (c = nkeep1) */
    int64_t *s1p_group;       /* [n_s1p] global G_I group index of S1' node k */
    uint64_t *M2k;            /* [n_s1p x nkeep2] columns keep2[] of the pass-II matrix */
    or_groups G2k;            /* G_II restricted to trials keep2[] */
    uint64_t *dig_G2k;        /* [nkeep2] */
} or_stream;

static int in_list(const int32_t *l, int32_t n, int32_t x)
{
    for (int32_t i = 0; i < n; i++)
        if (l[i] == x) return i;
    return -1;
}

void or_stream_free(or_stream *S);

or_stream *or_shingling_stream(int64_t n, int64_t nnz, const int64_t *row_ptr, const int32_t *col,
                               int32_t s1, int32_t c1, uint64_t seed1,
                               int32_t s2, int32_t c2, uint64_t seed2,
                               const int32_t *keep1, int32_t nkeep1,
                               const int32_t *keep2, int32_t nkeep2)
{
    or_stream *S = (or_stream *)calloc(1, sizeof(or_stream));
    if (!S) return NULL;
    S->c1 = c1; S->c2 = c2; S->nkeep1 = nkeep1; S->nkeep2 = nkeep2;
    if (s1 < 1 || s1 > 16 || s2 < 1 || s2 > 16 || c1 < 1 || c2 < 1 || nkeep1 < 0 || nkeep2 < 0 ||
        or_validate(n, nnz, row_ptr, col)) {
        S->status = 1;
        return S;
    }
    uint32_t *A1 = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)c1);
    uint32_t *B1 = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)c1);
    uint32_t *A2 = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)c2);
    uint32_t *B2 = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)c2);
    or_hash_params(seed1, c1, A1, B1);
    or_hash_params(seed2, c2, A2, B2);

    /* pass-I rows: vertices with >= s1 links */
    int64_t n_e = 0;
    for (int64_t u = 0; u < n; u++)
        if (row_ptr[u + 1] - row_ptr[u] >= s1) n_e++;
    S->n_e = n_e;
    S->rows1 = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)(n_e > 0 ? n_e : 1));
    for (int64_t u = 0, r = 0; u < n; u++)
        if (row_ptr[u + 1] - row_ptr[u] >= s1) S->rows1[r++] = (uint32_t)u;
    S->dig_M1 = (uint64_t *)calloc((size_t)c1, sizeof(uint64_t));
    S->dig_G1 = (uint64_t *)calloc((size_t)c1, sizeof(uint64_t));
    S->M1k = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(n_e * nkeep1 > 0 ? n_e * nkeep1 : 1));
    or_pair *pairs = (or_pair *)malloc((size_t)(n_e > 0 ? n_e : 1) * sizeof(or_pair));
    or_pair *tmp = (or_pair *)malloc((size_t)(n_e > 0 ? n_e : 1) * sizeof(or_pair));
    /* kept G_I trials (grown as they are cut) */
    or_vec g1ids = {0, 0, NULL, sizeof(uint64_t)}, g1offs = {0, 0, NULL, sizeof(int64_t)};
    or_vec g1mem = {0, 0, NULL, sizeof(uint32_t)};
    S->G1k.c = nkeep1;
    S->G1k.trial_goffs = (int64_t *)calloc((size_t)nkeep1 + 1, sizeof(int64_t));
    /* S1' map and the kept pass-II columns */
    or_vec s1p = {0, 0, NULL, sizeof(int64_t)};
    or_vec m2 = {0, 0, NULL, sizeof(uint64_t) * (size_t)(nkeep2 > 0 ? nkeep2 : 1)};
    uint64_t *m2row = (uint64_t *)calloc((size_t)(nkeep2 > 0 ? nkeep2 : 1), sizeof(uint64_t));
    if (!A1 || !B1 || !A2 || !B2 || !S->rows1 || !S->dig_M1 || !S->dig_G1 || !S->M1k || !pairs ||
        !tmp || !S->G1k.trial_goffs || !m2row) {
        S->status = 2;
        goto done;
    }
    int64_t g_glob = 0;    /* global G_I group index */
    for (int32_t j = 0; j < c1; j++) {
        const int32_t kj = in_list(keep1, nkeep1, j);
        uint64_t dm = 0;
        for (int64_t r = 0; r < n_e; r++) {                   /* emission order */
            const uint32_t u = S->rows1[r];
            const uint64_t id = row_trial_id((const uint32_t *)(col + row_ptr[u]),
                                             row_ptr[u + 1] - row_ptr[u], s1, seed1, j, A1[j], B1[j]);
            dm += dig_col_term(id, (uint64_t)r);
            if (kj >= 0) S->M1k[r * nkeep1 + kj] = id;
            pairs[r].id = id;
            pairs[r].key = or_mix64(id);
            pairs[r].member = u;
        }
        S->dig_M1[j] = dm;
        merge_sort_by_key(pairs, tmp, 0, n_e);                  /* per-trial sorting (AMB-5) */
        if (kj >= 0) S->G1k.trial_goffs[kj] = g1ids.n;           /* keep1 is given ascending */
        uint64_t dg = 0;
        int64_t gl = -1;       /* local group index within trial j */
        for (int64_t r = 0; r < n_e;) {
            int64_t e = r + 1;
            while (e < n_e && pairs[e].key == pairs[r].key) e++;
            gl++;
            dg += dig_gid_term(pairs[r].id, (uint64_t)gl);
            for (int64_t x = r; x < e; x++) dg += dig_mem_term(pairs[x].member, x == r, (uint64_t)x);
            if (kj >= 0) {
                int64_t off = g1mem.n;
                if (vec_push(&g1ids, &pairs[r].id) || vec_push(&g1offs, &off)) { S->status = 2; goto done; }
                for (int64_t x = r; x < e; x++)
                    if (vec_push(&g1mem, &pairs[x].member)) { S->status = 2; goto done; }
            }
            const int64_t len = e - r;
            if (len >= s2) {                                      /* S1' */
                /* L(s): the generators, ascending (stable sort of ascending rows) */
                uint32_t *L = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)len);
                if (!L) { S->status = 2; goto done; }
                for (int64_t x = r; x < e; x++) L[x - r] = pairs[x].member;
                for (int32_t t2 = 0; t2 < nkeep2; t2++) {
                    const int32_t t = keep2[t2];
                    m2row[t2] = row_trial_id(L, len, s2, seed2, t, A2[t], B2[t]);
                }
                free(L);
                if (vec_push(&s1p, &g_glob) || (nkeep2 > 0 && vec_push(&m2, m2row))) { S->status = 2; goto done; }
                S->e2 += len;
            }
            g_glob++;
            r = e;
        }
        S->dig_G1[j] = dg;
        S->groups1 += gl + 1;
        S->pairs1 += n_e;
    }
    S->G1k.trial_goffs[nkeep1] = g1ids.n;
    S->G1k.ngroups = g1ids.n;
    S->G1k.npairs = g1mem.n;
    {
        int64_t endoff = g1mem.n;
        if (vec_push(&g1offs, &endoff)) { S->status = 2; goto done; }
    }
    S->G1k.ids = (uint64_t *)g1ids.p;
    S->G1k.offs = (int64_t *)g1offs.p;
    S->G1k.members = (uint32_t *)g1mem.p;
    g1ids.p = g1offs.p = g1mem.p = NULL;
    S->n_s1p = s1p.n;
    S->s1p_group = (int64_t *)s1p.p;
    s1p.p = NULL;
    S->M2k = (uint64_t *)m2.p;
    m2.p = NULL;
    /* G_II for the kept pass-II trials: the same grouping (member = k) */
    {
        const int64_t nk = S->n_s1p;
        uint64_t *col2 = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(nk * (nkeep2 > 0 ? nkeep2 : 1) + 1));
        uint32_t *kk = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)(nk > 0 ? nk : 1));
        S->dig_G2k = (uint64_t *)calloc((size_t)(nkeep2 > 0 ? nkeep2 : 1), sizeof(uint64_t));
        if (!col2 || !kk || !S->dig_G2k) { free(col2); free(kk); S->status = 2; goto done; }
        for (int64_t k = 0; k < nk; k++) kk[k] = (uint32_t)k;
        /* group_pass wants the [rows x c] matrix: M2k already is [nk x nkeep2] */
        if (nkeep2 > 0 && group_pass(nk, nkeep2, S->M2k, kk, &S->G2k)) {
            free(col2); free(kk); S->status = 2; goto done;
        }
        if (nkeep2 == 0) {
            S->G2k.trial_goffs = (int64_t *)calloc(1, sizeof(int64_t));
            S->G2k.offs = (int64_t *)calloc(1, sizeof(int64_t));
        }
        for (int32_t t2 = 0; t2 < nkeep2; t2++) {
            uint64_t d = 0;
            const int64_t g0 = S->G2k.trial_goffs[t2], g1 = S->G2k.trial_goffs[t2 + 1];
            const int64_t p0 = S->G2k.offs[g0];
            for (int64_t g = g0; g < g1; g++) {
                d += dig_gid_term(S->G2k.ids[g], (uint64_t)(g - g0));
                for (int64_t p = S->G2k.offs[g]; p < S->G2k.offs[g + 1]; p++)
                    d += dig_mem_term(S->G2k.members[p], p == S->G2k.offs[g], (uint64_t)(p - p0));
            }
            S->dig_G2k[t2] = d;
        }
        free(col2);
        free(kk);
    }
    S->status = 0;
done:
    free(A1); free(B1); free(A2); free(B2);
    free(pairs); free(tmp); free(m2row);
    free(g1ids.p); free(g1offs.p); free(g1mem.p); free(s1p.p); free(m2.p);
    return S;
}

void or_stream_free(or_stream *S)
{
    if (!S) return;
    free(S->rows1); free(S->dig_M1); free(S->dig_G1); free(S->M1k);
    free_groups(&S->G1k);
    free(S->s1p_group); free(S->M2k);
    free_groups(&S->G2k);
    free(S->dig_G2k);
    free(S);
}

/* Plain accessors (oracle/__init__.py). */
int32_t or_st_status(const or_stream *S) { return S->status; }
void or_st_counts(const or_stream *S, int64_t out[5])
{
    out[0] = S->n_e; out[1] = S->groups1; out[2] = S->pairs1; out[3] = S->n_s1p; out[4] = S->e2;
}
const uint32_t *or_st_rows1(const or_stream *S) { return S->rows1; }
const uint64_t *or_st_dig(const or_stream *S, int32_t which)
{
    return which == 0 ? S->dig_M1 : which == 1 ? S->dig_G1 : S->dig_G2k;
}
const uint64_t *or_st_M(const or_stream *S, int32_t level) { return level == 1 ? S->M1k : S->M2k; }
const int64_t *or_st_s1p_group(const or_stream *S) { return S->s1p_group; }
static const or_groups *st_pick(const or_stream *S, int32_t level) { return level == 1 ? &S->G1k : &S->G2k; }
int64_t or_st_g_ngroups(const or_stream *S, int32_t level) { return st_pick(S, level)->ngroups; }
int64_t or_st_g_npairs(const or_stream *S, int32_t level) { return st_pick(S, level)->npairs; }
const int64_t *or_st_g_trial_goffs(const or_stream *S, int32_t level) { return st_pick(S, level)->trial_goffs; }
const uint64_t *or_st_g_ids(const or_stream *S, int32_t level) { return st_pick(S, level)->ids; }
const int64_t *or_st_g_offs(const or_stream *S, int32_t level) { return st_pick(S, level)->offs; }
const uint32_t *or_st_g_members(const or_stream *S, int32_t level) { return st_pick(S, level)->members; }
