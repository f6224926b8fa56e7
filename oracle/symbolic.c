/*
 * oracle/symbolic.c -- CPU ORACLE, symbolic part.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this code.  It
 * shares no code, header, table or helper with the CUDA product path
 * (paper_conf_ipps_georgesgsc11_b200/); neither includes the other.
 *
 * What it computes: the symbolic structure the multifrontal method runs on
 * [PAPER.md L27, Sec. II-A]: "The algorithm performs a postorder traversal of
 * the supernodal elimination tree ... k is the size (number of consecutive rows
 * and columns with the same nonzero pattern in L) of the supernode n".  The
 * paper does not specify the symbolic algorithms or WSMP's amalgamation, so this
 * file follows the plain DEFINITIONS, step by step, in the order of SURVEY.md
 * Sec. 8(c) "Oracle algorithm" steps 1-6 and the exact amalgamation rule of
 * SURVEY.md Appendix B (readings C2, C5 in DESIGN.md):
 *
 *   1. B = P A P^T, lower pattern (upper entries of A ignored, duplicates merged).
 *   2. For j = 0..n-1 ascending:
 *        struct(L_j) = {j} U {i > j : B(i,j) != 0} U  U_{c : parent(c) = j} (struct(L_c) \ {c})
 *        parent(j)   = min(struct(L_j) \ {j}), or -1.
 *      (the definition of the column structures and of the elimination tree;
 *       no Liu's algorithm, no row-subtree counting -- the product path uses
 *       those, this file must not.)
 *   3. Postorder (iterative DFS, roots and children ascending).  If it is not
 *      the identity, relabel (compose perm) and redo 1-2.
 *   4. cc_j = |struct(L_j)|, nnz(L) = sum cc_j, flops = sum cc_j^2.
 *   5. Fundamental supernodes: j, j+1 together iff parent(j) = j+1, j+1 has
 *      exactly one child and cc_j = cc_{j+1} + 1.
 *   6. Relaxed amalgamation (Appendix B rule, verbatim) and row lists
 *      R_s = U_{j in cols(s)} struct(L_j).
 *
 * Parity pins for this file live in tests/test_oracle_symbolic.py (brute-force
 * boolean elimination, closed forms, hand examples, Appendix-A integers).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OS_OK 0
#define OS_ERR_ARG (-1)
#define OS_ERR_NOMEM (-3)

typedef struct {
    int64_t n;
    int32_t status;
    int32_t postorder_was_identity;
    /* final labels: perm[new] = old = input perm composed with the postorder */
    int32_t *perm;
    int32_t *parent;     /* elimination tree, -1 for roots */
    int64_t *cc;         /* column counts incl. diagonal */
    int64_t *Lp;         /* n+1 */
    int32_t *Li;         /* struct(L_j), ascending, first entry = j */
    int64_t nnzL;
    int64_t flops;       /* sum cc^2 */
    int32_t nfund;
    int32_t *fund_first; /* nfund+1 */
    int32_t nsuper;
    int32_t *sn_first;   /* nsuper+1 */
    int32_t *sn_parent;  /* relaxed supernodal parent, -1 for roots */
    int64_t *sn_rowptr;  /* nsuper+1 */
    int32_t *sn_rows;    /* R_s ascending; first k entries = cols(s) */
    int64_t stored_L;    /* sum k(k+1)/2 + k m */
    int64_t exec_flops;  /* sum over fronts of k m^2 + m k(k+1) + k(k+1)(2k+1)/6 */
} osym;

void oracle_sym_free(osym *h) {
    if (!h) return;
    free(h->perm); free(h->parent); free(h->cc); free(h->Lp); free(h->Li);
    free(h->fund_first); free(h->sn_first); free(h->sn_parent);
    free(h->sn_rowptr); free(h->sn_rows);
    free(h);
}

static int cmp_i32(const void *a, const void *b) {
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

/* Step 1: lower pattern of B = P A P^T as CSC (sorted, no duplicates, no diagonal). */
static int build_B(int64_t n, const int64_t *colptr, const int32_t *rowind, const int32_t *perm,
                   int64_t **Bp_out, int32_t **Bi_out) {
    int32_t *iperm = malloc(sizeof(int32_t) * (size_t)(n ? n : 1));
    int64_t *cnt = calloc((size_t)n + 1, sizeof(int64_t));
    if (!iperm || !cnt) { free(iperm); free(cnt); return OS_ERR_NOMEM; }
    for (int64_t k = 0; k < n; k++) iperm[perm[k]] = (int32_t)k;
    for (int64_t c = 0; c < n; c++)
        for (int64_t p = colptr[c]; p < colptr[c + 1]; p++) {
            int64_t r = rowind[p];
            if (r <= c) continue;                 /* upper entries ignored; diagonal implicit */
            int32_t i = iperm[r], j = iperm[c];
            int32_t lo = i < j ? i : j;
            cnt[lo + 1]++;
        }
    for (int64_t j = 0; j < n; j++) cnt[j + 1] += cnt[j];
    int32_t *Bi = malloc(sizeof(int32_t) * (size_t)(cnt[n] ? cnt[n] : 1));
    int64_t *fill = malloc(sizeof(int64_t) * (size_t)(n ? n : 1));
    if (!Bi || !fill) { free(iperm); free(cnt); free(Bi); free(fill); return OS_ERR_NOMEM; }
    for (int64_t j = 0; j < n; j++) fill[j] = cnt[j];
    for (int64_t c = 0; c < n; c++)
        for (int64_t p = colptr[c]; p < colptr[c + 1]; p++) {
            int64_t r = rowind[p];
            if (r <= c) continue;
            int32_t i = iperm[r], j = iperm[c];
            int32_t lo = i < j ? i : j, hi = i < j ? j : i;
            Bi[fill[lo]++] = hi;
        }
    /* sort + dedupe each column, compact */
    int64_t w = 0;
    for (int64_t j = 0; j < n; j++) {
        int64_t b = cnt[j], e = cnt[j + 1];
        qsort(Bi + b, (size_t)(e - b), sizeof(int32_t), cmp_i32);
        cnt[j] = w;
        for (int64_t p = b; p < e; p++)
            if (p == b || Bi[p] != Bi[p - 1]) Bi[w++] = Bi[p];
    }
    cnt[n] = w;
    free(iperm); free(fill);
    *Bp_out = cnt; *Bi_out = Bi;
    return OS_OK;
}

/* Step 2: column structures and the etree by their definition. */
static int column_structures(int64_t n, const int64_t *Bp, const int32_t *Bi,
                             int32_t *parent, int64_t **Lp_out, int32_t **Li_out) {
    int64_t cap = Bp[n] + 2 * n + 16, len = 0;
    int64_t *Lp = malloc(sizeof(int64_t) * (size_t)(n + 1));
    int32_t *Li = malloc(sizeof(int32_t) * (size_t)cap);
    int32_t *cur = malloc(sizeof(int32_t) * (size_t)(n + 1));
    int32_t *tmp = malloc(sizeof(int32_t) * (size_t)(n + 1));
    int32_t *head = malloc(sizeof(int32_t) * (size_t)(n ? n : 1));   /* first child */
    int32_t *tail = malloc(sizeof(int32_t) * (size_t)(n ? n : 1));   /* last child */
    int32_t *next = malloc(sizeof(int32_t) * (size_t)(n ? n : 1));   /* next sibling */
    if (!Lp || !Li || !cur || !tmp || !head || !tail || !next) goto nomem;
    for (int64_t j = 0; j < n; j++) head[j] = tail[j] = next[j] = -1;
    Lp[0] = 0;
    for (int64_t j = 0; j < n; j++) {
        /* {i > j : B(i,j) != 0}, already sorted */
        int64_t nc = 0;
        for (int64_t p = Bp[j]; p < Bp[j + 1]; p++) cur[nc++] = Bi[p];
        /* union with struct(L_c) \ {c} for every child c, in ascending c */
        for (int32_t c = head[j]; c >= 0; c = next[c]) {
            const int32_t *s = Li + Lp[c] + 1;
            int64_t ns = Lp[c + 1] - Lp[c] - 1, a = 0, b = 0, t = 0;
            while (b < ns && s[b] <= j) b++;   /* j itself (= parent(c)) is added below */
            while (a < nc || b < ns) {
                int32_t v;
                if (b >= ns || (a < nc && cur[a] < s[b])) v = cur[a++];
                else if (a >= nc || s[b] < cur[a]) v = s[b++];
                else { v = cur[a]; a++; b++; }
                tmp[t++] = v;
            }
            memcpy(cur, tmp, sizeof(int32_t) * (size_t)t);
            nc = t;
        }
        if (len + nc + 1 > cap) {
            int64_t ncap = cap + cap / 2 + nc + 1;
            int32_t *nl = realloc(Li, sizeof(int32_t) * (size_t)ncap);
            if (!nl) goto nomem;
            Li = nl; cap = ncap;
        }
        Li[len++] = (int32_t)j;
        memcpy(Li + len, cur, sizeof(int32_t) * (size_t)nc);
        len += nc;
        Lp[j + 1] = len;
        parent[j] = nc ? cur[0] : -1;
        if (nc) {
            int32_t pj = cur[0];
            if (tail[pj] < 0) head[pj] = (int32_t)j; else next[tail[pj]] = (int32_t)j;
            tail[pj] = (int32_t)j;
        }
    }
    free(cur); free(tmp); free(head); free(tail); free(next);
    *Lp_out = Lp; *Li_out = Li;
    return OS_OK;
nomem:
    free(Lp); free(Li); free(cur); free(tmp); free(head); free(tail); free(next);
    return OS_ERR_NOMEM;
}

/* Step 3: postorder by iterative DFS; roots and children in ascending index. */
static int postorder(int64_t n, const int32_t *parent, int32_t *post) {
    int32_t *head = malloc(sizeof(int32_t) * (size_t)(n ? n : 1));
    int32_t *next = malloc(sizeof(int32_t) * (size_t)(n ? n : 1));
    int32_t *stack = malloc(sizeof(int32_t) * (size_t)(n ? n : 1));
    if (!head || !next || !stack) { free(head); free(next); free(stack); return OS_ERR_NOMEM; }
    for (int64_t j = 0; j < n; j++) head[j] = -1;
    /* build child lists in ascending order: insert in descending j at the front */
    for (int64_t j = n - 1; j >= 0; j--)
        if (parent[j] >= 0) { next[j] = head[parent[j]]; head[parent[j]] = (int32_t)j; }
    int64_t k = 0;
    for (int64_t r = 0; r < n; r++) {
        if (parent[r] >= 0) continue;
        int64_t top = 0;
        stack[top++] = (int32_t)r;
        while (top) {
            int32_t v = stack[top - 1];
            int32_t c = head[v];
            if (c >= 0) {            /* descend into the first unvisited child */
                head[v] = next[c];
                stack[top++] = c;
            } else {
                post[k++] = v;
                top--;
            }
        }
    }
    free(head); free(next); free(stack);
    return k == n ? OS_OK : OS_ERR_ARG;
}

osym *oracle_symbolic(int64_t n, const int64_t *colptr, const int32_t *rowind, const int32_t *perm_in,
                      const int32_t *nrelax, const double *zrelax, int32_t amalgamate) {
    osym *h = calloc(1, sizeof(osym));
    if (!h) return NULL;
    h->n = n;
    /* --- validate (SURVEY.md Sec. 8(b) conventions) --- */
    if (n < 0 || !colptr || (n > 0 && colptr[0] != 0)) { h->status = OS_ERR_ARG; return h; }
    for (int64_t c = 0; c < n; c++) if (colptr[c + 1] < colptr[c]) { h->status = OS_ERR_ARG; return h; }
    for (int64_t p = 0; p < (n ? colptr[n] : 0); p++)
        if (rowind[p] < 0 || rowind[p] >= n) { h->status = OS_ERR_ARG; return h; }
    h->perm = malloc(sizeof(int32_t) * (size_t)(n ? n : 1));
    if (!h->perm) { h->status = OS_ERR_NOMEM; return h; }
    {
        char *seen = calloc((size_t)(n ? n : 1), 1);
        if (!seen) { h->status = OS_ERR_NOMEM; return h; }
        for (int64_t k = 0; k < n; k++) {
            int32_t v = perm_in ? perm_in[k] : (int32_t)k;
            if (v < 0 || v >= n || seen[v]) { free(seen); h->status = OS_ERR_ARG; return h; }
            seen[v] = 1; h->perm[k] = v;
        }
        free(seen);
    }
    h->parent = malloc(sizeof(int32_t) * (size_t)(n ? n : 1));
    int32_t *post = malloc(sizeof(int32_t) * (size_t)(n ? n : 1));
    if (!h->parent || !post) { free(post); h->status = OS_ERR_NOMEM; return h; }

    h->postorder_was_identity = 1;
    for (int pass = 0; pass < 2; pass++) {
        int64_t *Bp; int32_t *Bi;
        int st = build_B(n, colptr, rowind, h->perm, &Bp, &Bi);
        if (st) { free(post); h->status = st; return h; }
        st = column_structures(n, Bp, Bi, h->parent, &h->Lp, &h->Li);
        free(Bp); free(Bi);
        if (st) { free(post); h->status = st; return h; }
        st = postorder(n, h->parent, post);
        if (st) { free(post); h->status = st; return h; }
        int ident = 1;
        for (int64_t k = 0; k < n; k++) if (post[k] != k) { ident = 0; break; }
        if (ident) break;
        /* relabel: new perm[k] = perm[post[k]], then redo steps 1-2 */
        h->postorder_was_identity = 0;
        int32_t *np = malloc(sizeof(int32_t) * (size_t)n);
        if (!np) { free(post); h->status = OS_ERR_NOMEM; return h; }
        for (int64_t k = 0; k < n; k++) np[k] = h->perm[post[k]];
        free(h->perm); h->perm = np;
        free(h->Lp); free(h->Li); h->Lp = NULL; h->Li = NULL;
    }
    free(post);

    /* --- Step 4: counts --- */
    h->cc = malloc(sizeof(int64_t) * (size_t)(n ? n : 1));
    if (!h->cc) { h->status = OS_ERR_NOMEM; return h; }
    h->nnzL = 0; h->flops = 0;
    for (int64_t j = 0; j < n; j++) {
        h->cc[j] = h->Lp[j + 1] - h->Lp[j];
        h->nnzL += h->cc[j];
        h->flops += h->cc[j] * h->cc[j];
    }

    /* --- Step 5: fundamental supernodes --- */
    int32_t *nchild = calloc((size_t)(n ? n : 1), sizeof(int32_t));
    h->fund_first = malloc(sizeof(int32_t) * (size_t)(n + 1));
    if (!nchild || !h->fund_first) { free(nchild); h->status = OS_ERR_NOMEM; return h; }
    for (int64_t j = 0; j < n; j++) if (h->parent[j] >= 0) nchild[h->parent[j]]++;
    int32_t S = 0;
    for (int64_t j = 0; j < n; j++) {
        int same = j > 0 && h->parent[j - 1] == j && nchild[j] == 1 && h->cc[j - 1] == h->cc[j] + 1;
        if (!same) h->fund_first[S++] = (int32_t)j;
    }
    h->fund_first[S] = (int32_t)n;
    h->nfund = S;
    free(nchild);

    /* --- Step 6: relaxed amalgamation, SURVEY.md Appendix B "Amalgamation rule" --- */
    int32_t nr0 = nrelax ? nrelax[0] : 4, nr1 = nrelax ? nrelax[1] : 16, nr2 = nrelax ? nrelax[2] : 48;
    double z0 = zrelax ? zrelax[0] : 0.8, z1 = zrelax ? zrelax[1] : 0.1, z2 = zrelax ? zrelax[2] : 0.05;
    int32_t *col2fund = malloc(sizeof(int32_t) * (size_t)(n ? n : 1));
    int64_t *ks = malloc(sizeof(int64_t) * (size_t)(S ? S : 1));
    int64_t *ms = malloc(sizeof(int64_t) * (size_t)(S ? S : 1));
    int32_t *sp = malloc(sizeof(int32_t) * (size_t)(S ? S : 1));
    int64_t *K = malloc(sizeof(int64_t) * (size_t)(S ? S : 1));
    int64_t *F = malloc(sizeof(int64_t) * (size_t)(S ? S : 1));
    int64_t *Z = malloc(sizeof(int64_t) * (size_t)(S ? S : 1));
    char *merge_next = calloc((size_t)(S ? S : 1), 1);   /* fundamental s joined the group of s+1 */
    if (!col2fund || !ks || !ms || !sp || !K || !F || !Z || !merge_next) { h->status = OS_ERR_NOMEM; return h; }
    for (int32_t s = 0; s < S; s++) {
        for (int32_t j = h->fund_first[s]; j < h->fund_first[s + 1]; j++) col2fund[j] = s;
        ks[s] = h->fund_first[s + 1] - h->fund_first[s];
        ms[s] = h->cc[h->fund_first[s]] - ks[s];
    }
    for (int32_t s = 0; s < S; s++) {
        int32_t last = h->fund_first[s + 1] - 1;
        sp[s] = h->parent[last] >= 0 ? col2fund[h->parent[last]] : -1;
        K[s] = ks[s]; F[s] = ks[s] + ms[s]; Z[s] = 0;
    }
    for (int32_t j = S - 2; j >= 0 && amalgamate; j--) {
        if (sp[j] != j + 1) continue;
        int32_t g = j + 1;                          /* lowest member of the group of j+1 */
        int64_t ns = ks[j] + K[g];
        int64_t newz = ks[j] * (F[g] - ms[j]);
        int64_t num = Z[g] + newz;
        int64_t den = ns * (ns + 1) / 2 + ns * (F[g] - K[g]);
        double z = (double)num / (double)den;
        int merge = ns <= nr0 || newz == 0 || (ns <= nr1 && z < z0) || (ns <= nr2 && z < z1) || z < z2;
        if (merge) {
            merge_next[j] = 1;
            K[j] = ns; F[j] = F[g] + ks[j]; Z[j] = Z[g] + newz;
        }
    }
    /* relaxed supernodes = maximal runs of fundamental supernodes linked by merge_next */
    h->sn_first = malloc(sizeof(int32_t) * (size_t)(S + 1));
    int32_t *col2sn = malloc(sizeof(int32_t) * (size_t)(n ? n : 1));
    if (!h->sn_first || !col2sn) { h->status = OS_ERR_NOMEM; return h; }
    int32_t R = 0;
    for (int32_t s = 0; s < S; s++)
        if (s == 0 || !merge_next[s - 1]) h->sn_first[R++] = h->fund_first[s];
    h->sn_first[R] = (int32_t)n;
    h->nsuper = R;
    for (int32_t s = 0; s < R; s++)
        for (int32_t j = h->sn_first[s]; j < h->sn_first[s + 1]; j++) col2sn[j] = s;
    h->sn_parent = malloc(sizeof(int32_t) * (size_t)(R ? R : 1));
    h->sn_rowptr = malloc(sizeof(int64_t) * (size_t)(R + 1));
    if (!h->sn_parent || !h->sn_rowptr) { h->status = OS_ERR_NOMEM; return h; }
    for (int32_t s = 0; s < R; s++) {
        int32_t last = h->sn_first[s + 1] - 1;
        h->sn_parent[s] = h->parent[last] >= 0 ? col2sn[h->parent[last]] : -1;
    }
    /* R_s = union of struct(L_j) over the columns of s */
    int32_t *mark = malloc(sizeof(int32_t) * (size_t)(n ? n : 1));
    int64_t cap = 2 * n + 16, len = 0;
    h->sn_rows = malloc(sizeof(int32_t) * (size_t)cap);
    if (!mark || !h->sn_rows) { free(mark); h->status = OS_ERR_NOMEM; return h; }
    for (int64_t i = 0; i < n; i++) mark[i] = -1;
    h->sn_rowptr[0] = 0;
    h->stored_L = 0; h->exec_flops = 0;
    for (int32_t s = 0; s < R; s++) {
        for (int32_t j = h->sn_first[s]; j < h->sn_first[s + 1]; j++)
            for (int64_t p = h->Lp[j]; p < h->Lp[j + 1]; p++) {
                int32_t i = h->Li[p];
                if (mark[i] == s) continue;
                mark[i] = s;
                if (len + 1 > cap) {
                    int64_t ncap = cap * 2;
                    int32_t *nr = realloc(h->sn_rows, sizeof(int32_t) * (size_t)ncap);
                    if (!nr) { free(mark); h->status = OS_ERR_NOMEM; return h; }
                    h->sn_rows = nr; cap = ncap;
                }
                h->sn_rows[len++] = i;
            }
        qsort(h->sn_rows + h->sn_rowptr[s], (size_t)(len - h->sn_rowptr[s]), sizeof(int32_t), cmp_i32);
        h->sn_rowptr[s + 1] = len;
        int64_t k = h->sn_first[s + 1] - h->sn_first[s];
        int64_t m = (h->sn_rowptr[s + 1] - h->sn_rowptr[s]) - k;
        h->stored_L += k * (k + 1) / 2 + k * m;
        h->exec_flops += k * m * m + m * k * (k + 1) + k * (k + 1) * (2 * k + 1) / 6;
    }
    free(mark); free(col2sn); free(col2fund); free(ks); free(ms); free(sp);
    free(K); free(F); free(Z); free(merge_next);
    h->status = OS_OK;
    return h;
}
