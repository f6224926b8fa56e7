// symbolic.cpp -- host symbolic analysis for the multifrontal hot path (row a0 of
// SURVEY.md Sec. 8(a)).  Feeds the postorder traversal of the supernodal
// elimination tree described in PAPER.md L27 (Sec. II-A).
//
// Algorithms (chosen to differ from the oracle's plain definitions):
//   * B = P A P^T lower, built by two stable counting sorts (no comparison sort),
//     keeping the input-order list of value indices of every unique entry;
//   * elimination tree: Liu's algorithm with path compression over the rows of B;
//   * postorder: iterative DFS, children ascending (reading C5); if it is not the
//     identity the order is composed and the analysis redone;
//   * column counts: row-subtree traversal (each row k walks up from the columns
//     of its off-diagonal entries until it meets a node already marked k);
//   * fundamental supernodes (reading C2) and the Appendix-B relaxed amalgamation
//     rule (verbatim -- both sides must agree bit-exactly);
//   * row lists: supernodal merge R_s = cols(s) U rows(B(:, cols(s))) U
//     (U_{children t} R_t), with a marker array;
//   * perm == NULL: the library's own host-side ordering, METIS nested dissection
//     (METIS_NodeND of the static METIS that ships with the CUDA toolkit, the one
//     behind cusolverSpXcsrmetisndHost) on the graph of A + A^T without the
//     diagonal (reading C4; the paper used WSMP's own
//     ordering).
#include <algorithm>
#include <cstring>

#include "mf.h"
#include "mf_plan.h"

// METIS 5 (libmetis_static.a of the CUDA toolkit, built with 64-bit idx_t);
// declared here because the toolkit ships the library without metis.h.
extern "C" {
int METIS_SetDefaultOptions(int64_t *options);
int METIS_NodeND(int64_t *nvtxs, int64_t *xadj, int64_t *adjncy, int64_t *vwgt, int64_t *options, int64_t *perm,
                 int64_t *iperm);
}

namespace mf {

namespace {

constexpr int kMetisOk = 1, kMetisNoptions = 40;

// Fill-reducing nested-dissection order (new -> old) of the pattern's graph.
int order_metis(int64_t n, const int64_t *colptr, const int32_t *rowind, std::vector<int32_t> &perm) {
    perm.resize(n);
    if (n == 0) return MF_OK;
    // symmetric adjacency without the diagonal: count, fill, then sort + dedup per vertex
    std::vector<int64_t> deg(n + 1, 0);
    for (int64_t c = 0; c < n; c++)
        for (int64_t p = colptr[c]; p < colptr[c + 1]; p++)
            if (rowind[p] != c) {
                deg[rowind[p] + 1]++;
                deg[c + 1]++;
            }
    for (int64_t v = 0; v < n; v++) deg[v + 1] += deg[v];
    std::vector<int64_t> adj(deg[n]), fill(deg.begin(), deg.end() - 1);
    for (int64_t c = 0; c < n; c++)
        for (int64_t p = colptr[c]; p < colptr[c + 1]; p++)
            if (rowind[p] != c) {
                adj[fill[rowind[p]]++] = c;
                adj[fill[c]++] = rowind[p];
            }
    std::vector<int64_t> xadj(n + 1, 0);
    int64_t e = 0;
    for (int64_t v = 0; v < n; v++) {
        int64_t *b = adj.data() + deg[v], *t = adj.data() + deg[v + 1];
        std::sort(b, t);
        t = std::unique(b, t);
        xadj[v] = e;
        for (int64_t *q = b; q < t; q++) adj[e++] = *q;
    }
    xadj[n] = e;
    if (e == 0) {   // no edges (diagonal matrix): any order is fill-free
        for (int64_t v = 0; v < n; v++) perm[v] = (int32_t)v;
        return MF_OK;
    }
    int64_t opts[kMetisNoptions];
    METIS_SetDefaultOptions(opts);
    int64_t nv = n;
    std::vector<int64_t> p(n), ip(n);
    if (METIS_NodeND(&nv, xadj.data(), adj.data(), nullptr, opts, p.data(), ip.data()) != kMetisOk)
        return MF_ERR_NOMEM;
    for (int64_t k = 0; k < n; k++) perm[k] = (int32_t)p[k];   // row k of P A P^T is row p[k] of A
    return MF_OK;
}

// B = P A P^T restricted to lower entries, duplicates grouped (input order kept).
int build_B(int64_t n, const int64_t *colptr, const int32_t *rowind, const std::vector<int32_t> &perm,
            Symbolic &S) {
    std::vector<int32_t> iperm(n);
    for (int64_t k = 0; k < n; k++) iperm[perm[k]] = (int32_t)k;
    // collect (lo, hi, src) for every read entry
    int64_t nread = 0;
    for (int64_t c = 0; c < n; c++)
        for (int64_t p = colptr[c]; p < colptr[c + 1]; p++)
            if (rowind[p] >= c) nread++;
    S.nnzA_read = nread;
    S.nnz_in = colptr[n];
    std::vector<int32_t> lo(nread), hi(nread);
    std::vector<int64_t> src(nread);
    int64_t w = 0;
    for (int64_t c = 0; c < n; c++)
        for (int64_t p = colptr[c]; p < colptr[c + 1]; p++) {
            int64_t r = rowind[p];
            if (r < c) continue;
            int32_t i = iperm[r], j = iperm[c];
            lo[w] = std::min(i, j);
            hi[w] = std::max(i, j);
            src[w] = p;
            w++;
        }
    // pass 1: stable counting sort by hi
    std::vector<int64_t> cnt(n + 1, 0);
    for (int64_t e = 0; e < nread; e++) cnt[hi[e] + 1]++;
    for (int64_t i = 0; i < n; i++) cnt[i + 1] += cnt[i];
    std::vector<int64_t> ord1(nread);
    for (int64_t e = 0; e < nread; e++) ord1[cnt[hi[e]]++] = e;
    // pass 2: stable counting sort by lo  => sorted by (lo, hi, input position)
    std::fill(cnt.begin(), cnt.end(), 0);
    for (int64_t e = 0; e < nread; e++) cnt[lo[e] + 1]++;
    for (int64_t i = 0; i < n; i++) cnt[i + 1] += cnt[i];
    std::vector<int64_t> ord(nread);
    for (int64_t q = 0; q < nread; q++) {
        int64_t e = ord1[q];
        ord[cnt[lo[e]]++] = e;
    }
    // unique entries
    S.bcolptr.assign(n + 1, 0);
    S.brow.clear();
    S.bvptr.clear();
    S.bvidx.resize(nread);
    S.brow.reserve(nread);
    S.bvptr.reserve(nread + 1);
    int32_t plo = -1, phi = -1;
    for (int64_t q = 0; q < nread; q++) {
        int64_t e = ord[q];
        if (lo[e] != plo || hi[e] != phi) {
            S.brow.push_back(hi[e]);
            S.bvptr.push_back(q);
            S.bcolptr[lo[e] + 1]++;
            plo = lo[e];
            phi = hi[e];
        }
        S.bvidx[q] = src[e];
    }
    S.bvptr.push_back(nread);
    for (int64_t i = 0; i < n; i++) S.bcolptr[i + 1] += S.bcolptr[i];
    return MF_OK;
}

// Liu's elimination-tree algorithm with path compression.
void etree_liu(int64_t n, const Symbolic &S, std::vector<int32_t> &parent,
               std::vector<int64_t> &rowptr, std::vector<int32_t> &rowcols) {
    // rows of the strictly lower part of B: row hi lists columns lo < hi
    rowptr.assign(n + 1, 0);
    for (int64_t j = 0; j < n; j++)
        for (int64_t e = S.bcolptr[j]; e < S.bcolptr[j + 1]; e++)
            if (S.brow[e] != j) rowptr[S.brow[e] + 1]++;
    for (int64_t i = 0; i < n; i++) rowptr[i + 1] += rowptr[i];
    rowcols.resize(rowptr[n]);
    std::vector<int64_t> fill(rowptr.begin(), rowptr.end() - 1);
    for (int64_t j = 0; j < n; j++)
        for (int64_t e = S.bcolptr[j]; e < S.bcolptr[j + 1]; e++)
            if (S.brow[e] != j) rowcols[fill[S.brow[e]]++] = (int32_t)j;
    parent.assign(n, -1);
    std::vector<int32_t> anc(n, -1);
    for (int64_t k = 0; k < n; k++) {
        for (int64_t p = rowptr[k]; p < rowptr[k + 1]; p++) {
            int32_t r = rowcols[p];
            while (anc[r] != -1 && anc[r] != k) {
                int32_t t = anc[r];
                anc[r] = (int32_t)k;
                r = t;
            }
            if (anc[r] == -1) {
                anc[r] = (int32_t)k;
                parent[r] = (int32_t)k;
            }
        }
    }
}

void tree_postorder(int64_t n, const std::vector<int32_t> &parent, std::vector<int32_t> &post) {
    std::vector<int32_t> head(n, -1), next(n, -1), stack;
    for (int64_t j = n - 1; j >= 0; j--)
        if (parent[j] >= 0) {
            next[j] = head[parent[j]];
            head[parent[j]] = (int32_t)j;
        }
    post.clear();
    post.reserve(n);
    stack.reserve(64);
    for (int64_t r = 0; r < n; r++) {
        if (parent[r] >= 0) continue;
        stack.push_back((int32_t)r);
        while (!stack.empty()) {
            int32_t v = stack.back();
            int32_t c = head[v];
            if (c >= 0) {
                head[v] = next[c];
                stack.push_back(c);
            } else {
                post.push_back(v);
                stack.pop_back();
            }
        }
    }
}

}  // namespace

int analyze_symbolic(int64_t n, const int64_t *colptr, const int32_t *rowind, const int32_t *perm_in,
                     const Options &opt, Symbolic &S) {
    // ---------------- validation
    if (n < 0 || n >= (int64_t)INT32_MAX || !colptr) return MF_ERR_ARG;
    if (n > 0 && !rowind && colptr[n] > 0) return MF_ERR_ARG;
    if (colptr[0] != 0) return MF_ERR_ARG;
    for (int64_t c = 0; c < n; c++)
        if (colptr[c + 1] < colptr[c]) return MF_ERR_ARG;
    for (int64_t p = 0; p < colptr[n]; p++)
        if (rowind[p] < 0 || rowind[p] >= n) return MF_ERR_ARG;
    std::vector<int32_t> lib_perm;
    if (!perm_in) {   // the library's own ordering
        if (int st = order_metis(n, colptr, rowind, lib_perm)) return st;
        perm_in = lib_perm.data();
    }
    {
        std::vector<char> seen(n, 0);
        for (int64_t k = 0; k < n; k++) {
            int32_t v = perm_in[k];
            if (v < 0 || v >= n || seen[v]) return MF_ERR_ARG;
            seen[v] = 1;
        }
    }
    S = Symbolic();
    S.n = n;
    S.perm.assign(perm_in, perm_in + n);
    std::vector<int64_t> rowptr;
    std::vector<int32_t> rowcols;
    for (int pass = 0;; pass++) {
        int st = build_B(n, colptr, rowind, S.perm, S);
        if (st) return st;
        etree_liu(n, S, S.parent, rowptr, rowcols);
        std::vector<int32_t> post;
        tree_postorder(n, S.parent, post);
        bool ident = true;
        for (int64_t k = 0; k < n; k++)
            if (post[k] != k) {
                ident = false;
                break;
            }
        if (ident) break;
        if (pass >= 1) return MF_ERR_ARG;  // a postorder of a postordered tree is the identity
        std::vector<int32_t> np(n);
        for (int64_t k = 0; k < n; k++) np[k] = S.perm[post[k]];
        S.perm.swap(np);
    }
    // ---------------- column counts by row-subtree traversal
    S.cc.assign(n, 1);
    {
        std::vector<int32_t> mark(n, -1);
        for (int64_t k = 0; k < n; k++) {
            mark[k] = (int32_t)k;
            for (int64_t p = rowptr[k]; p < rowptr[k + 1]; p++) {
                int32_t r = rowcols[p];
                while (mark[r] != k) {
                    S.cc[r]++;
                    mark[r] = (int32_t)k;
                    r = S.parent[r];
                }
            }
        }
    }
    S.nnzL = 0;
    S.flops = 0;
    for (int64_t j = 0; j < n; j++) {
        S.nnzL += S.cc[j];
        S.flops += S.cc[j] * S.cc[j];
    }
    // ---------------- fundamental supernodes
    std::vector<int32_t> nkids(n, 0);
    for (int64_t j = 0; j < n; j++)
        if (S.parent[j] >= 0) nkids[S.parent[j]]++;
    S.fund_first.clear();
    for (int64_t j = 0; j < n; j++) {
        bool cont = j > 0 && S.parent[j - 1] == j && nkids[j] == 1 && S.cc[j - 1] == S.cc[j] + 1;
        if (!cont) S.fund_first.push_back((int32_t)j);
    }
    const int32_t nf = (int32_t)S.fund_first.size();
    S.fund_first.push_back((int32_t)n);
    // ---------------- relaxed amalgamation, SURVEY.md Appendix B
    std::vector<int32_t> fund_of(n);
    for (int32_t s = 0; s < nf; s++)
        for (int32_t j = S.fund_first[s]; j < S.fund_first[s + 1]; j++) fund_of[j] = s;
    struct Grp {
        int64_t K, F, Z;
    };
    std::vector<Grp> g(nf);
    std::vector<int64_t> kf(nf), mfund(nf);
    std::vector<int32_t> spar(nf);
    for (int32_t s = 0; s < nf; s++) {
        kf[s] = S.fund_first[s + 1] - S.fund_first[s];
        mfund[s] = S.cc[S.fund_first[s]] - kf[s];
        int32_t pl = S.parent[S.fund_first[s + 1] - 1];
        spar[s] = pl < 0 ? -1 : fund_of[pl];
        g[s] = {kf[s], kf[s] + mfund[s], 0};
    }
    std::vector<char> joins_next(nf, 0);
    if (opt.amalgamate) {
        for (int32_t j = nf - 2; j >= 0; j--) {
            if (spar[j] != j + 1) continue;
            const Grp &G = g[j + 1];
            int64_t ns = kf[j] + G.K;
            int64_t newz = kf[j] * (G.F - mfund[j]);
            int64_t den = ns * (ns + 1) / 2 + ns * (G.F - G.K);
            double z = (double)(G.Z + newz) / (double)den;
            bool merge = ns <= opt.nrelax[0] || newz == 0 || (ns <= opt.nrelax[1] && z < opt.zrelax[0]) ||
                         (ns <= opt.nrelax[2] && z < opt.zrelax[1]) || z < opt.zrelax[2];
            if (merge) {
                joins_next[j] = 1;
                g[j] = {ns, G.F + kf[j], G.Z + newz};
            }
        }
    }
    S.sn_first.clear();
    for (int32_t s = 0; s < nf; s++)
        if (s == 0 || !joins_next[s - 1]) S.sn_first.push_back(S.fund_first[s]);
    const int32_t ns_ = (int32_t)S.sn_first.size();
    S.sn_first.push_back((int32_t)n);
    std::vector<int32_t> sn_of(n);
    for (int32_t s = 0; s < ns_; s++)
        for (int32_t j = S.sn_first[s]; j < S.sn_first[s + 1]; j++) sn_of[j] = s;
    S.sn_parent.resize(ns_);
    for (int32_t s = 0; s < ns_; s++) {
        int32_t pl = S.parent[S.sn_first[s + 1] - 1];
        S.sn_parent[s] = pl < 0 ? -1 : sn_of[pl];
    }
    // ---------------- supernodal row lists
    std::vector<int32_t> chead(ns_, -1), cnext(ns_, -1), ctail(ns_, -1);
    for (int32_t s = 0; s < ns_; s++) {
        int32_t p = S.sn_parent[s];
        if (p < 0) continue;
        if (ctail[p] < 0) chead[p] = s; else cnext[ctail[p]] = s;
        ctail[p] = s;
    }
    S.sn_rowptr.assign(ns_ + 1, 0);
    S.sn_rows.clear();
    S.sn_rows.reserve(3 * n);
    std::vector<int32_t> mark(n, -1);
    S.stored_L = 0;
    S.exec_flops = 0;
    for (int32_t s = 0; s < ns_; s++) {
        const int32_t f0 = S.sn_first[s], f1 = S.sn_first[s + 1];
        const size_t base = S.sn_rows.size();
        for (int32_t j = f0; j < f1; j++) S.sn_rows.push_back(j);
        for (int32_t j = f0; j < f1; j++)
            for (int64_t e = S.bcolptr[j]; e < S.bcolptr[j + 1]; e++) {
                int32_t r = S.brow[e];
                if (r >= f1 && mark[r] != s) {
                    mark[r] = s;
                    S.sn_rows.push_back(r);
                }
            }
        for (int32_t t = chead[s]; t >= 0; t = cnext[t])
            for (int64_t q = S.sn_rowptr[t]; q < S.sn_rowptr[t + 1]; q++) {
                int32_t r = S.sn_rows[q];
                if (r >= f1 && mark[r] != s) {
                    mark[r] = s;
                    S.sn_rows.push_back(r);
                }
            }
        std::sort(S.sn_rows.begin() + base + (f1 - f0), S.sn_rows.end());
        S.sn_rowptr[s + 1] = (int64_t)S.sn_rows.size();
        int64_t k = f1 - f0, m = (int64_t)(S.sn_rows.size() - base) - k;
        S.stored_L += k * (k + 1) / 2 + k * m;
        S.exec_flops += k * m * m + m * k * (k + 1) + k * (k + 1) * (2 * k + 1) / 6;
    }
    return MF_OK;
}

}  // namespace mf
