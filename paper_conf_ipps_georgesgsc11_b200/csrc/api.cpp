// api.cpp -- the C ABI (include/mf.h): state machine, device arena, and the
// level-by-level driver of the factor-update hot path.
//
// mf_factor is the postorder traversal of PAPER.md L27 (Sec. II-A) realised as
// a bottom-up level schedule (children always in a lower level than their
// parent): per level, the small fronts run in one batched fused launch per size
// class, the large fronts in the blocked path (assembly; per diagonal block:
// potrf, trsm, DMMA trailing update; then the DMMA syrk on U^n).  Everything
// stays resident in HBM; the only host<->device traffic is the optional upload
// of `values` and the 4-byte NOT_SPD flag.
#include <algorithm>
#include <chrono>
#include <climits>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <new>
#include <map>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "kernels.cuh"
#include "mf.h"
#include "mf_plan.h"

using namespace mf;

// One extra solve pipeline (mf_solve_nrhs, single GPU): its own vectors, dataflow
// flags / partial sums, solve epoch and ticket counters, a stream and a captured graph,
// so several right-hand sides run concurrently -- the block chains of the large
// supernodes are latency-bound, so overlapping them raises the throughput.
struct SolveSlot {
    mf::DevPlan d{};
    double *y = nullptr, *bx = nullptr;
    unsigned *tickets = nullptr;
    cudaStream_t st = nullptr;
    cudaEvent_t done = nullptr;
    cudaGraph_t graph = nullptr;
    cudaGraphExec_t exec = nullptr;
};
constexpr int kSolveSlots = 8;   // measured nrhs = 8: c5 2 / 4 / 8 slots 69.9 / 62.8 / 61.6 ms, c3 16.2 / 12.4 / 10.7 ms

struct mf_ctx {
    Options opt;
    std::vector<SolveSlot> slots;
    int device = 0;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    int state = 0;   // 0 created, 1 analyzed, 2 factored (ok), 3 factor failed
    bool host_only = false;
    Symbolic S;
    Plan P;
    mf_info info{};
    std::vector<void *> allocs;
    DevPlan d{};
    // device copies of schedule arrays
    int32_t *d_small = nullptr, *d_large = nullptr, *d_asm = nullptr, *d_trsm = nullptr, *d_levels = nullptr;
    int32_t *d_panel = nullptr;
    int32_t *d_sn_rows = nullptr;
    int64_t *d_sn_rowptr = nullptr;
    GemmProb *d_probs = nullptr;
    TileTask *d_tiles = nullptr;
    double *d_values = nullptr;
    double *d_y = nullptr, *d_bx = nullptr;
    int *d_failed = nullptr;
    int32_t *d_solve_list = nullptr, *d_df_tasks = nullptr;
    unsigned *d_tickets = nullptr;   // ticket-counter pair per dataflow launch slot (kernels.cu take_ticket)
    int32_t *d_dinv_tasks = nullptr; // solve setup: (supernode, 64-block) pairs whose inverse the solves use
    bool dinv_stale = true;          // set by mf_factor; the next solve recomputes the block inverses
    cudaEvent_t ev0 = nullptr, ev1 = nullptr, ev_in = nullptr;
    int64_t launches = 0;
    int profiling = 0;               // 1: eager per-launch events; 2: timeline (events captured in the graph)
    cudaGraph_t graph_tl = nullptr;  // the timeline-mode graph of the local program (events after every launch)
    cudaGraphExec_t graph_tl_exec = nullptr;
    cudaEvent_t tl_base = nullptr;   // timeline zero: recorded after the init launch
    bool use_graph = true;
    cudaGraph_t graph = nullptr, graph_top = nullptr, solve_graph = nullptr;
    cudaGraphExec_t graph_exec = nullptr, graph_top_exec = nullptr, solve_exec = nullptr;
    mf_exchange_fn xfn = nullptr;
    void *xuser = nullptr;
    double *d_ytmp = nullptr;
    int32_t *d_top_list = nullptr, *d_own_list = nullptr;
    std::vector<cudaEvent_t> prof_events;
    // single GPU: one stream per subtree branch, forked from / joined into `stream`
    std::vector<cudaStream_t> bstreams;
    std::vector<cudaEvent_t> bevents;   // [0] fork, [1 + b] join of branch b
    // look-ahead: the main path of the top fronts on a high-priority stream, the
    // split-off trailing updates on a low-priority side stream
    cudaStream_t la_hi = nullptr, la_side = nullptr;
    cudaEvent_t la_ev[4] = {nullptr, nullptr, nullptr, nullptr};   // hi fork, side fork, side join, hi join
    mf_kernel_stat kstats[KC_COUNT];
    int64_t prof_factors = 0;
    // device-memory hooks (mf_options.dev_alloc / dev_free; NULL = cudaMalloc / cudaFree)
    // Ozaki-scheme Schur updates (ozaki_slices > 0): problem / tile / split lists, scratch
    OzProb *d_oz_probs = nullptr;
    OzTile *d_oz_tiles = nullptr;
    int32_t *d_oz_split = nullptr;
    int8_t *d_oz_scratch = nullptr;
    int32_t *d_oz_expo = nullptr;
    // fp64 iterative refinement (refine_iters > 0): symmetric CSR of B, B values, vectors
    int64_t *d_rs_ptr = nullptr;
    int32_t *d_rs_col = nullptr, *d_rs_ent = nullptr;
    double *d_bval = nullptr, *d_rb = nullptr, *d_rx = nullptr, *d_norms = nullptr;
    void *(*halloc)(size_t, void *) = nullptr;
    void (*hfree)(void *, void *) = nullptr;
    void *huser = nullptr;
};

namespace {

// NVTX ranges around the host-side phases of every call (header-only NVTX v3: a
// no-op unless a tool such as nsys / ncu injects itself), for timelines.
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

int cuda_err(cudaError_t e) {
    if (e == cudaSuccess) return MF_OK;
    fprintf(stderr, "[libmf] CUDA error: %s\n", cudaGetErrorString(e));
    return e == cudaErrorMemoryAllocation ? MF_ERR_NOMEM : MF_ERR_CUDA;
}

#define CK(x)                            \
    do {                                 \
        int _r = cuda_err(x);            \
        if (_r != MF_OK) return _r;      \
    } while (0)

// Every device buffer of the ctx comes from here: the caller's hooks or cudaMalloc.
int dev_alloc(mf_ctx *c, void **dst, size_t bytes) {
    void *p = nullptr;
    bytes = std::max<size_t>(bytes, 16);
    if (c->halloc) {
        p = c->halloc(bytes, c->huser);
        if (!p) return MF_ERR_NOMEM;
    } else {
        CK(cudaMalloc(&p, bytes));
    }
    c->allocs.push_back(p);
    *dst = p;
    return MF_OK;
}

template <class T>
int dev_upload(mf_ctx *c, T **dst, const std::vector<T> &src) {
    void *p = nullptr;
    if (int r = dev_alloc(c, &p, std::max<size_t>(src.size(), 1) * sizeof(T))) return r;
    if (!src.empty()) CK(cudaMemcpy(p, src.data(), src.size() * sizeof(T), cudaMemcpyHostToDevice));
    *dst = (T *)p;
    return MF_OK;
}

void drop_graph(mf_ctx *c) {
    if (c->graph_exec) cudaGraphExecDestroy(c->graph_exec);
    if (c->graph) cudaGraphDestroy(c->graph);
    if (c->graph_tl_exec) cudaGraphExecDestroy(c->graph_tl_exec);
    if (c->graph_tl) cudaGraphDestroy(c->graph_tl);
    if (c->tl_base) cudaEventDestroy(c->tl_base);
    if (c->graph_top_exec) cudaGraphExecDestroy(c->graph_top_exec);
    if (c->graph_top) cudaGraphDestroy(c->graph_top);
    c->graph_exec = nullptr;
    c->graph = nullptr;
    c->graph_top_exec = nullptr;
    c->graph_top = nullptr;
    if (c->solve_exec) cudaGraphExecDestroy(c->solve_exec);
    if (c->solve_graph) cudaGraphDestroy(c->solve_graph);
    c->solve_exec = nullptr;
    c->solve_graph = nullptr;
    for (SolveSlot &q : c->slots) {
        if (q.exec) cudaGraphExecDestroy(q.exec);
        if (q.graph) cudaGraphDestroy(q.graph);
        q.exec = nullptr;
        q.graph = nullptr;
    }
}

void free_device(mf_ctx *c) {
    drop_graph(c);
    for (SolveSlot &q : c->slots) {   // buffers are in c->allocs
        if (q.st) cudaStreamDestroy(q.st);
        if (q.done) cudaEventDestroy(q.done);
    }
    c->slots.clear();
    for (void *p : c->allocs) {
        if (c->hfree) c->hfree(p, c->huser);
        else cudaFree(p);
    }
    c->allocs.clear();
    c->d = DevPlan{};
}

// Device inputs (values, b) were produced on some caller stream.  A ctx that
// created its own non-blocking stream orders its first read after all work
// already queued on the legacy default stream (where torch's default stream and
// plain cudaMemcpy land); a caller that passed mf_options.stream orders its own
// producers on that stream (include/mf.h, "Pointers").
int order_after_caller(mf_ctx *c) {
    if (!c->own_stream) return MF_OK;
    CK(cudaEventRecord(c->ev_in, cudaStreamLegacy));
    CK(cudaStreamWaitEvent(c->stream, c->ev_in, 0));
    return MF_OK;
}

bool is_device_ptr(const void *p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}


void fill_info(mf_ctx *c, int64_t n, int with_device) {
    const Symbolic &S = c->S;
    const Plan &P = c->P;
    mf_info &I = c->info;
    I = mf_info{};
    I.n = n;
    I.nnzA = S.nnzA_read;
    I.nnzL = S.nnzL;
    I.nnzL_stored = S.stored_L;
    I.panel_words = P.L_words - 2;
    I.flops_true = S.flops;
    I.flops_exec = S.exec_flops;
    I.nfund = (int32_t)S.fund_first.size() - 1;
    I.nsuper = P.nsuper;
    I.nlevels = P.nlevels;
    I.max_front = P.max_front;
    I.nbranch = P.nbranch;
    I.rows_total = P.rows_total;
    I.failed_col = -1;
    I.ozaki_slices = P.oz_slices;
    I.refine_steps = 0;
    I.solve_berr = -1.0;
    I.launches_ozaki = 0;
    for (const Launch &L : P.program) I.launches_ozaki += L.oz;
    for (const Launch &L : P.program_top) I.launches_ozaki += L.oz;
    int64_t ws = 0;
    ws += (P.L_words + P.U_words + P.fv_words + 2 * std::max<int64_t>(n, 1) + S.nnz_in) * 8;
    ws += (int64_t)P.tiles.size() * sizeof(TileTask) + (int64_t)P.probs.size() * sizeof(GemmProb);
    ws += (int64_t)(S.bvidx.size() * 16 + S.brow.size() * 16 + P.relmap.size() * 4);
    ws += P.oz_scratch_bytes + P.oz_expo_words * 4 + (int64_t)P.oz_tiles.size() * sizeof(OzTile);
    I.workspace_bytes = with_device ? ws : 0;
}

}  // namespace

extern "C" {

const char *mf_strerror(int code) {
    switch (code) {
        case MF_OK: return "ok";
        case MF_NOT_SPD: return "matrix is not symmetric positive definite";
        case MF_ERR_ARG: return "invalid argument";
        case MF_ERR_STATE: return "call out of order";
        case MF_ERR_NOMEM: return "out of memory";
        case MF_ERR_CUDA: return "CUDA error";
        case MF_ERR_NCCL: return "NCCL error";
        default: return "unknown error";
    }
}

int mf_default_options(mf_options *o) {
    if (!o) return MF_ERR_ARG;
    Options d;
    o->amalgamate = d.amalgamate;
    for (int i = 0; i < 3; i++) {
        o->nrelax[i] = d.nrelax[i];
        o->zrelax[i] = d.zrelax[i];
    }
    o->small_front_max = d.small_front_max;
    o->panel_w = d.panel_w;
    o->device = -1;
    o->host_only = 0;
    o->nranks = 1;
    o->rank = 0;
    o->stream = nullptr;
    o->split_all = 0;
    o->nbranch = d.nbranch;
    o->fuse_ea = d.fuse_ea;
    o->lookahead = d.lookahead;
    o->dev_alloc = nullptr;
    o->dev_free = nullptr;
    o->alloc_user = nullptr;
    o->ozaki_slices = 0;
    o->refine_iters = -1;
    return MF_OK;
}

int mf_create(mf_ctx **out, const mf_options *o) {
    if (!out) return MF_ERR_ARG;
    *out = nullptr;
    mf_options def;
    mf_default_options(&def);
    if (!o) o = &def;
    if (o->panel_w < 16 || o->panel_w > 64 || (o->panel_w % 16)) return MF_ERR_ARG;
    if (o->small_front_max < 8 || !small_front_smem_ok(o->small_front_max)) return MF_ERR_ARG;
    mf_ctx *c = new (std::nothrow) mf_ctx();
    if (!c) return MF_ERR_NOMEM;
    c->opt.amalgamate = o->amalgamate;
    for (int i = 0; i < 3; i++) {
        c->opt.nrelax[i] = o->nrelax[i];
        c->opt.zrelax[i] = o->zrelax[i];
    }
    c->opt.small_front_max = o->small_front_max;
    c->opt.panel_w = o->panel_w;
    if (o->nranks < 1 || o->rank < 0 || o->rank >= o->nranks) {
        delete c;
        return MF_ERR_ARG;
    }
    c->opt.nranks = o->nranks;
    c->opt.split_all = o->split_all;
    if (o->nbranch < 1 || o->nbranch > 64) {
        delete c;
        return MF_ERR_ARG;
    }
    c->opt.nbranch = o->nbranch;
    c->opt.fuse_ea = o->fuse_ea != 0;
    c->opt.lookahead = o->lookahead != 0;
    if (o->ozaki_slices != 0 && (o->ozaki_slices < 3 || o->ozaki_slices > 8)) {
        delete c;
        return MF_ERR_ARG;
    }
    c->opt.ozaki_slices = o->ozaki_slices;
    c->opt.refine_iters = o->refine_iters < 0 ? ((o->ozaki_slices == 0 || o->ozaki_slices == 8) ? 0 : 10)
                                              : o->refine_iters;
    if (c->opt.ozaki_slices) c->opt.lookahead = 0;   // the Ozaki scratch is per stream: no side stream
    c->opt.rank = o->rank;
    c->host_only = o->host_only != 0;
    if ((o->dev_alloc == nullptr) != (o->dev_free == nullptr)) {
        delete c;
        return MF_ERR_ARG;
    }
    c->halloc = o->dev_alloc;
    c->hfree = o->dev_free;
    c->huser = o->alloc_user;
    c->info.failed_col = -1;
    if (c->host_only) {   // symbolic analysis + plan only; never touches CUDA
        *out = c;
        return MF_OK;
    }
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        delete c;
        fprintf(stderr, "[libmf] no CUDA device: the product path has no CPU fallback\n");
        return MF_ERR_CUDA;
    }
    if (o->device >= 0) {
        if (cudaSetDevice(o->device) != cudaSuccess) {
            delete c;
            return MF_ERR_CUDA;
        }
    }
    cudaGetDevice(&c->device);
    if (o->stream) {
        c->stream = (cudaStream_t)o->stream;
    } else {
        if (cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking) != cudaSuccess) {
            delete c;
            return MF_ERR_CUDA;
        }
        c->own_stream = true;
    }
    cudaEventCreate(&c->ev0);
    cudaEventCreate(&c->ev1);
    cudaEventCreateWithFlags(&c->ev_in, cudaEventDisableTiming);
    c->info.failed_col = -1;
    *out = c;
    return MF_OK;
}

void mf_destroy(mf_ctx *c) {
    if (!c) return;
    if (c->host_only) {
        delete c;
        return;
    }
    cudaSetDevice(c->device);
    if (c->stream) cudaStreamSynchronize(c->stream);
    free_device(c);
    for (cudaEvent_t e : c->prof_events) cudaEventDestroy(e);
    for (cudaEvent_t e : c->bevents) cudaEventDestroy(e);
    for (cudaEvent_t e : c->la_ev)
        if (e) cudaEventDestroy(e);
    if (c->la_hi) cudaStreamDestroy(c->la_hi);
    if (c->la_side) cudaStreamDestroy(c->la_side);
    for (cudaStream_t bs : c->bstreams) cudaStreamDestroy(bs);
    if (c->ev0) cudaEventDestroy(c->ev0);
    if (c->ev1) cudaEventDestroy(c->ev1);
    if (c->ev_in) cudaEventDestroy(c->ev_in);
    if (c->own_stream) cudaStreamDestroy(c->stream);
    delete c;
}

int mf_analyze(mf_ctx *c, int64_t n, const int64_t *colptr, const int32_t *rowind, const int32_t *perm) {
    if (!c) return MF_ERR_ARG;
    NvtxRange nvtx_("mf_analyze");
    auto t0 = std::chrono::steady_clock::now();
    if (!c->host_only) {
        CK(cudaSetDevice(c->device));
        cudaStreamSynchronize(c->stream);
        free_device(c);
        if (kernels_init()) return MF_ERR_CUDA;
    }
    c->state = 0;
    int st;
    {
        NvtxRange r("mf_analyze: symbolic");
        st = analyze_symbolic(n, colptr, rowind, perm, c->opt, c->S);
    }
    if (st) return st;
    {
        NvtxRange r("mf_analyze: plan");
        st = build_plan(c->S, c->opt, c->P);
    }
    if (st) return st;
    if (c->host_only) {
        fill_info(c, n, 0);
        c->info.t_analyze = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
        c->state = 1;
        return MF_OK;
    }
    const Symbolic &S = c->S;
    const Plan &P = c->P;
    DevPlan &d = c->d;
    int r;
    void *p0 = nullptr;
#define UP(dst, vec)                                   \
    if ((r = dev_upload(c, dst, vec)) != MF_OK) return r;
    int32_t *sn_first, *sn_k, *sn_f, *sn_ld, *child_ptr, *child_list, *relmap, *blrow, *perm_d;
    int64_t *L_off, *U_off, *fv_off, *relmap_ptr, *bcolptr, *bvptr, *bvidx;
    UP(&sn_first, S.sn_first);
    UP(&sn_k, P.sn_k);
    UP(&sn_f, P.sn_f);
    UP(&sn_ld, P.sn_ld);
    UP(&L_off, P.L_off);
    UP(&U_off, P.U_off);
    UP(&fv_off, P.fv_off);
    UP(&child_ptr, P.child_ptr);
    UP(&child_list, P.child_list);
    UP(&relmap_ptr, P.relmap_ptr);
    UP(&relmap, P.relmap);
    UP(&bcolptr, S.bcolptr);
    UP(&blrow, P.blrow);
    UP(&bvptr, S.bvptr);
    UP(&bvidx, S.bvidx);
    UP(&perm_d, S.perm);
    UP(&c->d_small, P.small_list);
    UP(&c->d_large, P.large_list);
    UP(&c->d_asm, P.asm_tasks);
    UP(&c->d_trsm, P.trsm_tasks);
    UP(&c->d_panel, P.panel_tasks);
    UP(&c->d_levels, P.level_list);
    UP(&c->d_sn_rows, S.sn_rows);
    UP(&c->d_sn_rowptr, S.sn_rowptr);
    UP(&c->d_probs, P.probs);
    UP(&c->d_tiles, P.tiles);
    UP(&c->d_solve_list, P.solve_list);
    UP(&c->d_df_tasks, P.df_tasks);
    int64_t *df_part_off = nullptr, *df_seg_off = nullptr, *dinv_off = nullptr;
    UP(&df_part_off, P.df_part_off);
    UP(&df_seg_off, P.df_seg_off);
    UP(&dinv_off, P.dinv_off);
    UP(&c->d_dinv_tasks, P.dinv_tasks);
    int32_t *ea_qs = nullptr;
    UP(&ea_qs, P.ea_qs);
    UP(&c->d_top_list, P.top_list);
    UP(&c->d_own_list, P.own_list);
    UP(&c->d_oz_probs, P.oz_probs);
    UP(&c->d_oz_tiles, P.oz_tiles);
    UP(&c->d_oz_split, P.oz_split);
    if (c->opt.refine_iters > 0) {
        // row k of B = P A P^T (final labels): (column, entry) of every stored entry of
        // row k and of column k -- the residual of the refinement walks whole rows
        const int64_t nb = (int64_t)S.brow.size();
        std::vector<int64_t> rp(n + 1, 0);
        for (int64_t j = 0; j < n; j++)
            for (int64_t e = S.bcolptr[j]; e < S.bcolptr[j + 1]; e++) {
                rp[S.brow[e] + 1]++;
                if (S.brow[e] != j) rp[j + 1]++;
            }
        for (int64_t k = 0; k < n; k++) rp[k + 1] += rp[k];
        std::vector<int32_t> rc(rp[n]), re(rp[n]);
        std::vector<int64_t> fill(rp.begin(), rp.end() - 1);
        for (int64_t j = 0; j < n; j++)
            for (int64_t e = S.bcolptr[j]; e < S.bcolptr[j + 1]; e++) {
                const int32_t i = S.brow[e];
                rc[fill[i]] = (int32_t)j;
                re[fill[i]++] = (int32_t)e;
                if (i != j) {
                    rc[fill[j]] = i;
                    re[fill[j]++] = (int32_t)e;
                }
            }
        if (nb >= INT32_MAX) return MF_ERR_ARG;
        UP(&c->d_rs_ptr, rp);
        UP(&c->d_rs_col, rc);
        UP(&c->d_rs_ent, re);
        if ((r = dev_alloc(c, &p0, (size_t)std::max<int64_t>(nb, 1) * sizeof(double)))) return r;
        c->d_bval = (double *)p0;
        if ((r = dev_alloc(c, &p0, (size_t)std::max<int64_t>(n, 1) * sizeof(double)))) return r;
        c->d_rb = (double *)p0;
        if ((r = dev_alloc(c, &p0, (size_t)std::max<int64_t>(n, 1) * sizeof(double)))) return r;
        c->d_rx = (double *)p0;
        if ((r = dev_alloc(c, &p0, 4 * sizeof(double)))) return r;
        c->d_norms = (double *)p0;
    }
    if (P.oz_slices > 0) {
        if ((r = dev_alloc(c, &p0, (size_t)std::max<int64_t>(P.oz_scratch_bytes, 16)))) return r;
        c->d_oz_scratch = (int8_t *)p0;
        if ((r = dev_alloc(c, &p0, (size_t)std::max<int64_t>(P.oz_expo_words, 4) * sizeof(int32_t)))) return r;
        c->d_oz_expo = (int32_t *)p0;
    }
#undef UP
    d.sn_first = sn_first;
    d.sn_k = sn_k;
    d.sn_f = sn_f;
    d.sn_ld = sn_ld;
    d.L_off = L_off;
    d.U_off = U_off;
    d.fv_off = fv_off;
    d.child_ptr = child_ptr;
    d.child_list = child_list;
    d.relmap_ptr = relmap_ptr;
    d.relmap = relmap;
    d.bcolptr = bcolptr;
    d.blrow = blrow;
    d.bvptr = bvptr;
    d.bvidx = bvidx;
    d.perm = perm_d;
    d.df_part_off = df_part_off;
    d.df_seg_off = df_seg_off;
    d.dinv_off = dinv_off;
    d.ea_qs = ea_qs;
    d.fuse_ea = P.fuse_ea;
    void *p;
    // + kTileM words: the bulk-copy Schur update stages whole 64-row operand columns,
    // so the last tile row of the last panel may read past its f rows
    if ((r = dev_alloc(c, &p, (P.L_words + kTileM) * sizeof(double))) != MF_OK) return r;
    d.L = (double *)p;
    if ((r = dev_alloc(c, &p, P.U_words * sizeof(double))) != MF_OK) return r;
    d.U = (double *)p;
    if ((r = dev_alloc(c, &p, P.fv_words * sizeof(double))) != MF_OK) return r;
    d.fv = (double *)p;
    if ((r = dev_alloc(c, &p, sizeof(int) * 4)) != MF_OK) return r;
    c->d_failed = (int *)p;
    {   // one counter pair per launch slot of every program (factor local / top, solves)
        const size_t slots = P.program.size() + P.program_top.size() + P.fsolve.size() + P.bsolve.size() +
                             P.fsolve_top.size() + P.bsolve_top.size() + 1;
        if ((r = dev_alloc(c, &p, kTkWords * slots * sizeof(unsigned))) != MF_OK) return r;
        c->d_tickets = (unsigned *)p;
        CK(cudaMemsetAsync(p, 0, kTkWords * slots * sizeof(unsigned), c->stream));
    }
    if ((r = dev_alloc(c, &p, (size_t)std::max<int64_t>(P.df_nparts, 1) * sizeof(double))) != MF_OK) return r;
    d.df_parts = (double *)p;
    if ((r = dev_alloc(c, &p, (size_t)std::max<int64_t>(P.df_nseg_words, 1) * sizeof(double))) != MF_OK) return r;
    d.df_seg = (double *)p;
    launch_fill_pending(d.df_seg, P.df_nseg_words, c->stream);   // tail-segment partials: not yet written
    if ((r = dev_alloc(c, &p, (size_t)std::max<int64_t>(P.dinv_words, 1) * sizeof(double))) != MF_OK) return r;
    d.dinv = (double *)p;
    c->dinv_stale = true;
    d.failed = c->d_failed;
    d.epoch = reinterpret_cast<const unsigned *>(c->d_failed + 1);
    if ((r = dev_alloc(c, &p, std::max<int32_t>(P.nsuper, 1) * sizeof(unsigned))) != MF_OK) return r;
    d.leaf_flag = (unsigned *)p;
    CK(cudaMemsetAsync(d.leaf_flag, 0, std::max<int32_t>(P.nsuper, 1) * sizeof(unsigned), c->stream));
    {
        const size_t nf = (size_t)std::max<int32_t>(P.nsuper, 1) * kPanelFlags;
        if ((r = dev_alloc(c, &p, nf * sizeof(unsigned))) != MF_OK) return r;
        d.panel_flag = (unsigned *)p;
        CK(cudaMemsetAsync(d.panel_flag, 0, nf * sizeof(unsigned), c->stream));
    }
    CK(cudaMemsetAsync(c->d_failed, 0, sizeof(int) * 4, c->stream));
    if ((r = dev_alloc(c, &p, std::max<int64_t>(S.nnz_in, 1) * sizeof(double))) != MF_OK) return r;
    c->d_values = (double *)p;
    if ((r = dev_alloc(c, &p, (size_t)std::max<int64_t>(n, 1) * sizeof(double))) != MF_OK) return r;
    c->d_y = (double *)p;
    if ((r = dev_alloc(c, &p, (size_t)std::max<int64_t>(n, 1) * sizeof(double))) != MF_OK) return r;
    c->d_ytmp = (double *)p;
    if ((r = dev_alloc(c, &p, (size_t)std::max<int64_t>(n, 1) * sizeof(double))) != MF_OK) return r;
    c->d_bx = (double *)p;
    // subtree-branch streams (single GPU), created once per ctx
    while ((int)c->bstreams.size() < P.nbranch) {
        cudaStream_t bs;
        CK(cudaStreamCreateWithFlags(&bs, cudaStreamNonBlocking));
        c->bstreams.push_back(bs);
    }
    while ((int)c->bevents.size() < 1 + P.nbranch) {
        cudaEvent_t e;
        CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        c->bevents.push_back(e);
    }
    if (P.nside > 0 && !c->la_hi) {
        int least = 0, greatest = 0;
        CK(cudaDeviceGetStreamPriorityRange(&least, &greatest));
        CK(cudaStreamCreateWithPriority(&c->la_hi, cudaStreamNonBlocking, greatest));
        CK(cudaStreamCreateWithPriority(&c->la_side, cudaStreamNonBlocking, least));
        for (cudaEvent_t &e : c->la_ev) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    }
    // the L arena starts zeroed once so that never-written padding words are defined.
    // MF_DEBUG_NANFILL=1 (debug): fill the L / U / front-vector arenas with NaN
    // instead -- every word a kernel reads into a real output must have been written
    // by this factorization first (tests/test_gpu_parity.py runs it bitwise vs 0-fill)
    const char *nanfill = getenv("MF_DEBUG_NANFILL");
    const int fillb = (nanfill && atoi(nanfill) == 1) ? 0xff : 0;
    CK(cudaMemsetAsync(d.L, fillb, (P.L_words + kTileM) * sizeof(double), c->stream));
    if (fillb) {
        CK(cudaMemsetAsync(d.U, fillb, P.U_words * sizeof(double), c->stream));
        CK(cudaMemsetAsync(d.fv, fillb, P.fv_words * sizeof(double), c->stream));
    }
    CK(cudaStreamSynchronize(c->stream));

    fill_info(c, n, 1);
    mf_info &I = c->info;
    I.t_analyze = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    c->state = 1;
    return MF_OK;
}

namespace {

// Run one launch program (the whole factorization for one rank, or rank 0's top
// part) on the ctx stream: eagerly with per-launch events when profiling,
// otherwise as a CUDA graph captured on first use.
int run_program(mf_ctx *c, const std::vector<Launch> &prog, size_t i0, size_t i1, const double *vals, bool with_init,
                size_t ev_base, cudaGraph_t *graph, cudaGraphExec_t *exec) {
    const Plan &P = c->P;
    const DevPlan &d = c->d;
    cudaStream_t st = c->stream;
    unsigned *tk0 = c->d_tickets + kTkWords * (&prog == &P.program ? 0 : P.program.size());   // this program's slots
    // tl: timeline mode -- the graph keeps its branches and streams, with a timing
    // event recorded before and after every launch on the launch's own stream
    auto issue = [&](const double *v, bool with_events, bool tl = false) -> int {
        if (with_init) launch_init_failed(c->d_failed, st);
        // (captured timing events must be external record nodes: a plain record in a
        // capture only tracks a dependency and is never executed)
        if (tl) CK(cudaEventRecordWithFlags(c->tl_base, st, cudaEventRecordExternal));
        // subtree branches run on their own streams (forked after the init launch,
        // joined before the first top launch); profiled runs stay on one stream
        const bool branches = !with_events && P.nbranch > 1 && (int)c->bstreams.size() >= P.nbranch;
        bool forked = false, joined = false;
        auto join = [&]() -> int {
            for (int b = 0; b < P.nbranch; b++) {
                CK(cudaEventRecord(c->bevents[1 + b], c->bstreams[b]));
                CK(cudaStreamWaitEvent(st, c->bevents[1 + b], 0));
            }
            joined = true;
            return MF_OK;
        };
        // look-ahead streams (graph replay only; profiled runs stay on one stream)
        const bool la = !with_events && c->la_hi != nullptr;
        cudaStream_t mainst = st;
        for (size_t li = i0; li < i1; li++) {
            const Launch &L = prog[li];
            cudaStream_t ls = st;
            if (branches && L.stream >= 0) {
                if (!forked) {
                    CK(cudaEventRecord(c->bevents[0], st));
                    for (int b = 0; b < P.nbranch; b++) CK(cudaStreamWaitEvent(c->bstreams[b], c->bevents[0], 0));
                    forked = true;
                }
                ls = c->bstreams[L.stream];
            } else if (branches && forked && !joined) {
                if (int r = join()) return r;
            }
            if (la && L.stream < 0) {
                if (mainst == st) {   // the main path moves to the high-priority stream
                    CK(cudaEventRecord(c->la_ev[0], st));
                    CK(cudaStreamWaitEvent(c->la_hi, c->la_ev[0], 0));
                    mainst = c->la_hi;
                }
                ls = mainst;
                if (L.side) {
                    CK(cudaEventRecord(c->la_ev[1], mainst));
                    CK(cudaStreamWaitEvent(c->la_side, c->la_ev[1], 0));
                    ls = c->la_side;
                } else if (L.join) {
                    CK(cudaEventRecord(c->la_ev[2], c->la_side));
                    CK(cudaStreamWaitEvent(mainst, c->la_ev[2], 0));
                }
            }
            auto launch = [&](cudaStream_t st) -> int {
            if (with_events) CK(cudaEventRecord(c->prof_events[ev_base + 2 * li], st));
            if (tl) CK(cudaEventRecordWithFlags(c->prof_events[ev_base + 2 * li], st, cudaEventRecordExternal));
            switch (L.kind) {
                case KC_SMALL: launch_small_fronts(d, c->d_small + L.off, (int)L.count, L.param, v, st); break;
                case KC_ASSEMBLE: launch_assemble(d, c->d_asm + 2 * L.off, L.count, v, st); break;
                case KC_POTRF: launch_potrf_diag(d, c->d_large + L.off, (int)L.count, L.param, P.w, st); break;
                case KC_TRSM: launch_trsm_panel(d, c->d_trsm + 2 * L.off, L.count, L.param, P.w, st); break;
                case KC_UPDATE:   // long-K launches of many waves take the bulk-copy pipeline
                    if (L.oz)   // int8 tensor cores, Ozaki scheme
                        launch_update_oz(d, c->d_probs, c->d_oz_probs, c->d_oz_split + 3 * L.oz_s, L.oz_ns,
                                         c->d_oz_tiles + L.oz_t, L.oz_nt, c->d_oz_scratch, c->d_oz_expo + L.oz_e,
                                         L.oz_ne, P.oz_slices, L.oz_wide, st);
                    else
                        launch_update(d, c->d_probs, c->d_tiles + L.off, L.count,
                                      L.count > 0 ? L.flops / (2.0 * kTileM * kTileN * L.count) : 0.0, st);
                    break;
                case KC_PANEL:
                    launch_panel(d, c->d_panel + 2 * L.off, L.count, L.param, (int)L.count2, tk0 + kTkWords * li, st);
                    break;
                case KC_LEAF:
                    launch_leaf(d, c->d_large + L.off, (int)L.count, c->d_trsm + 2 * L.off2, L.count2, L.param, P.w,
                                tk0 + kTkWords * li, st);
                    break;
                default: return MF_ERR_STATE;   // exchange points are handled by run_with_exchanges
            }
            if (with_events) CK(cudaEventRecord(c->prof_events[ev_base + 2 * li + 1], st));
            if (tl) CK(cudaEventRecordWithFlags(c->prof_events[ev_base + 2 * li + 1], st, cudaEventRecordExternal));
            return MF_OK;
            };
            if (int r = launch(ls)) return r;
        }
        if (forked && !joined) {
            if (int r = join()) return r;
        }
        if (mainst != st) {
            CK(cudaEventRecord(c->la_ev[3], mainst));
            CK(cudaStreamWaitEvent(st, c->la_ev[3], 0));
        }
        return MF_OK;
    };
    // (timeline mode: the local program as a graph with captured events; anything else
    // -- the multi-GPU top program's segments, or no graph -- eagerly with events)
    if (c->profiling == 1 || (c->profiling == 2 && (!c->use_graph || !graph || &prog != &P.program)))
        return issue(vals, true);
    if (!c->use_graph || !graph) return issue(vals, false);
    if (c->profiling == 2) {   // timeline: its own graph of the local program, events captured into it
        if (vals != c->d_values && c->S.nnz_in > 0 && with_init)
            CK(cudaMemcpyAsync(c->d_values, vals, c->S.nnz_in * sizeof(double), cudaMemcpyDeviceToDevice, st));
        if (!c->graph_tl_exec) {
            if (!c->tl_base) CK(cudaEventCreate(&c->tl_base));
            CK(cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal));
            int r = issue(c->d_values, false, true);
            cudaGraph_t g = nullptr;
            cudaError_t e = cudaStreamEndCapture(st, &g);
            if (r) return r;
            CK(e);
            c->graph_tl = g;
            CK(cudaGraphInstantiateWithFlags(&c->graph_tl_exec, g, cudaGraphInstantiateFlagUseNodePriority));
        }
        CK(cudaGraphLaunch(c->graph_tl_exec, st));
        return MF_OK;
    }
    // the graph always reads the ctx's value buffer
    if (vals != c->d_values && c->S.nnz_in > 0 && with_init)
        CK(cudaMemcpyAsync(c->d_values, vals, c->S.nnz_in * sizeof(double), cudaMemcpyDeviceToDevice, st));
    if (!*exec) {
        CK(cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal));
        int r = issue(c->d_values, false);
        cudaGraph_t g = nullptr;
        cudaError_t e = cudaStreamEndCapture(st, &g);
        if (r) return r;
        CK(e);
        *graph = g;
        // node priorities (captured from the look-ahead streams) decide which ready
        // kernel gets free SM slots first: the panel path before the side updates
        if (getenv("MF_DEBUG_GRAPH")) {   // node priorities as captured (look-ahead check)
            size_t nn = 0;
            cudaGraphGetNodes(g, nullptr, &nn);
            std::vector<cudaGraphNode_t> nodes(nn);
            cudaGraphGetNodes(g, nodes.data(), &nn);
            std::map<int, int> hist;
            for (cudaGraphNode_t nd : nodes) {
                cudaGraphNodeType t;
                cudaGraphNodeGetType(nd, &t);
                if (t != cudaGraphNodeTypeKernel) continue;
                cudaLaunchAttributeValue v{};
                if (cudaGraphKernelNodeGetAttribute(nd, cudaLaunchAttributePriority, &v) == cudaSuccess) hist[v.priority]++;
                else hist[999]++;
            }
            for (auto &kv : hist) fprintf(stderr, "[libmf] graph kernel nodes with priority %d: %d\n", kv.first, kv.second);
        }
        CK(cudaGraphInstantiateWithFlags(exec, g, cudaGraphInstantiateFlagUseNodePriority));
    }
    CK(cudaGraphLaunch(*exec, st));
    return MF_OK;
}

// Hand a list of transfers to the caller's exchange callback (multi-GPU only);
// the ctx stream is drained first, so the buffers are final.
int exchange(mf_ctx *c, std::vector<mf_xfer> &ops) {
    NvtxRange nvtx_("mf exchange");
    // every rank calls the callback at every exchange point, even with nothing to
    // move, so the caller's collectives stay aligned across ranks
    if (!c->xfn) return MF_ERR_STATE;
    CK(cudaStreamSynchronize(c->stream));
    const int r = c->xfn(c->xuser, ops.empty() ? nullptr : ops.data(), (int64_t)ops.size());
    return r ? MF_ERR_NCCL : MF_OK;
}

// A program with exchange points (the multi-GPU top): kernel segments run eagerly
// on the ctx stream, each exchange point hands its transfer group (pointers into
// the L / U arenas) to the callback.
int run_with_exchanges(mf_ctx *c, const std::vector<Launch> &prog, const double *vals, size_t ev_base) {
    const Plan &P = c->P;
    size_t i0 = 0;
    while (i0 < prog.size()) {
        size_t i1 = i0;
        while (i1 < prog.size() && prog[i1].kind != KC_EXCHANGE) i1++;
        if (i1 > i0) {
            const int r = run_program(c, prog, i0, i1, vals, false, ev_base, nullptr, nullptr);
            if (r) return r;
        }
        if (i1 == prog.size()) break;
        std::vector<mf_xfer> ops;
        for (const XferSpec &x : P.xfers[prog[i1].param])
            ops.push_back(mf_xfer{x.op, x.peer, (x.in_U ? c->d.U : c->d.L) + x.off, x.words * (int64_t)sizeof(double)});
        const int r = exchange(c, ops);
        if (r) return r;
        i0 = i1 + 1;
    }
    return MF_OK;
}

void accumulate_stats(mf_ctx *c, const std::vector<Launch> &prog, size_t ev_base) {
    for (size_t li = 0; li < prog.size(); li++) {
        const Launch &L = prog[li];
        if (L.kind < 0 || L.kind >= KC_COUNT) continue;
        float t = 0.f;
        cudaEventElapsedTime(&t, c->prof_events[ev_base + 2 * li], c->prof_events[ev_base + 2 * li + 1]);
        mf_kernel_stat &K = c->kstats[L.kind];
        K.launches += 1;
        K.ms += t;
        K.flops += L.flops;
        K.bytes += L.bytes;
    }
}

}  // namespace

int mf_factor(mf_ctx *c, const double *values) {
    if (!c || !values) return MF_ERR_ARG;
    NvtxRange nvtx_("mf_factor");
    if (c->state < 1 || c->host_only) return MF_ERR_STATE;
    CK(cudaSetDevice(c->device));
    const Plan &P = c->P;
    cudaStream_t st = c->stream;
    const bool multi = P.nranks > 1;
    if (multi && !c->xfn) return MF_ERR_STATE;
    const double *vals = values;
    const bool vdev = is_device_ptr(values);
    if (vdev) {
        if (int r = order_after_caller(c)) return r;
    }
    CK(cudaEventRecord(c->ev0, st));
    if (!vdev || multi) {
        // bvidx indexes the caller's array; copy the whole array (colptr[n] entries)
        if (c->S.nnz_in > 0)
            CK(cudaMemcpyAsync(c->d_values, values, c->S.nnz_in * sizeof(double),
                               vdev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, st));
        vals = c->d_values;
    }
    if (multi && c->S.nnz_in > 0) {   // rank 0's values are the matrix (include/mf.h)
        std::vector<mf_xfer> bc{mf_xfer{MF_XFER_BCAST, 0, c->d_values, c->S.nnz_in * (int64_t)sizeof(double)}};
        if (int r = exchange(c, bc)) return r;
    }
    const bool prof = c->profiling != 0;
    const size_t nev = 2 * (P.program.size() + P.program_top.size());
    if (prof && c->prof_events.size() < nev) {
        for (size_t i = c->prof_events.size(); i < nev; i++) {
            cudaEvent_t e;
            CK(cudaEventCreate(&e));
            c->prof_events.push_back(e);
        }
    }
    int r = run_program(c, P.program, 0, P.program.size(), vals, true, 0, &c->graph, &c->graph_exec);
    if (r) return r;
    int64_t launches = 1 + (int64_t)P.program.size();
    if (multi) {
        // (1) the frontier roots' update matrices are broadcast by their owners: every
        // rank holds a replica of the top fronts
        std::vector<mf_xfer> ops;
        for (int32_t root : P.frontier_roots) {
            const int32_t m = P.sn_f[root] - P.sn_k[root];
            if (m <= 0) continue;
            ops.push_back(mf_xfer{MF_XFER_BCAST, P.owner[root], c->d.U + P.U_off[root],   // packed lower U^c
                                  (int64_t)m * (m + 1) / 2 * (int64_t)sizeof(double)});
        }
        if ((r = exchange(c, ops))) return r;
        // (2) every rank factors the top: replicated small fronts, cooperative large ones
        if (!P.program_top.empty()) {
            r = run_with_exchanges(c, P.program_top, vals, 2 * P.program.size());
            if (r) return r;
            for (const Launch &L : P.program_top) launches += L.kind != KC_EXCHANGE;
        }
        // (3) first failing pivot over all ranks
        std::vector<mf_xfer> red{mf_xfer{MF_XFER_ALLREDUCE_MIN_I32, 0, c->d_failed, (int64_t)sizeof(int)}};
        if ((r = exchange(c, red))) return r;
    }
    if (c->d_bval) launch_refine_bval(c->d, vals, c->d_bval, (int64_t)c->S.brow.size(), st);   // for mf_solve's residuals
    c->dinv_stale = true;
    CK(cudaGetLastError());
    int failed = INT_MAX;
    CK(cudaMemcpyAsync(&failed, c->d_failed, sizeof(int), cudaMemcpyDeviceToHost, st));
    CK(cudaEventRecord(c->ev1, st));
    CK(cudaStreamSynchronize(st));
    float ms = 0.f;
    cudaEventElapsedTime(&ms, c->ev0, c->ev1);
    c->info.t_factor = ms * 1e-3;
    c->info.launches_factor = launches;
    if (prof) {
        accumulate_stats(c, P.program, 0);
        accumulate_stats(c, P.program_top, 2 * P.program.size());
        c->prof_factors++;
    }
    if (failed != INT_MAX) {
        c->info.failed_col = c->S.perm[failed];
        c->state = 3;
        return MF_NOT_SPD;
    }
    c->info.failed_col = -1;
    c->state = 2;
    return MF_OK;
}

namespace {
// One solve program on (d, y, tickets, st): the ctx's own pipeline or a SolveSlot's.
void run_solve_program(mf_ctx *c, const std::vector<SolveLaunch> &prog, const DevPlan &d, double *y,
                       unsigned *tickets, cudaStream_t st) {
    const Plan &P = c->P;
    size_t base = P.program.size() + P.program_top.size();   // ticket slots of this solve program
    for (const std::vector<SolveLaunch> *q : {&P.fsolve, &P.bsolve, &P.fsolve_top, &P.bsolve_top}) {
        if (q == &prog) break;
        base += q->size();
    }
    unsigned *tk0 = tickets + kTkWords * base;
    for (size_t li = 0; li < prog.size(); li++) {
        const SolveLaunch &L = prog[li];
        switch (L.kind) {
            case SK_SMALL_F: launch_fwd_solve(d, c->d_solve_list + L.off, (int)L.count, y, st); break;
            case SK_INIT_F: launch_fsolve_init(d, c->d_df_tasks + 2 * L.off, L.count, y, st); break;
            case SK_INIT_B:
                launch_bsolve_init(d, c->d_df_tasks + 2 * L.off, L.count, y, c->d_sn_rows, c->d_sn_rowptr, st);
                break;
            case SK_DF_F:
                launch_fsolve_df(d, c->d_df_tasks + 2 * L.off, L.count, c->d_df_tasks + 2 * L.off2, L.count2, P.w, L.j0,
                                 y, tk0 + kTkWords * li, st);
                break;
            case SK_SMALL_B:
                launch_bwd_solve(d, c->d_solve_list + L.off, (int)L.count, y, c->d_sn_rows, c->d_sn_rowptr, st);
                break;
            case SK_DF_B:
                launch_bsolve_df(d, c->d_df_tasks + 2 * L.off, L.count, c->d_df_tasks + 2 * L.off2, L.count2, P.w, L.j0,
                                 y, c->d_sn_rows, c->d_sn_rowptr, tk0 + kTkWords * li, st);
                break;
        }
    }
}
}  // namespace

int mf_solve(mf_ctx *c, const double *b, double *x) {
    if (!c || !b || !x || b == x) return MF_ERR_ARG;
    NvtxRange nvtx_("mf_solve");
    if (c->state != 2 || c->host_only) return MF_ERR_STATE;
    CK(cudaSetDevice(c->device));
    const Plan &P = c->P;
    const DevPlan &d = c->d;
    cudaStream_t st = c->stream;
    const int64_t n = c->S.n;
    const bool multi = P.nranks > 1;
    const bool bdev = is_device_ptr(b), xdev = is_device_ptr(x);
    if (bdev || xdev) {
        if (int r = order_after_caller(c)) return r;
    }
    CK(cudaEventRecord(c->ev0, st));
    if (c->dinv_stale) {   // solve setup, once per factorization: inverses of the 64 x 64 diagonal blocks
        launch_diag_inv(d, c->d_dinv_tasks, (int64_t)P.dinv_tasks.size() / 2, P.w, st);
        c->dinv_stale = false;
    }
    if (!multi && c->use_graph) {
        // single GPU: the whole solve is one CUDA graph over the ctx buffers
        // (b -> d_bx, permute, forward, backward, permute back into d_bx -> x)
        CK(cudaMemcpyAsync(c->d_bx, b, n * sizeof(double), bdev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice,
                           st));
        if (!c->solve_exec) {
            CK(cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal));
            launch_permute_in(d, c->d_bx, c->d_y, n, st);
            run_solve_program(c, P.fsolve, d, c->d_y, c->d_tickets, st);
            run_solve_program(c, P.bsolve, d, c->d_y, c->d_tickets, st);
            launch_permute_out(d, c->d_y, c->d_bx, n, st);
            cudaGraph_t g = nullptr;
            cudaError_t e2 = cudaStreamEndCapture(st, &g);
            CK(e2);
            c->solve_graph = g;
            CK(cudaGraphInstantiate(&c->solve_exec, g, 0));
        }
        CK(cudaGraphLaunch(c->solve_exec, st));
        const double *xsrc = c->d_bx;
        if (c->opt.refine_iters > 0 && c->d_rx) {
            // fp64 iterative refinement on the (reduced-precision) factor: r = b - A x
            // with the caller's values, dx = A^{-1} r through the same solve graph
            CK(cudaMemcpyAsync(c->d_rb, b, n * sizeof(double), bdev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice,
                               st));
            CK(cudaMemcpyAsync(c->d_rx, c->d_bx, n * sizeof(double), cudaMemcpyDeviceToDevice, st));
            double prev = 1e300, berr = 0.0;
            int steps = 0;
            for (;;) {
                launch_refine_resid(d, c->d_rs_ptr, c->d_rs_col, c->d_rs_ent, c->d_bval, c->d_rb, c->d_rx, c->d_bx,
                                    c->d_norms, n, st);
                double nrm[4];
                CK(cudaMemcpyAsync(nrm, c->d_norms, sizeof nrm, cudaMemcpyDeviceToHost, st));
                CK(cudaStreamSynchronize(st));
                const double den = nrm[3] * nrm[1] + nrm[2];
                berr = den > 0 ? nrm[0] / den : 0.0;
                if (berr <= 0x1p-52 || steps >= c->opt.refine_iters || berr > 0.5 * prev) break;
                prev = berr;
                CK(cudaGraphLaunch(c->solve_exec, st));   // d_bx: r -> dx
                launch_refine_axpy(c->d_rx, c->d_bx, n, st);
                steps++;
            }
            c->info.refine_steps = steps;
            c->info.solve_berr = berr;
            xsrc = c->d_rx;
        }
        CK(cudaMemcpyAsync(x, xsrc, n * sizeof(double), xdev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost,
                           st));
        CK(cudaGetLastError());
        CK(cudaEventRecord(c->ev1, st));
        CK(cudaStreamSynchronize(st));
        float ms = 0.f;
        cudaEventElapsedTime(&ms, c->ev0, c->ev1);
        c->info.t_solve = ms * 1e-3;
        return MF_OK;
    }
    const double *bd = b;
    if (!bdev || multi) {
        CK(cudaMemcpyAsync(c->d_bx, b, n * sizeof(double), bdev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice,
                           st));
        bd = c->d_bx;
    }
    if (multi && n > 0) {   // rank 0's right-hand side (include/mf.h)
        std::vector<mf_xfer> bc{mf_xfer{MF_XFER_BCAST, 0, c->d_bx, n * (int64_t)sizeof(double)}};
        if (int r = exchange(c, bc)) return r;
    }
    launch_permute_in(d, bd, c->d_y, n, st);
    int r;
    run_solve_program(c, P.fsolve, d, c->d_y, c->d_tickets, st);   // forward, own subtrees
    if (multi) {
        std::vector<mf_xfer> ops;                      // frontier roots' update vectors -> rank 0
        for (int32_t root : P.frontier_roots) {
            const int32_t own = P.owner[root];
            if (own == 0 || P.sn_f[root] == P.sn_k[root]) continue;
            if (P.rank == own || P.rank == 0)
                ops.push_back(mf_xfer{P.rank == own ? MF_XFER_SEND : MF_XFER_RECV, P.rank == own ? 0 : own,
                                      c->d.fv + P.fv_off[root], (int64_t)P.sn_f[root] * (int64_t)sizeof(double)});
        }
        if ((r = exchange(c, ops))) return r;
        run_solve_program(c, P.fsolve_top, d, c->d_y, c->d_tickets, st);   // rank 0: forward + backward on the top
        run_solve_program(c, P.bsolve_top, d, c->d_y, c->d_tickets, st);
        // rank 0's top solution -> every rank (y columns of the top supernodes)
        if (P.rank == 0) CK(cudaMemcpyAsync(c->d_ytmp, c->d_y, n * sizeof(double), cudaMemcpyDeviceToDevice, st));
        std::vector<mf_xfer> bc{mf_xfer{MF_XFER_BCAST, 0, c->d_ytmp, n * (int64_t)sizeof(double)}};
        if ((r = exchange(c, bc))) return r;
        if (P.rank != 0) launch_copy_cols(d, c->d_top_list, (int)P.top_list.size(), c->d_ytmp, c->d_y, st);
    }
    run_solve_program(c, P.bsolve, d, c->d_y, c->d_tickets, st);   // backward, own subtrees
    if (multi) {   // every rank contributes its own columns; the sum is the full solution
        CK(cudaMemsetAsync(c->d_ytmp, 0, n * sizeof(double), st));
        launch_copy_cols(d, c->d_own_list, (int)P.own_list.size(), c->d_y, c->d_ytmp, st);
        std::vector<mf_xfer> ar{mf_xfer{MF_XFER_ALLREDUCE_SUM, 0, c->d_ytmp, n * (int64_t)sizeof(double)}};
        if ((r = exchange(c, ar))) return r;
        CK(cudaMemcpyAsync(c->d_y, c->d_ytmp, n * sizeof(double), cudaMemcpyDeviceToDevice, st));
    }
    double *xd = xdev ? x : c->d_bx;
    launch_permute_out(d, c->d_y, xd, n, st);
    if (!xdev) CK(cudaMemcpyAsync(x, c->d_bx, n * sizeof(double), cudaMemcpyDeviceToHost, st));
    CK(cudaGetLastError());
    CK(cudaEventRecord(c->ev1, st));
    CK(cudaStreamSynchronize(st));
    float ms = 0.f;
    cudaEventElapsedTime(&ms, c->ev0, c->ev1);
    c->info.t_solve = ms * 1e-3;
    return MF_OK;
}

namespace {
// Extra solve pipelines for mf_solve_nrhs (allocated on first use; freed with the plan).
int ensure_slots(mf_ctx *c, int ns) {
    const Plan &P = c->P;
    const int64_t n = c->S.n;
    const size_t tk_words = kTkWords * (P.program.size() + P.program_top.size() + P.fsolve.size() + P.bsolve.size() +
                                 P.fsolve_top.size() + P.bsolve_top.size() + 1);
    while ((int)c->slots.size() < ns) {
        SolveSlot q;
        q.d = c->d;
        void *p = nullptr;
        int r;
        if ((r = dev_alloc(c, &p, (size_t)std::max<int64_t>(n, 1) * sizeof(double)))) return r;
        q.y = (double *)p;
        if ((r = dev_alloc(c, &p, (size_t)std::max<int64_t>(n, 1) * sizeof(double)))) return r;
        q.bx = (double *)p;
        if ((r = dev_alloc(c, &p, (size_t)P.fv_words * sizeof(double)))) return r;
        q.d.fv = (double *)p;
        if ((r = dev_alloc(c, &p, (size_t)std::max<int64_t>(P.df_nparts, 1) * sizeof(double)))) return r;
        q.d.df_parts = (double *)p;
        if ((r = dev_alloc(c, &p, (size_t)std::max<int64_t>(P.df_nseg_words, 1) * sizeof(double)))) return r;
        q.d.df_seg = (double *)p;
        launch_fill_pending(q.d.df_seg, P.df_nseg_words, c->stream);
        if ((r = dev_alloc(c, &p, tk_words * sizeof(unsigned)))) return r;
        CK(cudaMemsetAsync(p, 0, tk_words * sizeof(unsigned), c->stream));
        q.tickets = (unsigned *)p;
        CK(cudaStreamCreateWithFlags(&q.st, cudaStreamNonBlocking));
        CK(cudaEventCreateWithFlags(&q.done, cudaEventDisableTiming));
        // the same program as mf_solve's graph, on the slot's buffers and stream
        CK(cudaStreamBeginCapture(q.st, cudaStreamCaptureModeThreadLocal));
        launch_permute_in(q.d, q.bx, q.y, n, q.st);
        run_solve_program(c, P.fsolve, q.d, q.y, q.tickets, q.st);
        run_solve_program(c, P.bsolve, q.d, q.y, q.tickets, q.st);
        launch_permute_out(q.d, q.y, q.bx, n, q.st);
        cudaError_t e = cudaStreamEndCapture(q.st, &q.graph);
        CK(e);
        CK(cudaGraphInstantiate(&q.exec, q.graph, 0));
        c->slots.push_back(q);
    }
    CK(cudaStreamSynchronize(c->stream));   // zeroed flags / tickets before first use
    return MF_OK;
}
}  // namespace

int mf_solve_nrhs(mf_ctx *c, int32_t nrhs, const double *B, int64_t ldb, double *X, int64_t ldx) {
    if (!c || nrhs < 0) return MF_ERR_ARG;
    NvtxRange nvtx_("mf_solve_nrhs");
    if (c->state != 2 || c->host_only) return MF_ERR_STATE;
    const int64_t n = c->S.n;
    if (nrhs == 0) return MF_OK;
    if (!B || !X || ldb < n || ldx < n) return MF_ERR_ARG;
    if ((const void *)B == (const void *)X) return MF_ERR_ARG;
    if (c->P.nranks > 1 || !c->use_graph || c->opt.refine_iters > 0 || nrhs == 1) {
        for (int32_t r = 0; r < nrhs; r++)   // one column at a time through mf_solve
            if (int e = mf_solve(c, B + r * ldb, X + r * ldx)) return e;
        return MF_OK;
    }
    CK(cudaSetDevice(c->device));
    cudaStream_t st = c->stream;
    const bool bdev = is_device_ptr(B), xdev = is_device_ptr(X);
    if (bdev || xdev) {
        if (int r = order_after_caller(c)) return r;
    }
    if (c->dinv_stale) {   // solve setup (inverses of the diagonal blocks), once per factorization
        launch_diag_inv(c->d, c->d_dinv_tasks, (int64_t)c->P.dinv_tasks.size() / 2, c->P.w, st);
        c->dinv_stale = false;
    }
    static const int max_slots = [] {   // MF_SOLVE_SLOTS: tuning override of kSolveSlots
        const char *e = getenv("MF_SOLVE_SLOTS");
        return e ? std::max(1, std::min(16, atoi(e))) : kSolveSlots;
    }();
    const int ns = std::min<int>(max_slots, nrhs);
    if (int r = ensure_slots(c, ns)) return r;
    CK(cudaEventRecord(c->ev0, st));
    for (int q = 0; q < ns; q++) CK(cudaStreamWaitEvent(c->slots[q].st, c->ev0, 0));
    // right-hand side r on slot r mod ns: each slot's columns run in order on its stream,
    // the slots concurrently (same kernels and order as mf_solve: bitwise the same x)
    for (int32_t r = 0; r < nrhs; r++) {
        SolveSlot &q = c->slots[r % ns];
        CK(cudaMemcpyAsync(q.bx, B + r * ldb, n * sizeof(double),
                           bdev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, q.st));
        CK(cudaGraphLaunch(q.exec, q.st));
        CK(cudaMemcpyAsync(X + r * ldx, q.bx, n * sizeof(double),
                           xdev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, q.st));
    }
    for (int q = 0; q < ns; q++) {
        CK(cudaEventRecord(c->slots[q].done, c->slots[q].st));
        CK(cudaStreamWaitEvent(st, c->slots[q].done, 0));
    }
    CK(cudaGetLastError());
    CK(cudaEventRecord(c->ev1, st));
    CK(cudaStreamSynchronize(st));
    float ms = 0.f;
    cudaEventElapsedTime(&ms, c->ev0, c->ev1);
    c->info.t_solve = ms * 1e-3;
    return MF_OK;
}

int mf_set_exchange(mf_ctx *c, mf_exchange_fn fn, void *user) {
    if (!c) return MF_ERR_ARG;
    c->xfn = fn;
    c->xuser = user;
    return MF_OK;
}

int mf_get_info(const mf_ctx *c, mf_info *out) {
    if (!c || !out) return MF_ERR_ARG;
    *out = c->info;
    return MF_OK;
}

int mf_get_perm(const mf_ctx *c, int32_t *out) {
    if (!c || !out) return MF_ERR_ARG;
    if (c->state < 1) return MF_ERR_STATE;
    std::memcpy(out, c->S.perm.data(), c->S.perm.size() * sizeof(int32_t));
    return MF_OK;
}

int mf_get_etree(const mf_ctx *c, int32_t *parent, int64_t *cc) {
    if (!c) return MF_ERR_ARG;
    if (c->state < 1) return MF_ERR_STATE;
    if (parent) std::memcpy(parent, c->S.parent.data(), c->S.parent.size() * sizeof(int32_t));
    if (cc) std::memcpy(cc, c->S.cc.data(), c->S.cc.size() * sizeof(int64_t));
    return MF_OK;
}

int mf_get_supernodes(const mf_ctx *c, int32_t *sn_first, int32_t *sn_parent, int64_t *sn_rowptr, int32_t *sn_rows,
                      int32_t *fund_first) {
    if (!c) return MF_ERR_ARG;
    if (c->state < 1) return MF_ERR_STATE;
    const Symbolic &S = c->S;
    if (sn_first) std::memcpy(sn_first, S.sn_first.data(), S.sn_first.size() * sizeof(int32_t));
    if (sn_parent) std::memcpy(sn_parent, S.sn_parent.data(), S.sn_parent.size() * sizeof(int32_t));
    if (sn_rowptr) std::memcpy(sn_rowptr, S.sn_rowptr.data(), S.sn_rowptr.size() * sizeof(int64_t));
    if (sn_rows) std::memcpy(sn_rows, S.sn_rows.data(), S.sn_rows.size() * sizeof(int32_t));
    if (fund_first) std::memcpy(fund_first, S.fund_first.data(), S.fund_first.size() * sizeof(int32_t));
    return MF_OK;
}

int mf_export_panel(const mf_ctx *c, int32_t s, double *out) {
    if (!c || !out) return MF_ERR_ARG;
    if (c->state != 2) return MF_ERR_STATE;
    if (s < 0 || s >= c->P.nsuper) return MF_ERR_ARG;
    CK(cudaSetDevice(c->device));
    const int f = c->P.sn_f[s], k = c->P.sn_k[s], ld = c->P.sn_ld[s];
    CK(cudaMemcpy2DAsync(out, f * sizeof(double), c->d.L + c->P.L_off[s], ld * sizeof(double), f * sizeof(double), k,
                         cudaMemcpyDeviceToHost, c->stream));
    CK(cudaStreamSynchronize(c->stream));
    return MF_OK;
}

static const char *kKernelNames[KC_COUNT] = {"small_front_fused", "assemble_extend_add", "potrf_diag",
                                             "trsm_panel", "dmma_schur_update", "leaf_potrf_trsm",
                                             "dataflow_panel"};

int mf_set_profiling(mf_ctx *c, int enable) {
    if (!c) return MF_ERR_ARG;
    if (enable < 0 || enable > 2) return MF_ERR_ARG;
    c->profiling = enable;
    for (int k = 0; k < KC_COUNT; k++) {
        c->kstats[k] = mf_kernel_stat{};
        snprintf(c->kstats[k].name, sizeof(c->kstats[k].name), "%s", kKernelNames[k]);
    }
    c->prof_factors = 0;
    return MF_OK;
}

int mf_get_mapping(const mf_ctx *c, int32_t *owner, int8_t *top, double *rank_load, double *top_load) {
    if (!c) return MF_ERR_ARG;
    if (c->state < 1) return MF_ERR_STATE;
    const Plan &P = c->P;
    if (owner) std::memcpy(owner, P.owner.data(), P.owner.size() * sizeof(int32_t));
    if (top)
        for (size_t i = 0; i < P.top.size(); i++) top[i] = P.top[i] ? (P.dist[i] ? 2 : 1) : 0;
    if (rank_load) std::memcpy(rank_load, P.rank_load.data(), P.rank_load.size() * sizeof(double));
    if (top_load) *top_load = P.top_load;
    return MF_OK;
}

int mf_get_program(const mf_ctx *c, mf_launch_info *out, int64_t max, int64_t *count) {
    if (!c || !count) return MF_ERR_ARG;
    if (c->state < 1) return MF_ERR_STATE;
    const auto &prog = c->P.program;
    *count = (int64_t)prog.size();
    if (out)
        for (int64_t i = 0; i < std::min<int64_t>(max, (int64_t)prog.size()); i++)
            out[i] = mf_launch_info{prog[i].kind,     prog[i].level, prog[i].count, prog[i].flops, prog[i].bytes,
                                    prog[i].int8_ops, prog[i].stream, 0};
    return MF_OK;
}

int mf_get_launch_times(const mf_ctx *c, double *out, int64_t max, int64_t *count) {
    if (!c || !count) return MF_ERR_ARG;
    const int64_t n = (int64_t)c->P.program.size();
    *count = n;
    if (!out) return MF_OK;
    if (c->host_only || c->prof_factors == 0 || (int64_t)c->prof_events.size() < 2 * n) return MF_ERR_STATE;
    for (int64_t i = 0; i < std::min(n, max); i++) {
        float t = 0.f;
        cudaEventElapsedTime(&t, c->prof_events[2 * i], c->prof_events[2 * i + 1]);
        out[i] = t;
    }
    return MF_OK;
}

int mf_get_launch_timeline(const mf_ctx *c, double *start_ms, double *end_ms, int64_t max, int64_t *count) {
    if (!c || !count) return MF_ERR_ARG;
    const int64_t n = (int64_t)c->P.program.size();
    *count = n;
    if (!start_ms && !end_ms) return MF_OK;
    if (c->host_only || c->profiling != 2 || c->prof_factors == 0 || !c->tl_base || !c->graph_tl_exec ||
        (int64_t)c->prof_events.size() < 2 * n)
        return MF_ERR_STATE;
    for (int64_t i = 0; i < std::min(n, max); i++) {
        float t0 = 0.f, t1 = 0.f;
        cudaEventElapsedTime(&t0, c->tl_base, c->prof_events[2 * i]);
        cudaEventElapsedTime(&t1, c->tl_base, c->prof_events[2 * i + 1]);
        if (start_ms) start_ms[i] = t0;
        if (end_ms) end_ms[i] = t1;
    }
    return MF_OK;
}

int mf_set_variant_model(mf_ctx *c, const double *theta, int32_t nfeatures, int32_t nclasses, int32_t force) {
    if (!c) return MF_ERR_ARG;
    if (c->state != 0) return MF_ERR_STATE;
    if (force < -1 || force >= kVariants) return MF_ERR_ARG;
    if (theta && (nfeatures != kVariantFeatures || nclasses != kVariants)) return MF_ERR_ARG;
    c->opt.variant_theta.clear();
    if (theta) c->opt.variant_theta.assign(theta, theta + kVariantFeatures * kVariants);
    c->opt.force_variant = force;
    return MF_OK;
}

int mf_get_variants(const mf_ctx *c, int32_t *out) {
    if (!c || !out) return MF_ERR_ARG;
    if (c->state < 1) return MF_ERR_STATE;
    std::copy(c->P.variant.begin(), c->P.variant.end(), out);
    return MF_OK;
}

int mf_get_kernel_stats(const mf_ctx *c, mf_kernel_stat *out, int32_t *count) {
    if (!c || !out || !count) return MF_ERR_ARG;
    for (int k = 0; k < KC_COUNT; k++) out[k] = c->kstats[k];
    *count = KC_COUNT;
    return MF_OK;
}

int mf_export_diag(const mf_ctx *c, double *out) {
    if (!c || !out) return MF_ERR_ARG;
    if (c->state != 2) return MF_ERR_STATE;
    CK(cudaSetDevice(c->device));
    const int64_t n = c->S.n;
    launch_export_diag(c->d, c->P.nsuper, c->d_bx, c->stream);
    CK(cudaMemcpyAsync(out, c->d_bx, n * sizeof(double), cudaMemcpyDeviceToHost, c->stream));
    CK(cudaStreamSynchronize(c->stream));
    return MF_OK;
}

int mf_export_panels(const mf_ctx *c, double *out) {
    if (!c || !out) return MF_ERR_ARG;
    if (c->state != 2) return MF_ERR_STATE;
    int64_t o = 0;
    for (int32_t s = 0; s < c->P.nsuper; s++) {
        int r = mf_export_panel(c, s, out + o);
        if (r) return r;
        o += (int64_t)c->P.sn_f[s] * c->P.sn_k[s];
    }
    return MF_OK;
}

int mf_export_L(const mf_ctx *c, int64_t *Lp, int32_t *Li, double *Lx) {
    if (!c) return MF_ERR_ARG;
    if (c->state < 1) return MF_ERR_STATE;
    if (Lx && c->state != 2) return MF_ERR_STATE;
    const Symbolic &S = c->S;
    const Plan &P = c->P;
    const int64_t n = S.n;
    if (Lp) {   // column j of supernode s (local jj): rows R_s[jj..f)
        Lp[0] = 0;
        for (int32_t s = 0; s < P.nsuper; s++)
            for (int32_t jj = 0; jj < P.sn_k[s]; jj++) {
                const int64_t j = S.sn_first[s] + jj;
                Lp[j + 1] = Lp[j] + (P.sn_f[s] - jj);
            }
    }
    if (!Li && !Lx) return MF_OK;
    std::vector<double> panel;
    int64_t o = 0;
    for (int32_t s = 0; s < P.nsuper; s++) {
        const int32_t f = P.sn_f[s], k = P.sn_k[s];
        const int32_t *R = S.sn_rows.data() + S.sn_rowptr[s];
        if (Lx) {
            panel.resize((size_t)f * k);
            if (int r = mf_export_panel(c, s, panel.data())) return r;
        }
        for (int32_t jj = 0; jj < k; jj++) {
            if (Li) std::memcpy(Li + o, R + jj, (size_t)(f - jj) * sizeof(int32_t));
            if (Lx) std::memcpy(Lx + o, panel.data() + (size_t)jj * f + jj, (size_t)(f - jj) * sizeof(double));
            o += f - jj;
        }
    }
    (void)n;
    return MF_OK;
}

}  // extern "C"
