// kernels.cuh -- device-side plan view and kernel launchers (internal to libmf).
#pragma once
#include <cuda_runtime.h>
#include <cstdint>

#include "mf_plan.h"

namespace mf {

// Flat device arrays of the plan (uploaded once by mf_analyze).
struct DevPlan {
    double *L;            // L arena (panels)
    double *U;            // U arena (update matrices)
    double *fv;           // solve: one front vector per supernode
    const int32_t *sn_first, *sn_k, *sn_f, *sn_ld;
    const int64_t *L_off, *U_off, *fv_off;
    const int32_t *child_ptr, *child_list;
    const int64_t *relmap_ptr;
    const int32_t *relmap;
    const int64_t *bcolptr;  // B entries per column (final labels)
    const int32_t *blrow;    // local row of each B entry in its front
    const int64_t *bvptr;    // value-index list per B entry
    const int64_t *bvidx;
    const int32_t *perm;     // final perm (new -> old)
    int *failed;             // min failing pivot column (final labels); INT_MAX = none
    const unsigned *epoch;   // factorization counter (= failed + 1), bumped by the init kernel
    unsigned *leaf_flag;     // per supernode: fused-leaf "diagonal block done" flag
    unsigned *panel_flag;    // per supernode: kPanelFlags dataflow-panel tile flags
    double *df_parts;        // dataflow backward sweep: published x of the pivot columns (value = flag)
    const int64_t *df_part_off;
    double *df_seg;          // dataflow backward sweep: column partials of the tail segments (value = flag)
    const int64_t *df_seg_off;
    double *dinv;            // dataflow solve: inverses of the 64 x 64 diagonal blocks (solve setup)
    const int64_t *dinv_off; // per supernode: word offset of its blocks in dinv (-1: none)
    const int32_t *ea_qs;    // fused extend-add: tile-row start tables of the syrk problems
    int fuse_ea;             // 1: large-front assembly covers the panel columns only
};

// launchers (all asynchronous on `st`)
void launch_init_failed(int *failed, cudaStream_t st);
void launch_small_fronts(const DevPlan &d, const int32_t *list, int count, int fmax, const double *values,
                         cudaStream_t st);
void launch_assemble(const DevPlan &d, const int32_t *tasks, int64_t count, const double *values, cudaStream_t st);
// tk: the launch slot's ticket-counter pair (zeroed at analyze; see take_ticket in kernels.cu)
void launch_leaf(const DevPlan &d, const int32_t *fronts, int npotrf, const int32_t *tasks, int64_t ntrsm, int j0,
                 int w, unsigned *tk, cudaStream_t st);
void launch_panel(const DevPlan &d, const int32_t *tasks, int64_t count, int j0, int nbk, unsigned *tk,
                  cudaStream_t st);
void launch_potrf_diag(const DevPlan &d, const int32_t *fronts, int count, int j0, int w, cudaStream_t st);
void launch_trsm_panel(const DevPlan &d, const int32_t *tasks, int64_t count, int j0, int w, cudaStream_t st);
// kavg = the launch's average inner dimension.  Variant per launch (measured per
// launch with tools/level_breakdown.py and MF_UPD_BULK / MF_UPD_LOWK = 0/1):
//  * many waves of long-K tiles: mbarrier + bulk-copy staging (c5 -4 ms);
//  * short K (latency-bound on the C gather / store): 2-stage ring, 5 CTAs/SM;
//  * otherwise the 3-stage cp.async pipeline, 4 CTAs/SM.
constexpr int64_t kBulkMinTiles = 4 * 592;   // 4 waves of 148 SMs x 4 CTAs
constexpr double kBulkMinK = 512;
constexpr double kLowKMax = 256;
void launch_update(const DevPlan &d, const GemmProb *probs, const TileTask *tiles, int64_t ntiles, double kavg,
                   cudaStream_t st);
// Schur update of one launch on the int8 tensor cores (Ozaki scheme, S slices)
void launch_update_oz(const DevPlan &d, const GemmProb *probs, const OzProb *oprobs, const int32_t *split,
                      int64_t nsplit, const OzTile *tiles, int64_t ntiles, int8_t *scratch, int32_t *expo,
                      int64_t expo_words, int S, int wide, cudaStream_t st);
// fp64 iterative refinement (mixed-precision mode): B entry values, residual + norms, x += dx
void launch_refine_bval(const DevPlan &d, const double *values, double *bval, int64_t nb, cudaStream_t st);
void launch_refine_resid(const DevPlan &d, const int64_t *rs_ptr, const int32_t *rs_col, const int32_t *rs_ent,
                         const double *bval, const double *b, const double *x, double *r, double *norms, int64_t n,
                         cudaStream_t st);
void launch_refine_axpy(double *x, const double *dx, int64_t n, cudaStream_t st);
void launch_permute_in(const DevPlan &d, const double *b, double *y, int64_t n, cudaStream_t st);
void launch_permute_out(const DevPlan &d, const double *xf, double *x, int64_t n, cudaStream_t st);
void launch_fwd_solve(const DevPlan &d, const int32_t *list, int count, double *y, cudaStream_t st);
void launch_bwd_solve(const DevPlan &d, const int32_t *list, int count, double *y, const int32_t *sn_rows,
                      const int64_t *sn_rowptr, cudaStream_t st);
// solve setup: inverses of the 64 x 64 diagonal blocks of the dataflow-solved supernodes
void launch_diag_inv(const DevPlan &d, const int32_t *tasks, int64_t count, int w, cudaStream_t st);
void launch_fill_pending(double *p, int64_t n, cudaStream_t st);   // dataflow-solve slots: not yet written

// deep = 1: the levels with multi-block fronts (register ring of MF_DF_BUF blocks, 1 CTA / SM)
// the init tasks of a level (front vectors, pending slots) as a launch of their own ...
void launch_fsolve_init(const DevPlan &d, const int32_t *tasks, int64_t count, double *y, cudaStream_t st);
void launch_bsolve_init(const DevPlan &d, const int32_t *tasks, int64_t count, const double *y,
                        const int32_t *sn_rows, const int64_t *sn_rowptr, cudaStream_t st);
// ... or (itasks / ninit) run first in the level's dataflow launch
void launch_fsolve_df(const DevPlan &d, const int32_t *tasks, int64_t count, const int32_t *itasks, int64_t ninit,
                      int w, int deep, double *y, unsigned *tk, cudaStream_t st);
void launch_bsolve_df(const DevPlan &d, const int32_t *tasks, int64_t count, const int32_t *itasks, int64_t ninit,
                      int w, int deep, double *y, const int32_t *sn_rows, const int64_t *sn_rowptr, unsigned *tk,
                      cudaStream_t st);


int small_front_smem_ok(int fmax);
int kernels_init();
void launch_copy_cols(const DevPlan &d, const int32_t *list, int count, const double *src, double *dst,
                      cudaStream_t st);
void launch_export_diag(const DevPlan &d, int nsuper, double *out, cudaStream_t st);

}  // namespace mf
