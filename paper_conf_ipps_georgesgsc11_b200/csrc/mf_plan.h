// mf_plan.h -- host-side symbolic analysis + device plan of the multifrontal
// factor-update hot path (internal to libmf; the public ABI is include/mf.h).
//
// The symbolic layer feeds PAPER.md L27 (Sec. II-A): supernodal elimination
// tree in postorder, front row lists R_s (front order f = k + m, reading C1),
// child -> parent extend-add index maps, A-entry -> front maps.  Algorithms
// (Liu's etree with path compression, row-subtree column counts, supernodal
// row-list merge) are deliberately different from the oracle's definitions
// (oracle/symbolic.c) so that bit-exact agreement is a real check.
#pragma once
#include <cstdint>
#include <vector>

#ifdef __CUDACC__
#define MF_HD __host__ __device__ __forceinline__
#else
#define MF_HD inline
#endif

namespace mf {

// Update matrices U^s (m x m, lower triangle) are stored PACKED, column-major lower:
// column j (its diagonal first) starts at word j (2m - j + 1) / 2; element (i, j),
// i >= j, is word upk_col(j, m) + i - j.  m (m + 1) / 2 words per front, half the
// full square (workspace, and the bytes a multi-GPU exchange moves).
MF_HD int64_t upk_col(int64_t j, int64_t m) { return j * (2 * m - j + 1) / 2; }
MF_HD int64_t upk(int64_t i, int64_t j, int64_t m) { return upk_col(j, m) + (i - j); }

struct Options {
    int amalgamate = 1;
    int nrelax[3] = {4, 16, 48};
    double zrelax[3] = {0.8, 0.1, 0.05};
    int small_front_max = 128;
    int panel_w = 64;
    int nranks = 1;   // GPUs sharing one factorization (one process per GPU)
    int rank = 0;
    int split_all = 0;   // multi-GPU mapping ignores the exchange-cost model
    int fuse_ea = 1;     // extend-add into the U^s part fused into the syrk prologue (NEXT-1)
    int nbranch = 4;     // single GPU: concurrent subtree branches (graph branches on their own streams)
    int lookahead = 0;   // single GPU, main stream: trailing update split so the next panel overlaps its rest (measured: no gain; off)
    // learned kernel-variant selector (Sec. VI, Eqs. 3-5):
    // theta is kVariantFeatures x kVariants (column j = class j); empty = the fixed
    // front-order thresholds.  force_variant >= 0 forces that class wherever feasible.
    std::vector<double> variant_theta;
    int force_variant = -1;
    // Schur updates on the int8 tensor cores (Ozaki scheme):
    // 0 = FP64 DMMA; 8 = FP64-class emulation; 3..7 = reduced precision (mf_solve
    // then refines in fp64).  refine_iters: max refinement steps (-1 = auto).
    int ozaki_slices = 0;
    int refine_iters = -1;
};

// Kernel variants a front can be factored with (the GPU-only policy classes that
// replace the paper's CPU/GPU policies P1-P4, Table VI): one warp per
// front (f <= 16, f <= 32), one CTA per front with the front in shared memory
// (f <= 64, 96, 128, 160), or the tiled large-front path.  kVariantFmax = the
// largest front order a class accepts (0 = any: tiled).
constexpr int kVariants = 7;
constexpr int kVariantTiled = 6;
constexpr int kVariantFmax[kVariants] = {16, 32, 64, 96, 128, 160, 0};
// Features of a front (m off-diagonal rows, k pivot columns): the paper's
// [m, k, m/k, m^2, mk, k^2, k^3, mk^2] after a constant 1, with
// m and k measured in units of 64 (reading R3 in DESIGN.md).
constexpr int kVariantFeatures = 9;
inline void variant_features(double m, double k, double *x) {
    const double a = m / 64.0, b = k / 64.0;
    x[0] = 1.0;
    x[1] = a;
    x[2] = b;
    x[3] = m / k;
    x[4] = a * a;
    x[5] = a * b;
    x[6] = b * b;
    x[7] = b * b * b;
    x[8] = a * b * b;
}

// ---------------------------------------------------------------- symbolic
struct Symbolic {
    int64_t n = 0;
    int64_t nnzA_read = 0;
    int64_t nnz_in = 0;              // colptr[n]: length of the caller's values array
    std::vector<int32_t> perm;       // final perm (new -> old)
    std::vector<int32_t> parent;     // elimination tree
    std::vector<int64_t> cc;         // column counts
    int64_t nnzL = 0, flops = 0, stored_L = 0, exec_flops = 0;
    std::vector<int32_t> fund_first;
    std::vector<int32_t> sn_first, sn_parent;
    std::vector<int64_t> sn_rowptr;
    std::vector<int32_t> sn_rows;
    // unique entries of B = P A P^T (lower incl. diagonal), sorted (col, row);
    // value of entry e = sum of values[bvidx[bvptr[e] .. bvptr[e+1])] in input order
    std::vector<int64_t> bcolptr;    // n+1
    std::vector<int32_t> brow;
    std::vector<int64_t> bvptr;
    std::vector<int64_t> bvidx;
};

// returns 0 or a negative MF_ERR_* code
int analyze_symbolic(int64_t n, const int64_t *colptr, const int32_t *rowind, const int32_t *perm,
                     const Options &opt, Symbolic &S);

// ---------------------------------------------------------------- device plan
// A (lower-trapezoidal) Schur update problem:  C[i][j] -= sum_p A[i][p] * A[j][p]
// for 0 <= j < N, j <= i < M (only entries with i >= j are written).
// A: M x K, column-major, leading dim lda, inside the L arena.
// C: column-major, leading dim ldc, inside the L arena (flags bit 0 = 0), or packed
// lower of order ldc (upk) inside the U arena (1).  flags bit 1: the problem is shifted one row / column up-left so that
// its first A row is even (16-byte staging); row / column 0 of the shifted space
// are padding: C(i, j) of the kernel is C_orig(i - 1, j - 1).
// flags bit 2 (the syrk on U^s with the extend-add fused into its prologue,
// SURVEY.md NEXT-1): C starts from 0 + the children's U^c in ascending order,
// gathered through their relative maps, instead of from a U^s assembled in HBM;
// s = the front, ea_qs[qs_off + j (ntr + 1) + t] = first row of child j whose
// parent row falls in tile row t or below (ntr = tile rows of the problem).
struct GemmProb {
    int64_t a_off;
    int64_t c_off;
    int32_t lda, ldc;
    int32_t M, N, K;
    int32_t flags;
    int32_t s = -1;
    int32_t qs_off = 0;
};
static_assert(sizeof(GemmProb) == 48, "GemmProb layout");
constexpr int32_t kProbU = 1, kProbShift = 2, kProbGather = 4;

struct TileTask {       // one kTileM x kTileN output tile of a GemmProb
    int32_t prob;
    int32_t tij;        // (ti << 16) | tj
};

constexpr int kOzBM = 128, kOzBN = 64, kOzBK = 64;   // Ozaki tile rows, tile columns, int8 k per stage
constexpr int kOzMaxK = 16000;                       // int32-exact inner dimension (S <= 8)
constexpr int kOzSeg = 256;                          // k values per split task
// Ozaki-scheme form of a GemmProb (csrc/ozaki_update.cuh): its A rows are cut into
// int8 digit slices in a per-stream scratch before the int8 tensor-core update.
struct OzProb {
    int32_t prob;       // GemmProb index
    int32_t Mpad;       // rows padded to kOzBM (128)
    int32_t Kpad;       // inner dimension padded to kOzBK (64)
    int32_t pad_;
    int64_t sl_off;     // byte offset of its slices in the scratch: [S][Kpad/16][Mpad][16 bytes]
    int64_t ex_off;     // int32 offset of its row exponents E_i
};
static_assert(sizeof(OzProb) == 32, "OzProb layout");
struct OzTile {         // one 128 x 64 output tile
    int32_t oprob;
    int32_t tij;        // (ti << 16) | tj
};

// The factorization is a static launch program built once per pattern
// (mf_analyze) and replayed by every mf_factor.
enum KernelClass : int32_t {
    KC_SMALL = 0,     // batched fused small-front kernel (assembly + potrf + trsm + syrk in SMEM)
    KC_ASSEMBLE = 1,  // large-front assembly (A scatter + extend-add)
    KC_POTRF = 2,     // w x w diagonal-block potrf
    KC_TRSM = 3,      // panel trsm below the diagonal block
    KC_UPDATE = 4,    // DMMA Schur update (panel trailing update and the syrk on U^n)
    KC_LEAF = 5,      // fused potrf + trsm of one diagonal block (few active fronts)
    KC_PANEL = 6,     // dataflow panel: potrf + trsm + inner updates of up to kPanelMaxBlocks blocks of 64 columns
    KC_COUNT = 7,
    KC_EXCHANGE = 16  // multi-GPU: hand the transfer group Plan::xfers[param] to the exchange callback
};
constexpr int kFuseLeafMaxFronts = 8;
// Dataflow panel (KC_PANEL, w = 64 only): base case of the recursive blocked
// factorization; per front kPanelFlags epoch-tagged flags (band tiles + diagonal tiles).
constexpr int kPanelMaxBlocks = 8;   // 8 x 64 columns per panel launch (A/B: 4 -> 8 c5 -0.6%, c3 -1.6%, c4 -1%; 16 worse on c2/c3)
constexpr int kPanelFlags = kPanelMaxBlocks * (kPanelMaxBlocks + 1) / 2;

// One transfer of a multi-GPU exchange point, relative to the L or U arena.
struct XferSpec {
    int32_t op;         // MF_XFER_*
    int32_t peer;       // root of a broadcast / peer of a send or receive
    int32_t in_U;       // 0: L arena, 1: U arena
    int64_t off, words; // fp64 words
};
constexpr int32_t kDistLeaves = 4;   // distribution block of a top front = kDistLeaves leaves of w columns

struct Launch {
    int32_t kind;       // KernelClass
    int32_t param;      // KC_SMALL: class fmax; KC_POTRF/KC_TRSM: j0
    int64_t off, count; // offset/count into the kind's task array
    double flops;       // algorithmic flops of this launch
    double bytes;       // algorithmic HBM bytes of this launch
    int32_t level;
    int64_t off2 = 0, count2 = 0;   // KC_LEAF: the trsm tasks (off/count = the fronts); KC_PANEL: count2 = blocks
    int32_t stream = -1;            // single GPU: subtree branch (its own stream), -1 = the main stream
    // look-ahead (main stream only): side = 1 runs this launch on the low-priority
    // side stream, forked from the main stream at this point; join = 1 makes the
    // main stream wait for the side stream before this launch
    int32_t side = 0, join = 0;
    // KC_UPDATE on the int8 tensor cores (Ozaki): oprobs [oz_p, oz_p + oz_np), split
    // tasks (triples) [oz_s, oz_s + oz_ns), tiles [oz_t, oz_t + oz_nt); exponent
    // words [oz_e, oz_e + oz_ne) of the scratch
    int32_t oz = 0;
    int32_t oz_wide = 0;   // Ozaki tiles of 128 x 128 (two-pass kernel) instead of 128 x 64
    double int8_ops = 0;   // int8 MMA operations of an Ozaki launch
    int64_t oz_p = 0, oz_np = 0, oz_s = 0, oz_ns = 0, oz_t = 0, oz_nt = 0, oz_e = 0, oz_ne = 0;
};

// Triangular-solve program (forward sweep bottom-up, backward sweep top-down).
enum SolveKind : int32_t {
    SK_SMALL_F = 0,   // one CTA per small supernode: gather, trsv, gemv
    SK_INIT_F = 1,    // large supernodes: v = [y(cols); 0] + children's update vectors (levels of many fronts;
                      // otherwise the init tasks run in the SK_DF_F launch)
    SK_DF_F = 2,      // all large supernodes of a level, one launch: 256-row chunks, per-block flags
    SK_SMALL_B = 3,
    SK_INIT_B = 4,    // large supernodes: v(k:f) = x(R(k:f)) (idem, SK_DF_B)
    SK_DF_B = 5       // all large supernodes of a level, one launch: chunk partials, owner reduces + trsv
};
struct SolveLaunch {
    int32_t kind;
    int32_t j0;   // factor launches: first column; SK_DF_*: 1 = deep register ring
    int64_t off, count;
    // SK_DF_*: the level's init tasks [off2, off2 + count2) run in the same launch
    // (lower tickets; the dataflow tasks wait for their completion count)
    int64_t off2 = 0, count2 = 0;
};
constexpr int kTkWords = 4;   // words per launch slot: ticket, finished CTAs, fused-init count, (spare)

struct Plan {
    int32_t nsuper = 0, nlevels = 0, w = 64, small_max = 128, max_front = 0;
    int64_t L_words = 0, U_words = 0, rows_total = 0, relmap_total = 0, fv_words = 0;
    // per supernode (host copies; device mirrors in the ctx)
    std::vector<int32_t> sn_k, sn_f, sn_ld, sn_level;
    std::vector<int64_t> L_off, U_off, fv_off;
    std::vector<int32_t> child_ptr, child_list;      // children ascending
    std::vector<int64_t> relmap_ptr;                 // per supernode (as a child)
    std::vector<int32_t> relmap;                     // positions of R_c[k_c:] in R_parent
    std::vector<int32_t> blrow;                      // local row in the front of each B entry
    // schedule
    std::vector<int32_t> level_ptr, level_list;      // all supernodes by level (solve)
    std::vector<int32_t> small_list, small_class_fmax;
    std::vector<int32_t> variant;                    // per supernode: kernel-variant class (kVariantFmax)
    std::vector<int32_t> large_list;
    std::vector<int32_t> asm_tasks;                  // pairs (front, c0)
    std::vector<int32_t> trsm_tasks;                 // pairs (front, row0)
    std::vector<int32_t> panel_tasks;                // pairs (front, 64-row tile row), row-major over the fronts
    std::vector<GemmProb> probs;
    std::vector<TileTask> tiles;
    std::vector<int32_t> ea_qs;                      // fused extend-add: per (syrk problem, child) tile-row starts
    int32_t fuse_ea = 0;
    int32_t nside = 0;                               // look-ahead forks in the program
    std::vector<Launch> program;
    // solve
    std::vector<int32_t> solve_list;                 // supernode lists (small / large) per launch
    std::vector<int32_t> df_tasks;                   // dataflow solve: (front, chunk) pairs
    std::vector<int64_t> df_part_off;                // per supernode: base of its backward x slots (k words)
    int64_t df_nparts = 0;                           // fp64 x-slot words
    std::vector<int64_t> df_seg_off;                 // per supernode: backward tail-segment partials (-1: none)
    int64_t df_nseg_words = 0;
    // inverses of the 64 x 64 diagonal blocks of the dataflow-solved supernodes (solve setup,
    // computed once per factorization by the first solve): per supernode the word offset of
    // its ceil(k / 64) column-major 64 x 64 blocks; (supernode, block) task pairs
    std::vector<int64_t> dinv_off;
    std::vector<int32_t> dinv_tasks;
    int64_t dinv_words = 0;
    std::vector<SolveLaunch> fsolve, bsolve;
    // ---- multi-GPU: subtree-to-GPU mapping.  Subtrees below a
    // frontier are factored by their owner; the supernodes above the frontier ("top")
    // are replicated on every rank after the frontier roots' update matrices are
    // broadcast, and the large ones are factored cooperatively (block-cyclic pivot
    // columns, split trailing updates, all-gathered U^n).
    int32_t nranks = 1, rank = 0, split_all = 0;
    int32_t nbranch = 1;                             // single GPU: subtree branches actually used
    std::vector<int32_t> branch;                     // per supernode: its branch, -1 = top (main stream)
    std::vector<int32_t> owner;                      // rank factoring each supernode
    std::vector<char> top;                           // above the frontier (replicated)
    std::vector<char> dist;                          // top fronts factored cooperatively
    std::vector<int32_t> frontier_roots;             // subtree roots whose parent is top
    std::vector<double> rank_load;                   // executed flops per rank (subtrees)
    double top_load = 0;
    std::vector<Launch> program_top;                 // every rank: top supernodes, with exchange points
    std::vector<std::vector<XferSpec>> xfers;        // transfer groups of the KC_EXCHANGE entries
    std::vector<SolveLaunch> fsolve_top, bsolve_top; // rank 0: top supernodes
    // ---- Ozaki-scheme Schur updates (ozaki_slices > 0)
    int32_t oz_slices = 0;
    std::vector<OzProb> oz_probs;
    std::vector<OzTile> oz_tiles;
    std::vector<int32_t> oz_split;                   // (oprob, 128-row block, k segment) triples
    int64_t oz_scratch_bytes = 0, oz_expo_words = 0; // per-stream regions, summed
    std::vector<int32_t> top_list, own_list;         // supernode lists (copy / mask kernels)
};

constexpr int kTileM = 64, kTileN = 64;
constexpr int kAsmCols = 16;
constexpr int kAsmRowBlock = 2048;   // assembly tasks split tall fronts into row blocks of this many rows
constexpr int kTrsmRows = 128;
constexpr int kSmallClasses = 5;
constexpr int kSolveRowBlock = 64;    // dataflow forward solve: rows per task (a multiple of the block width w)
// solve: one warp per front for f <= 128, and for f <= kSolveSmallMax when k <= kSolveSmallK
// (tools/gpu/job_solve_small.sh: c5 6.43 -> 5.73 ms, c2 1.74 -> 1.66, c3 unchanged)
constexpr int kSolveSmallMax = 256, kSolveSmallK = 32;
constexpr int kSolveDeepK = 256;      // dataflow solve: levels with a front of k >= this take the deep ring
constexpr int kSolveInitRows = 2048;
constexpr int kSolveFuseInitMax = 256;   // levels with at most this many init tasks run them in the dataflow launch
constexpr int kSolveSegSlabs = 16;    // dataflow backward solve: 64-row tail slabs per segment task  // solve init: front-vector rows per task (kernels.cu kInitRows)

int build_plan(const Symbolic &S, const Options &opt, Plan &P);

}  // namespace mf
