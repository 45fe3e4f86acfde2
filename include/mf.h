/*
 * mf.h -- C ABI of libmf, the B200 (sm_100a) implementation of the Mille-feuille hot path:
 * a tile-grained mixed-precision, single-kernel CG / BiCGSTAB solver
 * (Yang et al., SC'24; "P:<n>" cites /root/reference/PAPER.md line n).
 *
 * Conventions (every entry point):
 *  - Plain C types only.  Pointers are DEVICE pointers unless marked "host".
 *  - Every call is ordered on `stream` (a cudaStream_t; NULL = the legacy default stream).
 *    Calls that return results to the host (info / export / solve) synchronise `stream`.
 *  - Nothing throws.  A non-OK mf_status is returned; mf_last_error() gives a thread-local
 *    detail string.  Argument and CSR validation happen before any device work.
 *  - The caller owns every input buffer; buffers are read, never retained, and must stay
 *    valid until `stream` has passed the call.  The library owns handles (mf_tile_matrix,
 *    mf_precond) and their workspaces; *_destroy frees them.  Workspace memory
 *    comes from the allocator installed with mf_set_allocator (default: cudaMallocAsync).
 *  - At most one solve may be in flight per mf_tile_matrix.
 *  - Requires compute capability 10.0 (B200, sm_100a); otherwise MF_ERR_UNSUPPORTED_DEVICE.
 */
#ifndef MF_H
#define MF_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* mf_stream; /* ABI-identical to cudaStream_t */

typedef enum {
    MF_OK = 0,
    MF_ERR_INVALID_ARG = 1,        /* bad sizes / NULL / rowptr not 0..nnz monotone / col out of range */
    MF_ERR_UNSORTED_CSR = 2,       /* columns not strictly increasing within a row */
    MF_ERR_NONFINITE = 3,          /* a NaN / Inf value in the matrix */
    MF_ERR_OOM = 4,
    MF_ERR_CUDA = 5,
    MF_ERR_NCCL = 6,
    MF_ERR_BREAKDOWN = 7,          /* CG: (mu,p) <= 0 or non-finite; BiCGSTAB: (mu,r^), omega, rho == 0 */
    MF_ERR_ZERO_PIVOT = 8,         /* ILU(0): zero or missing diagonal */
    MF_ERR_DEADLOCK = 9,           /* a grid-barrier spin watchdog expired */
    MF_ERR_UNSUPPORTED_DEVICE = 10,
    MF_ERR_NOT_IMPLEMENTED = 11,
    MF_ERR_UNSUPPORTED = 12        /* a structural limit (e.g. > 4096 tiles in one tile row) */
} mf_status;

/* Precision codes; larger = lower precision (P:58 four data types; FP8 = OCP E4M3FN). */
typedef enum { MF_FP64 = 0, MF_FP32 = 1, MF_FP16 = 2, MF_FP8_E4M3 = 3, MF_BYPASS = 4 } mf_prec;

/* MF_MODE_FP64 and MF_MODE_STATIC_MIXED both compute every tile at its stored precision
 * TilePrec (they differ only in how the matrix was converted: convert_opts.classify = 0 makes
 * every tile FP64).  MF_MODE_DYNAMIC_MIXED adds the partial-convergence switch of Section III-D
 * (P:170-239): per SpMV, each tile column is lowered or bypassed from the level of its
 * 16-element segment of the SpMV input vector. */
typedef enum { MF_MODE_FP64 = 0, MF_MODE_STATIC_MIXED = 1, MF_MODE_DYNAMIC_MIXED = 2 } mf_mode;

typedef enum { MF_PRECOND_NONE = 0, MF_PRECOND_ILU0 = 1 } mf_precond_kind;

typedef struct mf_tile_matrix mf_tile_matrix;
typedef struct mf_precond mf_precond;

/* ---------------------------------------------------------------- conversion */
typedef struct {
    int32_t classify;     /* 1 (default): per-nonzero criterion of P:58; 0: every tile FP64 */
    double loss_tol;      /* 1e-15: relative loss below which a lower precision is "good enough" */
    int32_t grid_ctas;    /* persistent-kernel CTAs G; 0 = auto.  Fixes the dot-reduction tree. */
    int32_t block_threads;/* threads per CTA B (multiple of 32, <= 1024); 0 = auto */
    int32_t layout;       /* kernel slice layout: 0 auto, 1 compact (row-packed), 2 tile-synchronous */
} mf_convert_opts;

typedef struct {
    int64_t n_rows, n_cols, nnz;
    int32_t T;                 /* tile size: 16 */
    int64_t tilenum;           /* tiles (P:118 tilenumA) */
    int64_t rownum;            /* non-empty tile rows (P:124 rownumA) */
    int64_t n_tile_rows;       /* ceil(n_rows / 16) */
    int64_t tiles_per_prec[4]; /* tiles by TilePrec, [FP64, FP32, FP16, FP8] */
    int64_t nval[4];           /* nonzeros stored in each typed value array */
    int64_t max_tiles_per_tile_row;
    int64_t slots;             /* padded nonzero slots of the kernel layout (16 per slice column) */
    int64_t canonical_bytes;   /* bytes of the canonical arrays (Fig. 13 analog) */
    int64_t csr_bytes;         /* bytes of the input CSR (int64 rowptr, int32 col, f64 val) */
    int64_t kernel_bytes;      /* bytes of the kernel layout (index + value planes) */
    int32_t plan_G, plan_B;    /* launch plan: G CTAs of B threads; CTA g owns rows [R_g, R_{g+1}) */
    double convert_ms;         /* device time of the conversion (Fig. 14 analog) */
    int64_t convert_launches;  /* kernels the conversion launched */
    int32_t layout;            /* 1 compact, 2 tile-synchronous */
} mf_tile_info;

/* Canonical arrays (bit-exact contract).  HOST buffers,
 * allocated by the caller with the sizes from mf_tile_info; a NULL pointer skips that array. */
typedef struct {
    int32_t* TileRowidx;  /* [tilenum] tile row, tiles sorted by (row, col) */
    int32_t* TileColidx;  /* [tilenum] tile column */
    uint8_t* TilePrec;    /* [tilenum] mf_prec of the stored values */
    uint8_t* Floor;       /* [tilenum] range floor: lowest precision allowed by the value range */
    int64_t* TileNnz;     /* [tilenum+1] exclusive prefix of nonzeros per tile */
    int64_t* Nonrow;      /* [tilenum+1] exclusive prefix of non-empty rows per tile */
    int64_t* ValOff;      /* [tilenum] element offset of the tile's values in its precision's array */
    int64_t* TileRowPtr;  /* [n_tile_rows+1] CSR-of-tiles */
    uint8_t* RowIndex;    /* [rownum] local row (0..15) of each non-empty tile row */
    uint8_t* CsrRowptr;   /* [rownum] tile-local offset of the row's first nonzero */
    uint8_t* CsrColidx;   /* [nnz] local column (0..15) */
    double* Val64;        /* [nval[0]] */
    float* Val32;         /* [nval[1]] */
    uint16_t* Val16;      /* [nval[2]] IEEE binary16 bits */
    uint8_t* Val8;        /* [nval[3]] E4M3FN bits */
    int64_t* PlanRows;    /* [plan_G+1] R_g (row boundaries of the launch plan) */
} mf_tile_export;

/* ---------------------------------------------------------------- solves (Alg. 1-3) */
typedef struct {
    double tol;                 /* stop when ||r_j|| / ||b|| < tol (1e-10) */
    int64_t max_iter;           /* 1000 */
    mf_mode mode;               /* default MF_MODE_DYNAMIC_MIXED */
    double switch_eps;          /* eps of P:174; < 0 = default (= tol, reading R8); tau = eps*||v0||_2 */
    int32_t switch_absolute;    /* 0: tau = eps*||v0||_2 (reading R8); 1: tau = eps (Alg. 1 l.3) */
    int32_t sticky;             /* 1 (dynamic mode): one-time in-place downgrade (P:237 literal) -- a tile
                                   lowered to e_t keeps its values rounded to e_t for the rest of the solve
                                   (successive RNE, oracle spmv_tiles).  Both kernel layouts; not combined
                                   with level statistics (MF_ERR_NOT_IMPLEMENTED) */
    int32_t range_guard;        /* 1 (default): never lower a tile below its range floor */
    const mf_precond* M;        /* NULL = no preconditioner; else PCG / right-preconditioned PBiCGSTAB */
    double* residual_history;   /* host, optional: relres_0 .. relres_k (k+1 values) */
    int64_t history_cap;
    int64_t* tile_level_counts; /* host, optional: 5 per SpMV: tiles at FP64,FP32,FP16,FP8, bypassed */
    int64_t level_counts_cap;   /* number of SpMVs that fit */
    int32_t collect_stats;      /* 1: count tiles / nonzeros per effective precision in every SpMV
                                   (exact dynamic byte model; costs ALU in the SpMV loop).
                                   Implied when tile_level_counts != NULL. */
    int32_t watchdog_ms;        /* spin watchdog of the grid barriers / ready flags / SpTRSV (0 = 60000 ms);
                                   expiry returns MF_ERR_DEADLOCK */
    int32_t cg_variant;         /* mf_cg_solve: 0 (default) Alg. 1 (two grid reductions per iteration);
                                   1 single-reduction CG (Chronopoulos-Gear; one reduction, the dynamic
                                   switch watching r, the SpMV input of that variant) */
    int32_t dist_mode;          /* *_solve_dist only: 0 (default) auto = the device-initiated single kernel
                                   for CG (2 below), the host-orchestrated path for BiCGSTAB; 1 host-
                                   orchestrated kernels + NCCL between them; 2 device-
                                   initiated: ONE persistent kernel per rank that stores the halo
                                   into the peers' windows over NVLink and reduces across ranks
                                   itself (Finding 2, across GPUs) */
} mf_solve_opts;

typedef struct {
    int64_t iterations;        /* iterations performed (CG: SpMVs in the loop; BiCGSTAB: 2 SpMVs each) */
    int32_t converged;
    mf_status status;          /* MF_OK or MF_ERR_BREAKDOWN / MF_ERR_DEADLOCK (also the return value) */
    double rel_residual;       /* last recurrence ||r||/||b|| */
    double kernel_ms;          /* device time of the solve (persistent kernel, CUDA events) */
    double model_bytes;        /* algorithmic bytes moved */
    int64_t n_spmv;
    int64_t launches;          /* kernels launched by the solve */
    double barrier_ms;         /* mean over CTAs of time spent spinning in grid barriers / ready flags */
    double phase_ms[12];       /* mean over CTAs of time per kernel phase */
    int32_t ring_slots;        /* TMA ring depth of the SpMV (tile-synchronous layout) */
    int32_t mu_onchip;         /* 1: the SpMV outputs stayed in shared memory across the barrier */
} mf_solve_info;

void mf_default_convert_opts(mf_convert_opts* o);
void mf_default_solve_opts(mf_solve_opts* o);

/* Device-memory hook (torch's caching allocator in the Python binding). */
mf_status mf_set_allocator(void* (*alloc)(size_t bytes, mf_stream s, void* ctx),
                           void (*dealloc)(void* ptr, mf_stream s, void* ctx), void* ctx);

/* CSR -> two-level tiles with per-tile precision; rowptr int64[n_rows+1],
 * colidx int32[nnz] strictly increasing per row, vals f64[nnz]; all DEVICE pointers. */
mf_status mf_tile_matrix_from_csr(int64_t n_rows, int64_t n_cols, int64_t nnz, const int64_t* rowptr,
                                  const int32_t* colidx, const double* vals, const mf_convert_opts* opts,
                                  mf_stream stream, mf_tile_matrix** out);
mf_status mf_tile_matrix_destroy(mf_tile_matrix* A);
mf_status mf_tile_matrix_info(const mf_tile_matrix* A, mf_tile_info* out /* host */);
mf_status mf_tile_matrix_export(const mf_tile_matrix* A, mf_tile_export* host, mf_stream stream);

/* y = A~ x (Alg. 5).  level: per 16-element segment of x (mf_prec or MF_BYPASS), NULL = every
 * tile at TilePrec.  range_guard as in mf_solve_opts.  counts: host, optional, 5 int64. */
mf_status mf_spmv(const mf_tile_matrix* A, const double* x, double* y, const uint8_t* level,
                  int32_t range_guard, int64_t* counts, mf_stream stream);
/* Convergent-element retrieval (Alg. 4): level[J] of each 16-element segment of v
 * from thresholds th (host, 4 non-decreasing doubles; otherwise MF_ERR_INVALID_ARG). */
mf_status mf_levels(const double* v, int64_t n, const double* th, uint8_t* level, mf_stream stream);
/* (u, v) with the matrix's launch-plan reduction tree; host result. */
mf_status mf_dot(const mf_tile_matrix* A, const double* u, const double* v, double* out, mf_stream stream);

/* ILU(0) preconditioner of the stored matrix.  z = M^-1 r via SpTRSV kernels.
 * Factorisation on the host (IKJ order, FP64 factors of the stored values; setup, not per iteration).
 * Triangular solves (mf_precond_opts.sptrsv):
 *  - MF_SPTRSV_SYNC_FREE: row-by-row substitution, rows grabbed in chunks, per-row ready flags;
 *  - MF_SPTRSV_RECURSIVE_BLOCK: the recursive block SpTRSV of P:166 ([41]): each triangle of rows
 *    [lo, hi) splits at mid = lo + 16*floor((hi-lo)/32) into two triangles (solved recursively,
 *    rb_depth levels; leaves by the sync-free solve) and one square block (an SpMV s = T v, then
 *    rhs -= s).  mf_precond_apply runs it as one kernel per node (the paper's multi-kernel method);
 *    the persistent PCG / PBiCGSTAB kernels run the same node sequence with grid barriers between
 *    nodes.  rb_depth 0 = auto (leaves of about 2^14 rows).  Results equal the oracle's
 *    rb_lower / rb_upper bit for bit (reading R27).
 * mf_precond_create(A, kind, ...) == mf_precond_create_ex with sptrsv = MF_SPTRSV_SYNC_FREE. */
typedef enum { MF_SPTRSV_SYNC_FREE = 0, MF_SPTRSV_RECURSIVE_BLOCK = 1 } mf_sptrsv_algo;
typedef struct {
    mf_precond_kind kind;   /* MF_PRECOND_ILU0 */
    int32_t sptrsv;         /* mf_sptrsv_algo */
    int32_t rb_depth;       /* recursive block levels, 1..24; 0 = auto */
} mf_precond_opts;
mf_status mf_precond_create(const mf_tile_matrix* A, mf_precond_kind kind, mf_stream stream, mf_precond** out);
mf_status mf_precond_create_ex(const mf_tile_matrix* A, const mf_precond_opts* opts, mf_stream stream, mf_precond** out);
/* Scheduling of the triangular solves (either algorithm above): the library measures the depth of
 * the L and U dependency DAGs at creation; with fewer than 64 rows per level on average (e.g. C4:
 * 2^20 rows, 2.8e5 levels) the triangles -- or the recursive-block leaves -- are solved by ONE CTA
 * sweeping 32-row windows (warp shuffles inside a window, shared-memory ready counters between
 * windows) instead of grid-wide chunks with global ready flags; the arithmetic is identical.
 * Every fma chain runs in the order the substitution produces the unknowns: forward ascending
 * column, backward descending column (reading R20). */
typedef struct {
    int32_t rb_depth;           /* 0: substitution over the whole factor */
    int32_t nodes_l, nodes_u;   /* recursive block nodes (0 without) */
    int32_t sweep;              /* 1: one-CTA sweep schedule */
    int64_t depth_l, depth_u;   /* levels of the L / U dependency DAGs */
    int64_t nnz_l, nnz_u;       /* strict-triangle entries of the factors */
} mf_precond_stats;
mf_status mf_precond_info(const mf_precond* M, mf_precond_stats* out /* host */);
mf_status mf_precond_destroy(mf_precond* M);
mf_status mf_precond_apply(const mf_precond* M, const double* r, double* z, mf_stream stream);

/* Solve A x = b.  x: in x0, out x (device, n).  info: host.  CG for SPD, BiCGSTAB otherwise. */
mf_status mf_cg_solve(const mf_tile_matrix* A, const double* b, double* x, const mf_solve_opts* opts,
                      mf_solve_info* info, mf_stream stream);
mf_status mf_bicgstab_solve(const mf_tile_matrix* A, const double* b, double* x, const mf_solve_opts* opts,
                            mf_solve_info* info, mf_stream stream);

/* ---------------------------------------------------------------- multi-GPU (row blocks)
 * The paper's solver is single-GPU; the build partitions matrices too large for one GPU
 * (BASELINE configs[4]) into contiguous blocks of whole 16-row tile rows, one block per GPU, one
 * process per GPU.  Communication is inside libmf (NCCL communicator, NVLink): the caller only
 * ships the 128-byte unique id from rank 0 to the other ranks (e.g. with torch.distributed).
 *
 * Rank k owns rows [row_begin, row_end) (row_begin a multiple of 16; the blocks of all ranks are
 * contiguous, in rank order, and cover the matrix).  It converts its rows as a local tile matrix
 * whose columns are [the halo segments of lower ranks | its own segments | the halo segments of
 * higher ranks], each part ascending: one-to-one with global segments and in global order, so
 * tiles, TilePrec, the dynamic levels of Alg. 4 AND every row's fma order are the global
 * matrix's.  Every dot is the sum, in rank order from +0, of the rank partials (each the launch
 * plan's tree over the rank's CTAs): identical on every rank, deterministic, and equal to the
 * oracle's rank-partitioned plan.  Two executions (mf_solve_opts.dist_mode):
 *  - device-initiated (CG default): one cooperative persistent kernel per rank; producers store
 *    their boundary segments into the peers' windows (NCCL symmetric windows, peer pointers from
 *    the NCCL device API) and count arrivals with system-scope release adds; rank partials are
 *    stored, tagged, into every rank's window; no host involvement per iteration;
 *  - host-orchestrated: the same steps as separate kernels with ncclSend/Recv and ncclAllGather
 *    between them, iterations enqueued as CUDA graphs with a device stop flag.
 * All calls are collective over the communicator's ranks. */
typedef struct mf_comm mf_comm;
/* host: 128 bytes (ncclUniqueId), created on rank 0 and broadcast to the others by the caller */
mf_status mf_nccl_unique_id(void* out);
mf_status mf_comm_create(const void* nccl_unique_id, int32_t nranks, int32_t rank, mf_comm** out);
mf_status mf_comm_destroy(mf_comm* comm);
mf_status mf_comm_info(const mf_comm* comm, int32_t* nranks, int32_t* rank);
/* In-process rank group: nranks host threads of ONE process each drive one rank, all ranks on the
 * current device (their windows are same-device buffers).  Runs the device-initiated kernel only
 * (each rank's thread must use its own stream; the kernels run concurrently, so the plan's CTAs of
 * all ranks must fit the device together: convert with grid_ctas <= SMs / nranks).  Verifies the
 * multi-rank exchange on a single GPU.  The group outlives its comms. */
typedef struct mf_local_group mf_local_group;
mf_status mf_local_group_create(int32_t nranks, mf_local_group** out);
mf_status mf_local_group_destroy(mf_local_group* g);
mf_status mf_comm_create_local(mf_local_group* g, int32_t rank, mf_comm** out);
/* rowptr int64[row_end-row_begin+1] (local, from 0), colidx int32[nnz_local] GLOBAL columns
 * (strictly increasing per row), vals f64[nnz_local]; device pointers.  The handle is freed with
 * mf_tile_matrix_destroy; mf_tile_matrix_info / export describe the LOCAL matrix. */
mf_status mf_tile_matrix_from_csr_dist(mf_comm* comm, int64_t n_global, int64_t row_begin, int64_t row_end,
                                       int64_t nnz_local, const int64_t* rowptr, const int32_t* colidx,
                                       const double* vals, const mf_convert_opts* opts, mf_stream stream,
                                       mf_tile_matrix** out);
/* local slices: b[row_end-row_begin], x (in x0, out x); info (host) is the global solve's (every
 * rank gets the same iterations / residual history).  Preconditioning / sticky / level
 * statistics: MF_ERR_NOT_IMPLEMENTED. */
mf_status mf_cg_solve_dist(const mf_tile_matrix* A, const double* b, double* x, const mf_solve_opts* opts,
                           mf_solve_info* info, mf_stream stream);
mf_status mf_bicgstab_solve_dist(const mf_tile_matrix* A, const double* b, double* x, const mf_solve_opts* opts,
                                 mf_solve_info* info, mf_stream stream);
/* host: this rank's row block, halo segments received and own segments sent per exchange */
mf_status mf_dist_info(const mf_tile_matrix* A, int64_t* row_begin, int64_t* row_end, int64_t* halo_segments,
                       int64_t* send_segments);

/* Host-only planner (no GPU): the global 16-element column segments that rank `rank`'s rows gather
 * outside its own block (ascending; the first halo_cap written to halo_segments, host, nullable),
 * their count (*nhalo) and how many each rank owns (recv_counts[nranks], host).  rank_rows
 * [nranks+1] host row boundaries; colidx host, global.  The device plan of
 * mf_tile_matrix_from_csr_dist is the same. */
mf_status mf_dist_plan(int64_t n_global, int32_t nranks, const int64_t* rank_rows, int32_t rank, int64_t nnz,
                       const int32_t* colidx, int64_t* recv_counts, int32_t* halo_segments, int64_t halo_cap,
                       int64_t* nhalo);

/* Per-rank steps of the classic multi-kernel CG (Alg. 1 steps C and D) on a
 * matrix's rows, with the launch plan's reduction tree: the comparison path of SURVEY 8(f) f3. */
/* x += alpha p ; r = fma(-alpha, mu, r) on the matrix's rows; *rr (host) = (r, r), plan tree. */
mf_status mf_cg_update_xr(const mf_tile_matrix* A, double alpha, const double* p, const double* mu, double* x,
                          double* r, double* rr, mf_stream stream);
/* p = fma(beta, p, r) on the matrix's rows. */
mf_status mf_cg_update_p(const mf_tile_matrix* A, double beta, const double* r, double* p, mf_stream stream);

const char* mf_status_string(mf_status s);
const char* mf_last_error(void);
int32_t mf_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* MF_H */
