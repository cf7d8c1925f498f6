/*
 * tqr.h -- C ABI of the B200-native tiled Householder QR (Kim & Park, ICPP'13).
 *
 * Problem statement: A = QR with Q orthogonal (Q^T Q = Q Q^T = I) and R upper
 * triangular, Eq. (1); A x = b solved as R x = Q^T b, Eqs. (2)-(3) P:L181-188,
 * P:L242.  The method is the tiled QR of Sec. II.B: Triangulation (GEQRT,
 * Eqs. 4-5), update for triangulation (UNMQR, Eq. 6, applied as Q^T -- reading Q5),
 * Elimination (TSQRT, Eqs. 7-8) and update for elimination (TSMQR, Eq. 9), over square
 * nb x nb tiles.  Column tiles are distributed to devices by the distribution
 * guide array, Eq. (12) P:L1026 (Algorithm 4).
 *
 * Conventions for every entry point:
 *   - Every call returns tqr_status (TQR_OK = 0).  No C++ exception, abort or exit crosses
 *     the ABI.  A failed call leaves a message retrievable with tqr_last_error().
 *   - Matrices are column-major: element (i, j) of X with leading dimension ldx is
 *     X[i + j*ldx], in the plan's dtype.
 *   - Pointers may be host memory (pageable or pinned) or device memory of the plan's
 *     first device; the library detects which with cudaPointerGetAttributes.  The caller
 *     owns its buffers; the plan never frees or retains them past the call.
 *   - Calls are synchronous: each call that touches a caller buffer first waits for all work
 *     already queued on the buffer's / plan's devices (any stream), and on return every result
 *     is in the caller's buffer.
 *   - A CUDA or NCCL failure poisons the plan: later calls return TQR_ERR_STATE until
 *     tqr_destroy.  A plan is not thread-safe; distinct plans are independent.
 */
#ifndef TQR_H_
#define TQR_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct tqr_plan_s* tqr_plan;

typedef enum { TQR_F64 = 0, TQR_F32 = 1 } tqr_dtype;

typedef enum {
    TQR_OK = 0,
    TQR_ERR_ARG = 1,         /* invalid argument (sizes, guide entries, NULL pointer, ld < m) */
    TQR_ERR_ALLOC = 2,       /* device or pinned-host allocation failed */
    TQR_ERR_CUDA = 3,        /* a CUDA runtime call or kernel failed (plan is poisoned) */
    TQR_ERR_NCCL = 4,        /* NCCL missing or an NCCL call failed (plan is poisoned) */
    TQR_ERR_STATE = 5,       /* call not valid in the plan's state (e.g. apply before factor) */
    TQR_ERR_SINGULAR = 6,    /* solve: some R_ii == 0 exactly (LAPACK dtrtrs convention) */
    TQR_ERR_UNSUPPORTED = 7  /* valid request this build does not implement (dtype/nb/ib combo) */
} tqr_status;

/* Options for tqr_create_ex.  Zero-initialise, then set what you need. */
typedef struct {
    /* 1: all ndev column owners live on the calling thread's current CUDA device
     * ("logical devices"); panel broadcasts become device-to-device copies.  Exercises the
     * guide-array partition and broadcast ordering on one GPU.  0: owner d uses CUDA
     * device d (single-process) or this process's device (multi-process). */
    int32_t logical_devices;
    /* Multi-process mode, one process per owner: world > 1 (or world <= 1 with a non-NULL
     * nccl_id: a single-rank NCCL communicator), this process is `rank`; ndev must equal
     * max(world, 1).  The panel transport is chosen by `transport` (below): NCCL needs nccl_id,
     * the 128-byte ncclUniqueId produced by tqr_nccl_unique_id() on rank 0 and shared out of band
     * (e.g. torch.distributed); IPC needs the tqr_ipc_handle / tqr_ipc_connect exchange. */
    int32_t rank;
    int32_t world;
    const void* nccl_id;
    /* 0 = disable the one-panel lookahead (plain step order), otherwise enabled (default). */
    int32_t no_lookahead;
    /* 1: record CUDA events around every update-kernel launch so tqr_kernel_stats() can
     * report the dominant kernel's device time (bench.py roofline). */
    int32_t profile;
    /* Elimination tree (the paper's TT elimination): every panel
     * column is split into TS domains of L tiles, each factored (GEQRT of its head + TSQRT chain)
     * by one CTA concurrently, and the domain heads' R factors are merged by a TT chain; updates
     * and tqr_apply_qt replay the same tree.  0 = auto (tree for a single column tile, q == 1,
     * with L = ceil(p / SM count)), -1 = always flat TS, L > 0 = domains of L tiles (FP64 only). */
    int32_t tree_domain;
    /* Tree mode: how the D domain heads are merged.  0 = auto (two-level when D >= 16, groups of
     * ceil(sqrt(D))), -1 = one flat TT chain of D - 1 merges, G > 1 = two-level: the heads of each
     * group of G consecutive domains are merged into the group's first head by concurrent TT
     * chains, then the group heads into head 0 by one chain (G - 1 + ceil(D/G) - 1 sequential
     * merges instead of D - 1). */
    int32_t tree_group;
    /* Row split (NEXT-1 across devices; the paper's TT elimination P:L409-419 / TSQR): a single
     * column tile (n <= nb) is split into ndev contiguous row blocks, one per owner (device or
     * process); each owner factors its block (TS domains + merges), the owners' R factors are
     * gathered to owner 0 (NCCL all-gather in multi-process mode) and merged there by one more
     * factorisation of the stacked triu(R_g).  0 = auto (n <= nb, FP64, ndev > 1, >= 2 tiles per
     * owner), 1 = force, -1 = off (column partition: owner(0) does all the work).  Row-split
     * plans support tqr_factor / tqr_load / tqr_factor_tiles / tqr_store_r only. */
    int32_t row_split;
    /* Multi-process panel transport.  TQR_TRANSPORT_AUTO (0): NCCL when nccl_id is
     * given, otherwise IPC.  TQR_TRANSPORT_NCCL (1): ncclBroadcast of every panel from its owner
     * on a comm stream (one GPU per rank).  TQR_TRANSPORT_IPC (2): the panel owner copies V/T
     * straight into each receiving rank's CUDA-IPC-mapped receive slot (NVLink peer memory, or the
     * same HBM when several ranks share one GPU) and orders the copy with stream-ordered 64-bit
     * flags (cuStreamWaitValue64 / cuStreamWriteValue64): no NCCL, no SM spent on the transfer,
     * any number of ranks per GPU.  An IPC plan must be connected (tqr_ipc_handle on every rank,
     * all blobs exchanged out of band, tqr_ipc_connect) before its first factor. */
    int32_t transport;
} tqr_options;

#define TQR_TRANSPORT_AUTO 0
#define TQR_TRANSPORT_NCCL 1
#define TQR_TRANSPORT_IPC 2

/*
 * Create a plan for the QR factorisation of an m x n matrix.
 *   m, n      : matrix size, m >= n >= 1.  Any sizes: the tile grid is p = ceil(m/nb) x
 *               q = ceil(n/nb) and the ragged tails are zero-padded inside the plan (a zero
 *               padded column gets tau = 0 and padded rows stay zero, so R(0:n,0:n) and
 *               Q = diag(Q_m, I) restricted to the caller's m rows are unchanged).
 *   nb        : tile size (square tiles); supported 64, 128, 256, 512.
 *   ib        : inner blocking of the compact-WY T factors; 1 <= ib <= nb, nb % ib == 0;
 *               supported 16, 32.
 *   dtype     : TQR_F64 or TQR_F32 (FP32 tiles and updates; each panel is factored in FP64 and
 *               rounded once, reading Q9).  Tree mode (tree_domain > 0) is FP64 only.
 *   ndev      : number of column-tile owners (devices).
 *   guide     : distribution guide array (Alg. 4), entries in [0, ndev); column tile j is
 *               owned by guide[j % guide_len] (Eq. 12).  NULL -> {0, 1, ..., ndev-1}.
 *   out       : receives the plan (owned by the caller, release with tqr_destroy).
 * The plan owns all device memory (tile storage, T factors, panel receive buffers),
 * streams, events and (multi-process) the NCCL communicator.
 * Errors: TQR_ERR_ARG on invalid sizes/guide, TQR_ERR_UNSUPPORTED on unsupported combos,
 * TQR_ERR_ALLOC / TQR_ERR_CUDA / TQR_ERR_NCCL on resource failures (nothing is leaked).
 */
tqr_status tqr_create(int64_t m, int64_t n, int32_t nb, int32_t ib, tqr_dtype dtype,
                      int32_t ndev, const int32_t* guide, int32_t guide_len, tqr_plan* out);

/* As tqr_create with explicit options (opt may be NULL = all defaults). */
tqr_status tqr_create_ex(int64_t m, int64_t n, int32_t nb, int32_t ib, tqr_dtype dtype,
                         int32_t ndev, const int32_t* guide, int32_t guide_len,
                         const tqr_options* opt, tqr_plan* out);

/*
 * Factor A (m x n, lda >= m) in place: A = QR (Eq. 1).  On return A(0:n, 0:n) holds R in
 * its upper triangle and every entry below the diagonal of A is zero (the reflectors stay
 * inside the plan in tile layout for tqr_apply_qt / tqr_solve_ls).  In multi-process mode
 * A is the full matrix on every rank and each rank writes back the columns it owns.
 * The call runs a1 (layout convert), a2-a7 (tiled factorisation) and a8 (R out).  When A is
 * not resident on the owning device (host memory or another GPU), the column loads and the R
 * stores are pipelined with the factorisation (column k is written back as soon as its panel
 * is factored); the result is bitwise the same.
 */
tqr_status tqr_factor(tqr_plan h, void* A, int64_t lda);

/* The three phases of tqr_factor, for timing: tiles <- A; factor the resident tiles;
 * A <- R.  tqr_factor == tqr_load + tqr_factor_tiles + tqr_store_r. */
tqr_status tqr_load(tqr_plan h, const void* A, int64_t lda);
tqr_status tqr_factor_tiles(tqr_plan h);
tqr_status tqr_store_r(tqr_plan h, void* A, int64_t lda);

/*
 * B (m x nrhs, ldb >= m) <- Q^T B (trans 'T') or Q B (trans 'N'), with Q from the last
 * tqr_factor (Alg. 1 lines 13-14 read for the tiled factorisation).  Rows 0..n-1 of Q^T B
 * (and Q [C; 0]) are unique; rows n..m-1 of Q^T B depend on the tile algorithm.
 * TQR_ERR_STATE before a successful factor.
 * Several owners (logical devices, several GPUs, or ranks): the first apply/solve after a factor
 * gathers every panel's reflectors, T factors and R tiles onto the caller's device (peer copies;
 * ncclBroadcast from each column's owner; or IPC pulls from the owners' memory), then applies
 * there.  Multi-process plans: a collective -- every rank calls it with its own full B and gets
 * the full result; an IPC plan returns only when every rank has finished its pulls, so the next
 * factor cannot overwrite reflectors a peer is still reading.  Row-split plans: the owners apply
 * their blocks' Q_g, then the stage-2 plan's Q to the stacked top rows (single process only).
 */
tqr_status tqr_apply_qt(tqr_plan h, char trans, void* B, int64_t ldb, int64_t nrhs);

/*
 * Least squares min ||A X - B||_F via Eqs. (2)-(3): B <- Q^T B, then R X = B(0:n, :) by tile
 * back substitution on the resident R tiles; X is returned in B(0:n, :) (rows
 * n..m-1 unspecified).  B may be host or device memory (ldb >= m).
 * TQR_ERR_SINGULAR if some R_ii == 0 exactly (B unspecified).
 */
tqr_status tqr_solve_ls(tqr_plan h, void* B, int64_t ldb, int64_t nrhs);

/* Release everything the plan owns.  NULL-safe; always TQR_OK for a valid or NULL plan. */
tqr_status tqr_destroy(tqr_plan h);

/* Static description of a status code. */
const char* tqr_status_string(tqr_status s);

/* Message of the last failed call on h (or of the last failed tqr_create when h is NULL). */
const char* tqr_last_error(tqr_plan h);

/* Write a fresh 128-byte ncclUniqueId into id[0..127] (rank 0 of a multi-process plan).
 * TQR_ERR_NCCL if libnccl.so.2 cannot be loaded. */
tqr_status tqr_nccl_unique_id(void* id128);

/* CUDA-IPC transport handshake (tqr_options.transport = TQR_TRANSPORT_IPC, multi-process).
 * tqr_ipc_handle writes this rank's export blob (IPC handles of its receive slots, flag block and
 * reflector storage) into buf (capacity cap bytes; buf NULL = size query) and its size to *len
 * (the same on every rank).  The application all-gathers the blobs in rank order (e.g.
 * torch.distributed.all_gather_object) and passes the world * len concatenation to
 * tqr_ipc_connect, which opens every peer's memory (cudaIpcMemLazyEnablePeerAccess) and arms
 * the transfer flags.  TQR_ERR_STATE on a non-IPC plan or a second connect; TQR_ERR_ARG on a
 * blob of the wrong size or rank order; TQR_ERR_CUDA if a handle cannot be opened. */
tqr_status tqr_ipc_handle(tqr_plan h, void* buf, int64_t cap, int64_t* len);
tqr_status tqr_ipc_connect(tqr_plan h, const void* all, int64_t len);

/* The operations the last tqr_factor_tiles issued on this rank, in issue order, as the same
 * 5-int32 records tqr_schedule produces ({op, k, i, j, root}; UPDATE records one per column, in
 * the order the columns' launches were enqueued).  The executor consumes tqr_schedule's list,
 * so per step k the records are the schedule's (tests compare them).  cap/count as tqr_schedule. */
tqr_status tqr_issued_ops(tqr_plan h, int32_t* ops, int64_t cap, int64_t* count);

/* How the plan executes, as a bit mask (0 for NULL): TQR_PLAN_ROW_SPLIT (single column tile split by
 * rows across the owners), TQR_PLAN_TREE (TS domains + TT merges), TQR_PLAN_MULTIPROC (one process
 * per owner), TQR_PLAN_IPC / TQR_PLAN_NCCL (its panel transport), TQR_PLAN_F32. */
#define TQR_PLAN_ROW_SPLIT 1
#define TQR_PLAN_TREE 2
#define TQR_PLAN_MULTIPROC 4
#define TQR_PLAN_IPC 8
#define TQR_PLAN_NCCL 16
#define TQR_PLAN_F32 32
int32_t tqr_plan_flags(tqr_plan h);

/* Owner of column tile j under the plan's guide array (Eq. 12), or -1 if j is out of range. */
int32_t tqr_owner(tqr_plan h, int64_t j);

/*
 * Host-side schedule of the tiled DAG (Fig. 3) for rank `rank`: writes up to
 * cap records of 5 int32 {op, k, i, j, root} into ops and the total count into *count.
 * op: 0 = PANEL (GEQRT(k,k) + TSQRT(i,k) chain, on owner(k)), 1 = BCAST (panel k from
 * root = owner(k)), 2 = UPDATE (UNMQR(k,j) + TSMQR(i,j,k) chain for column j).  Pure host
 * logic (no GPU needed); used by the multi-process CPU tests.
 */
tqr_status tqr_schedule(int64_t m, int64_t n, int32_t nb, int32_t ndev, const int32_t* guide,
                        int32_t guide_len, int32_t rank, int32_t* ops, int64_t cap, int64_t* count);

/* Distribution guide array from integer per-device tile-update rates (Alg. 4 GET_RATIO +
 * GENERATE_ARRAY; ties -> lowest ID).  Writes sum(ratio) entries to guide
 * (capacity cap) and the length to *len. */
tqr_status tqr_generate_guide(const int32_t* rates, int32_t ndev, int32_t* guide, int32_t cap, int32_t* len);

/* Row split (tqr_options.row_split): owner g of ndev holds rows [r0[g], r0[g] + rows[g]) of an
 * m-row single-column-tile matrix -- the contiguous tile rows [g p / ndev, (g+1) p / ndev),
 * p = ceil(m / nb).  Host-only (used by tqr_create_ex and the multi-process CPU tests). */
tqr_status tqr_row_split_ranges(int64_t m, int32_t nb, int32_t ndev, int64_t* r0, int64_t* rows);

/* Measured average time (seconds) of one tile operation on a device (the paper's time_i(op),
 * P:L878-881): T = triangulation (GEQRT), E = elimination (TSQRT), UT = update for
 * triangulation (UNMQR), UE = update for elimination (TSMQR). */
typedef struct {
    double t_T, t_E, t_UT, t_UE;
} tqr_tile_times;

/* Main computing device selection, Algorithm 2 (reading Q22): the candidates can
 * finish T before every other device's UE and E before every other device's UT; the candidate
 * with the minimum update speed 1/(t_UT + t_UE) is returned (lowest ID on ties); no candidate
 * -> the fastest updater.  Host-only.  TQR_ERR_ARG on ndev < 1 / negative times. */
tqr_status tqr_select_main(int32_t ndev, const tqr_tile_times* t, int32_t* main_dev);

/* Number-of-devices selection, Algorithm 3 with Eqs. (10)-(11) (readings
 * Q23-Q25).  M x N tile grid of T x T tiles, elem_size bytes per element; t[ndev] per-tile
 * times; speed = ndev x ndev row-major link speeds in bytes/s (speed[x*ndev + y]: x -> y, > 0
 * off the diagonal; the diagonal is ignored = infinite); main_dev from tqr_select_main.
 * Outputs: order[ndev] (optional) = the device list (main first, then descending update
 * speed); Tp[ndev] (optional) = the predicted first-iteration time T(p) = Top(p) + Tcomm(p) for
 * p = 1..ndev (seconds); *pbest = the p minimising T(p): the first p devices of `order`
 * participate, distributed by tqr_generate_guide over their rates.  Host-only. */
tqr_status tqr_select_ndev(int32_t M, int32_t N, int32_t T, int32_t elem_size, int32_t ndev,
                           const tqr_tile_times* t, const double* speed, int32_t main_dev, int32_t* order,
                           double* Tp, int32_t* pbest);

/* Device-time statistics of the plan's kernels since the last reset (opt.profile = 1):
 * which = 0 update (UNMQR+TSMQR) kernel, 1 panel (GEQRT+TSQRT) kernel, 2 layout kernels (a1
 * to_tiles in tqr_load, a8 from_tiles in tqr_store_r), 3 panel transfers (BCAST: NCCL
 * broadcast, IPC copies or peer copies, from the transfer's start to the receive completing).
 * *count launches (transfers), *ms device-busy CUDA-event milliseconds (union of the intervals:
 * overlapping launches are not double counted), *flops algorithmic flops (which = 0, 1) or
 * bytes moved (which = 2, 3).  reset != 0 clears after reading. */
tqr_status tqr_kernel_stats(tqr_plan h, int32_t which, int64_t* count, double* ms, double* flops, int32_t reset);

/* Number of kernel launches the plan issued since the last call (then resets). */
int64_t tqr_launch_count(tqr_plan h);

#ifdef __cplusplus
}
#endif
#endif /* TQR_H_ */
