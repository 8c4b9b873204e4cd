/*
 * mpspmm.h -- C ABI of libmpspmm.so, a B200 (sm_100a) MergePath-SpMM.
 *
 * Computes the GCN aggregation C = A * B (the row-wise product of PAPER.md P:41-43,
 * sec. II) for a sparse m x n CSR matrix A and a dense, tall and thin n x K matrix B
 * (the paper's XW), scheduled by the merge path of Alg. 1 and
 * Alg. 2.  Citations "P:<line>" are lines of the paper text; DESIGN.md
 * lists every reading taken where the paper is garbled or silent ("R<k>").
 *
 * Conventions (all entry points):
 *  - Plain C: no C++ types, no exceptions cross this boundary.  Every function
 *    returns an mps_status; mps_last_error() gives a thread-local detail string.
 *  - Ownership: the caller allocates and frees every buffer (A, B, C, coordinates,
 *    workspace, tails).  The library keeps no global state and allocates nothing
 *    persistent; all functions are reentrant.  Everything a launch needs beyond its
 *    arguments lives in the caller's workspace -- including the counters from which
 *    the segment kernel's warps claim segments (one 32-bit word per column tile,
 *    zeroed on the stream by the call that uses them) -- so two calls (or two captured
 *    CUDA graphs) running concurrently must use different workspaces, and never
 *    interfere otherwise.  Host-side caches are per device and hold only occupancy
 *    and attribute queries.
 *  - Pointers are DEVICE pointers unless the parameter name ends in _host.
 *  - Streams: every device call is asynchronous on `stream` (a cudaStream_t passed
 *    as void*; NULL = the legacy default stream).  Only mps_validate_csr
 *    synchronises.
 *  - Index type: int32 row_ptr / col_idx through mps_csr (M = m + nnz must be < 2^31,
 *    else MPS_ERR_UNSUPPORTED, reading R16); int64 row_ptr through mps_csr64 and the
 *    *64 entry points (NEXT-4).
 *  - Multi-GPU calls (mps_spmm_shard*, mps_xw_bf16_bcast, mps_peer_*) take peer
 *    pointers mapped with the mps_ipc_* calls; collectives stay outside the library.
 *  - Errors: MPS_ERR_INVALID for NULL pointers with non-zero sizes, negative sizes,
 *    ldb < K, ldc < K, num_parts < 1, rank outside [0, world); MPS_ERR_UNSUPPORTED
 *    for M >= 2^31 or an unknown dtype; MPS_ERR_WORKSPACE if workspace_bytes is too
 *    small; MPS_ERR_CUDA if a launch or copy fails.  K == 0 or m == 0 is a no-op
 *    returning MPS_OK.  Misaligned B or C selects a narrower vector path, never an
 *    error.  CSR *content* (monotone row_ptr, columns in range) is NOT checked on the
 *    hot path -- the method needs no preprocessing; mps_validate_csr does it.
 */
#ifndef MPSPMM_H
#define MPSPMM_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t mps_status;
enum {
    MPS_OK = 0,
    MPS_ERR_INVALID = 1,
    MPS_ERR_UNSUPPORTED = 2,
    MPS_ERR_CUDA = 3,
    MPS_ERR_WORKSPACE = 4,
    MPS_ERR_COMM = 5
};

/* How rows split across merge-path segments are settled (a4). */
enum {
    MPS_FIXUP_AUTO = 0,   /* library choice: CARRY on the small-graph fused path
                           * (mps_spmm_online_path), ATOMIC otherwise                   */
    MPS_FIXUP_ATOMIC = 1, /* zero split rows, then one vector red.add per partial row  */
    MPS_FIXUP_CARRY = 2   /* partial rows to workspace, fixed-order reduction; deterministic */
};

/* Element type of B.  C is always fp32, accumulation always fp32 (reading R15). */
enum { MPS_DT_F32 = 0, MPS_DT_BF16 = 1 };

/* Fused epilogue applied to C (the GCN layer's sigma; NEXT-3 in SURVEY.md):
 * RELU stores max(C, 0).  Complete rows get it in the store; rows cut by a schedule
 * boundary get it after all their partial sums landed.                            */
enum { MPS_EPI_NONE = 0, MPS_EPI_RELU = 1 };

/* A: m x n CSR.  row_ptr[m+1] (row_ptr[0] = 0, row_ptr[m] = nnz), col_idx[nnz],
 * val[nnz]; columns need not be sorted, duplicates are summed (CSR).        */
typedef struct {
    int64_t m, n, nnz;
    const int32_t *row_ptr;
    const int32_t *col_idx;
    const float *val;
} mps_csr;

int mps_abi_version(void);
const char *mps_status_string(mps_status s);
const char *mps_last_error(void);

/* a1 -- schedule sizing (host only, no GPU needed).  Alg. 1 lines 2-3 and
 * sec. III-C: M = m + nnz; P = max(ceil(M / cost), min_parts);
 * L = ceil(M / P) (reading R1).  items_per_part (the paper's merge-path cost,
 * P:137) == 0 selects the library default, tuned on B200 (NEXT-1 sweep):
 * max(64, min(clamp(next_pow2(4*ceil(nnz/m)), 512, 2048),
 *             pow2_floor(M / (1.5 * resident warps of the current device))))
 * items per warp segment; min_parts (the paper's thread threshold) == 0
 * selects 1184 (8 per SM of 148).  Outputs P and L.                               */
mps_status mps_plan(int64_t m, int64_t nnz, int32_t K, int32_t b_dtype, int64_t items_per_part,
                    int64_t min_parts, int64_t *num_parts_out, int64_t *items_per_part_out);

/* a2 -- merge-path partition, Alg. 1 lines 4-7.  For p = 0..num_parts it
 * writes the coordinate of diagonal d_p = diag_begin + min(p*L, diag_end - diag_begin)
 * (L = items_per_part): x = max{x : x + row_ptr[x] <= d_p}, y = d_p - x
 * (readings R4, R5).  coord_x / coord_y: caller-owned device int32[num_parts+1].
 * Bit-exact; asynchronous on stream.                                              */
mps_status mps_partition(const int32_t *row_ptr, int64_t m, int64_t nnz, int64_t diag_begin,
                         int64_t diag_end, int64_t num_parts, int64_t items_per_part,
                         int32_t *coord_x, int32_t *coord_y, void *stream);

/* a2 + the atomic fix-up's precondition in ONE launch: mps_partition, and every row cut
 * by one of the diagonals (x_p < m, y_p > row_ptr[x_p]) gets its K floats of C zeroed
 * (C row r at C + r*ldc).  Equivalent to mps_partition followed by mps_zero_split_rows
 * (reading R10).  Asynchronous on stream.                                          */
mps_status mps_partition_split(const int32_t *row_ptr, int64_t m, int64_t nnz,
                               int64_t num_parts, int64_t items_per_part, int32_t *coord_x,
                               int32_t *coord_y, float *C, int64_t ldc, int32_t K,
                               void *stream);

/* a3+a4 -- offline SpMM with a precomputed schedule (computed once, reused).
 * C = A * B; C is overwritten entirely (it need not be initialised: complete rows
 * are stored, split rows are zeroed first or stored by the carry pass, empty rows
 * get 0).  B: n rows, leading dimension ldb elements (b_dtype); C: m rows, leading
 * dimension ldc floats.  workspace: caller-owned device memory of at least
 * mps_spmm_workspace_bytes(...) bytes (>= 256: the segment-claim counters, then the
 * carry records in carry mode); its content on entry does not matter.           */
mps_status mps_spmm_workspace_bytes(const mps_csr *A, int32_t K, int32_t b_dtype,
                                    int64_t num_parts, int32_t fixup, size_t *bytes);
mps_status mps_spmm(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb, int32_t K,
                    float *C, int64_t ldc, const int32_t *coord_x, const int32_t *coord_y,
                    int64_t num_parts, int32_t fixup, void *workspace, size_t workspace_bytes,
                    void *stream);

/* The two launches mps_spmm is made of, for callers that time or overlap them:
 * mps_zero_split_rows zeroes the rows cut by a boundary of the schedule (x_p < m,
 * y_p > row_ptr[x_p]; the atomic fix-up's precondition, reading R10);
 * mps_spmm_segments runs a3 (+ the a4 carry reduction) and, in atomic mode,
 * REQUIRES that mps_zero_split_rows ran earlier on the same C and schedule.  Its
 * workspace is sized by mps_spmm_workspace_bytes; for long schedules it zeroes the
 * claim counters there with one cudaMemsetAsync before the segment kernel.       */
mps_status mps_zero_split_rows(const mps_csr *A, const int32_t *coord_x, const int32_t *coord_y,
                               int64_t num_parts, float *C, int64_t ldc, int32_t K,
                               void *stream);
mps_status mps_spmm_segments(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                             int32_t K, float *C, int64_t ldc, const int32_t *coord_x,
                             const int32_t *coord_y, int64_t num_parts, int32_t fixup,
                             void *workspace, size_t workspace_bytes, void *stream);

/* The Fig. 5 statistic counted where the segment kernel writes: mps_spmm
 * (zeroing of the cut rows in atomic mode, then the segment kernel with its debug
 * counters on) writing C as mps_spmm does, and counts (device int64[3], zeroed first):
 *   [0] partial-row updates issued (Alg. 2 lines 5, 9, 13: red.add in atomic mode, a
 *       carry record in carry mode),
 *   [1] partial start pieces that are empty (the segment starts on a row's end item),
 *       whose add the kernel elides -- Alg. 2 counts them as updates, so [0] + [1] is
 *       the paper's #atomic,
 *   [2] complete-row stores (Alg. 2 line 15), the paper's #regular.
 * Column tile 0 is counted.  Same workspace as mps_spmm.                           */
mps_status mps_spmm_write_counts(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                                 int32_t K, float *C, int64_t ldc, const int32_t *coord_x,
                                 const int32_t *coord_y, int64_t num_parts, int32_t fixup,
                                 int64_t *counts, void *workspace, size_t workspace_bytes,
                                 void *stream);

/* Degree-aware L2 residency (a B200 addition, not in the paper).  When B does not fit
 * in L2, the B rows gathered most often (hub columns of a power-law A) should stay in
 * L2 and the long tail should stream.  mps_hot_rows counts the non-zeros of every
 * column of A and writes hot_bitmap (caller-owned uint32[(n+31)/32], bit c of word
 * c/32 set) for the columns with the largest counts such that at most budget_rows rows
 * are hot (power-of-two count threshold; no host synchronisation).  workspace:
 * mps_hot_rows_workspace_bytes(n) bytes.  mps_spmm_segments_hot is mps_spmm_segments
 * with that bitmap: hot rows are gathered with L2 evict_last, the others evict_first.
 * mps_spmm_online / mps_spmm_host do this automatically when MPS_HOT_FRAC (fraction
 * of the L2 given to hot rows) is set > 0 and the gathered B exceeds half the L2.
 * Default off: on B200 the static split gained <= 5% over plain evict_last LRU and
 * its per-call pre-pass costs more than that online (profiles/r01/hot_rows.md).    */
mps_status mps_hot_rows_workspace_bytes(int64_t n, size_t *bytes);
/* The library's choice for (A, K, b_dtype) on the current device: *budget_rows_out =
 * -1 when B fits in half of the L2 (no hot-row split), else the hot-row budget.     */
mps_status mps_hot_budget_rows(const mps_csr *A, int32_t K, int32_t b_dtype,
                               int64_t *budget_rows_out);
mps_status mps_hot_rows(const mps_csr *A, int64_t budget_rows, uint32_t *hot_bitmap,
                        void *workspace, size_t workspace_bytes, void *stream);
mps_status mps_spmm_segments_hot(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                                 int32_t K, float *C, int64_t ldc, const int32_t *coord_x,
                                 const int32_t *coord_y, int64_t num_parts, int32_t fixup,
                                 const uint32_t *hot_bitmap, void *workspace,
                                 size_t workspace_bytes, void *stream);

/* mps_spmm with a fused epilogue (MPS_EPI_*) and an optional hot-row bitmap (NULL =
 * none, see mps_hot_rows).  mps_spmm(...) == mps_spmm_ex(..., MPS_EPI_NONE, NULL, ...). */
mps_status mps_spmm_ex(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb, int32_t K,
                       float *C, int64_t ldc, const int32_t *coord_x, const int32_t *coord_y,
                       int64_t num_parts, int32_t fixup, int32_t epilogue,
                       const uint32_t *hot_bitmap, void *workspace, size_t workspace_bytes,
                       void *stream);

/* Online convenience: a1 + a2 + a3 + a4 in one call; the partition is
 * written into the workspace.  items_per_part / min_parts as in mps_plan.         */
mps_status mps_spmm_online_workspace_bytes(const mps_csr *A, int32_t K, int32_t b_dtype,
                                           int64_t items_per_part, int64_t min_parts,
                                           int32_t fixup, size_t *bytes);
mps_status mps_spmm_online(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                           int32_t K, float *C, int64_t ldc, int64_t items_per_part,
                           int64_t min_parts, int32_t fixup, void *workspace,
                           size_t workspace_bytes, void *stream);
mps_status mps_spmm_online_ex(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                              int32_t K, float *C, int64_t ldc, int64_t items_per_part,
                              int64_t min_parts, int32_t fixup, int32_t epilogue,
                              void *workspace, size_t workspace_bytes, void *stream);

/* Which kernels mps_spmm_online(_ex) launches for these arguments (same K, strides,
 * pointers' alignment, items_per_part, min_parts and fixup as the call):
 *  - MPS_PATH_PARTITION_SEGMENTS: the partition kernel (a2, plus the cut-row zeroing in
 *    atomic mode), then the segment kernel per column tile (+ the carry reduction);
 *  - MPS_PATH_SMALL_FUSED: small graphs -- row_ptr (m + 1 int32) and the segment staging
 *    fit in one CTA's shared memory (<= 112 KB), L <= 512 items, one column tile
 *    (K <= 32 x the lane vector width), int32 indices, fixup AUTO or CARRY: ONE kernel in
 *    which every CTA stages the whole row_ptr and every warp computes its own segment's
 *    coordinates (written to the workspace like the partition kernel's), walks it and
 *    leaves the cut rows' pieces as carry records, then the carry reduction sums each cut
 *    row in segment order (deterministic).  Both launches use programmatic dependent
 *    launch.  MPS_SMALL=0 in the environment disables this path.                      */
enum { MPS_PATH_PARTITION_SEGMENTS = 0, MPS_PATH_SMALL_FUSED = 1 };
mps_status mps_spmm_online_path(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                                int32_t K, const float *C, int64_t ldc, int64_t items_per_part,
                                int64_t min_parts, int32_t fixup, int32_t *path_out);

/* End-to-end call on HOST buffers: copies A and B host->device, runs the online path
 * and copies C device->host, all enqueued on `stream` (pinned host memory gives
 * true async copies).  A_host holds HOST pointers.  device_workspace: caller-owned
 * device memory of mps_spmm_host_workspace_bytes(...) bytes.  The caller
 * synchronises the stream before reading C_host.  Only the K valid columns of each
 * row are copied: with ldb > K or ldc > K the padding of B_host is never read and
 * the padding of C_host never written.  In atomic mode the call pipelines the H2D of
 * A (merge-path chunks) with the segment kernels and the D2H of finished rows on two
 * streams it creates for the call and releases when the call's work completes; the
 * whole call is ordered after earlier work on `stream` and later work on `stream`
 * waits for it.                                                                  */
mps_status mps_spmm_host_workspace_bytes(const mps_csr *A_host, int32_t K, int32_t b_dtype,
                                         int64_t ldb, int64_t ldc, int64_t items_per_part,
                                         int64_t min_parts, int32_t fixup, size_t *bytes);
mps_status mps_spmm_host(const mps_csr *A_host, const void *B_host, int32_t b_dtype,
                         int64_t ldb, int32_t K, float *C_host, int64_t ldc,
                         int64_t items_per_part, int64_t min_parts, int32_t fixup,
                         void *device_workspace, size_t workspace_bytes, void *stream);

/* End to end with the graph resident and the dense operands on the host (the paper's
 * offline setting: A -- like its schedule -- stays on the device across
 * inferences; the features B and the output C move every call).  A: DEVICE CSR;
 * B_host, C_host: host buffers (pinned for asynchronous copies).  Enqueues H2D of B,
 * the online path and D2H of C on `stream`; the caller synchronises before reading
 * C_host.  device_workspace: mps_spmm_host_dense_workspace_bytes(...) bytes.        */
mps_status mps_spmm_host_dense_workspace_bytes(const mps_csr *A, int32_t K, int32_t b_dtype,
                                               int64_t ldb, int64_t ldc, int64_t items_per_part,
                                               int64_t min_parts, int32_t fixup, size_t *bytes);
mps_status mps_spmm_host_dense(const mps_csr *A, const void *B_host, int32_t b_dtype,
                               int64_t ldb, int32_t K, float *C_host, int64_t ldc,
                               int64_t items_per_part, int64_t min_parts, int32_t fixup,
                               void *device_workspace, size_t workspace_bytes, void *stream);

/* NEXT-3: the GCN combination B = X * W (A*(X*W) order) on the sm_100
 * tensor cores (tcgen05.mma kind::f16, fp32 accumulation in TMEM, TMA-fed), writing B in
 * bf16 into the row-major layout the SpMM gathers (MPS_DT_BF16, ldb).
 * X: bf16 [n][ldx] (first F columns used); Wt: bf16 [N][ldw] = W transposed (first F
 * columns used); B: bf16 [n][ldb].  Requires 16 <= N <= 256, N % 16 == 0, ldx, ldw,
 * ldb multiples of 8 and 16-B aligned pointers, else MPS_ERR_UNSUPPORTED.           */
mps_status mps_xw_bf16(const void *X, int64_t n, int64_t F, int64_t ldx, const void *Wt,
                       int32_t N, int64_t ldw, void *B, int64_t ldb, void *stream);

/* NEXT-3, multi-GPU: the combination fused with the replication of B over NVLink.  This
 * rank's row block X (n_rows x F) times W is written as bf16 rows row_offset ..
 * row_offset + n_rows - 1 of EVERY B replica in B_dsts_host (a HOST array of ndst
 * device pointers, each to a full [n][ldb] bf16 replica; entry 0 should be this rank's
 * own replica, the others peer replicas mapped with mps_ipc_open_handle).  One kernel:
 * the epilogue of each tile stores it to all destinations, so the all-gather of B
 * overlaps the GEMM.  Same shape rules as mps_xw_bf16, 1 <= ndst <= 16.  Completion on
 * a peer is only guaranteed after this stream is synchronised and the ranks have met
 * at a barrier (the caller's process group).                                        */
mps_status mps_xw_bf16_bcast(const void *X, int64_t n_rows, int64_t F, int64_t ldx,
                             const void *Wt, int32_t N, int64_t ldw, void *const *B_dsts_host,
                             int32_t ndst, int64_t row_offset, int64_t ldb, void *stream);

/* GCN glue between layers (sigma = ReLU): H[r][c] = bf16(max(C[r][c], 0)) for
 * rows x K (C fp32 with leading dimension ldc, H bf16 with ldh) -- the next layer's
 * combination input.  Asynchronous on stream.                                        */
mps_status mps_relu_to_bf16(const float *C, int64_t rows, int32_t K, int64_t ldc, void *H,
                            int64_t ldh, void *stream);

/* Cross-GPU signals over peer memory, used to pipeline the replication of B (written
 * tile by tile by mps_xw_bf16_bcast) with the SpMM of the tiles that have arrived.
 * Signal buffer of every rank: mps_signal_bytes() bytes, zeroed once, flags
 * [64 slots][16 ranks] uint32.  mps_peer_signal: after everything enqueued earlier on
 * `stream`, raises flag[slot][rank] to `epoch` in every rank's buffer
 * (signal_bufs_host: HOST array of `world` device pointers, peers mapped with
 * mps_ipc_open_handle).  mps_peer_wait: work enqueued after it on `stream` starts once
 * every rank raised flag[slot][*] to >= epoch in this rank's buffer (bounded wait,
 * ~20 s, then the kernel traps).  world <= 16, 0 <= slot < 64, epoch >= 1.          */
size_t mps_signal_bytes(void);
mps_status mps_peer_signal(void *const *signal_bufs_host, int32_t world, int32_t rank,
                           int32_t slot, uint32_t epoch, void *stream);
mps_status mps_peer_wait(const void *my_signal_buf, int32_t world, int32_t slot, uint32_t epoch,
                         void *stream);

/* CUDA IPC between the ranks of one node (peer access over NVLink is enabled lazily).
 * mps_ipc_get_handle: handle_out (mps_ipc_handle_bytes() bytes, caller-owned) names the
 * device allocation that contains dev_ptr; *offset_out = dev_ptr - its base.  The peer
 * opens it with mps_ipc_open_handle (base address in this process; add the offset) and
 * unmaps it with mps_ipc_close_handle.  Errors: MPS_ERR_INVALID for NULL or non-device
 * pointers, MPS_ERR_CUDA if the runtime refuses (e.g. a handle opened in its own
 * process).                                                                         */
size_t mps_ipc_handle_bytes(void);
mps_status mps_ipc_get_handle(const void *dev_ptr, void *handle_out, int64_t *offset_out);
mps_status mps_ipc_open_handle(const void *handle, void **base_out);
mps_status mps_ipc_close_handle(void *base);

/* Fig. 5 statistic: with the Alg. 2 write rules (lines 5, 9, 13 atomic,
 * line 15 regular) for the given schedule, counts_out[0] = #atomic row updates,
 * counts_out[1] = #regular row stores.  counts_out: device int64[2], overwritten. */
mps_status mps_write_stats(const mps_csr *A, const int32_t *coord_x, const int32_t *coord_y,
                           int64_t num_parts, int64_t *counts_out, void *stream);

/* a6 -- multi-GPU merge-path sharding (north-star stage 4; not in the paper).
 * Host closed form: shard g covers diagonals [D_g, D_{g+1}), D_g = min(g*ceil(M/G), M);
 * (X_g, Y_g) = coordinate of D_g.  Shard g owns C rows [X_g, X_{g+1}); its tail row
 * is X_{g+1} if that row is cut (Y_{g+1} > row_ptr[X_{g+1}]), else -1.
 * row_ptr_host: host copy of row_ptr.  X, Y: host int32[world+1];
 * tail_rows: host int32[world].                                                   */
mps_status mps_shard_bounds(const int32_t *row_ptr_host, int64_t m, int64_t nnz, int32_t world,
                            int32_t *X, int32_t *Y, int32_t *tail_rows);

/* Rank-local SpMM of shard `rank`.  A->row_ptr is the GLOBAL row_ptr (device);
 * A->col_idx / A->val point at the rank's slice, which starts at global nnz index
 * Y[rank] (A->nnz stays the global nnz).  C_local: rows X[rank] .. X[rank+1]-1
 * (leading dimension ldc), overwritten.  tail_out: device float[K], overwritten
 * with the shard's partial sum of row tail_rows[rank] (zeros if there is none).
 * X, Y, tail_rows: host arrays from mps_shard_bounds.                            */
mps_status mps_spmm_shard_workspace_bytes(const mps_csr *A, int32_t K, int32_t b_dtype,
                                          const int32_t *X, int32_t rank, int32_t world,
                                          int64_t items_per_part, int64_t min_parts,
                                          int32_t fixup, size_t *bytes);
mps_status mps_spmm_shard(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                          int32_t K, const int32_t *X, const int32_t *Y,
                          const int32_t *tail_rows, int32_t rank, int32_t world,
                          int64_t items_per_part, int64_t min_parts, float *C_local,
                          int64_t ldc, float *tail_out, int32_t fixup, void *workspace,
                          size_t workspace_bytes, void *stream);

/* a6 with the tail exchange over peer memory instead of a collective (fused into the
 * kernel that finalises the tail: the last column tile's segment kernel in atomic mode,
 * the carry reduction in carry mode).  The LAST CTA of that kernel
 *   - pushes this rank's tail (row tail_rows[rank]) into the mailbox of the row's owner
 *     (owner(r) = max{g : X_g <= r}) and raises flag[rank] there to `epoch`;
 *   - if other ranks' tails belong to this rank's first row, waits for their flags to
 *     reach `epoch` and adds them to the row in ascending rank order, then acknowledges.
 * No mps_apply_tails / all-gather is needed.  mailboxes_host: HOST array of `world`
 * device pointers, entry g = rank g's mailbox of mps_shard_mailbox_bytes(K) bytes
 * (this rank's own, peers' mapped with mps_ipc_open_handle); every mailbox must be
 * zeroed once before the first call.  epoch: 1 for the first call, +1 per call (two
 * inbox slots alternate; a push waits for the owner's acknowledgement of epoch - 2).
 * world <= 16.  Waits are bounded (~20 s), after which the kernel traps
 * (MPS_ERR_CUDA on the next call) rather than hang.  Other arguments: mps_spmm_shard. */
size_t mps_shard_mailbox_bytes(int32_t K);
mps_status mps_spmm_shard_p2p(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                              int32_t K, const int32_t *X, const int32_t *Y,
                              const int32_t *tail_rows, int32_t rank, int32_t world,
                              int64_t items_per_part, int64_t min_parts, float *C_local,
                              int64_t ldc, float *tail_out, int32_t fixup,
                              void *const *mailboxes_host, uint32_t epoch, void *workspace,
                              size_t workspace_bytes, void *stream);

/* After an all-gather of every rank's tail_out into tails (device float[world*K],
 * rank-major): add the tails whose row this rank owns (owner(r) = max{g : X_g <= r})
 * into C_local, in ascending rank order (deterministic).                         */
mps_status mps_apply_tails(const float *tails, const int32_t *X, const int32_t *tail_rows,
                           int32_t world, int32_t rank, int32_t K, float *C_local,
                           int64_t ldc, void *stream);

/* NEXT-4 -- 64-bit non-zero indices, for graphs with
 * M = m + nnz >= 2^31 (the paper motivates billion-edge graphs).  Rows and
 * columns stay below 2^31, so coord_x and col_idx stay int32; row_ptr and the nnz
 * coordinate y are int64.  The method is unchanged: the same a1-a4 steps run with
 * 64-bit y (x = max{x : x + row_ptr[x] <= d} on int64 diagonals d).
 * A: row_ptr int64[m+1], col_idx int32[nnz], val fp32[nnz]; m, n < 2^31,
 * nnz < 2^62, else MPS_ERR_UNSUPPORTED.  Every other convention (ownership, streams,
 * errors, overwrite of C, fix-up modes, epilogues) is that of the int32 calls above:
 *   mps_plan64           = mps_plan without the 2^31 limit on M;
 *   mps_partition64      = mps_partition, coord_y int64[num_parts+1];
 *   mps_spmm64           = mps_spmm_ex (no hot-row bitmap), coord_y int64;
 *   mps_spmm64_online    = mps_spmm_online_ex;
 *   mps_write_stats64, mps_validate_csr64 = mps_write_stats, mps_validate_csr.      */
typedef struct {
    int64_t m, n, nnz;
    const int64_t *row_ptr;
    const int32_t *col_idx;
    const float *val;
} mps_csr64;

mps_status mps_plan64(int64_t m, int64_t nnz, int32_t K, int32_t b_dtype, int64_t items_per_part,
                      int64_t min_parts, int64_t *num_parts_out, int64_t *items_per_part_out);
mps_status mps_partition64(const int64_t *row_ptr, int64_t m, int64_t nnz, int64_t diag_begin,
                           int64_t diag_end, int64_t num_parts, int64_t items_per_part,
                           int32_t *coord_x, int64_t *coord_y, void *stream);
mps_status mps_spmm64_workspace_bytes(const mps_csr64 *A, int32_t K, int32_t b_dtype,
                                      int64_t num_parts, int32_t fixup, size_t *bytes);
mps_status mps_spmm64(const mps_csr64 *A, const void *B, int32_t b_dtype, int64_t ldb,
                      int32_t K, float *C, int64_t ldc, const int32_t *coord_x,
                      const int64_t *coord_y, int64_t num_parts, int32_t fixup,
                      int32_t epilogue, void *workspace, size_t workspace_bytes, void *stream);
mps_status mps_spmm64_online_workspace_bytes(const mps_csr64 *A, int32_t K, int32_t b_dtype,
                                             int64_t items_per_part, int64_t min_parts,
                                             int32_t fixup, size_t *bytes);
mps_status mps_spmm64_online(const mps_csr64 *A, const void *B, int32_t b_dtype, int64_t ldb,
                             int32_t K, float *C, int64_t ldc, int64_t items_per_part,
                             int64_t min_parts, int32_t fixup, int32_t epilogue,
                             void *workspace, size_t workspace_bytes, void *stream);
/* a6 sharding with 64-bit indices (NEXT-4 scale-out): Y int64[world+1]; the same
 * closed form, ownership and tail rules as mps_shard_bounds / mps_spmm_shard(_p2p).
 * mps_spmm_shard64 takes the peer-memory tail exchange's mailboxes_host/epoch (NULL/0 =
 * none: exchange the tails with an all-gather and mps_apply_tails instead).          */
mps_status mps_shard_bounds64(const int64_t *row_ptr_host, int64_t m, int64_t nnz,
                              int32_t world, int32_t *X, int64_t *Y, int32_t *tail_rows);
mps_status mps_spmm_shard64_workspace_bytes(const mps_csr64 *A, int32_t K, int32_t b_dtype,
                                            const int32_t *X, int32_t rank, int32_t world,
                                            int64_t items_per_part, int64_t min_parts,
                                            int32_t fixup, size_t *bytes);
mps_status mps_spmm_shard64(const mps_csr64 *A, const void *B, int32_t b_dtype, int64_t ldb,
                            int32_t K, const int32_t *X, const int64_t *Y,
                            const int32_t *tail_rows, int32_t rank, int32_t world,
                            int64_t items_per_part, int64_t min_parts, float *C_local,
                            int64_t ldc, float *tail_out, int32_t fixup,
                            void *const *mailboxes_host, uint32_t epoch, void *workspace,
                            size_t workspace_bytes, void *stream);
mps_status mps_write_stats64(const mps_csr64 *A, const int32_t *coord_x, const int64_t *coord_y,
                             int64_t num_parts, int64_t *counts_out, void *stream);
mps_status mps_validate_csr64(const mps_csr64 *A, int64_t *first_bad_host, void *stream);

/* Debug-only validation of CSR content on the device (synchronises).  Checks
 * row_ptr[0] == 0, row_ptr non-decreasing, row_ptr[m] == nnz, 0 <= col < n.
 * *first_bad_host = -1 if valid, else the first offending row_ptr index (< m+1) or
 * m + 1 + the first offending nnz index.                                          */
mps_status mps_validate_csr(const mps_csr *A, int64_t *first_bad_host, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* MPSPMM_H */
