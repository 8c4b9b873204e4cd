// capi.cu -- the extern "C" boundary of libmpspmm.so (include/mpspmm.h): argument
// validation, schedule sizing (a1), workspace layout, column tiling and launch order.
#include <cstdio>
#include <cstring>
#include <cstdarg>
#include <cstdlib>
#include <type_traits>
#include <vector>

#include <cuda.h>

#include "mps_internal.cuh"

namespace mps { int num_sms(); }

namespace {

thread_local char g_err[512] = "";

mps_status fail(mps_status st, const char *fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return st;
}

mps_status cuda_fail(cudaError_t e, const char *where) {
    return fail(MPS_ERR_CUDA, "%s: %s", where, cudaGetErrorString(e));
}

#define MPS_CUDA(call, where)                                   \
    do {                                                        \
        cudaError_t e__ = (call);                               \
        if (e__ != cudaSuccess) return cuda_fail(e__, where);   \
    } while (0)

constexpr int64_t kMaxIndex = (int64_t)1 << 31;
constexpr int64_t kDefaultMinParts = 8 * 148;  // ~ the paper's 1024-thread floor

inline size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

inline int elt_bytes(int32_t dt) { return dt == MPS_DT_BF16 ? 2 : 4; }

// Default merge-path cost (items per warp segment).  The paper tunes this per K on an
// RTX 6000 (Fig. 6: 15-50 items per thread).  On B200 the NEXT-1 sweep over
// the 22 Table-II-shaped graphs and the BASELINE graphs (profiles/r01/sensitivity.md)
// finds the optimum set by two things rather than K: long rows want long segments
// (fewer cut rows: ~4 rows per segment, 512..2048 items), and the schedule must keep
// >= 1.5 waves of resident warps busy, which caps the cost on mid-size graphs:
//   cost = max(64, min(clamp(next_pow2(4*ceil(nnz/m)), 512, 2048),
//                      pow2_floor(M / (1.5 * resident_warps))))
// (geomean 0.974 of the per-graph best on Table II, 0.998 on Reddit/products/R-MAT).
// Resident warps: 24 per SM for fp32, 20 for bf16 (the 128-thread bf16 CTAs of round 2's
// second session; with 16 the bf16 Table-II score fell to 0.933, with 20 it is 0.966 --
// profiles/r03/sensitivity.md; the BASELINE graphs' costs do not change).
int64_t default_cost(int64_t m, int64_t nnz, int32_t K, int32_t dt) {
    (void)K;
    const int64_t avg = m > 0 ? (nnz + m - 1) / m : 1;
    int64_t deg = 1;
    while (deg < 4 * avg) deg <<= 1;
    deg = deg < 512 ? 512 : (deg > 2048 ? 2048 : deg);
    const int64_t resident = (int64_t)mps::num_sms() * (dt == MPS_DT_BF16 ? 20 : 24);
    const double target = (double)(m + nnz) / (1.5 * (double)resident);
    int64_t cap = 1;
    while ((double)(cap * 2) <= target) cap <<= 1;
    int64_t c = deg < cap ? deg : cap;
    return c < 64 ? 64 : c;
}

struct Vec {
    int W = 1;     // elements per lane access
    int tile = 0;  // columns per launch (multiple of 32*W)
    bool deep = false;  // DRAM-bound gathers: the deep-gather instantiation (see below)
    bool dram = false;  // a column tile's B slice exceeds half the L2 (gathers miss L2)
};

static int64_t l2_bytes() {
    static int64_t cache = 0;
    if (cache == 0) {
        int dev = 0, l2 = 0;
        if (cudaGetDevice(&dev) != cudaSuccess ||
            cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev) != cudaSuccess || l2 <= 0)
            l2 = 126 << 20;
        cache = l2;
    }
    return cache;
}

// Widest lane vector (16 B when possible) that the alignment of B and C allows.  Rows
// narrower than 32*W columns are gathered NR at a time per warp instruction.
// Column tiling (B200, measured in profiles/r01/tiling.md): when the gathered B (b_rows
// rows) exceeds half the L2, each pass covers 256-byte slices of the B rows, so the L2
// holds a larger share of every pass's working set (Reddit K=256 fp32: 8.1 -> 6.5 ms).
Vec choose_vec(int32_t K, int32_t dt, const void *B, int64_t ldb, const float *C, int64_t ldc,
               int64_t b_rows = 0, int64_t m = 0, int64_t nnz = 0) {
    const int eb = elt_bytes(dt);
    const int cand_f32[3] = {4, 2, 1};
    const int cand_bf[4] = {8, 4, 2, 1};
    const int *cand = dt == MPS_DT_BF16 ? cand_bf : cand_f32;
    const int nc = dt == MPS_DT_BF16 ? 4 : 3;
    auto ok = [&](int W) {
        const int cw = W < 4 ? W : 4;  // C is written in float(W<=4) or float4 pieces
        return K % W == 0 && ldb % W == 0 && ((uintptr_t)B % (size_t)(W * eb)) == 0 &&
               ldc % cw == 0 && ((uintptr_t)C % (size_t)(cw * 4)) == 0;
    };
    // MPS_MAX_W: debug/tuning cap on the lane vector width (elements)
    static const int max_w = [] {
        const char *e = getenv("MPS_MAX_W");
        return e ? atoi(e) : 16;
    }();
    // MPS_MAX_V: debug/tuning cap on slots per lane, i.e. the column-tile width 32*W*V
    static const int max_v = [] {
        const char *e = getenv("MPS_MAX_V");
        const int v = e ? atoi(e) : 4;
        return v < 1 ? 1 : (v > 4 ? 4 : v);
    }();
    // narrow K: keep >= 4 lanes per B row (NR <= 8 rows per warp instruction).  Fewer
    // rows per instruction mean shorter row-end butterflies and fewer predicated passes
    // per batch; measured on the 22 Table-II graphs (CUDA-graph replay) over 16-B
    // gathers with 16-32 rows per instruction: fp32 K=2/4/8 +4/12/8%, bf16 K=4/8/16
    // +11/35/16% (profiles/r01/narrow_k/; 8 lanes: within 1% except bf16 K=32 +6%).
    // MPS_NARROW = minimum lanes per row (0 disables).
    int wcap = max_w;
    const char *en = getenv("MPS_NARROW");    // minimum lanes per row (default 4; 0: off)
    const int min_lanes = en ? atoi(en) : 4;
    if (min_lanes > 0) {
        int lim = K / min_lanes < 1 ? 1 : K / min_lanes;
        int p2 = 1;
        while (p2 * 2 <= lim) p2 *= 2;
        if (p2 < wcap) wcap = p2;
    }
    Vec v;
    for (int i = 0; i < nc && v.tile == 0; ++i)
        if (cand[i] <= wcap && ok(cand[i])) { v.W = cand[i]; v.tile = 32 * cand[i] * max_v; }
    if (v.tile == 0) { v.W = 1; v.tile = 32 * max_v; }
    // MPS_TILE: tuning override of the column-tile width (0 = rule below, -1 = no tiling)
    const char *et = getenv("MPS_TILE");   // read per call (tests vary it)
    const int env_tile = et ? atoi(et) : 0;
    int tile = 0;
    if (env_tile > 0) tile = env_tile;
    else if (env_tile == 0 && b_rows > 0 &&
             (double)b_rows * K * eb > 0.5 * (double)l2_bytes())
        tile = 256 / eb;
    if (tile > 0 && tile < v.tile && tile < K) v.tile = (tile / v.W > 0 ? tile / v.W : 1) * v.W;
    // Deep gathers (2x the 16-B gathers in flight per lane, 2 CTAs/SM at 128 registers)
    // for fp32 256-B row slices when a pass's B slice exceeds half the L2 and rows are
    // long enough (>= 32 non-zeros on average) for the larger batches to stay on the
    // fast path: DRAM-bound gathers want more bytes in flight (products K=128 -3.2%);
    // L2-resident B (Reddit K=64: +1.7%) and short rows (R-MAT: +10%) lose with it
    // (profiles/r01/deep_gathers/).  MPS_DEEP=0/1 overrides.
    const char *ed = getenv("MPS_DEEP");
    const int kt = v.tile < K ? v.tile : K;
    v.dram = b_rows > 0 && (double)b_rows * kt * eb > 0.5 * (double)l2_bytes();
    if (ed) v.deep = atoi(ed) != 0;
    else v.deep = b_rows > 0 && m > 0 && nnz >= 32 * m &&
                  (double)b_rows * kt * eb > 0.5 * (double)l2_bytes();
    v.deep = v.deep && dt == MPS_DT_F32 && v.W == 4 && kt == 64;
    return v;
}

// Lane geometry of one column tile of kt columns: V slots per lane, NR rows per warp
// instruction (NR > 1 only when a row needs fewer than 32 lanes).
void tile_geometry(int32_t kt, int W, int *V, int *NR) {
    const int lanes = (kt + W - 1) / W;
    if (lanes >= 32) {
        *NR = 1;
        *V = (kt + 32 * W - 1) / (32 * W);
    } else {
        int lr = 1;
        while (lr < lanes) lr <<= 1;
        *NR = 32 / lr;
        *V = 1;
    }
}

// Index type of a CSR struct: int32_t (mps_csr) or int64_t (mps_csr64, NEXT-4).
template <typename CSR>
using idx_t = std::remove_const_t<std::remove_pointer_t<decltype(CSR::row_ptr)>>;

constexpr int64_t kMaxIndex64 = (int64_t)1 << 62;

template <typename CSR>
mps_status check_csr(const CSR *A, bool device_ptrs_needed = true) {
    if (!A) return fail(MPS_ERR_INVALID, "A is NULL");
    if (A->m < 0 || A->n < 0 || A->nnz < 0) return fail(MPS_ERR_INVALID, "negative CSR size");
    if (sizeof(*A->row_ptr) == 4 && (A->m + A->nnz >= kMaxIndex || A->n >= kMaxIndex))
        return fail(MPS_ERR_UNSUPPORTED, "m + nnz = %lld >= 2^31 (int32 indices; use mps_csr64)",
                    (long long)(A->m + A->nnz));
    if (sizeof(*A->row_ptr) == 8 &&
        (A->m >= kMaxIndex || A->n >= kMaxIndex || A->nnz >= kMaxIndex64))
        return fail(MPS_ERR_UNSUPPORTED, "mps_csr64 needs m, n < 2^31 and nnz < 2^62");
    if (device_ptrs_needed && A->m > 0 && !A->row_ptr) return fail(MPS_ERR_INVALID, "row_ptr NULL");
    if (device_ptrs_needed && A->nnz > 0 && (!A->col_idx || !A->val))
        return fail(MPS_ERR_INVALID, "col_idx/val NULL");
    return MPS_OK;
}

template <typename CSR>
mps_status check_dense(const void *B, int32_t dt, int64_t ldb, int32_t K, const float *C,
                       int64_t ldc, const CSR *A) {
    if (dt != MPS_DT_F32 && dt != MPS_DT_BF16) return fail(MPS_ERR_UNSUPPORTED, "b_dtype %d", dt);
    if (K < 0) return fail(MPS_ERR_INVALID, "K < 0");
    if (K > 0 && (ldb < K || ldc < K)) return fail(MPS_ERR_INVALID, "ldb/ldc < K");
    if (K > 0 && A->m > 0 && !C) return fail(MPS_ERR_INVALID, "C NULL");
    if (K > 0 && A->nnz > 0 && !B) return fail(MPS_ERR_INVALID, "B NULL");
    return MPS_OK;
}

int64_t carry_kpad(int32_t K, const Vec &v) {
    const int64_t kt = K < v.tile ? K : v.tile;
    return (int64_t)align_up((size_t)kt, 8);
}

size_t carry_bytes(int64_t P, int32_t K, const Vec &v) {
    return (size_t)P * 2 * (size_t)carry_kpad(K, v) * sizeof(float);
}

// Dynamic segment claims: one 32-bit counter per column tile, in the caller's workspace
// (no library state: every workspace, and so every captured CUDA graph, owns its
// counters).  Sized for the worst case of one column per tile.
size_t claim_bytes(int32_t K) { return align_up((size_t)(K > 0 ? K : 1) * 4, 256); }
int32_t num_tiles(int32_t K, const Vec &v) { return K > 0 ? (K + v.tile - 1) / v.tile : 0; }
// claim counters a kernel preceding the segment kernel can zero (one per thread of a CTA)
int32_t zeroable_claims(int32_t K, const Vec &v) {
    const int32_t t = num_tiles(K, v);
    return t <= mps::kBlock ? t : 0;
}

int resolve_fix(int32_t fixup) { return fixup == MPS_FIXUP_CARRY ? mps::FIX_CARRY : mps::FIX_ATOMIC; }

// host coordinate of diagonal d (shard bounds): x = max{x : x + rp[x] <= d}
template <typename IT>
int64_t host_diag_x(const IT *rp, int64_t m, int64_t nnz, int64_t d) {
    int64_t lo = (d > nnz ? d - nnz : 0) + 1, hi = (d < m ? d : m) + 1;
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (mid + (int64_t)rp[mid] > d) hi = mid;
        else lo = mid + 1;
    }
    return lo - 1;
}

// Run a3 (+ a4 carry reduction) over all column tiles for a ready schedule.
// claims: the per-tile claim counters (workspace; NULL: static segment assignment);
// claims_zeroed: a kernel earlier on the stream already zeroed them, else they are
// zeroed here when the schedule is long enough for dynamic claims.
template <typename IT>
mps_status run_segments(mps::SegArgsT<IT> base, int32_t dt, int32_t K, const Vec &v, int fix,
                        void *workspace, unsigned *claims, bool claims_zeroed,
                        cudaStream_t s) {
    const int eb = elt_bytes(dt);
    if (claims && !claims_zeroed && base.P >= mps::seg_dynamic_min_parts())
        MPS_CUDA(cudaMemsetAsync(claims, 0, (size_t)num_tiles(K, v) * 4, s), "zero claims");
    if (claims && !claims_zeroed && base.P < mps::seg_dynamic_min_parts()) claims = nullptr;
    for (int32_t c0 = 0; c0 < K; c0 += v.tile) {
        mps::SegArgsT<IT> a = base;
        // the tail exchange rides on the launch that finalises the tail: the last tile's
        // segment kernel (atomic) or carry reduction (carry)
        if (c0 + v.tile < K) a.mail.on = 0;
        const int32_t kt = (K - c0) < v.tile ? (K - c0) : v.tile;
        a.K = kt;
        a.B = (const char *)base.B + (size_t)c0 * eb;
        a.C = base.C ? base.C + c0 : nullptr;
        a.tail = base.tail ? base.tail + c0 : nullptr;
        a.rec = (float *)workspace;
        a.kpad = (int32_t)carry_kpad(K, v);
        a.claim = claims ? claims + c0 / v.tile : nullptr;
        if (c0 > 0) a.wstat = nullptr;      // the write statistic counts column tile 0
        // TMA staging needs col and val equally aligned modulo 16 B
        a.direct = ((((uintptr_t)base.col) ^ ((uintptr_t)base.val)) & 15u) != 0;
        static const int hints = [] {
            const char *e = getenv("MPS_L2_HINTS");
            return e ? atoi(e) : 1;
        }();
        a.l2_hints = hints;
        int V, NR;
        tile_geometry(kt, v.W, &V, &NR);
        a.deep = v.deep && kt == 64 ? 1 : 0;
        // next-batch L2 prefetch of B rows (bf16 dynamic kernels) where the tile's B slice
        // exceeds half the L2; MPS_PF (read per call) 0/1 overrides
        const char *ep = getenv("MPS_PF");
        const int pfm = ep ? atoi(ep) : -1;
        a.pf = pfm >= 0 ? pfm : (v.dram && dt == MPS_DT_BF16 ? 1 : 0);
        {
            int lines = (kt * eb + 127) / 128, sh = 0;
            while ((1 << sh) < lines) ++sh;
            a.pf_shift = sh;
        }
        mps::SegArgsT<IT> seg_only = a;
        seg_only.mail.on = 0;
        MPS_CUDA(mps::launch_segments(fix == mps::FIX_CARRY ? seg_only : a, dt, v.W, V, NR, fix,
                                      s), "segment kernel");
        if (fix == mps::FIX_CARRY) MPS_CUDA(mps::launch_carry_reduce(a, s), "carry reduce");
        else if (a.relu) MPS_CUDA(mps::launch_relu_split(a, s), "relu on cut rows");
    }
    return MPS_OK;
}

}  // namespace

namespace mps {
int num_sms() {
    static int cache[64] = {0};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 148;
    if (cache[dev] == 0) {
        int v = 0;
        if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || v <= 0)
            v = 148;
        cache[dev] = v;
    }
    return cache[dev];
}
}  // namespace mps

extern "C" {

int mps_abi_version(void) { return 2; }  // 2: claim counters in the workspace

const char *mps_status_string(mps_status s) {
    switch (s) {
    case MPS_OK: return "MPS_OK";
    case MPS_ERR_INVALID: return "MPS_ERR_INVALID";
    case MPS_ERR_UNSUPPORTED: return "MPS_ERR_UNSUPPORTED";
    case MPS_ERR_CUDA: return "MPS_ERR_CUDA";
    case MPS_ERR_WORKSPACE: return "MPS_ERR_WORKSPACE";
    case MPS_ERR_COMM: return "MPS_ERR_COMM";
    default: return "MPS_ERR_UNKNOWN";
    }
}

const char *mps_last_error(void) { return g_err; }

}  // extern "C"

static mps_status plan_impl(int64_t m, int64_t nnz, int32_t K, int32_t b_dtype,
                            int64_t items_per_part, int64_t min_parts, int64_t *num_parts_out,
                            int64_t *items_per_part_out, bool wide) {
    if (m < 0 || nnz < 0 || K < 0 || items_per_part < 0 || min_parts < 0)
        return fail(MPS_ERR_INVALID, "negative plan argument");
    if (!num_parts_out || !items_per_part_out) return fail(MPS_ERR_INVALID, "NULL output");
    if (b_dtype != MPS_DT_F32 && b_dtype != MPS_DT_BF16)
        return fail(MPS_ERR_UNSUPPORTED, "b_dtype %d", b_dtype);
    if (!wide && m + nnz >= kMaxIndex) return fail(MPS_ERR_UNSUPPORTED, "m + nnz >= 2^31");
    if (wide && (m >= kMaxIndex || nnz >= kMaxIndex64))
        return fail(MPS_ERR_UNSUPPORTED, "m >= 2^31 or nnz >= 2^62");
    const int64_t cost = items_per_part ? items_per_part : default_cost(m, nnz, K, b_dtype);
    const int64_t pmin = min_parts ? min_parts : kDefaultMinParts;
    const int64_t M = m + nnz;                      // Alg. 1 line 2
    int64_t P = (M + cost - 1) / cost;              // threads = merge_items / cost
    if (P < pmin) P = pmin;                         // thread floor
    *num_parts_out = P;
    *items_per_part_out = (M + P - 1) / P;          // Alg. 1 line 3 (reading R1)
    return MPS_OK;
}

template <typename IT>
static mps_status partition_impl(const IT *row_ptr, int64_t m, int64_t nnz, int64_t diag_begin,
                                 int64_t diag_end, int64_t num_parts, int64_t items_per_part,
                                 int32_t *coord_x, IT *coord_y, void *stream) {
    if (m < 0 || nnz < 0 || num_parts < 1 || items_per_part < 0)
        return fail(MPS_ERR_INVALID, "bad partition sizes");
    if (sizeof(IT) == 4 && m + nnz >= kMaxIndex)
        return fail(MPS_ERR_UNSUPPORTED, "m + nnz >= 2^31");
    if (sizeof(IT) == 8 && (m >= kMaxIndex || nnz >= kMaxIndex64))
        return fail(MPS_ERR_UNSUPPORTED, "m >= 2^31 or nnz >= 2^62");
    if (diag_begin < 0 || diag_end < diag_begin || diag_end > m + nnz)
        return fail(MPS_ERR_INVALID, "diagonal range outside [0, m + nnz]");
    if (!row_ptr || !coord_x || !coord_y) return fail(MPS_ERR_INVALID, "NULL pointer");
    MPS_CUDA(mps::launch_partition<IT>(row_ptr, m, nnz, diag_begin, diag_end - diag_begin,
                                       num_parts, items_per_part, coord_x, coord_y, nullptr, 0, 0,
                                       0, -1, nullptr, nullptr, 0, (cudaStream_t)stream),
             "partition kernel");
    return MPS_OK;
}

extern "C" {

mps_status mps_plan(int64_t m, int64_t nnz, int32_t K, int32_t b_dtype, int64_t items_per_part,
                    int64_t min_parts, int64_t *num_parts_out, int64_t *items_per_part_out) {
    return plan_impl(m, nnz, K, b_dtype, items_per_part, min_parts, num_parts_out,
                     items_per_part_out, false);
}

mps_status mps_plan64(int64_t m, int64_t nnz, int32_t K, int32_t b_dtype, int64_t items_per_part,
                      int64_t min_parts, int64_t *num_parts_out, int64_t *items_per_part_out) {
    return plan_impl(m, nnz, K, b_dtype, items_per_part, min_parts, num_parts_out,
                     items_per_part_out, true);
}

mps_status mps_partition64(const int64_t *row_ptr, int64_t m, int64_t nnz, int64_t diag_begin,
                           int64_t diag_end, int64_t num_parts, int64_t items_per_part,
                           int32_t *coord_x, int64_t *coord_y, void *stream) {
    return partition_impl<int64_t>(row_ptr, m, nnz, diag_begin, diag_end, num_parts,
                                   items_per_part, coord_x, coord_y, stream);
}

mps_status mps_partition(const int32_t *row_ptr, int64_t m, int64_t nnz, int64_t diag_begin,
                         int64_t diag_end, int64_t num_parts, int64_t items_per_part,
                         int32_t *coord_x, int32_t *coord_y, void *stream) {
    return partition_impl<int32_t>(row_ptr, m, nnz, diag_begin, diag_end, num_parts,
                                   items_per_part, coord_x, coord_y, stream);
}

mps_status mps_partition_split(const int32_t *row_ptr, int64_t m, int64_t nnz,
                               int64_t num_parts, int64_t items_per_part, int32_t *coord_x,
                               int32_t *coord_y, float *C, int64_t ldc, int32_t K,
                               void *stream) {
    if (m < 0 || nnz < 0 || num_parts < 1 || items_per_part < 0 || K < 0 || (K > 0 && ldc < K))
        return fail(MPS_ERR_INVALID, "bad partition sizes");
    if (m + nnz >= kMaxIndex) return fail(MPS_ERR_UNSUPPORTED, "m + nnz >= 2^31");
    if (!row_ptr || !coord_x || !coord_y || (K > 0 && m > 0 && !C))
        return fail(MPS_ERR_INVALID, "NULL pointer");
    MPS_CUDA(mps::launch_partition(row_ptr, m, nnz, 0, m + nnz, num_parts, items_per_part, coord_x,
                                   coord_y, K > 0 ? C : nullptr, ldc, 0, K, -1, nullptr,
                                   nullptr, 0, (cudaStream_t)stream),
             "partition kernel");
    return MPS_OK;
}

}  // extern "C"

// ---------------------------------------------------------------------------------
// a3 + a4 implementations shared by the int32 (mps_csr) and int64 (mps_csr64, NEXT-4)
// entry points.  CSR is the public struct; its row_ptr type is the index type IT.
// ---------------------------------------------------------------------------------
namespace {

template <typename CSR>
mps_status spmm_ws_impl(const CSR *A, int32_t K, int32_t b_dtype, int64_t num_parts,
                        int32_t fixup, size_t *bytes) {
    mps_status st = check_csr(A, false);
    if (st) return st;
    if (!bytes || num_parts < 1 || K < 0) return fail(MPS_ERR_INVALID, "bad arguments");
    if (b_dtype != MPS_DT_F32 && b_dtype != MPS_DT_BF16)
        return fail(MPS_ERR_UNSUPPORTED, "b_dtype %d", b_dtype);
    // worst case over alignments: the narrowest vector gives the smallest tile
    Vec v = choose_vec(K, b_dtype, nullptr, K ? K : 1, nullptr, K ? K : 1);
    Vec vmin;
    vmin.W = 1;
    vmin.tile = 128;
    size_t need = resolve_fix(fixup) == mps::FIX_CARRY
                      ? (carry_bytes(num_parts, K, v) > carry_bytes(num_parts, K, vmin)
                             ? carry_bytes(num_parts, K, v) : carry_bytes(num_parts, K, vmin))
                      : 0;
    *bytes = claim_bytes(K) + need;   // [claim counters][carry records]
    return MPS_OK;
}

template <typename CSR>
mps_status zero_split_impl(const CSR *A, const int32_t *coord_x, const idx_t<CSR> *coord_y,
                           int64_t num_parts, float *C, int64_t ldc, int32_t K, void *stream,
                           unsigned *claims = nullptr, int32_t nclaims = 0) {
    mps_status st = check_csr(A);
    if (st) return st;
    if (num_parts < 1 || K < 0 || (K > 0 && ldc < K)) return fail(MPS_ERR_INVALID, "bad arguments");
    if (K == 0 || A->m == 0) return MPS_OK;
    if (!coord_x || !coord_y || !C) return fail(MPS_ERR_INVALID, "NULL pointer");
    MPS_CUDA(mps::launch_zero_split(A->row_ptr, (int32_t)A->m, coord_x, coord_y, num_parts, C,
                                    ldc, 0, K, -1, nullptr, claims, nclaims,
                                    (cudaStream_t)stream),
             "zero split rows");
    return MPS_OK;
}

template <typename CSR>
mps_status segments_impl(const CSR *A, const void *B, int32_t b_dtype, int64_t ldb, int32_t K,
                         float *C, int64_t ldc, const int32_t *coord_x,
                         const idx_t<CSR> *coord_y, int64_t num_parts, int32_t fixup,
                         const uint32_t *hot_bitmap, int32_t relu, void *workspace,
                         size_t workspace_bytes, void *stream, bool claims_zeroed = false,
                         unsigned long long *wstat = nullptr) {
    mps_status st = check_csr(A);
    if (st) return st;
    if ((st = check_dense(B, b_dtype, ldb, K, C, ldc, A))) return st;
    if (num_parts < 1) return fail(MPS_ERR_INVALID, "num_parts < 1");
    if (K == 0 || A->m == 0) return MPS_OK;
    if (!coord_x || !coord_y) return fail(MPS_ERR_INVALID, "NULL coordinates");
    const int fix = resolve_fix(fixup);
    const Vec v = choose_vec(K, b_dtype, B, ldb, C, ldc, A->n, A->m, A->nnz);
    // workspace: [claim counters][carry records (carry mode)]
    const size_t need = claim_bytes(K) + (fix == mps::FIX_CARRY ? carry_bytes(num_parts, K, v) : 0);
    if (!workspace || workspace_bytes < need)
        return fail(MPS_ERR_WORKSPACE, "workspace %zu < %zu", workspace_bytes, need);
    mps::SegArgsT<idx_t<CSR>> a{};
    a.rp = A->row_ptr;
    a.col = A->col_idx;
    a.val = A->val;
    a.B = B;
    a.ldb = ldb;
    a.C = C;
    a.ldc = ldc;
    a.row_base = 0;
    a.m = (int32_t)A->m;
    a.cx = coord_x;
    a.cy = coord_y;
    a.P = num_parts;
    a.tail_row = -1;
    a.tail = nullptr;
    a.nnz_end = A->nnz;
    a.hot = hot_bitmap;
    a.relu = relu;
    a.wstat = wstat;
    return run_segments(a, b_dtype, K, v, fix, (char *)workspace + claim_bytes(K),
                        (unsigned *)workspace, claims_zeroed, (cudaStream_t)stream);
}

template <typename CSR>
mps_status spmm_ex_impl(const CSR *A, const void *B, int32_t b_dtype, int64_t ldb, int32_t K,
                        float *C, int64_t ldc, const int32_t *coord_x,
                        const idx_t<CSR> *coord_y, int64_t num_parts, int32_t fixup,
                        int32_t epilogue, const uint32_t *hot_bitmap, void *workspace,
                        size_t workspace_bytes, void *stream) {
    if (epilogue != MPS_EPI_NONE && epilogue != MPS_EPI_RELU)
        return fail(MPS_ERR_UNSUPPORTED, "epilogue %d", epilogue);
    if (resolve_fix(fixup) == mps::FIX_ATOMIC) {
        mps_status st = check_csr(A);
        if (st) return st;
        if ((st = check_dense(B, b_dtype, ldb, K, C, ldc, A))) return st;
        if (num_parts < 1) return fail(MPS_ERR_INVALID, "num_parts < 1");
        if (K == 0 || A->m == 0) return MPS_OK;
        const Vec v = choose_vec(K, b_dtype, B, ldb, C, ldc, A->n, A->m, A->nnz);
        const int32_t nz = zeroable_claims(K, v);
        if (!workspace || workspace_bytes < claim_bytes(K))
            return fail(MPS_ERR_WORKSPACE, "workspace %zu < %zu", workspace_bytes, claim_bytes(K));
        if ((st = zero_split_impl(A, coord_x, coord_y, num_parts, C, ldc, K, stream,
                                  (unsigned *)workspace, nz)))
            return st;
        return segments_impl(A, B, b_dtype, ldb, K, C, ldc, coord_x, coord_y, num_parts, fixup,
                             hot_bitmap, epilogue == MPS_EPI_RELU, workspace, workspace_bytes,
                             stream, nz > 0);
    }
    return segments_impl(A, B, b_dtype, ldb, K, C, ldc, coord_x, coord_y, num_parts, fixup,
                         hot_bitmap, epilogue == MPS_EPI_RELU, workspace, workspace_bytes,
                         stream);
}

size_t hot_scratch_bytes(int64_t n) {
    return align_up((size_t)n * 4, 256) + align_up(34 * 4, 256);
}
size_t hot_bitmap_bytes(int64_t n) { return align_up((size_t)((n + 31) / 32) * 4, 256); }

template <typename CSR>
mps_status hot_rows_impl(const CSR *A, int64_t budget_rows, uint32_t *hot_bitmap,
                         void *workspace, size_t workspace_bytes, void *stream) {
    mps_status st = check_csr(A);
    if (st) return st;
    if (budget_rows < 0 || (A->n > 0 && !hot_bitmap)) return fail(MPS_ERR_INVALID, "bad arguments");
    if (workspace_bytes < hot_scratch_bytes(A->n) || (A->n > 0 && !workspace))
        return fail(MPS_ERR_WORKSPACE, "workspace %zu < %zu", workspace_bytes,
                    hot_scratch_bytes(A->n));
    if (A->n == 0) return MPS_OK;
    int32_t *counts = (int32_t *)workspace;
    uint32_t *hist = (uint32_t *)((char *)workspace + align_up((size_t)A->n * 4, 256));
    MPS_CUDA(mps::launch_hot_columns(A->col_idx, A->nnz, A->n, budget_rows, counts, hist,
                                     hot_bitmap, (cudaStream_t)stream),
             "hot rows");
    return MPS_OK;
}

// Use degree-aware L2 residency when the gathered B is larger than half the L2.
int64_t hot_budget_rows(int64_t n, int32_t K, int32_t dt) {
    const double row = (double)K * elt_bytes(dt);
    if ((double)n * row <= 0.5 * (double)l2_bytes()) return -1;     // B fits: plain evict_last
    // Off by default: measured on B200 (profiles/r01/hot_rows.md) the static hub policy
    // gains <= 5% in the segment kernel and its per-call pre-pass costs more online.
    static const double frac = [] {
        const char *e = getenv("MPS_HOT_FRAC");
        return e ? atof(e) : 0.0;
    }();
    if (frac <= 0) return -1;
    return (int64_t)(frac * (double)l2_bytes() / row);
}

// online workspace: coord_x int32[P+1], coord_y IT[P+1], claim counters, carry records,
// hot-row scratch
size_t online_bytes(int64_t P, int32_t K, const Vec &v, int fix, int64_t n = 0,
                    size_t ysize = 4) {
    size_t b = align_up((size_t)(P + 1) * 4, 256) + align_up((size_t)(P + 1) * ysize, 256) +
               claim_bytes(K);
    if (fix == mps::FIX_CARRY) b += carry_bytes(P, K, v);
    if (n > 0) b += hot_bitmap_bytes(n) + hot_scratch_bytes(n);
    return b;
}

// The one-launch small-graph path (small.cu): row_ptr and the col/val staging fit in one
// CTA's shared memory, one column tile, int32 indices, no hot-row bitmap; chosen for
// MPS_FIXUP_AUTO and MPS_FIXUP_CARRY (it settles cut rows with the carry records).
// MPS_SMALL=0 disables it.
bool small_possible(int64_t m, int64_t L) {
    static const int on = [] {
        const char *e = getenv("MPS_SMALL");
        return e ? atoi(e) : 1;
    }();
    return on && L <= mps::kSmallMaxL && m + 1 < ((int64_t)1 << 30) &&
           mps::small_smem_bytes(m, L) <= (size_t)mps::kSmallMaxSmem;
}

template <typename CSR>
bool small_path_ok(const CSR *A, int32_t K, const Vec &v, int32_t fixup, int64_t L,
                   int64_t hot_rows) {
    if (sizeof(idx_t<CSR>) != 4 || fixup == MPS_FIXUP_ATOMIC || hot_rows >= 0) return false;
    if (!small_possible(A->m, L) || A->nnz >= kMaxIndex) return false;
    if (((uintptr_t)A->row_ptr) & 15u) return false;
    int V, NR;
    tile_geometry(K, v.W, &V, &NR);
    return V == 1 && v.tile >= K;
}

template <typename CSR>
mps_status online_ws_impl(const CSR *A, int32_t K, int32_t b_dtype, int64_t items_per_part,
                          int64_t min_parts, int32_t fixup, size_t *bytes) {
    mps_status st = check_csr(A, false);
    if (st) return st;
    if (!bytes) return fail(MPS_ERR_INVALID, "bytes NULL");
    int64_t P, L;
    if ((st = plan_impl(A->m, A->nnz, K, b_dtype, items_per_part, min_parts, &P, &L,
                        sizeof(idx_t<CSR>) == 8)))
        return st;
    Vec vmin;
    vmin.W = 1;
    vmin.tile = 128;
    const Vec v = choose_vec(K, b_dtype, nullptr, K ? K : 1, nullptr, K ? K : 1);
    // AUTO may take the small path, which needs the carry records
    const int fix = (fixup == MPS_FIXUP_AUTO && sizeof(idx_t<CSR>) == 4 &&
                     small_possible(A->m, L)) ? mps::FIX_CARRY : resolve_fix(fixup);
    const int64_t nh = hot_budget_rows(A->n, K, b_dtype) >= 0 ? A->n : 0;
    const size_t ys = sizeof(idx_t<CSR>);
    size_t a = online_bytes(P, K, v, fix, nh, ys), b = online_bytes(P, K, vmin, fix, nh, ys);
    *bytes = a > b ? a : b;
    return MPS_OK;
}

template <typename CSR>
mps_status small_online_impl(const CSR *A, const void *B, int32_t b_dtype, int64_t ldb,
                             int32_t K, float *C, int64_t ldc, int64_t P, int64_t L,
                             const Vec &v, int32_t epilogue, void *workspace,
                             size_t workspace_bytes, cudaStream_t s) {
    const size_t need = online_bytes(P, K, v, mps::FIX_CARRY, 0, 4);
    if (!workspace || workspace_bytes < need)
        return fail(MPS_ERR_WORKSPACE, "workspace %zu < %zu", workspace_bytes, need);
    const size_t xb = align_up((size_t)(P + 1) * 4, 256);
    int32_t *cx = (int32_t *)workspace;
    int32_t *cy = (int32_t *)((char *)workspace + xb);
    float *rec = (float *)((char *)workspace + 2 * xb + claim_bytes(K));
    int V, NR;
    tile_geometry(K, v.W, &V, &NR);
    static const int hints = [] {
        const char *e = getenv("MPS_L2_HINTS");
        return e ? atoi(e) : 1;
    }();
    mps::SmallArgs sa{};
    sa.rp = (const int32_t *)A->row_ptr;
    sa.col = A->col_idx;
    sa.val = A->val;
    sa.B = B;
    sa.ldb = ldb;
    sa.K = K;
    sa.C = C;
    sa.ldc = ldc;
    sa.m = (int32_t)A->m;
    sa.nnz = (int32_t)A->nnz;
    sa.P = (int32_t)P;
    sa.L = (int32_t)L;
    sa.cx = cx;
    sa.cy = cy;
    sa.rec = rec;
    sa.kpad = (int32_t)carry_kpad(K, v);
    sa.relu = epilogue == MPS_EPI_RELU;
    sa.l2_hints = hints;
    MPS_CUDA(mps::launch_small_online(sa, b_dtype, v.W, NR, s), "small online kernel");
    mps::SegArgsT<int32_t> a{};
    a.rp = (const int32_t *)A->row_ptr;
    a.C = C;
    a.ldc = ldc;
    a.K = K;
    a.m = (int32_t)A->m;
    a.cx = cx;
    a.cy = cy;
    a.P = P;
    a.tail_row = -1;
    a.rec = rec;
    a.kpad = sa.kpad;
    a.relu = sa.relu;
    MPS_CUDA(mps::launch_carry_reduce(a, s), "carry reduce");
    return MPS_OK;
}

// Which kernels the online call launches (mps_spmm_online_path).
template <typename CSR>
mps_status online_path_impl(const CSR *A, const void *B, int32_t b_dtype, int64_t ldb,
                            int32_t K, const float *C, int64_t ldc, int64_t items_per_part,
                            int64_t min_parts, int32_t fixup, int32_t *path) {
    mps_status st = check_csr(A, false);
    if (st) return st;
    if (!path) return fail(MPS_ERR_INVALID, "path_out NULL");
    *path = MPS_PATH_PARTITION_SEGMENTS;
    if (K <= 0 || A->m == 0) return MPS_OK;
    int64_t P, L;
    if ((st = plan_impl(A->m, A->nnz, K, b_dtype, items_per_part, min_parts, &P, &L,
                        sizeof(idx_t<CSR>) == 8)))
        return st;
    const Vec v = choose_vec(K, b_dtype, B, ldb, C, ldc, A->n, A->m, A->nnz);
    if (small_path_ok(A, K, v, fixup, L, hot_budget_rows(A->n, K, b_dtype)))
        *path = MPS_PATH_SMALL_FUSED;
    return MPS_OK;
}

template <typename CSR>
mps_status online_ex_impl(const CSR *A, const void *B, int32_t b_dtype, int64_t ldb, int32_t K,
                          float *C, int64_t ldc, int64_t items_per_part, int64_t min_parts,
                          int32_t fixup, int32_t epilogue, void *workspace,
                          size_t workspace_bytes, void *stream) {
    using IT = idx_t<CSR>;
    if (epilogue != MPS_EPI_NONE && epilogue != MPS_EPI_RELU)
        return fail(MPS_ERR_UNSUPPORTED, "epilogue %d", epilogue);
    mps_status st = check_csr(A);
    if (st) return st;
    if ((st = check_dense(B, b_dtype, ldb, K, C, ldc, A))) return st;
    if (K == 0 || A->m == 0) return MPS_OK;
    int64_t P, L;
    if ((st = plan_impl(A->m, A->nnz, K, b_dtype, items_per_part, min_parts, &P, &L,
                        sizeof(IT) == 8)))
        return st;
    const Vec v = choose_vec(K, b_dtype, B, ldb, C, ldc, A->n, A->m, A->nnz);
    const int64_t hot_rows = hot_budget_rows(A->n, K, b_dtype);
    if (small_path_ok(A, K, v, fixup, L, hot_rows))
        return small_online_impl(A, B, b_dtype, ldb, K, C, ldc, P, L, v, epilogue, workspace,
                                 workspace_bytes, (cudaStream_t)stream);
    const int fix = resolve_fix(fixup);
    const int64_t nh = hot_rows >= 0 ? A->n : 0;
    const size_t need = online_bytes(P, K, v, fix, nh, sizeof(IT));
    if (!workspace || workspace_bytes < need)
        return fail(MPS_ERR_WORKSPACE, "workspace %zu < %zu", workspace_bytes, need);
    cudaStream_t s = (cudaStream_t)stream;
    const size_t xb = align_up((size_t)(P + 1) * 4, 256);
    const size_t yb = align_up((size_t)(P + 1) * sizeof(IT), 256);
    int32_t *cx = (int32_t *)workspace;
    IT *cy = (IT *)((char *)workspace + xb);
    unsigned *claims = (unsigned *)((char *)workspace + xb + yb);
    void *rec = (char *)workspace + xb + yb + claim_bytes(K);
    const int32_t nz = zeroable_claims(K, v);
    uint32_t *bitmap = nullptr;
    if (nh > 0) {
        char *hb = (char *)workspace + online_bytes(P, K, v, fix, 0, sizeof(IT));
        bitmap = (uint32_t *)hb;
        mps_status hs = hot_rows_impl(A, hot_rows, bitmap, hb + hot_bitmap_bytes(A->n),
                                      hot_scratch_bytes(A->n), stream);
        if (hs) return hs;
    }
    MPS_CUDA(mps::launch_partition<IT>(A->row_ptr, A->m, A->nnz, 0, A->m + A->nnz, P, L, cx, cy,
                                       fix == mps::FIX_ATOMIC ? C : nullptr, ldc, 0, K, -1,
                                       nullptr, claims, nz, s),
             "partition kernel");
    mps::SegArgsT<IT> a{};
    a.rp = A->row_ptr;
    a.col = A->col_idx;
    a.val = A->val;
    a.B = B;
    a.ldb = ldb;
    a.C = C;
    a.ldc = ldc;
    a.row_base = 0;
    a.m = (int32_t)A->m;
    a.cx = cx;
    a.cy = cy;
    a.P = P;
    a.tail_row = -1;
    a.tail = nullptr;
    a.nnz_end = A->nnz;
    a.hot = bitmap;
    a.relu = epilogue == MPS_EPI_RELU;
    return run_segments(a, b_dtype, K, v, fix, rec, claims, nz > 0, s);
}

template <typename CSR>
mps_status write_stats_impl(const CSR *A, const int32_t *coord_x, const idx_t<CSR> *coord_y,
                            int64_t num_parts, int64_t *counts_out, void *stream) {
    mps_status st = check_csr(A);
    if (st) return st;
    if (num_parts < 1 || !coord_x || !coord_y || !counts_out)
        return fail(MPS_ERR_INVALID, "bad arguments");
    MPS_CUDA(mps::launch_write_stats(A->row_ptr, (int32_t)A->m, coord_x, coord_y, num_parts,
                                     counts_out, (cudaStream_t)stream),
             "write stats");
    return MPS_OK;
}

template <typename CSR>
mps_status validate_impl(const CSR *A, int64_t *first_bad_host, void *stream) {
    mps_status st = check_csr(A);
    if (st) return st;
    if (!first_bad_host) return fail(MPS_ERR_INVALID, "first_bad_host NULL");
    *first_bad_host = -1;
    if (A->m == 0 && A->nnz == 0) return MPS_OK;
    cudaStream_t s = (cudaStream_t)stream;
    unsigned long long *d = nullptr;
    MPS_CUDA(cudaMallocAsync((void **)&d, sizeof(*d), s), "alloc");
    const unsigned long long init = ~0ull;
    MPS_CUDA(cudaMemcpyAsync(d, &init, sizeof(init), cudaMemcpyHostToDevice, s), "H2D");
    MPS_CUDA(mps::launch_validate(A->row_ptr, A->col_idx, A->m, A->n, A->nnz, d, s), "validate");
    unsigned long long h = 0;
    MPS_CUDA(cudaMemcpyAsync(&h, d, sizeof(h), cudaMemcpyDeviceToHost, s), "D2H");
    MPS_CUDA(cudaFreeAsync(d, s), "free");
    MPS_CUDA(cudaStreamSynchronize(s), "sync");
    *first_bad_host = (h == ~0ull) ? -1 : (int64_t)h;
    return MPS_OK;
}

}  // namespace

extern "C" {

// ---- int32 entry points (mps_csr) ----------------------------------------------------
mps_status mps_spmm_workspace_bytes(const mps_csr *A, int32_t K, int32_t b_dtype,
                                    int64_t num_parts, int32_t fixup, size_t *bytes) {
    return spmm_ws_impl(A, K, b_dtype, num_parts, fixup, bytes);
}

mps_status mps_zero_split_rows(const mps_csr *A, const int32_t *coord_x, const int32_t *coord_y,
                               int64_t num_parts, float *C, int64_t ldc, int32_t K,
                               void *stream) {
    return zero_split_impl(A, coord_x, coord_y, num_parts, C, ldc, K, stream);
}

mps_status mps_spmm(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb, int32_t K,
                    float *C, int64_t ldc, const int32_t *coord_x, const int32_t *coord_y,
                    int64_t num_parts, int32_t fixup, void *workspace, size_t workspace_bytes,
                    void *stream) {
    return spmm_ex_impl(A, B, b_dtype, ldb, K, C, ldc, coord_x, coord_y, num_parts, fixup,
                        MPS_EPI_NONE, nullptr, workspace, workspace_bytes, stream);
}

mps_status mps_spmm_segments(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                             int32_t K, float *C, int64_t ldc, const int32_t *coord_x,
                             const int32_t *coord_y, int64_t num_parts, int32_t fixup,
                             void *workspace, size_t workspace_bytes, void *stream) {
    return segments_impl(A, B, b_dtype, ldb, K, C, ldc, coord_x, coord_y, num_parts, fixup,
                         nullptr, 0, workspace, workspace_bytes, stream);
}

mps_status mps_spmm_write_counts(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                                 int32_t K, float *C, int64_t ldc, const int32_t *coord_x,
                                 const int32_t *coord_y, int64_t num_parts, int32_t fixup,
                                 int64_t *counts, void *workspace, size_t workspace_bytes,
                                 void *stream) {
    if (!counts) return fail(MPS_ERR_INVALID, "counts NULL");
    cudaStream_t s = (cudaStream_t)stream;
    MPS_CUDA(cudaMemsetAsync(counts, 0, 3 * sizeof(int64_t), s), "zero counts");
    mps_status st = check_csr(A);
    if (st) return st;
    if (resolve_fix(fixup) == mps::FIX_ATOMIC && K > 0 && A->m > 0 &&
        (st = zero_split_impl(A, coord_x, coord_y, num_parts, C, ldc, K, stream)))
        return st;
    return segments_impl(A, B, b_dtype, ldb, K, C, ldc, coord_x, coord_y, num_parts, fixup,
                         nullptr, 0, workspace, workspace_bytes, stream, false,
                         reinterpret_cast<unsigned long long *>(counts));
}

mps_status mps_spmm_segments_hot(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                                 int32_t K, float *C, int64_t ldc, const int32_t *coord_x,
                                 const int32_t *coord_y, int64_t num_parts, int32_t fixup,
                                 const uint32_t *hot_bitmap, void *workspace,
                                 size_t workspace_bytes, void *stream) {
    return segments_impl(A, B, b_dtype, ldb, K, C, ldc, coord_x, coord_y, num_parts, fixup,
                         hot_bitmap, 0, workspace, workspace_bytes, stream);
}

mps_status mps_spmm_ex(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb, int32_t K,
                       float *C, int64_t ldc, const int32_t *coord_x, const int32_t *coord_y,
                       int64_t num_parts, int32_t fixup, int32_t epilogue,
                       const uint32_t *hot_bitmap, void *workspace, size_t workspace_bytes,
                       void *stream) {
    return spmm_ex_impl(A, B, b_dtype, ldb, K, C, ldc, coord_x, coord_y, num_parts, fixup,
                        epilogue, hot_bitmap, workspace, workspace_bytes, stream);
}

mps_status mps_hot_rows_workspace_bytes(int64_t n, size_t *bytes) {
    if (n < 0 || !bytes) return fail(MPS_ERR_INVALID, "bad arguments");
    *bytes = hot_scratch_bytes(n);
    return MPS_OK;
}

mps_status mps_hot_rows(const mps_csr *A, int64_t budget_rows, uint32_t *hot_bitmap,
                        void *workspace, size_t workspace_bytes, void *stream) {
    return hot_rows_impl(A, budget_rows, hot_bitmap, workspace, workspace_bytes, stream);
}

mps_status mps_hot_budget_rows(const mps_csr *A, int32_t K, int32_t b_dtype,
                               int64_t *budget_rows_out) {
    mps_status st = check_csr(A, false);
    if (st) return st;
    if (!budget_rows_out || K < 0) return fail(MPS_ERR_INVALID, "bad arguments");
    if (b_dtype != MPS_DT_F32 && b_dtype != MPS_DT_BF16)
        return fail(MPS_ERR_UNSUPPORTED, "b_dtype %d", b_dtype);
    *budget_rows_out = K > 0 ? hot_budget_rows(A->n, K, b_dtype) : -1;
    return MPS_OK;
}

mps_status mps_spmm_online_workspace_bytes(const mps_csr *A, int32_t K, int32_t b_dtype,
                                           int64_t items_per_part, int64_t min_parts,
                                           int32_t fixup, size_t *bytes) {
    return online_ws_impl(A, K, b_dtype, items_per_part, min_parts, fixup, bytes);
}

mps_status mps_spmm_online(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                           int32_t K, float *C, int64_t ldc, int64_t items_per_part,
                           int64_t min_parts, int32_t fixup, void *workspace,
                           size_t workspace_bytes, void *stream) {
    return online_ex_impl(A, B, b_dtype, ldb, K, C, ldc, items_per_part, min_parts, fixup,
                          MPS_EPI_NONE, workspace, workspace_bytes, stream);
}

mps_status mps_spmm_online_path(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                                int32_t K, const float *C, int64_t ldc, int64_t items_per_part,
                                int64_t min_parts, int32_t fixup, int32_t *path_out) {
    return online_path_impl(A, B, b_dtype, ldb, K, C, ldc, items_per_part, min_parts, fixup,
                            path_out);
}

mps_status mps_spmm_online_ex(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                              int32_t K, float *C, int64_t ldc, int64_t items_per_part,
                              int64_t min_parts, int32_t fixup, int32_t epilogue,
                              void *workspace, size_t workspace_bytes, void *stream) {
    return online_ex_impl(A, B, b_dtype, ldb, K, C, ldc, items_per_part, min_parts, fixup,
                          epilogue, workspace, workspace_bytes, stream);
}

// ---- int64 entry points (mps_csr64, NEXT-4) ------------------------------------------
mps_status mps_spmm64_workspace_bytes(const mps_csr64 *A, int32_t K, int32_t b_dtype,
                                      int64_t num_parts, int32_t fixup, size_t *bytes) {
    return spmm_ws_impl(A, K, b_dtype, num_parts, fixup, bytes);
}

mps_status mps_spmm64(const mps_csr64 *A, const void *B, int32_t b_dtype, int64_t ldb,
                      int32_t K, float *C, int64_t ldc, const int32_t *coord_x,
                      const int64_t *coord_y, int64_t num_parts, int32_t fixup,
                      int32_t epilogue, void *workspace, size_t workspace_bytes, void *stream) {
    return spmm_ex_impl(A, B, b_dtype, ldb, K, C, ldc, coord_x, coord_y, num_parts, fixup,
                        epilogue, nullptr, workspace, workspace_bytes, stream);
}

mps_status mps_spmm64_online_workspace_bytes(const mps_csr64 *A, int32_t K, int32_t b_dtype,
                                             int64_t items_per_part, int64_t min_parts,
                                             int32_t fixup, size_t *bytes) {
    return online_ws_impl(A, K, b_dtype, items_per_part, min_parts, fixup, bytes);
}

mps_status mps_spmm64_online(const mps_csr64 *A, const void *B, int32_t b_dtype, int64_t ldb,
                             int32_t K, float *C, int64_t ldc, int64_t items_per_part,
                             int64_t min_parts, int32_t fixup, int32_t epilogue,
                             void *workspace, size_t workspace_bytes, void *stream) {
    return online_ex_impl(A, B, b_dtype, ldb, K, C, ldc, items_per_part, min_parts, fixup,
                          epilogue, workspace, workspace_bytes, stream);
}

mps_status mps_write_stats64(const mps_csr64 *A, const int32_t *coord_x, const int64_t *coord_y,
                             int64_t num_parts, int64_t *counts_out, void *stream) {
    return write_stats_impl(A, coord_x, coord_y, num_parts, counts_out, stream);
}

mps_status mps_validate_csr64(const mps_csr64 *A, int64_t *first_bad_host, void *stream) {
    return validate_impl(A, first_bad_host, stream);
}

// ----------------------------------------------------------------------------------
// host-buffer end-to-end call
// ----------------------------------------------------------------------------------
struct HostLayout {
    size_t rp, ci, val, B, C, ws, total;
};

static HostLayout host_layout(const mps_csr *A, int32_t dt, int64_t ldb, int64_t ldc,
                              size_t online) {
    HostLayout h;
    size_t o = 0;
    h.rp = o; o += align_up((size_t)(A->m + 1) * 4, 256);
    h.ci = o; o += align_up((size_t)A->nnz * 4, 256);
    h.val = o; o += align_up((size_t)A->nnz * 4, 256);
    h.B = o; o += align_up((size_t)A->n * (size_t)ldb * elt_bytes(dt), 256);
    h.C = o; o += align_up((size_t)A->m * (size_t)ldc * 4, 256);
    h.ws = o; o += online;
    h.total = o;
    return h;
}

mps_status mps_spmm_host_workspace_bytes(const mps_csr *A_host, int32_t K, int32_t b_dtype,
                                         int64_t ldb, int64_t ldc, int64_t items_per_part,
                                         int64_t min_parts, int32_t fixup, size_t *bytes) {
    size_t online = 0;
    mps_status st = mps_spmm_online_workspace_bytes(A_host, K, b_dtype, items_per_part,
                                                    min_parts, fixup, &online);
    if (st) return st;
    *bytes = host_layout(A_host, b_dtype, ldb, ldc, online).total;
    return MPS_OK;
}

// Pipelined end-to-end call (atomic fix-up): the H2D of A is cut into NC chunks at
// merge-path segment boundaries p_c, so the segment kernel of chunk c overlaps the copy
// of chunk c+1, and the rows chunk c finalises go back D2H while later chunks still
// copy in (PCIe is full duplex).  Chunk c covers diagonals [p_c L, p_{c+1} L); the host
// finds their coordinates (x_c, y_c) with the same search as the shard bounds, so the
// chunk's non-zeros are exactly [y_c, y_{c+1}) = [cy[p_c], cy[p_{c+1}]) of the device
// partition (Alg. 1 and its closed form, reading R2).  Rows [x_c, x_{c+1}) are final
// after chunks 0..c: a row's end item lies on a diagonal below d_{c+1}, and a row cut
// at x_{c+1} belongs to the next range.  One partition (+ cut-row zeroing) launch over
// all P segments serves every chunk, so the result is the one mps_spmm_online gives.
namespace {
// The pipelined host call's two auxiliary streams (compute, D2H) are created per call and
// released when the call's work completes: the library keeps no streams between calls.
struct AuxStreams {
    cudaStream_t comp = nullptr, d2h = nullptr;
    ~AuxStreams() {
        if (comp) cudaStreamDestroy(comp);   // deferred by the runtime until the work is done
        if (d2h) cudaStreamDestroy(d2h);
    }
};

// rows x width bytes between pitched buffers: only the K valid columns of a strided
// (ld > K) host matrix are read or written, never its padding
cudaError_t copy_rows(void *dst, const void *src, size_t pitch, size_t width, size_t rows,
                      cudaMemcpyKind kind, cudaStream_t s) {
    if (rows == 0 || width == 0) return cudaSuccess;
    if (pitch == width) return cudaMemcpyAsync(dst, src, rows * width, kind, s);
    return cudaMemcpy2DAsync(dst, pitch, src, pitch, width, rows, kind, s);
}

bool getenv_flag(const char *name) {
    const char *e = getenv(name);
    return e && atoi(e) != 0;
}

int64_t host_chunk_bytes() {
    const char *e = getenv("MPS_HOST_CHUNK_BYTES");   // read per call (tests vary it)
    const long long x = e ? atoll(e) : 0;
    return (int64_t)(x > 0 ? x : (32ll << 20));
}
}  // namespace

static mps_status host_pipelined(const mps_csr *A_host, const void *B_host, int32_t b_dtype,
                                 int64_t ldb, int32_t K, float *C_host, int64_t ldc,
                                 int64_t P, int64_t L, const Vec &v, const HostLayout &h,
                                 char *w, cudaStream_t s) {
    AuxStreams ax;
    if (cudaStreamCreateWithFlags(&ax.comp, cudaStreamNonBlocking) != cudaSuccess ||
        cudaStreamCreateWithFlags(&ax.d2h, cudaStreamNonBlocking) != cudaSuccess)
        return fail(MPS_ERR_CUDA, "auxiliary streams");
    const int64_t m = A_host->m, nnz = A_host->nnz, M = m + nnz;
    int64_t nc = (nnz * 8 + host_chunk_bytes() - 1) / host_chunk_bytes();
    if (nc < 1) nc = 1;
    if (nc > 64) nc = 64;
    if (nc > P) nc = P;
    std::vector<int64_t> pc(nc + 1), xc(nc + 1), yc(nc + 1);
    for (int64_t c = 0; c <= nc; ++c) {
        pc[c] = (P * c) / nc;
        const int64_t d = pc[c] * L < M ? pc[c] * L : M;
        xc[c] = host_diag_x(A_host->row_ptr, m, nnz, d);
        yc[c] = d - xc[c];
    }
    const size_t bbytes = (size_t)A_host->n * (size_t)ldb * elt_bytes(b_dtype);
    const size_t brow = (size_t)ldb * elt_bytes(b_dtype), bwidth = (size_t)K * elt_bytes(b_dtype);
    int32_t *rp = (int32_t *)(w + h.rp);
    int32_t *ci = (int32_t *)(w + h.ci);
    float *va = (float *)(w + h.val);
    float *C = (float *)(w + h.C);
    const size_t xb = align_up((size_t)(P + 1) * 4, 256);
    int32_t *cx = (int32_t *)(w + h.ws);
    int32_t *cy = (int32_t *)(w + h.ws + xb);

    std::vector<cudaEvent_t> ev(2 * nc + 3, nullptr);
    for (auto &e : ev)
        if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) {
            for (auto &f : ev) if (f) cudaEventDestroy(f);
            return fail(MPS_ERR_CUDA, "event create");
        }
    cudaEvent_t ev_rp = ev[0], ev_B = ev[1], ev_end = ev[2];
    cudaEvent_t *ev_A = &ev[3], *ev_done = &ev[3 + nc];
    mps_status st = MPS_OK;
    auto chk = [&](cudaError_t e, const char *where) {
        if (e != cudaSuccess && st == MPS_OK) st = cuda_fail(e, where);
        return st == MPS_OK;
    };
    // copy stream (the caller's): row_ptr, B, then A chunk by chunk
    chk(cudaMemcpyAsync(rp, A_host->row_ptr, (size_t)(m + 1) * 4, cudaMemcpyHostToDevice, s),
        "H2D row_ptr");
    chk(cudaEventRecord(ev_rp, s), "event");
    if (bbytes)
        chk(copy_rows(w + h.B, B_host, brow, bwidth, (size_t)A_host->n, cudaMemcpyHostToDevice, s),
            "H2D B");
    chk(cudaEventRecord(ev_B, s), "event");
    for (int64_t c = 0; c < nc && st == MPS_OK; ++c) {
        const size_t n = (size_t)(yc[c + 1] - yc[c]) * 4;
        if (n) {
            chk(cudaMemcpyAsync(ci + yc[c], A_host->col_idx + yc[c], n, cudaMemcpyHostToDevice, s),
                "H2D col_idx");
            chk(cudaMemcpyAsync(va + yc[c], A_host->val + yc[c], n, cudaMemcpyHostToDevice, s),
                "H2D val");
        }
        chk(cudaEventRecord(ev_A[c], s), "event");
    }
    // compute stream: one partition (+ cut-row zeroing), then the segments chunk by chunk
    chk(cudaStreamWaitEvent(ax.comp, ev_rp, 0), "wait");
    if (st == MPS_OK)
        chk(mps::launch_partition<int32_t>(rp, m, nnz, 0, M, P, L, cx, cy, C, ldc, 0, K, -1,
                                           nullptr, nullptr, 0, ax.comp), "partition kernel");
    chk(cudaStreamWaitEvent(ax.comp, ev_B, 0), "wait");
    for (int64_t c = 0; c < nc && st == MPS_OK; ++c) {
        chk(cudaStreamWaitEvent(ax.comp, ev_A[c], 0), "wait");
        if (pc[c + 1] > pc[c]) {
            mps::SegArgsT<int32_t> a{};
            a.rp = rp;
            a.col = ci;
            a.val = va;
            a.B = w + h.B;
            a.ldb = ldb;
            a.C = C;
            a.ldc = ldc;
            a.row_base = 0;
            a.m = (int32_t)m;
            a.cx = cx + pc[c];
            a.cy = cy + pc[c];
            a.P = pc[c + 1] - pc[c];
            a.tail_row = -1;
            a.tail = nullptr;
            a.nnz_end = nnz;
            a.hot = nullptr;
            a.relu = 0;
            // static segment assignment: the chunks' launches would each need their
            // own claim counters; this path is bound by the H2D copies anyway
            st = run_segments(a, b_dtype, K, v, mps::FIX_ATOMIC, nullptr, nullptr, true, ax.comp);
        }
        chk(cudaEventRecord(ev_done[c], ax.comp), "event");
    }
    // D2H stream: rows [x_c, x_{c+1}) once chunk c is done (the last chunk: up to m)
    for (int64_t c = 0; c < nc && st == MPS_OK; ++c) {
        const int64_t r0 = xc[c], r1 = (c + 1 == nc) ? m : xc[c + 1];
        chk(cudaStreamWaitEvent(ax.d2h, ev_done[c], 0), "wait");
        if (r1 > r0)
            chk(copy_rows(C_host + r0 * ldc, C + r0 * ldc, (size_t)ldc * 4, (size_t)K * 4,
                          (size_t)(r1 - r0), cudaMemcpyDeviceToHost, ax.d2h), "D2H C");
    }
    // join: the caller's stream sees the whole call
    chk(cudaEventRecord(ev_end, ax.d2h), "event");
    chk(cudaStreamWaitEvent(s, ev_end, 0), "wait");
    for (auto &e : ev) cudaEventDestroy(e);   // released once the recorded work completes
    return st;
}

mps_status mps_spmm_host(const mps_csr *A_host, const void *B_host, int32_t b_dtype,
                         int64_t ldb, int32_t K, float *C_host, int64_t ldc,
                         int64_t items_per_part, int64_t min_parts, int32_t fixup,
                         void *device_workspace, size_t workspace_bytes, void *stream) {
    mps_status st = check_csr(A_host);
    if (st) return st;
    if ((st = check_dense(B_host, b_dtype, ldb, K, C_host, ldc, A_host))) return st;
    if (K == 0 || A_host->m == 0) return MPS_OK;
    size_t online = 0;
    if ((st = mps_spmm_online_workspace_bytes(A_host, K, b_dtype, items_per_part, min_parts,
                                              fixup, &online)))
        return st;
    const HostLayout h = host_layout(A_host, b_dtype, ldb, ldc, online);
    if (!device_workspace || workspace_bytes < h.total)
        return fail(MPS_ERR_WORKSPACE, "workspace %zu < %zu", workspace_bytes, h.total);
    cudaStream_t s = (cudaStream_t)stream;
    char *w = (char *)device_workspace;
    if (resolve_fix(fixup) == mps::FIX_ATOMIC && hot_budget_rows(A_host->n, K, b_dtype) < 0 &&
        !getenv_flag("MPS_HOST_SERIAL")) {
        int64_t P, L;
        if ((st = plan_impl(A_host->m, A_host->nnz, K, b_dtype, items_per_part, min_parts, &P,
                            &L, false)))
            return st;
        const Vec v = choose_vec(K, b_dtype, w + h.B, ldb, (float *)(w + h.C), ldc, A_host->n,
                                 A_host->m, A_host->nnz);
        return host_pipelined(A_host, B_host, b_dtype, ldb, K, C_host, ldc, P, L, v, h, w, s);
    }
    const size_t bbytes = (size_t)A_host->n * (size_t)ldb * elt_bytes(b_dtype);
    MPS_CUDA(cudaMemcpyAsync(w + h.rp, A_host->row_ptr, (size_t)(A_host->m + 1) * 4,
                             cudaMemcpyHostToDevice, s), "H2D row_ptr");
    if (A_host->nnz) {
        MPS_CUDA(cudaMemcpyAsync(w + h.ci, A_host->col_idx, (size_t)A_host->nnz * 4,
                                 cudaMemcpyHostToDevice, s), "H2D col_idx");
        MPS_CUDA(cudaMemcpyAsync(w + h.val, A_host->val, (size_t)A_host->nnz * 4,
                                 cudaMemcpyHostToDevice, s), "H2D val");
    }
    if (bbytes)
        MPS_CUDA(copy_rows(w + h.B, B_host, (size_t)ldb * elt_bytes(b_dtype),
                           (size_t)K * elt_bytes(b_dtype), (size_t)A_host->n,
                           cudaMemcpyHostToDevice, s), "H2D B");
    mps_csr Ad = *A_host;
    Ad.row_ptr = (const int32_t *)(w + h.rp);
    Ad.col_idx = (const int32_t *)(w + h.ci);
    Ad.val = (const float *)(w + h.val);
    if ((st = mps_spmm_online(&Ad, w + h.B, b_dtype, ldb, K, (float *)(w + h.C), ldc,
                              items_per_part, min_parts, fixup, w + h.ws, online, stream)))
        return st;
    MPS_CUDA(copy_rows(C_host, w + h.C, (size_t)ldc * 4, (size_t)K * 4, (size_t)A_host->m,
                       cudaMemcpyDeviceToHost, s), "D2H C");
    return MPS_OK;
}

mps_status mps_spmm_host_dense_workspace_bytes(const mps_csr *A, int32_t K, int32_t b_dtype,
                                               int64_t ldb, int64_t ldc, int64_t items_per_part,
                                               int64_t min_parts, int32_t fixup, size_t *bytes) {
    if (!A || !bytes) return fail(MPS_ERR_INVALID, "NULL pointer");
    size_t online = 0;
    mps_status st = mps_spmm_online_workspace_bytes(A, K, b_dtype, items_per_part, min_parts,
                                                    fixup, &online);
    if (st) return st;
    *bytes = align_up((size_t)A->n * (size_t)ldb * elt_bytes(b_dtype), 256) +
             align_up((size_t)A->m * (size_t)ldc * 4, 256) + online;
    return MPS_OK;
}

mps_status mps_spmm_host_dense(const mps_csr *A, const void *B_host, int32_t b_dtype,
                               int64_t ldb, int32_t K, float *C_host, int64_t ldc,
                               int64_t items_per_part, int64_t min_parts, int32_t fixup,
                               void *device_workspace, size_t workspace_bytes, void *stream) {
    mps_status st = check_csr(A);
    if (st) return st;
    if ((st = check_dense(B_host, b_dtype, ldb, K, C_host, ldc, A))) return st;
    if (K == 0 || A->m == 0) return MPS_OK;
    size_t need = 0, online = 0;
    if ((st = mps_spmm_host_dense_workspace_bytes(A, K, b_dtype, ldb, ldc, items_per_part,
                                                  min_parts, fixup, &need)))
        return st;
    if ((st = mps_spmm_online_workspace_bytes(A, K, b_dtype, items_per_part, min_parts, fixup,
                                              &online)))
        return st;
    if (!device_workspace || workspace_bytes < need)
        return fail(MPS_ERR_WORKSPACE, "workspace %zu < %zu", workspace_bytes, need);
    cudaStream_t s = (cudaStream_t)stream;
    char *w = (char *)device_workspace;
    const size_t bbytes = (size_t)A->n * (size_t)ldb * elt_bytes(b_dtype);
    char *Bd = w;
    float *Cd = (float *)(w + align_up(bbytes, 256));
    char *ws = (char *)Cd + align_up((size_t)A->m * (size_t)ldc * 4, 256);
    if (bbytes)
        MPS_CUDA(copy_rows(Bd, B_host, (size_t)ldb * elt_bytes(b_dtype),
                           (size_t)K * elt_bytes(b_dtype), (size_t)A->n, cudaMemcpyHostToDevice,
                           s), "H2D B");
    if ((st = mps_spmm_online(A, Bd, b_dtype, ldb, K, Cd, ldc, items_per_part, min_parts, fixup,
                              ws, online, stream)))
        return st;
    MPS_CUDA(copy_rows(C_host, Cd, (size_t)ldc * 4, (size_t)K * 4, (size_t)A->m,
                       cudaMemcpyDeviceToHost, s), "D2H C");
    return MPS_OK;
}

mps_status mps_xw_bf16(const void *X, int64_t n, int64_t F, int64_t ldx, const void *Wt,
                       int32_t N, int64_t ldw, void *B, int64_t ldb, void *stream) {
    if (n < 0 || F < 0 || N < 0 || ldx < F || ldw < F || ldb < N)
        return fail(MPS_ERR_INVALID, "bad xw sizes");
    if (n == 0 || N == 0) return MPS_OK;
    if (!X || !Wt || !B) return fail(MPS_ERR_INVALID, "NULL pointer");
    const cudaError_t e = mps::launch_xw_bf16(X, n, F, ldx, Wt, N, ldw, B, ldb, (cudaStream_t)stream);
    if (e == cudaErrorNotSupported)
        return fail(MPS_ERR_UNSUPPORTED, "xw: need 16 <= N <= 256, N %% 16 == 0, ld %% 8 == 0, "
                    "16-B aligned pointers");
    MPS_CUDA(e, "xw gemm");
    return MPS_OK;
}

mps_status mps_xw_bf16_bcast(const void *X, int64_t n_rows, int64_t F, int64_t ldx,
                             const void *Wt, int32_t N, int64_t ldw, void *const *B_dsts_host,
                             int32_t ndst, int64_t row_offset, int64_t ldb, void *stream) {
    if (n_rows < 0 || F < 0 || N < 0 || ldx < F || ldw < F || ldb < N || row_offset < 0 ||
        ndst < 1)
        return fail(MPS_ERR_INVALID, "bad xw_bcast sizes");
    if (!B_dsts_host) return fail(MPS_ERR_INVALID, "B_dsts_host NULL");
    if (n_rows == 0 || N == 0) return MPS_OK;
    if (!X || !Wt) return fail(MPS_ERR_INVALID, "NULL pointer");
    const cudaError_t e = mps::launch_xw_bf16_bcast(X, n_rows, F, ldx, Wt, N, ldw, B_dsts_host,
                                                    ndst, row_offset, ldb, (cudaStream_t)stream);
    if (e == cudaErrorNotSupported)
        return fail(MPS_ERR_UNSUPPORTED, "xw_bcast: need 16 <= N <= 256, N %% 16 == 0, ld %% 8 "
                    "== 0, 16-B aligned non-NULL pointers, 1 <= ndst <= 16");
    MPS_CUDA(e, "xw gemm bcast");
    return MPS_OK;
}

mps_status mps_relu_to_bf16(const float *C, int64_t rows, int32_t K, int64_t ldc, void *H,
                            int64_t ldh, void *stream) {
    if (rows < 0 || K < 0 || (rows > 0 && K > 0 && (!C || !H || ldc < K || ldh < K)))
        return fail(MPS_ERR_INVALID, "bad relu_to_bf16 arguments");
    MPS_CUDA(mps::launch_relu_to_bf16(C, rows, K, ldc, H, ldh, (cudaStream_t)stream),
             "relu_to_bf16");
    return MPS_OK;
}

// ---- cross-GPU signals (pipelining the replication of B with the SpMM) ---------------
constexpr int kSignalSlots = 64;
size_t mps_signal_bytes(void) { return (size_t)kSignalSlots * mps::kMailMaxWorld * 4; }

mps_status mps_peer_signal(void *const *signal_bufs_host, int32_t world, int32_t rank,
                           int32_t slot, uint32_t epoch, void *stream) {
    if (!signal_bufs_host || world < 1 || world > mps::kMailMaxWorld || rank < 0 ||
        rank >= world || slot < 0 || slot >= kSignalSlots || epoch == 0)
        return fail(MPS_ERR_INVALID, "bad signal arguments");
    for (int32_t g = 0; g < world; ++g)
        if (!signal_bufs_host[g]) return fail(MPS_ERR_INVALID, "signal buffer %d NULL", g);
    MPS_CUDA(mps::launch_peer_signal(signal_bufs_host, world, rank, slot, epoch,
                                     (cudaStream_t)stream), "peer signal");
    return MPS_OK;
}

mps_status mps_peer_wait(const void *my_signal_buf, int32_t world, int32_t slot, uint32_t epoch,
                         void *stream) {
    if (!my_signal_buf || world < 1 || world > mps::kMailMaxWorld || slot < 0 ||
        slot >= kSignalSlots || epoch == 0)
        return fail(MPS_ERR_INVALID, "bad wait arguments");
    MPS_CUDA(mps::launch_peer_wait(my_signal_buf, world, slot, epoch, (cudaStream_t)stream),
             "peer wait");
    return MPS_OK;
}

// ---- CUDA IPC: map one rank's device buffer into another rank's address space --------
size_t mps_ipc_handle_bytes(void) { return sizeof(cudaIpcMemHandle_t); }

mps_status mps_ipc_get_handle(const void *dev_ptr, void *handle_out, int64_t *offset_out) {
    if (!dev_ptr || !handle_out || !offset_out) return fail(MPS_ERR_INVALID, "NULL pointer");
    // the handle names the whole allocation; report where dev_ptr sits inside it
    using RangeFn = CUresult (*)(CUdeviceptr *, size_t *, CUdeviceptr);
    static RangeFn range = nullptr;
    if (!range) {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &p, cudaEnableDefault, &q) !=
                cudaSuccess || q != cudaDriverEntryPointSuccess)
            return fail(MPS_ERR_CUDA, "cuMemGetAddressRange unavailable");
        range = reinterpret_cast<RangeFn>(p);
    }
    CUdeviceptr base = 0;
    size_t size = 0;
    if (range(&base, &size, (CUdeviceptr)(uintptr_t)dev_ptr) != CUDA_SUCCESS)
        return fail(MPS_ERR_INVALID, "not a device allocation");
    cudaIpcMemHandle_t h;
    MPS_CUDA(cudaIpcGetMemHandle(&h, (void *)(uintptr_t)base), "cudaIpcGetMemHandle");
    memcpy(handle_out, &h, sizeof(h));
    *offset_out = (int64_t)((uintptr_t)dev_ptr - (uintptr_t)base);
    return MPS_OK;
}

mps_status mps_ipc_open_handle(const void *handle, void **base_out) {
    if (!handle || !base_out) return fail(MPS_ERR_INVALID, "NULL pointer");
    cudaIpcMemHandle_t h;
    memcpy(&h, handle, sizeof(h));
    MPS_CUDA(cudaIpcOpenMemHandle(base_out, h, cudaIpcMemLazyEnablePeerAccess),
             "cudaIpcOpenMemHandle");
    return MPS_OK;
}

mps_status mps_ipc_close_handle(void *base) {
    if (!base) return fail(MPS_ERR_INVALID, "NULL pointer");
    MPS_CUDA(cudaIpcCloseMemHandle(base), "cudaIpcCloseMemHandle");
    return MPS_OK;
}

mps_status mps_write_stats(const mps_csr *A, const int32_t *coord_x, const int32_t *coord_y,
                           int64_t num_parts, int64_t *counts_out, void *stream) {
    return write_stats_impl(A, coord_x, coord_y, num_parts, counts_out, stream);
}

// ----------------------------------------------------------------------------------
// sharding (a6)
// ----------------------------------------------------------------------------------
}  // extern "C"

// ---------------------------------------------------------------------------------
// a6 sharding, shared by the int32 (mps_csr) and int64 (mps_csr64, NEXT-4) entry points.
// IT = row_ptr / Y type.
// ---------------------------------------------------------------------------------
template <typename IT>
static mps_status shard_bounds_impl(const IT *row_ptr_host, int64_t m, int64_t nnz,
                                    int32_t world, int32_t *X, IT *Y, int32_t *tail_rows) {
    if (m < 0 || nnz < 0 || world < 1) return fail(MPS_ERR_INVALID, "bad shard arguments");
    if (sizeof(IT) == 4 && m + nnz >= kMaxIndex)
        return fail(MPS_ERR_UNSUPPORTED, "m + nnz >= 2^31");
    if (sizeof(IT) == 8 && (m >= kMaxIndex || nnz >= kMaxIndex64))
        return fail(MPS_ERR_UNSUPPORTED, "m >= 2^31 or nnz >= 2^62");
    if (!row_ptr_host || !X || !Y || !tail_rows) return fail(MPS_ERR_INVALID, "NULL pointer");
    const int64_t M = m + nnz;
    const int64_t per = (M + world - 1) / world;
    for (int32_t g = 0; g <= world; ++g) {
        int64_t d = (int64_t)g * per;
        if (d > M) d = M;
        const int64_t x = host_diag_x(row_ptr_host, m, nnz, d);
        X[g] = (int32_t)x;
        Y[g] = (IT)(d - x);
    }
    for (int32_t g = 0; g < world; ++g) {
        const int32_t r = X[g + 1];
        tail_rows[g] = (r < m && Y[g + 1] > row_ptr_host[r]) ? r : -1;
    }
    return MPS_OK;
}

template <typename CSR>
static mps_status shard_plan(const CSR *A, const int32_t *X, const idx_t<CSR> *Y, int32_t rank,
                             int32_t K, int32_t dt, int64_t ipp, int64_t minp, int64_t *P,
                             int64_t *L, int64_t *D0, int64_t *span) {
    if (ipp == 0) ipp = default_cost(A->m, A->nnz, K, dt);  // the whole graph's row length
    *D0 = (int64_t)X[rank] + (int64_t)Y[rank];
    const int64_t D1 = (int64_t)X[rank + 1] + (int64_t)Y[rank + 1];
    *span = D1 - *D0;
    if (*span < 0) return fail(MPS_ERR_INVALID, "shard bounds not monotone");
    // local plan over the shard's merge items (items of rows counted as rows here)
    return plan_impl(*span, 0, K, dt, ipp, minp, P, L, sizeof(idx_t<CSR>) == 8);
}

template <typename CSR>
static mps_status shard_ws_impl(const CSR *A, int32_t K, int32_t b_dtype, const int32_t *X,
                                int32_t rank, int32_t world, int64_t items_per_part,
                                int64_t min_parts, int32_t fixup, size_t *bytes) {
    mps_status st = check_csr(A, false);
    if (st) return st;
    if (!X || !bytes || world < 1 || rank < 0 || rank >= world)
        return fail(MPS_ERR_INVALID, "bad shard arguments");
    // Y is not needed for the size: the span is at most ceil(M/world)
    const int64_t M = A->m + A->nnz;
    const int64_t span = (M + world - 1) / world;
    int64_t P, L;
    const int64_t ipp = items_per_part ? items_per_part : default_cost(A->m, A->nnz, K, b_dtype);
    if ((st = plan_impl(span, 0, K, b_dtype, ipp, min_parts, &P, &L,
                        sizeof(idx_t<CSR>) == 8)))
        return st;
    Vec vmin;
    vmin.W = 1;
    vmin.tile = 128;
    const Vec v = choose_vec(K, b_dtype, nullptr, K ? K : 1, nullptr, K ? K : 1);
    const int fix = resolve_fix(fixup);
    const size_t ys = sizeof(idx_t<CSR>);
    size_t a = online_bytes(P, K, v, fix, 0, ys), b = online_bytes(P, K, vmin, fix, 0, ys);
    *bytes = a > b ? a : b;
    return MPS_OK;
}

extern "C" {

mps_status mps_shard_bounds(const int32_t *row_ptr_host, int64_t m, int64_t nnz, int32_t world,
                            int32_t *X, int32_t *Y, int32_t *tail_rows) {
    return shard_bounds_impl(row_ptr_host, m, nnz, world, X, Y, tail_rows);
}

mps_status mps_shard_bounds64(const int64_t *row_ptr_host, int64_t m, int64_t nnz,
                              int32_t world, int32_t *X, int64_t *Y, int32_t *tail_rows) {
    return shard_bounds_impl(row_ptr_host, m, nnz, world, X, Y, tail_rows);
}

mps_status mps_spmm_shard_workspace_bytes(const mps_csr *A, int32_t K, int32_t b_dtype,
                                          const int32_t *X, int32_t rank, int32_t world,
                                          int64_t items_per_part, int64_t min_parts,
                                          int32_t fixup, size_t *bytes) {
    return shard_ws_impl(A, K, b_dtype, X, rank, world, items_per_part, min_parts, fixup,
                         bytes);
}

mps_status mps_spmm_shard64_workspace_bytes(const mps_csr64 *A, int32_t K, int32_t b_dtype,
                                            const int32_t *X, int32_t rank, int32_t world,
                                            int64_t items_per_part, int64_t min_parts,
                                            int32_t fixup, size_t *bytes) {
    return shard_ws_impl(A, K, b_dtype, X, rank, world, items_per_part, min_parts, fixup,
                         bytes);
}

}  // extern "C"

static int32_t owner_of(const int32_t *X, int32_t world, int32_t r) {
    int32_t owner = 0;
    for (int32_t g = 0; g < world; ++g)
        if (X[g] <= r) owner = g;
    return owner;
}

template <typename CSR>
static mps_status shard_impl(const CSR *A, const void *B, int32_t b_dtype, int64_t ldb,
                             int32_t K, const int32_t *X, const idx_t<CSR> *Y,
                             const int32_t *tail_rows, int32_t rank, int32_t world,
                             int64_t items_per_part, int64_t min_parts, float *C_local,
                             int64_t ldc, float *tail_out, int32_t fixup,
                             void *const *mailboxes_host, uint32_t epoch, void *workspace,
                             size_t workspace_bytes, void *stream) {
    using IT = idx_t<CSR>;
    if (!A) return fail(MPS_ERR_INVALID, "A is NULL");
    if (!X || !Y || !tail_rows || world < 1 || rank < 0 || rank >= world)
        return fail(MPS_ERR_INVALID, "bad shard arguments");
    // a shard without non-zeros may pass NULL col/val (an empty slice): never read
    CSR Aloc = *A;
    if (Y[rank + 1] == Y[rank] && A->row_ptr) {
        if (!Aloc.col_idx) Aloc.col_idx = (const int32_t *)A->row_ptr;
        if (!Aloc.val) Aloc.val = (const float *)A->row_ptr;
    }
    A = &Aloc;
    mps_status st = check_csr(A);
    if (st) return st;
    if ((st = check_dense(B, b_dtype, ldb, K, C_local ? C_local : (float *)B, ldc, A))) return st;
    if (mailboxes_host && (world > mps::kMailMaxWorld || epoch == 0))
        return fail(MPS_ERR_UNSUPPORTED, "p2p tails: world <= 16 and epoch >= 1");
    if (K == 0) return MPS_OK;
    if (!tail_out) return fail(MPS_ERR_INVALID, "tail_out NULL");
    cudaStream_t s = (cudaStream_t)stream;
    MPS_CUDA(cudaMemsetAsync(tail_out, 0, (size_t)K * 4, s), "zero tail");
    int64_t P, L, D0, span;
    if ((st = shard_plan(A, X, Y, rank, K, b_dtype, items_per_part, min_parts, &P, &L, &D0, &span)))
        return st;
    // a6 peer-memory tail exchange: who this rank pushes to and who pushes to it
    mps::TailMail mail{};
    if (mailboxes_host && world > 1) {
        for (int32_t g = 0; g < world; ++g)
            if (!mailboxes_host[g]) return fail(MPS_ERR_INVALID, "mailbox %d NULL", g);
        char *mine = (char *)mailboxes_host[rank];
        const size_t slot = epoch & 1u;
        mail.counter = (uint32_t *)mine;
        mail.epoch = epoch;
        mail.K = K;
        const int32_t trow = tail_rows[rank];
        if (trow >= 0) {
            const int32_t h = owner_of(X, world, trow);
            char *theirs = (char *)mailboxes_host[h];
            mail.tail = tail_out;
            mail.push_dst = (float *)(theirs + mps::kMailInboxOfs) +
                            (slot * mps::kMailMaxWorld + (size_t)rank) * K;
            mail.push_flag = (uint32_t *)(theirs + mps::kMailFlagsOfs) + rank;
            mail.push_ack = (const uint32_t *)(mine + mps::kMailAcksOfs) + h;
        }
        for (int32_t g = 0; g < world; ++g) {
            const int32_t r = tail_rows[g];
            if (g == rank || r < 0 || owner_of(X, world, r) != rank) continue;
            mail.pull_mask |= 1u << g;
            mail.pull_row = C_local + (int64_t)(r - X[rank]) * ldc;
            mail.ack_dst[g] = (uint32_t *)((char *)mailboxes_host[g] + mps::kMailAcksOfs) + rank;
        }
        mail.pull_src = (const float *)(mine + mps::kMailInboxOfs) + slot * mps::kMailMaxWorld * K;
        mail.pull_flags = (const uint32_t *)(mine + mps::kMailFlagsOfs);
        mail.on = (mail.push_dst || mail.pull_mask) ? 1 : 0;
        if (mail.pull_mask && !C_local) return fail(MPS_ERR_INVALID, "C_local NULL");
    }
    const int fix = resolve_fix(fixup);
    const Vec v = choose_vec(K, b_dtype, B, ldb, C_local ? C_local : tail_out, ldc, A->n, A->m,
                             A->nnz);
    if (span == 0) {
        // an empty shard still takes part in the exchange: run the final kernel empty
        if (!mail.on) return MPS_OK;
        P = 1;
        L = 0;
    }
    const size_t need = online_bytes(P, K, v, fix, 0, sizeof(IT));
    if (!workspace || workspace_bytes < need)
        return fail(MPS_ERR_WORKSPACE, "workspace %zu < %zu", workspace_bytes, need);
    const size_t xb = align_up((size_t)(P + 1) * 4, 256);
    const size_t yb = align_up((size_t)(P + 1) * sizeof(IT), 256);
    int32_t *cx = (int32_t *)workspace;
    IT *cy = (IT *)((char *)workspace + xb);
    unsigned *claims = (unsigned *)((char *)workspace + xb + yb);
    void *rec = (char *)workspace + xb + yb + claim_bytes(K);
    const int32_t nz = zeroable_claims(K, v);
    const int32_t trow = tail_rows[rank];
    MPS_CUDA(mps::launch_partition<IT>(A->row_ptr, A->m, A->nnz, D0, span, P, L, cx, cy,
                                       fix == mps::FIX_ATOMIC ? C_local : nullptr, ldc, X[rank],
                                       K, trow, fix == mps::FIX_ATOMIC ? tail_out : nullptr,
                                       claims, nz, s),
             "partition kernel");
    mps::SegArgsT<IT> a{};
    a.rp = A->row_ptr;
    // col/val hold global nnz [Y[rank], ...): shift so that col[j] is global nnz j
    a.col = (const int32_t *)((uintptr_t)A->col_idx - (uintptr_t)Y[rank] * 4);
    a.val = (const float *)((uintptr_t)A->val - (uintptr_t)Y[rank] * 4);
    a.B = B;
    a.ldb = ldb;
    a.C = C_local;
    a.ldc = ldc;
    a.row_base = X[rank];
    a.m = (int32_t)A->m;
    a.cx = cx;
    a.cy = cy;
    a.P = P;
    a.tail_row = trow;
    a.tail = tail_out;
    a.nnz_end = (int64_t)Y[rank + 1];
    a.mail = mail;
    return run_segments(a, b_dtype, K, v, fix, rec, claims, nz > 0, s);
}

extern "C" {

mps_status mps_spmm_shard(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                          int32_t K, const int32_t *X, const int32_t *Y,
                          const int32_t *tail_rows, int32_t rank, int32_t world,
                          int64_t items_per_part, int64_t min_parts, float *C_local,
                          int64_t ldc, float *tail_out, int32_t fixup, void *workspace,
                          size_t workspace_bytes, void *stream) {
    return shard_impl(A, B, b_dtype, ldb, K, X, Y, tail_rows, rank, world, items_per_part,
                      min_parts, C_local, ldc, tail_out, fixup, nullptr, 0, workspace,
                      workspace_bytes, stream);
}

mps_status mps_spmm_shard64(const mps_csr64 *A, const void *B, int32_t b_dtype, int64_t ldb,
                            int32_t K, const int32_t *X, const int64_t *Y,
                            const int32_t *tail_rows, int32_t rank, int32_t world,
                            int64_t items_per_part, int64_t min_parts, float *C_local,
                            int64_t ldc, float *tail_out, int32_t fixup,
                            void *const *mailboxes_host, uint32_t epoch, void *workspace,
                            size_t workspace_bytes, void *stream) {
    return shard_impl(A, B, b_dtype, ldb, K, X, Y, tail_rows, rank, world, items_per_part,
                      min_parts, C_local, ldc, tail_out, fixup, mailboxes_host, epoch,
                      workspace, workspace_bytes, stream);
}

size_t mps_shard_mailbox_bytes(int32_t K) {
    return align_up((size_t)mps::kMailInboxOfs +
                        2 * (size_t)mps::kMailMaxWorld * (size_t)(K > 0 ? K : 0) * 4, 256);
}

mps_status mps_spmm_shard_p2p(const mps_csr *A, const void *B, int32_t b_dtype, int64_t ldb,
                              int32_t K, const int32_t *X, const int32_t *Y,
                              const int32_t *tail_rows, int32_t rank, int32_t world,
                              int64_t items_per_part, int64_t min_parts, float *C_local,
                              int64_t ldc, float *tail_out, int32_t fixup,
                              void *const *mailboxes_host, uint32_t epoch, void *workspace,
                              size_t workspace_bytes, void *stream) {
    if (!mailboxes_host) return fail(MPS_ERR_INVALID, "mailboxes_host NULL");
    return shard_impl(A, B, b_dtype, ldb, K, X, Y, tail_rows, rank, world, items_per_part,
                      min_parts, C_local, ldc, tail_out, fixup, mailboxes_host, epoch,
                      workspace, workspace_bytes, stream);
}

mps_status mps_apply_tails(const float *tails, const int32_t *X, const int32_t *tail_rows,
                           int32_t world, int32_t rank, int32_t K, float *C_local,
                           int64_t ldc, void *stream) {
    if (!X || !tail_rows || world < 1 || rank < 0 || rank >= world || K < 0 || ldc < K)
        return fail(MPS_ERR_INVALID, "bad apply_tails arguments");
    std::vector<int32_t> mine;
    int32_t row = -1;
    for (int32_t h = 0; h < world; ++h) {
        const int32_t r = tail_rows[h];
        if (r < 0) continue;
        int32_t owner = 0;
        for (int32_t g = 0; g < world; ++g)
            if (X[g] <= r) owner = g;
        if (owner != rank) continue;
        mine.push_back(h);
        row = r;
    }
    if (mine.empty() || K == 0) return MPS_OK;
    if (!tails || !C_local) return fail(MPS_ERR_INVALID, "NULL pointer");
    MPS_CUDA(mps::launch_apply_tails(tails, K, mine.data(), (int32_t)mine.size(),
                                     C_local + (int64_t)(row - X[rank]) * ldc,
                                     (cudaStream_t)stream),
             "apply tails");
    return MPS_OK;
}

mps_status mps_validate_csr(const mps_csr *A, int64_t *first_bad_host, void *stream) {
    return validate_impl(A, first_bad_host, stream);
}

}  // extern "C"
