// partition.cu -- a2: merge-path partition (Alg. 1), the split-row
// zeroing of the atomic fix-up (a4), the Fig. 5 write statistic
// and the debug CSR validator.
#include "mps_internal.cuh"

namespace mps {

// Coordinate of diagonal d on the (row_ptr, nnz-index) merge grid (Alg. 1 lines 6-7).
// s(x) = x + rp[x] is strictly increasing with s(0) = 0; the point is
// x = max{x : s(x) <= d} (readings R4/R5), x in [max(0, d - nnz), min(d, m)].
// It is found by one warp with a 32-ary search: every round the lanes
// probe 32 points of the candidate range [a, b] (s(a) <= d holds throughout) and the
// ballot of s(q) <= d -- a prefix, s is increasing -- shrinks it ~32x, so a range of
// 2^21 rows takes 4-5 dependent loads instead of 21.
template <typename IT>
__device__ __forceinline__ int64_t diag_x_warp(const IT *__restrict__ rp, int64_t m,
                                               int64_t nnz, int64_t d, int lane) {
    int64_t a = d > nnz ? d - nnz : 0;          // s(a) = a + rp[a] <= d
    int64_t b = d < m ? d : m;                  // the answer is <= min(d, m)
    while (b > a) {
        const int64_t len = b - a;
        const int64_t q = a + (len * (lane + 1) + 31) / 32;   // in (a, b], q_31 = b
        const bool ok = q + (int64_t)__ldg(rp + q) <= d;
        const unsigned mask = __ballot_sync(0xffffffffu, ok);
        const int k = __popc(mask);             // probes q_0..q_{k-1} satisfy s <= d
        const int64_t qa = __shfl_sync(0xffffffffu, q, k > 0 ? k - 1 : 0);
        const int64_t qb = __shfl_sync(0xffffffffu, q, k < 32 ? k : 31);
        if (k > 0) a = qa;
        if (k < 32) b = qb - 1;
    }
    return a;
}

// One thread per diagonal p = 0..P, in blocks of consecutive diagonals.  x(d) is
// monotone, so warps 0 and 1 first find x of the block's first and last diagonal with
// the 32-ary search; the block's row_ptr window rp[x_first .. x_last] (if it fits) is
// staged in shared memory and every thread binary-searches only that window -- the
// partition costs a few dependent L2/DRAM round trips instead of ~log2(m).  With
// zero_C != nullptr (atomic fix-up, online) the warp then zeroes every destination row
// cut by one of its 32 diagonals (y_p > rp[x_p]): those rows receive only atomic
// partial sums (reading R10).
constexpr int kPartWin = 2048;   // row_ptr entries staged per block

template <typename IT>
__global__ void __launch_bounds__(kBlock)
partition_kernel(const IT *__restrict__ rp, int64_t m, int64_t nnz, int64_t d0,
                 int64_t span, int64_t P, int64_t L, int32_t *__restrict__ cx,
                 IT *__restrict__ cy, float *zero_C, int64_t ldc, int64_t row_base,
                 int32_t K, int32_t tail_row, float *tail, unsigned *claims, int32_t nclaims) {
    __shared__ IT s_rp[kPartWin];
    // the segment kernel that follows on the stream claims segments from these counters
    // (caller workspace); they start at zero
    if (blockIdx.x == 0 && (int)threadIdx.x < nclaims) claims[threadIdx.x] = 0u;
    __shared__ int64_t s_x[2];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t pb = (int64_t)blockIdx.x * blockDim.x;
    const int64_t pe = (pb + blockDim.x - 1 < P) ? pb + blockDim.x - 1 : P;
    auto diag = [&](int64_t q) {
        int64_t off = q * L;
        if (off > span) off = span;
        return d0 + off;
    };
    if (warp < 2) {
        const int64_t xw = diag_x_warp(rp, m, nnz, diag(warp == 0 ? pb : pe), lane);
        if (lane == 0) s_x[warp] = xw;
    }
    __syncthreads();
    const int64_t xlo = s_x[0], xhi = s_x[1];
    const int64_t wn = xhi - xlo + 1;           // candidates x in [xlo, xhi]
    const bool staged = wn <= kPartWin;
    if (staged) {
        // asynchronous copies, all in flight at once: one memory round trip for the window
        // (a load-then-store loop serialises one round trip per iteration)
        for (int64_t i = threadIdx.x; i < wn; i += blockDim.x) {
            if constexpr (sizeof(IT) == 8) cp_async8(s_rp + i, rp + xlo + i);
            else cp_async4(s_rp + i, rp + xlo + i);
        }
        cp_async_wait_all();
        __syncthreads();
    }
    const int64_t p = pb + threadIdx.x;
    const bool valid = p <= P;
    int64_t x = 0, y = 0;
    if (valid) {
        const int64_t d = diag(p);
        // x = max{x in [xlo, xhi] : x + rp[x] <= d}; s(xlo) <= d(pb) <= d
        int64_t a = xlo, b = xhi;
        while (b > a) {
            const int64_t mid = a + (b - a + 1) / 2;
            const int64_t r = staged ? (int64_t)s_rp[mid - xlo] : (int64_t)__ldg(rp + mid);
            if (mid + r <= d) a = mid;
            else b = mid - 1;
        }
        x = a;
        y = d - x;
        cx[p] = (int32_t)x;
        cy[p] = (IT)y;
    }
    if (zero_C == nullptr && tail == nullptr) return;  // uniform across the grid
    // x lies in [xlo, xhi]: rp[x] comes from the staged window when there is one
    const bool inside = valid && x < m &&
                        y > (staged ? (int64_t)s_rp[x - xlo] : (int64_t)__ldg(rp + x));
    unsigned todo = __ballot_sync(0xffffffffu, inside);
    while (todo) {
        const int src = __ffs(todo) - 1;
        todo &= todo - 1;
        const int64_t row = __shfl_sync(0xffffffffu, x, src);
        float *dst = (row == tail_row) ? tail : zero_C + (row - row_base) * ldc;
        for (int c = lane; c < K; c += 32) dst[c] = 0.f;
    }
}

template <typename IT>
cudaError_t launch_partition(const IT *rp, int64_t m, int64_t nnz, int64_t d0,
                             int64_t span, int64_t P, int64_t L, int32_t *cx, IT *cy,
                             float *zero_C, int64_t ldc, int64_t row_base, int32_t K,
                             int32_t tail_row, float *tail, unsigned *claims,
                             int32_t nclaims, cudaStream_t s) {
    const int64_t n = P + 1;
    const int64_t blocks = (n + kBlock - 1) / kBlock;
    if (nclaims > kBlock) return cudaErrorInvalidValue;
    partition_kernel<IT><<<(unsigned)blocks, kBlock, 0, s>>>(rp, m, nnz, d0, span, P, L, cx, cy,
                                                         zero_C, ldc, row_base, K, tail_row,
                                                         tail, claims, claims ? nclaims : 0);
    return cudaGetLastError();
}

// Offline atomic fix-up: zero the rows cut by a boundary of the given schedule; one
// warp per boundary, only the first boundary inside a row writes it.
template <typename IT>
__global__ void __launch_bounds__(kBlock)
zero_split_kernel(const IT *__restrict__ rp, int32_t m, const int32_t *__restrict__ cx,
                  const IT *__restrict__ cy, int64_t P, float *C, int64_t ldc,
                  int64_t row_base, int32_t K, int32_t tail_row, float *tail,
                  unsigned *claims, int32_t nclaims) {
    if (blockIdx.x == 0 && (int)threadIdx.x < nclaims) claims[threadIdx.x] = 0u;  // see above
    const int64_t p = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (p > P) return;
    const int32_t x = cx[p];
    if (x >= m) return;
    const IT start = __ldg(rp + x);
    if (cy[p] <= start) return;
    if (p > 0 && cx[p - 1] == x && cy[p - 1] > start) return;  // already zeroed
    float *dst = (x == tail_row) ? tail : C + ((int64_t)x - row_base) * ldc;
    for (int c = lane; c < K; c += 32) dst[c] = 0.f;
}

template <typename IT>
cudaError_t launch_zero_split(const IT *rp, int32_t m, const int32_t *cx,
                              const IT *cy, int64_t P, float *C, int64_t ldc,
                              int64_t row_base, int32_t K, int32_t tail_row, float *tail,
                              unsigned *claims, int32_t nclaims, cudaStream_t s) {
    const int64_t threads = (P + 1) * 32;
    const int64_t blocks = (threads + kBlock - 1) / kBlock;
    if (nclaims > kBlock) return cudaErrorInvalidValue;
    zero_split_kernel<IT><<<(unsigned)blocks, kBlock, 0, s>>>(rp, m, cx, cy, P, C, ldc, row_base,
                                                          K, tail_row, tail, claims,
                                                          claims ? nclaims : 0);
    return cudaGetLastError();
}

// Fig. 5 statistic: writes per Alg. 2 for each segment p:
//   start partial (line 2) and single row (line 3): 1 atomic (line 5);
//   else start partial: 1 atomic (line 9); end partial (line 11): 1 atomic (line 13);
//   rows [start_row, end_row): regular stores (line 15).
template <typename IT>
__global__ void __launch_bounds__(kBlock)
write_stats_kernel(const IT *__restrict__ rp, int32_t m, const int32_t *__restrict__ cx,
                   const IT *__restrict__ cy, int64_t P,
                   unsigned long long *counts) {
    __shared__ unsigned long long s_a, s_r;
    if (threadIdx.x == 0) { s_a = 0; s_r = 0; }
    __syncthreads();
    const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    unsigned long long na = 0, nr = 0;
    if (p < P) {
        const int32_t xs = cx[p], xe = cx[p + 1];
        const IT ys = cy[p], ye = cy[p + 1];
        const bool sp = xs < m && ys != __ldg(rp + xs);
        const bool ep = xe < m && ye != __ldg(rp + xe);
        if (sp && xs == xe) {
            na = 1;
        } else {
            const int32_t first = sp ? xs + 1 : xs;
            na = (sp ? 1 : 0) + (ep ? 1 : 0);
            nr = (unsigned long long)(xe - first);
        }
    }
    for (int o = 16; o > 0; o >>= 1) {
        na += __shfl_xor_sync(0xffffffffu, na, o);
        nr += __shfl_xor_sync(0xffffffffu, nr, o);
    }
    if ((threadIdx.x & 31) == 0) { atomicAdd(&s_a, na); atomicAdd(&s_r, nr); }
    __syncthreads();
    if (threadIdx.x == 0) { atomicAdd(counts, s_a); atomicAdd(counts + 1, s_r); }
}

template <typename IT>
cudaError_t launch_write_stats(const IT *rp, int32_t m, const int32_t *cx,
                               const IT *cy, int64_t P, int64_t *counts, cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(counts, 0, 2 * sizeof(int64_t), s);
    if (e != cudaSuccess) return e;
    const int64_t blocks = (P + kBlock - 1) / kBlock;
    if (blocks > 0)
        write_stats_kernel<IT><<<(unsigned)blocks, kBlock, 0, s>>>(
            rp, m, cx, cy, P, reinterpret_cast<unsigned long long *>(counts));
    return cudaGetLastError();
}

template <typename IT>
__global__ void __launch_bounds__(kBlock)
validate_kernel(const IT *__restrict__ rp, const int32_t *__restrict__ col, int64_t m,
                int64_t n, int64_t nnz, unsigned long long *first_bad) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i <= m) {
        const IT v = rp[i];
        bool bad = (i == 0 && v != 0) || (i == m && v != nnz) || v < 0 || v > nnz ||
                   (i > 0 && rp[i - 1] > v);
        if (bad) atomicMin(first_bad, (unsigned long long)i);
    }
    if (i < nnz) {
        const int32_t c = col[i];
        if (c < 0 || c >= n) atomicMin(first_bad, (unsigned long long)(m + 1 + i));
    }
}

template <typename IT>
cudaError_t launch_validate(const IT *rp, const int32_t *col, int64_t m, int64_t n,
                            int64_t nnz, unsigned long long *first_bad, cudaStream_t s) {
    const int64_t work = (m + 1 > nnz ? m + 1 : nnz);
    const int64_t blocks = (work + kBlock - 1) / kBlock;
    validate_kernel<IT><<<(unsigned)blocks, kBlock, 0, s>>>(rp, col, m, n, nnz, first_bad);
    return cudaGetLastError();
}

#define MPS_INST_PARTITION(IT)                                                               \
    template cudaError_t launch_partition<IT>(const IT *, int64_t, int64_t, int64_t, int64_t,  \
                                              int64_t, int64_t, int32_t *, IT *, float *,      \
                                              int64_t, int64_t, int32_t, int32_t, float *,     \
                                              unsigned *, int32_t, cudaStream_t);              \
    template cudaError_t launch_zero_split<IT>(const IT *, int32_t, const int32_t *,           \
                                               const IT *, int64_t, float *, int64_t, int64_t, \
                                               int32_t, int32_t, float *, unsigned *, int32_t, \
                                               cudaStream_t);                                  \
    template cudaError_t launch_write_stats<IT>(const IT *, int32_t, const int32_t *,          \
                                                const IT *, int64_t, int64_t *, cudaStream_t); \
    template cudaError_t launch_validate<IT>(const IT *, const int32_t *, int64_t, int64_t,    \
                                             int64_t, unsigned long long *, cudaStream_t);
MPS_INST_PARTITION(int32_t)
MPS_INST_PARTITION(int64_t)

}  // namespace mps
