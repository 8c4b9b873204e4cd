// hot.cu -- degree-aware L2 residency for the B gathers (a B200 addition, not in the
// paper): when B does not fit in L2, the rows gathered most often (the hubs of the
// power-law graph) are marked evict_last and the long tail evict_first, so the 126 MB
// L2 keeps the rows with the most re-use instead of an LRU mix.
//
// Three small kernels, no host synchronisation: (1) per-column non-zero counts,
// (2) a log2 histogram of the counts, (3) threshold = the smallest power of two t such
// that the columns with count >= t fit in `budget_rows`, then one bit per column.
#include "mps_internal.cuh"

namespace mps {

__global__ void __launch_bounds__(kBlock)
col_count_kernel(const int32_t *__restrict__ col, int64_t nnz, int32_t *counts) {
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nnz;
         j += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(counts + __ldg(col + j), 1);
}

__global__ void __launch_bounds__(kBlock)
count_hist_kernel(const int32_t *__restrict__ counts, int64_t n, uint32_t *hist) {
    __shared__ uint32_t h[33];
    if (threadIdx.x < 33) h[threadIdx.x] = 0;
    __syncthreads();
    for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n;
         c += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t v = (uint32_t)counts[c];
        atomicAdd(&h[v ? 32 - __clz(v) : 0], 1u);   // bin b holds counts in [2^(b-1), 2^b)
    }
    __syncthreads();
    if (threadIdx.x < 33 && h[threadIdx.x]) atomicAdd(hist + threadIdx.x, h[threadIdx.x]);
}

// hist[33] -> hist[33] = threshold count (columns with count >= threshold are hot)
__global__ void hot_threshold_kernel(uint32_t *hist, int64_t budget_rows) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    int64_t taken = 0;
    uint32_t thr = 0xffffffffu;
    for (int b = 32; b >= 1; --b) {
        if (taken + hist[b] > budget_rows) break;
        taken += hist[b];
        thr = 1u << (b - 1);
    }
    hist[33] = thr;
}

__global__ void __launch_bounds__(kBlock)
hot_bitmap_kernel(const int32_t *__restrict__ counts, int64_t n, const uint32_t *hist,
                  uint32_t *bitmap) {
    const uint32_t thr = hist[33];
    const int lane = threadIdx.x & 31;
    for (int64_t c0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) & ~31ll; c0 < n;
         c0 += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c = c0 + lane;
        const bool h = c < n && (uint32_t)counts[c] >= thr;
        const uint32_t word = __ballot_sync(0xffffffffu, h);
        if (lane == 0) bitmap[c0 >> 5] = word;
    }
}

cudaError_t launch_hot_columns(const int32_t *col, int64_t nnz, int64_t n, int64_t budget_rows,
                               int32_t *counts, uint32_t *hist, uint32_t *bitmap,
                               cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(counts, 0, (size_t)n * 4, s);
    if (e == cudaSuccess) e = cudaMemsetAsync(hist, 0, 34 * 4, s);
    if (e != cudaSuccess) return e;
    const int grid = num_sms() * 8;
    if (nnz > 0) col_count_kernel<<<grid, kBlock, 0, s>>>(col, nnz, counts);
    if (n > 0) count_hist_kernel<<<grid, kBlock, 0, s>>>(counts, n, hist);
    hot_threshold_kernel<<<1, 32, 0, s>>>(hist, budget_rows);
    if (n > 0) hot_bitmap_kernel<<<grid, kBlock, 0, s>>>(counts, n, hist, bitmap);
    return cudaGetLastError();
}

}  // namespace mps
