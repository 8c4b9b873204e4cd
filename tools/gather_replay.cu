// gather_replay.cu -- the attainable gather bandwidth of a workload's OWN access stream:
// the B-row gathers the segment kernel must make (row col_idx[j] of B for every non-zero
// j, in CSR order), issued with nothing else -- no row ends, no FMAs, no stores.  Warps
// take contiguous nnz ranges (like merge-path segments), read col_idx coalesced and keep
// 16 x 16-B gathers per lane in flight (L1 no_allocate, L2 evict_last as the kernel).
// The time of this replay is the roofline time of the segment kernel's dominant traffic
// on this box (L2 hits and DRAM misses as the real pattern produces them).  NOT part of
// the product: bench.py loads it for roofline.peak only.
#include <cuda_runtime.h>
#include <stdint.h>

namespace {
__device__ __forceinline__ uint4 ldg_b(const void *p, uint64_t pol) {
    uint4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p), "l"(pol));
    return v;
}

// row_bytes in {64, 128, 256, 512}: LR = row_bytes/16 lanes per row, NR = 32/LR rows per
// warp instruction; a batch = UL*NR non-zeros, UL gathers in flight per lane (UL = 32/NR
// by default: 16 for 256-B rows; ULC caps it, e.g. 8 = the segment kernel's own depth).
template <int LR, int ULC = 32>
__global__ void __launch_bounds__(256) replay_kernel(const int32_t *__restrict__ col, int64_t nnz,
                                                     const char *__restrict__ B, int64_t ldb_bytes,
                                                     int64_t per_warp, uint32_t *sink) {
    constexpr int NR = 32 / LR;
    constexpr int UL = (32 / NR) < ULC ? (32 / NR) : ULC;
    constexpr int U = UL * NR;
    const int lane = threadIdx.x & 31, grp = lane / LR, lr = lane % LR;
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    int64_t j0 = warp * per_warp;
    const int64_t j1 = j0 + per_warp < nnz ? j0 + per_warp : nnz;
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    uint32_t acc = 0;
    for (; j0 < j1; j0 += U) {
        const int64_t j = j0 + lane;
        const int c = (lane < U && j < j1) ? __ldg(col + j) : 0;
        uint4 v[UL];
#pragma unroll
        for (int i = 0; i < UL; ++i) {
            const int ci = __shfl_sync(0xffffffffu, c, i * NR + grp);
            v[i] = ldg_b(B + (int64_t)ci * ldb_bytes + lr * 16, pol);
        }
#pragma unroll
        for (int i = 0; i < UL; ++i) acc ^= v[i].x ^ v[i].y ^ v[i].z ^ v[i].w;
    }
    if (acc == 0x9e3779b9u) sink[0] = acc;
}
}  // namespace

template <int ULC>
static int replay_launch(int row_bytes, int64_t grid, const int32_t *col, int64_t nnz,
                         const void *B, int64_t ldb_bytes, int64_t per, uint32_t *sink) {
    switch (row_bytes) {
    case 64: replay_kernel<4, ULC><<<(unsigned)grid, 256>>>(col, nnz, (const char *)B, ldb_bytes, per, sink); break;
    case 128: replay_kernel<8, ULC><<<(unsigned)grid, 256>>>(col, nnz, (const char *)B, ldb_bytes, per, sink); break;
    case 256: replay_kernel<16, ULC><<<(unsigned)grid, 256>>>(col, nnz, (const char *)B, ldb_bytes, per, sink); break;
    case 512: replay_kernel<32, ULC><<<(unsigned)grid, 256>>>(col, nnz, (const char *)B, ldb_bytes, per, sink); break;
    default: return 3;
    }
    return 0;
}

// Gathers rows col[0..nnz) of B (row_bytes of each row, stride ldb_bytes) with the given
// resident CTAs (8 warps) per SM (0: best of 3, 4, 6) and gathers per lane (ul: 0 = 16
// for 256-B rows, or 8); returns the best time (ms) and the bytes it moved.
extern "C" int gather_replay_cfg(const int32_t *col, int64_t nnz, const void *B, int32_t row_bytes,
                                 int64_t ldb_bytes, int32_t reps, int32_t per_sm_only, int32_t ul,
                                 float *best_ms, double *bytes) {
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    uint32_t *sink = nullptr;
    if (cudaMalloc(&sink, 4) != cudaSuccess) return 1;
    // L2 flushed before every timed replay, as bench.py flushes before every step
    int l2 = 0;
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
    void *flush = nullptr;
    if (cudaMalloc(&flush, (size_t)l2 * 2) != cudaSuccess) return 1;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best = 1e30f;
    const int per_sm[3] = {3, 4, 6};
    int rc = 0;
    for (int c = 0; c < 3 && rc == 0; ++c) {
        const int psm = per_sm_only > 0 ? per_sm_only : per_sm[c];
        const int64_t warps = (int64_t)sms * psm * 8;
        int64_t per = (nnz + warps - 1) / warps;
        per = (per + 31) / 32 * 32;
        const int64_t nw = (nnz + per - 1) / per;
        const int64_t grid = (nw + 7) / 8;
        for (int r = 0; r < reps + 1 && rc == 0; ++r) {
            cudaMemsetAsync(flush, r & 1, (size_t)l2 * 2);
            cudaEventRecord(e0);
            rc = ul == 8 ? replay_launch<8>(row_bytes, grid, col, nnz, B, ldb_bytes, per, sink)
                         : replay_launch<32>(row_bytes, grid, col, nnz, B, ldb_bytes, per, sink);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float t = 0.f;
            cudaEventElapsedTime(&t, e0, e1);
            if (r > 0 && t < best) best = t;       // first launch: warm-up
        }
        if (per_sm_only > 0) break;
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(sink);
    cudaFree(flush);
    if (rc) return rc;
    *best_ms = best;
    *bytes = (double)nnz * row_bytes + (double)nnz * 4;
    return cudaGetLastError() == cudaSuccess ? 0 : 2;
}

// The attainable replay of bench.py's roofline: best of 3 / 4 / 6 CTAs per SM, 16 gathers
// of 16 B in flight per lane for 256-B rows.
extern "C" int gather_replay(const int32_t *col, int64_t nnz, const void *B, int32_t row_bytes,
                             int64_t ldb_bytes, int32_t reps, float *best_ms, double *bytes) {
    return gather_replay_cfg(col, nnz, B, row_bytes, ldb_bytes, reps, 0, 0, best_ms, bytes);
}
