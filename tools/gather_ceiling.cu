// gather_ceiling.cu -- B200 ceiling for random row gathers (the a3 access pattern without
// the SpMM bookkeeping): each warp reads NR rows of `row_bytes` per instruction group,
// rows chosen by a hash, from a table of `table_mb` MB.  Reports achieved GB/s.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gather_ceiling gather_ceiling.cu
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}
template <int UNROLL, int HINT>
__global__ void __launch_bounds__(256) gather(const char* __restrict__ tab, uint32_t nrows,
    uint32_t row_bytes, uint64_t iters, uint32_t* out) {
    const int lane = threadIdx.x & 31;
    const uint32_t lanes_per_row = row_bytes / 16;            // 16 B per lane
    const uint32_t rows_per_instr = 32 / lanes_per_row;
    const uint32_t grp = lane / lanes_per_row, lr = lane % lanes_per_row;
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    uint64_t pol;
    if (HINT) asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    uint32_t acc = 0;
    for (uint64_t it = 0; it < iters; ++it) {
        uint4 v[UNROLL];
#pragma unroll
        for (int u = 0; u < UNROLL; ++u) {
            uint32_t r = hash32((uint32_t)(warp * 0x9E3779B9u) ^ (uint32_t)((it * UNROLL + u) * rows_per_instr + grp)) % nrows;
            const char* p = tab + (uint64_t)r * row_bytes + lr * 16;
            if (HINT)
                asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                             : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(p), "l"(pol));
            else
                asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                             : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(p));
        }
#pragma unroll
        for (int u = 0; u < UNROLL; ++u) acc += v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
    }
    if (acc == 0x12345678) out[0] = acc;
}
int main(int argc, char** argv) {
    double table_mb = argc > 1 ? atof(argv[1]) : 60;
    uint32_t row_bytes = argc > 2 ? atoi(argv[2]) : 256;
    int blocks_per_sm = argc > 3 ? atoi(argv[3]) : 4;
    int hint = argc > 4 ? atoi(argv[4]) : 1;
    size_t bytes = (size_t)(table_mb * 1e6);
    uint32_t nrows = bytes / row_bytes;
    char* tab; uint32_t* out;
    cudaMalloc(&tab, (size_t)nrows * row_bytes); cudaMalloc(&out, 4);
    cudaMemset(tab, 1, (size_t)nrows * row_bytes);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int grid = sms * blocks_per_sm;
    uint64_t iters = 2000;
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto run = [&](auto kern) {
        kern<<<grid, 256>>>(tab, nrows, row_bytes, 50, out);
        cudaEventRecord(e0);
        kern<<<grid, 256>>>(tab, nrows, row_bytes, iters, out);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        return ms;
    };
    const int U = 8;
    float ms = hint ? run(gather<U, 1>) : run(gather<U, 0>);
    double total = (double)grid * 8 /*warps*/ * iters * U * 32 * 16;
    printf("table %.0f MB row %u B blocks/SM %d hint %d: %.3f ms  %.1f GB/s\n", table_mb, row_bytes,
           blocks_per_sm, hint, ms, total / ms / 1e6);
    return 0;
}
