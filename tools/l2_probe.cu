// l2_probe.cu -- live L2 -> SM read ceiling for the bench's roofline (SURVEY.md
// sec. 8(d): "L2->SM gather throughput" bounds the path where B fits in L2, e.g. Reddit
// K=64).  A table of `bytes` (< L2) is made resident, then every warp gathers rows of
// `row_bytes` at random (a hash of warp and iteration, 16 B per lane, L1 no_allocate,
// U gathers in flight per lane) -- the a3 access pattern without the SpMM's
// bookkeeping.  mode 1 streams the table instead (grid-stride, coalesced).  Reports the
// best read GB/s over a few grid shapes.  NOT part of the product: libmpspmm never
// links it; bench.py loads it only for roofline.units.
#include <cuda_runtime.h>
#include <stdint.h>

__device__ __forceinline__ uint32_t mix32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
    return x;
}

__device__ __forceinline__ uint4 ldg_na(const uint4 *p) {
    uint4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}

template <int U>
__global__ void __launch_bounds__(256) l2_gather(const uint4 *__restrict__ tab, uint32_t nrows,
                                                 uint32_t row16, int iters, uint32_t *sink) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t rows_per_instr = 32 / row16;            // row16 = 16-B words per row
    const uint32_t grp = lane / row16, lr = lane % row16;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    uint32_t acc = 0;
    uint32_t h = mix32(warp * 0x9E3779B9u + 1);
    for (int it = 0; it < iters; ++it) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint32_t r = mix32(h + (uint32_t)(u * rows_per_instr + grp)) % nrows;
            v[u] = ldg_na(tab + (uint64_t)r * row16 + lr);
        }
        h = mix32(h + (uint32_t)it);
#pragma unroll
        for (int u = 0; u < U; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
    }
    if (acc == 0x9e3779b9u) sink[0] = acc;
}

__global__ void __launch_bounds__(256) l2_stream(const uint4 *__restrict__ buf, int64_t n16,
                                                 int passes, uint32_t *sink) {
    uint32_t acc = 0;
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int p = 0; p < passes; ++p)
        for (int64_t i = tid; i < n16; i += stride) {
            const uint4 v = ldg_na(buf + i);
            acc ^= v.x ^ v.y ^ v.z ^ v.w;
        }
    if (acc == 0x9e3779b9u) sink[0] = acc;
}

// Lean probes (modes 2 and 3): the index arithmetic above (two multiplicative hashes
// and a runtime modulo per gather) costs more issue slots than the load itself, so
// those probes are issue-bound below the L2 rate.  Here a power-of-two row count lets
// one IMAD (LCG) + one shift pick a row, 16 gathers are in flight per lane, and the
// streaming read issues 8 independent coalesced 512-B warp loads per iteration.
template <int U>
__global__ void __launch_bounds__(256) l2_gather_lean(const uint4 *__restrict__ tab,
                                                      uint32_t shift, uint32_t row16,
                                                      int iters, uint32_t *sink) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t grp = lane / row16, lr = lane % row16;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    uint32_t x = mix32(warp * 0x9E3779B9u + grp * 0x85ebca6bu + 7u);
    uint32_t acc = 0;
    for (int it = 0; it < iters; ++it) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            x = x * 1664525u + 1013904223u;
            v[u] = ldg_na(tab + (uint64_t)(x >> shift) * row16 + lr);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
    }
    if (acc == 0x9e3779b9u) sink[0] = acc;
}

template <int U>
__global__ void __launch_bounds__(256) l2_stream_lean(const uint4 *__restrict__ buf,
                                                      uint32_t n16, int passes, uint32_t *sink) {
    uint32_t acc = 0;
    const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    const uint32_t stride = gridDim.x * blockDim.x;
    for (int p = 0; p < passes; ++p)
        for (uint32_t i = tid; i + (U - 1) * stride < n16; i += U * stride) {
            uint4 v[U];
#pragma unroll
            for (int u = 0; u < U; ++u) v[u] = ldg_na(buf + i + u * stride);
#pragma unroll
            for (int u = 0; u < U; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
        }
    if (acc == 0x9e3779b9u) sink[0] = acc;
}

// mode 4: lean random gathers through asynchronous copies (cp.async 16 B, LDGSTS) into
// a per-warp shared-memory ring of 2 batches: each lane issues 16 copies for batch b+1,
// then waits for batch b (cp.async.wait_group 1) and reads its own 16 B back (LDS) --
// the landing path a register-free pipelined gather would use.
template <int U>
__global__ void __launch_bounds__(256) l2_gather_async(const uint4 *__restrict__ tab,
                                                       uint32_t shift, uint32_t row16,
                                                       int iters, uint32_t *sink) {
    __shared__ uint4 ring[8][2][U][32];
    const uint32_t warp_in = threadIdx.x >> 5;
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t grp = lane / row16, lr = lane % row16;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    uint32_t x = mix32(warp * 0x9E3779B9u + grp * 0x85ebca6bu + 7u);
    uint32_t acc = 0;
    auto issue = [&](int slot) {
#pragma unroll
        for (int u = 0; u < U; ++u) {
            x = x * 1664525u + 1013904223u;
            const uint4 *src = tab + (uint64_t)(x >> shift) * row16 + lr;
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;"
                         :: "r"((uint32_t)__cvta_generic_to_shared(&ring[warp_in][slot][u][lane])),
                            "l"(src) : "memory");
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    issue(0);
    for (int it = 0; it < iters; ++it) {
        const int cur = it & 1;
        issue(cur ^ 1);
        asm volatile("cp.async.wait_group 1;" ::: "memory");
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint4 v = ring[warp_in][cur][u][lane];
            acc ^= v.x ^ v.y ^ v.z ^ v.w;
        }
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    if (acc == 0x9e3779b9u) sink[0] = acc;
}

// mode 0: random row gathers (row_bytes in {16..512}); mode 1: streaming read;
// mode 2: lean random gathers (power-of-two rows); mode 3: lean streaming read.
// Returns 0 on success; *gbs = best bytes read / time over the tried grid shapes.
extern "C" int l2_probe_read_gbs2(int64_t bytes, int32_t row_bytes, int32_t mode, float *gbs,
                                  float *ms) {
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (row_bytes < 16 || row_bytes > 512 || (row_bytes & (row_bytes - 1))) return 3;
    const int64_t n16 = bytes / 16;
    const uint32_t row16 = (uint32_t)row_bytes / 16;
    const uint32_t nrows = (uint32_t)(n16 / row16);
    uint4 *buf = nullptr;
    uint32_t *sink = nullptr;
    if (cudaMalloc(&buf, n16 * 16) != cudaSuccess) return 1;
    if (cudaMalloc(&sink, 4) != cudaSuccess) { cudaFree(buf); return 1; }
    cudaMemset(buf, 1, n16 * 16);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best = 0.f, best_ms = 0.f;
    const int per_sm[4] = {3, 4, 6, 8};
    uint32_t shift = 32;
    uint32_t nrows2 = 1;
    while (nrows2 * 2 <= nrows) { nrows2 *= 2; --shift; }
    for (int c = 0; c < 4; ++c) {
        const int grid = sms * per_sm[c];
        // lean stream: whole U*stride steps only (bytes counted exactly below)
        const uint32_t st = (uint32_t)grid * 256u;
        const uint32_t steps = (uint32_t)(n16 / (8ull * st));
        const int iters = 400;
        const int passes = 20;
        if (mode == 0) l2_gather<8><<<grid, 256>>>(buf, nrows, row16, 20, sink);
        else if (mode == 2) l2_gather_lean<16><<<grid, 256>>>(buf, shift, row16, 10, sink);
        else if (mode == 4) l2_gather_async<6><<<grid, 256>>>(buf, shift, row16, 10, sink);
        else l2_stream<<<grid, 256>>>(buf, n16, 1, sink);       // make it resident
        for (int rep = 0; rep < 3; ++rep) {
            cudaEventRecord(e0);
            double moved;
            if (mode == 0) {
                l2_gather<8><<<grid, 256>>>(buf, nrows, row16, iters, sink);
                moved = (double)grid * 256 * 16 * 8 * iters;   // 16 B per lane per gather
            } else if (mode == 2) {
                l2_gather_lean<16><<<grid, 256>>>(buf, shift, row16, iters / 2, sink);
                moved = (double)grid * 256 * 16 * 16 * (iters / 2);
            } else if (mode == 4) {
                l2_gather_async<6><<<grid, 256>>>(buf, shift, row16, iters, sink);
                moved = (double)grid * 256 * 16 * 6 * (iters + 1);
            } else if (mode == 3) {
                if (steps == 0) break;
                l2_stream_lean<8><<<grid, 256>>>(buf, (uint32_t)(steps * 8ull * st), passes, sink);
                moved = (double)steps * 8.0 * st * 16.0 * passes;
            } else {
                l2_stream<<<grid, 256>>>(buf, n16, passes, sink);
                moved = (double)n16 * 16 * passes;
            }
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float t = 0.f;
            cudaEventElapsedTime(&t, e0, e1);
            const float g = (float)(moved / (t * 1e-3) / 1e9);
            if (g > best) { best = g; best_ms = t; }
        }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(buf);
    cudaFree(sink);
    *gbs = best;
    *ms = best_ms;
    return cudaGetLastError() == cudaSuccess ? 0 : 2;
}

extern "C" int l2_probe_read_gbs(int64_t bytes, int passes, float *gbs, float *ms) {
    (void)passes;
    return l2_probe_read_gbs2(bytes, 256, 0, gbs, ms);
}
