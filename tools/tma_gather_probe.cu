// tma_gather_probe.cu -- how fast can TMA gather4 (cp.async.bulk.tensor.2d ... tile::gather4,
// sm_100) pull random 256-B rows of an L2-resident table into shared memory, compared
// with the LSU gathers of tools/l2_probe.cu (mode 2)?  NOT part of the product.
//
// Each warp owns a ring of SLOTS shared-memory slots of RPS rows; lane 0 issues RPS/4
// gather4 instructions per slot (random rows: one LCG step per row), the warp waits on
// the slot's mbarrier, every lane reads its 16 B of each row back (LDS.128), and the
// slot is refilled.  Reports GB/s of rows landed in shared memory.
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace {
constexpr int kRow = 256;                        // bytes per row (64 fp32)

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(b)), "r"(n));
}
__device__ __forceinline__ void mbar_expect(uint64_t *b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;"
                 :: "r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity) {
    asm volatile("{\n\t.reg .pred P;\n\tW_%=:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
                 "@!P bra W_%=;\n\t}" :: "r"(smem_u32(b)), "r"(parity) : "memory");
}
__device__ __forceinline__ void gather4(void *dst, const CUtensorMap *map, int r0, int r1, int r2,
                                        int r3, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
        :: "r"(smem_u32(dst)), "l"(map), "r"(0), "r"(r0), "r"(r1), "r"(r2), "r"(r3),
           "r"(smem_u32(bar)) : "memory");
}

template <int SLOTS, int RPS>
__global__ void __launch_bounds__(256, 1) tma_gather_kernel(const __grid_constant__ CUtensorMap map,
                                                            uint32_t shift, int iters, float *sink) {
    extern __shared__ __align__(1024) unsigned char smem[];
    __shared__ uint64_t bars[8][SLOTS];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned char *ring = smem + (size_t)warp * SLOTS * RPS * kRow;
    if (lane == 0)
        for (int s = 0; s < SLOTS; ++s) mbar_init(&bars[warp][s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncwarp();
    uint32_t x = (blockIdx.x * 8 + warp) * 0x9E3779B9u + 12345u;
    auto fill = [&](int s) {
        if (lane == 0) {
            mbar_expect(&bars[warp][s], RPS * kRow);
#pragma unroll
            for (int g = 0; g < RPS / 4; ++g) {
                int r[4];
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    x = x * 1664525u + 1013904223u;
                    r[k] = (int)(x >> shift);
                }
                gather4(ring + ((size_t)s * RPS + 4 * g) * kRow, &map, r[0], r[1], r[2], r[3],
                        &bars[warp][s]);
            }
        }
    };
    for (int s = 0; s < SLOTS; ++s) fill(s);
    float acc = 0.f;
    uint32_t phase = 0;
    for (int it = 0; it < iters; ++it) {
        for (int s = 0; s < SLOTS; ++s) {
            mbar_wait(&bars[warp][s], phase);
            const float4 *row = reinterpret_cast<const float4 *>(ring + (size_t)s * RPS * kRow);
#pragma unroll 4
            for (int i = 0; i < RPS; i += 2) {          // 2 rows per warp instruction
                const float4 v = row[(i + (lane >> 4)) * (kRow / 16) + (lane & 15)];
                acc += v.x + v.y + v.z + v.w;
            }
            __syncwarp();
            fill(s);
        }
        phase ^= 1u;
    }
    for (int s = 0; s < SLOTS; ++s) mbar_wait(&bars[warp][s], phase);
    if (acc == 1234.5f) sink[0] = acc;
}

using EncodeFn = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                              const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                              const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                              CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
}  // namespace

// Returns 0 on success; *gbs = best rows-landed GB/s over a few ring shapes.
extern "C" int tma_gather_probe_gbs(int64_t bytes, float *gbs, float *ms, int *best_cfg) {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
        return 4;
    EncodeFn enc = reinterpret_cast<EncodeFn>(p);
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    uint32_t rows = 1, shift = 32;
    while ((int64_t)(rows * 2) * kRow <= bytes) { rows *= 2; --shift; }
    float *tab = nullptr, *sink = nullptr;
    if (cudaMalloc(&tab, (size_t)rows * kRow) != cudaSuccess) return 1;
    cudaMalloc(&sink, 4);
    cudaMemset(tab, 0, (size_t)rows * kRow);
    CUtensorMap map;
    const cuuint64_t dims[2] = {64, rows};
    const cuuint64_t strides[1] = {kRow};
    const cuuint32_t box[2] = {64, 1};
    const cuuint32_t estr[2] = {1, 1};
    if (enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, tab, dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
        cudaFree(tab);
        return 5;
    }
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best = 0.f, best_ms = 0.f;
    int bc = -1;
    for (int cfg = 0; cfg < 3; ++cfg) {
        const int iters = 200;
        size_t smem = 0;
        void (*k)(CUtensorMap, uint32_t, int, float *) = nullptr;
        int slots = 0, rps = 0;
        if (cfg == 0) { k = tma_gather_kernel<4, 16>; slots = 4; rps = 16; }
        if (cfg == 1) { k = tma_gather_kernel<8, 8>; slots = 8; rps = 8; }
        if (cfg == 2) { k = tma_gather_kernel<6, 16>; slots = 6; rps = 16; }
        smem = (size_t)8 * slots * rps * kRow;
        if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
            cudaSuccess)
            continue;
        k<<<sms, 256, smem>>>(map, shift, 5, sink);           // warm-up, table resident
        for (int rep = 0; rep < 3; ++rep) {
            cudaEventRecord(e0);
            k<<<sms, 256, smem>>>(map, shift, iters, sink);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float t = 0.f;
            cudaEventElapsedTime(&t, e0, e1);
            const double moved = (double)sms * 8 * ((double)iters * slots + slots) * rps * kRow;
            const float g = (float)(moved / (t * 1e-3) / 1e9);
            if (g > best) { best = g; best_ms = t; bc = cfg; }
        }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(tab);
    cudaFree(sink);
    *gbs = best;
    *ms = best_ms;
    *best_cfg = bc;
    return cudaGetLastError() == cudaSuccess ? 0 : 2;
}
