// xw_gemm.cu -- NEXT-3: the GCN combination B = X * W (computed before
// the aggregation, A*(X*W)) on the 5th-generation tensor cores, writing B in bf16
// straight into the row-major layout the segment kernel gathers from.
//
// One CTA per 128-row tile of X, the whole output width N (<= 256) in TMEM:
//   warp 0 (one lane): TMA producer -- 2-D tensor loads of X[128 x 64] and Wt[N x 64]
//                      (bf16, 128-B swizzle) into a 2-4 stage smem ring (mbarrier full/empty),
//                      sized so that >= 2 CTAs share an SM;
//   warp 1 (one lane): MMA issuer -- tcgen05.mma.cta_group::1.kind::f16, M=128, N, K=16,
//                      fp32 accumulator in TMEM; tcgen05.commit frees each stage;
//   warps 0-3:         epilogue -- tcgen05.ld 32x32b (each thread one row), bf16 convert,
//                      16-B stores of the B row.
// The shape is tall and thin (n x F times F x N), so the kernel is HBM-bound on reading X;
// the tensor cores are far from busy, which is the point: the combination costs one read of
// X and one write of B.
//
// Multi-GPU (NEXT-3, the B replication of the sharder): the same kernel
// with several destinations.  Rank g computes its row block of B and the epilogue stores
// every tile into the B replica of EVERY rank (peer HBM over NVLink/NVSwitch, mapped with
// CUDA IPC), so the all-gather of B is fused into the GEMM that produces it and the NVLink
// transfer of one tile overlaps the TMA loads and MMAs of the next.
#include <cuda.h>
#include <cuda_bf16.h>

#include <cstdlib>
#include <cstring>

#include "mps_internal.cuh"

namespace mps {

namespace {

constexpr int kXwBM = 128;       // rows of X per CTA (UMMA M)
constexpr int kXwBK = 64;        // reduction chunk: 64 bf16 = 128 B = one swizzle row
constexpr int kXwMaxStages = 4;
constexpr int kXwMaxDst = 16;     // replicas one launch can write (ranks of one NVLink domain)
constexpr int kXwThreads = 128;

// Destinations of the epilogue: B row (row_offset + r) of each replica.
struct XwDst {
    __nv_bfloat16 *p[kXwMaxDst];
    int nd;
    int64_t row_offset;
};

__device__ __forceinline__ uint64_t smem_desc_sw128(uint32_t saddr) {
    // UMMA shared-memory descriptor, K-major, SWIZZLE_128B (cute::UMMA::SmemDescriptor):
    // start address >> 4 [0,14); LBO >> 4 [16,30) (unused for swizzled K-major, 1);
    // SBO >> 4 [32,46) = 1024 B between 8-row core-matrix groups; version 1 [46,48);
    // base offset 0 (1024-B aligned tiles); layout type 2 = SWIZZLE_128B [61,64).
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
    d |= (uint64_t)1u << 16;
    d |= (uint64_t)(1024u >> 4) << 32;
    d |= (uint64_t)1u << 46;
    d |= (uint64_t)2u << 61;
    return d;
}

__device__ __forceinline__ uint32_t instr_desc_bf16(int N) {
    // kind::f16 instruction descriptor: D fp32 (c_format 1, bits [4,6)), A and B bf16
    // (a_format 1 bits [7,10), b_format 1 bits [10,13)), both K-major, N >> 3 at [17,23),
    // M >> 4 at [24,29) with M = 128.
    return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(kXwBM >> 4) << 24);
}

__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap *map, int c0, int c1,
                                            uint32_t bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3}], [%4];"
        :: "r"(dst), "l"(map), "r"(c0), "r"(c1), "r"(bar) : "memory");
}

__device__ __forceinline__ void mbar_wait_u32(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred P;\n\t"
        "XW_WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
        "@!P bra XW_WAIT_%=;\n\t}"
        :: "r"(bar), "r"(parity) : "memory");
}

__global__ void __launch_bounds__(kXwThreads)
xw_gemm_kernel(const __grid_constant__ CUtensorMap map_x, const __grid_constant__ CUtensorMap map_w,
               int64_t n, int F, int N, int kXwStages, const XwDst dst, int64_t ldb) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    // 1024-B aligned carve-up: A stages, B stages, then barriers and the TMEM address
    uint8_t *base = (uint8_t *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    const uint32_t a_bytes = kXwBM * kXwBK * 2;                       // 16 KB
    const uint32_t b_bytes = (uint32_t)N * kXwBK * 2;                 // <= 32 KB
    uint8_t *sA = base;
    uint8_t *sB = base + kXwStages * a_bytes;
    uint64_t *full = (uint64_t *)(sB + kXwStages * b_bytes);
    uint64_t *empty = full + kXwMaxStages;
    uint64_t *done = empty + kXwMaxStages;
    uint32_t *tmem_slot = (uint32_t *)(done + 1);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t m0 = (int64_t)blockIdx.x * kXwBM;
    const int nk = (F + kXwBK - 1) / kXwBK;
    const uint32_t ncols = N <= 32 ? 32 : (N <= 64 ? 64 : (N <= 128 ? 128 : 256));

    if (threadIdx.x == 0) {
        for (int s = 0; s < kXwMaxStages; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], 1);
        }
        mbar_init(done, 1);
        asm volatile("prefetch.tensormap [%0];" :: "l"(&map_x) : "memory");
        asm volatile("prefetch.tensormap [%0];" :: "l"(&map_w) : "memory");
    }
    mbar_fence_init();
    if (warp == 2) {   // TMEM allocation: one warp, power-of-two columns >= 32
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                     :: "r"(smem_u32(tmem_slot)), "r"(ncols) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = *tmem_slot;

    if (warp == 0 && lane == 0) {
        // ---- TMA producer ----
        for (int kb = 0; kb < nk; ++kb) {
            const int s = kb % kXwStages;
            if (kb >= kXwStages) mbar_wait_u32(smem_u32(&empty[s]), ((kb / kXwStages) - 1) & 1);
            mbar_arrive_expect_tx(&full[s], a_bytes + b_bytes);
            tma_load_2d(smem_u32(sA + s * a_bytes), &map_x, kb * kXwBK, (int)m0, smem_u32(&full[s]));
            tma_load_2d(smem_u32(sB + s * b_bytes), &map_w, kb * kXwBK, 0, smem_u32(&full[s]));
        }
    } else if (warp == 1 && lane == 0) {
        // ---- MMA issuer (single thread) ----
        const uint32_t idesc = instr_desc_bf16(N);
        for (int kb = 0; kb < nk; ++kb) {
            const int s = kb % kXwStages;
            mbar_wait_u32(smem_u32(&full[s]), (kb / kXwStages) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            const uint64_t da = smem_desc_sw128(smem_u32(sA + s * a_bytes));
            const uint64_t db = smem_desc_sw128(smem_u32(sB + s * b_bytes));
#pragma unroll
            for (int k = 0; k < kXwBK / 16; ++k) {
                // advance 16 bf16 = 32 B inside the 128-B swizzle row (start address >> 4)
                const uint64_t a = da + (uint64_t)(k * 2);
                const uint64_t b = db + (uint64_t)(k * 2);
                const uint32_t acc = (kb > 0 || k > 0) ? 1u : 0u;
                asm volatile(
                    "{\n\t.reg .pred p;\n\t"
                    "setp.ne.b32 p, %4, 0;\n\t"
                    "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}"
                    :: "r"(tmem), "l"(a), "l"(b), "r"(idesc), "r"(acc) : "memory");
            }
            // frees the stage once these MMAs have read it
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                         :: "r"(smem_u32(&empty[s])) : "memory");
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                     :: "r"(smem_u32(done)) : "memory");
    }
    __syncwarp();

    // ---- epilogue: TMEM -> registers -> bf16 -> global ----
    mbar_wait_u32(smem_u32(done), 0);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const int64_t row = m0 + warp * 32 + lane;
    for (int c0 = 0; c0 < N; c0 += 32) {
        uint32_t v[32];
        const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)c0;
        asm volatile(
            "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
            "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
            "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
            : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]),
              "=r"(v[6]), "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]),
              "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]), "=r"(v[16]), "=r"(v[17]),
              "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
              "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]),
              "=r"(v[30]), "=r"(v[31])
            : "r"(taddr));
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        if (row < n) {
            const int cols = (N - c0) < 32 ? (N - c0) : 32;   // N % 16 == 0: 16 or 32
            uint32_t pk[16];
#pragma unroll
            for (int i = 0; i < 16; ++i) {
                __nv_bfloat162 h = __floats2bfloat162_rn(__uint_as_float(v[2 * i]),
                                                         __uint_as_float(v[2 * i + 1]));
                pk[i] = *reinterpret_cast<uint32_t *>(&h);
            }
            // local replica first, then the peers (rotated by block so that the ranks'
            // CTAs spread their NVLink stores over all destinations at once)
            for (int i = 0; i < dst.nd; ++i) {
                const int d = i == 0 ? 0 : 1 + (int)((blockIdx.x + i - 1) % (dst.nd - 1));
                uint4 *o = reinterpret_cast<uint4 *>(dst.p[d] + (dst.row_offset + row) * ldb + c0);
                o[0] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
                o[1] = make_uint4(pk[4], pk[5], pk[6], pk[7]);
                if (cols == 32) {
                    o[2] = make_uint4(pk[8], pk[9], pk[10], pk[11]);
                    o[3] = make_uint4(pk[12], pk[13], pk[14], pk[15]);
                }
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 2)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;"
                     :: "r"(tmem), "r"(ncols) : "memory");
}

// ---------------------------------------------------------------------------------
// Persistent variant, used whenever W fits in shared memory next to the X ring: W is
// loaded ONCE per CTA and stays resident; X tiles stream through an S-stage TMA ring; two
// TMEM accumulators (2 x N columns) let the epilogue of tile i overlap the MMAs of tile
// i+1.  Warp roles (320 threads): warp 0 = TMA producer, warp 1 = MMA issuer, warps 2-9 =
// epilogue (warp w reads TMEM lanes 32*(w%4)..+31; two warps per lane quarter split the
// columns).  The epilogue stages each 32x32 bf16 block in shared memory (XOR-swizzled)
// so that global stores write 64 contiguous bytes per row, 8 rows per instruction.
// ---------------------------------------------------------------------------------
constexpr int kXpThreads = 320;       // 2 + 8 epilogue warps (two per TMEM lane quarter)
constexpr int kXpMaxStages = 8;

__global__ void __launch_bounds__(kXpThreads, 1)
xw_persistent_kernel(const __grid_constant__ CUtensorMap map_x,
                     const __grid_constant__ CUtensorMap map_w,
                     const __grid_constant__ CUtensorMap map_b, int64_t n, int F, int N,
                     int stages, const XwDst dst, int64_t ldb, int staged, int nsplit,
                     int wstream) {
    // wstream = 1: W is NOT resident -- each ring stage carries the X chunk AND the
    // matching 64-wide chunk of W (re-read from L2 for every tile), for W too large for
    // shared memory (Reddit K=256: W = 256 x 602 bf16 = 308 KB)
    // N = the column slice this CTA computes; nsplit slices of W / B are spread over
    // consecutive CTAs (W too large for shared memory as a whole, or TMEM for 2 CTAs)
    const int slice = (int)(blockIdx.x % (unsigned)nsplit);
    const int64_t t0 = blockIdx.x / nsplit, tstride = gridDim.x / nsplit;
    const int col_off = slice * N;
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *base = (uint8_t *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    const int nk = (F + kXwBK - 1) / kXwBK;
    const uint32_t a_bytes = kXwBM * kXwBK * 2;            // 16 KB per X stage
    const uint32_t wchunk = (uint32_t)N * kXwBK * 2;        // one 64-wide chunk of W
    const uint32_t stage_bytes = a_bytes + (wstream ? wchunk : 0u);
    uint8_t *sW = base;
    uint8_t *sA = base + (wstream ? (size_t)0 : (size_t)nk * wchunk);
    // staging tiles right after the ring (1024-B aligned: every stage is a multiple of
    // 1 KB), barriers after them
    uint8_t *stg = sA + (size_t)stages * stage_bytes;       // 8 warps x 32 rows x 64 B
    uint64_t *full = (uint64_t *)(stg + 8 * 32 * 64);
    uint64_t *empty = full + kXpMaxStages;
    uint64_t *acc_full = empty + kXpMaxStages;              // [2]
    uint64_t *acc_empty = acc_full + 2;                     // [2]
    uint64_t *w_full = acc_empty + 2;
    uint32_t *tmem_slot = (uint32_t *)(w_full + 1);


    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t ntiles = (n + kXwBM - 1) / kXwBM;
    const uint32_t ncols = (2 * N) <= 32 ? 32 : ((2 * N) <= 64 ? 64 : ((2 * N) <= 128 ? 128
                           : ((2 * N) <= 256 ? 256 : 512)));

    if (threadIdx.x == 0) {
        for (int s = 0; s < kXpMaxStages; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], 1);
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(&acc_full[a], 1);
            mbar_init(&acc_empty[a], 8);                    // one arrival per epilogue warp
        }
        mbar_init(w_full, 1);
        asm volatile("prefetch.tensormap [%0];" :: "l"(&map_x) : "memory");
        asm volatile("prefetch.tensormap [%0];" :: "l"(&map_w) : "memory");
    }
    mbar_fence_init();
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                     :: "r"(smem_u32(tmem_slot)), "r"(ncols) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {
            // ---- TMA producer: W once (resident), then the X ring across this CTA's
            //      tiles; streamed W: every stage also carries its W chunk ----
            if (!wstream) {
                mbar_arrive_expect_tx(w_full, (uint32_t)nk * wchunk);
                for (int kb = 0; kb < nk; ++kb)
                    tma_load_2d(smem_u32(sW + (size_t)kb * wchunk), &map_w, kb * kXwBK, col_off,
                                smem_u32(w_full));
            }
            uint32_t it = 0;
            for (int64_t t = t0; t < ntiles; t += tstride) {
                for (int kb = 0; kb < nk; ++kb, ++it) {
                    const uint32_t s = it % (uint32_t)stages;
                    if (it >= (uint32_t)stages)
                        mbar_wait_u32(smem_u32(&empty[s]), ((it / stages) - 1) & 1);
                    uint8_t *st = sA + (size_t)s * stage_bytes;
                    mbar_arrive_expect_tx(&full[s], stage_bytes);
                    tma_load_2d(smem_u32(st), &map_x, kb * kXwBK, (int)(t * kXwBM),
                                smem_u32(&full[s]));
                    if (wstream)
                        tma_load_2d(smem_u32(st + a_bytes), &map_w, kb * kXwBK, col_off,
                                    smem_u32(&full[s]));
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {
            // ---- MMA issuer ----
            const uint32_t idesc = instr_desc_bf16(N);
            if (!wstream) mbar_wait_u32(smem_u32(w_full), 0);
            uint32_t it = 0, i = 0;
            for (int64_t t = t0; t < ntiles; t += tstride, ++i) {
                const uint32_t acc = i & 1u, use = i >> 1;
                if (use > 0) mbar_wait_u32(smem_u32(&acc_empty[acc]), (use - 1) & 1);
                asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                const uint32_t d = tmem + acc * (uint32_t)N;
                for (int kb = 0; kb < nk; ++kb, ++it) {
                    const uint32_t s = it % (uint32_t)stages;
                    mbar_wait_u32(smem_u32(&full[s]), (it / stages) & 1);
                    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                    uint8_t *st = sA + (size_t)s * stage_bytes;
                    const uint64_t da = smem_desc_sw128(smem_u32(st));
                    const uint64_t db = smem_desc_sw128(
                        smem_u32(wstream ? st + a_bytes : sW + (size_t)kb * wchunk));
#pragma unroll
                    for (int k = 0; k < kXwBK / 16; ++k) {
                        const uint32_t accum = (kb > 0 || k > 0) ? 1u : 0u;
                        asm volatile(
                            "{\n\t.reg .pred p;\n\t"
                            "setp.ne.b32 p, %4, 0;\n\t"
                            "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}"
                            :: "r"(d), "l"(da + (uint64_t)(k * 2)), "l"(db + (uint64_t)(k * 2)),
                               "r"(idesc), "r"(accum) : "memory");
                    }
                    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                                 :: "r"(smem_u32(&empty[s])) : "memory");
                }
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                             :: "r"(smem_u32(&acc_full[acc])) : "memory");
            }
        }
    } else {
        // ---- epilogue warps 2..9: TMEM -> registers -> bf16 -> every destination ----
        // warp w drains TMEM lane quarter w % 4 (the hardware's access rule), columns
        // chunks of 32 alternating between the two warps of a quarter
        const int q = warp & 3;                              // TMEM lane quarter
        const int half = (warp - 2) >> 2;
        uint8_t *wst = stg + (size_t)(warp - 2) * 32 * 64;  // this warp's staging tile
        uint32_t i = 0;
        for (int64_t t = t0; t < ntiles; t += tstride, ++i) {
            const uint32_t acc = i & 1u, use = i >> 1;
            mbar_wait_u32(smem_u32(&acc_full[acc]), use & 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            if (half * 32 >= N) {                            // no columns for this warp
                __syncwarp();
                if (lane == 0) mbar_arrive(&acc_empty[acc]);
                continue;
            }
            for (int c0 = half * 32; c0 < N; c0 += 64) {
                uint32_t v[32];
                const uint32_t taddr = tmem + ((uint32_t)(q * 32) << 16) + acc * (uint32_t)N +
                                       (uint32_t)c0;
                asm volatile(
                    "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
                    "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                    "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                    : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]),
                      "=r"(v[6]), "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]),
                      "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]), "=r"(v[16]), "=r"(v[17]),
                      "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
                      "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]),
                      "=r"(v[30]), "=r"(v[31])
                    : "r"(taddr));
                asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
                if (c0 + 64 >= N) {
                    // this warp's part is drained: hand it back to the MMA warp early
                    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&acc_empty[acc]);
                }
                if (!staged) {
                    if (t * kXwBM + q * 32 + lane < n) {
                        const int64_t row = t * kXwBM + q * 32 + lane;
                        const int cols = (N - c0) < 32 ? (N - c0) : 32;
                        uint32_t pk[16];
#pragma unroll
                        for (int j = 0; j < 16; ++j) {
                            __nv_bfloat162 h = __floats2bfloat162_rn(__uint_as_float(v[2 * j]),
                                                                     __uint_as_float(v[2 * j + 1]));
                            pk[j] = *reinterpret_cast<uint32_t *>(&h);
                        }
                        for (int e = 0; e < dst.nd; ++e) {
                            const int dd = e == 0 ? 0 : 1 + (int)((blockIdx.x + e - 1) % (dst.nd - 1));
                            uint4 *o = reinterpret_cast<uint4 *>(dst.p[dd] + (dst.row_offset + row) * ldb +
                                                                 col_off + c0);
                            o[0] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
                            o[1] = make_uint4(pk[4], pk[5], pk[6], pk[7]);
                            if (cols == 32) {
                                o[2] = make_uint4(pk[8], pk[9], pk[10], pk[11]);
                                o[3] = make_uint4(pk[12], pk[13], pk[14], pk[15]);
                            }
                        }
                    }
                    continue;
                }
                // bf16 row slice (64 B) -> this warp's staging tile, 16-B chunks XOR-swizzled
                // by (row >> 1) & 3 so that both the row-wise writes and the column-wise
                // reads below hit 8 distinct 16-B bank groups per 8 lanes
                uint32_t pk[16];
                if (staged == 2) {
                    // one destination, 32-column chunks: the 32 x 32 block leaves by a TMA
                    // tensor store (the pattern is the tensor map's 64-B swizzle), issued by
                    // one lane -- no per-lane address arithmetic or global stores
#pragma unroll
                    for (int j = 0; j < 16; ++j) {
                        __nv_bfloat162 h = __floats2bfloat162_rn(__uint_as_float(v[2 * j]),
                                                                 __uint_as_float(v[2 * j + 1]));
                        pk[j] = *reinterpret_cast<uint32_t *>(&h);
                    }
                    const uint32_t sb = smem_u32(wst);
                    if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
                    __syncwarp();
#pragma unroll
                    for (int j = 0; j < 4; ++j)
                        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};"
                                     :: "r"(sb + lane * 64 + ((j ^ ((lane >> 1) & 3)) << 4)),
                                        "r"(pk[4 * j]), "r"(pk[4 * j + 1]), "r"(pk[4 * j + 2]),
                                        "r"(pk[4 * j + 3]) : "memory");
                    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                    __syncwarp();
                    if (lane == 0) {
                        asm volatile(
                            "cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
                            :: "l"(&map_b), "r"(col_off + c0), "r"((int)(t * kXwBM) + q * 32), "r"(sb)
                            : "memory");
                        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
                    }
                    continue;
                }
#pragma unroll
                for (int j = 0; j < 16; ++j) {
                    __nv_bfloat162 h = __floats2bfloat162_rn(__uint_as_float(v[2 * j]),
                                                             __uint_as_float(v[2 * j + 1]));
                    pk[j] = *reinterpret_cast<uint32_t *>(&h);
                }
                uint4 *myst = reinterpret_cast<uint4 *>(wst) + lane * 4;
#pragma unroll
                for (int j = 0; j < 4; ++j)
                    myst[j ^ ((lane >> 1) & 3)] =
                        make_uint4(pk[4 * j], pk[4 * j + 1], pk[4 * j + 2], pk[4 * j + 3]);
                __syncwarp();
                // coalesced stores: each instruction writes 8 rows x 64 contiguous bytes
                const int cols = (N - c0) < 32 ? (N - c0) : 32;   // N % 16 == 0: 16 or 32
                const int j = lane & 3;
                if (j * 8 < cols) {
#pragma unroll
                    for (int k = 0; k < 4; ++k) {
                        const int r = k * 8 + (lane >> 2);
                        const int64_t grow = t * kXwBM + q * 32 + r;
                        if (grow < n) {
                            const uint4 val = reinterpret_cast<const uint4 *>(
                                wst)[r * 4 + (j ^ ((r >> 1) & 3))];
                            for (int e = 0; e < dst.nd; ++e) {
                                const int dd = e == 0 ? 0
                                               : 1 + (int)((blockIdx.x + e - 1) % (dst.nd - 1));
                                *reinterpret_cast<uint4 *>(dst.p[dd] + (dst.row_offset + grow) * ldb +
                                                           col_off + c0 + j * 8) = val;
                            }
                        }
                    }
                }
                __syncwarp();
            }
        }
    }
    if (staged == 2 && warp >= 2 && lane == 0)
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");   // the TMA stores
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 1)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;"
                     :: "r"(tmem), "r"(ncols) : "memory");
}

using EncodeFn = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                              const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                              const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                              CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeFn encode_fn() {
    static EncodeFn fn = nullptr;
    if (!fn) {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) ==
                cudaSuccess && q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<EncodeFn>(p);
    }
    return fn;
}

bool make_map(CUtensorMap *map, const void *ptr, int64_t rows, int64_t cols, int64_t ld_elems,
              int box_rows) {
    EncodeFn fn = encode_fn();
    if (!fn) return false;
    const cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
    const cuuint64_t strides[1] = {(cuuint64_t)ld_elems * 2};
    const cuuint32_t box[2] = {(cuuint32_t)kXwBK, (cuuint32_t)box_rows};
    const cuuint32_t estr[2] = {1, 1};
    return fn(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void *>(ptr), dims, strides,
              box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
              CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// B (bf16 [rows][ld], cols used) as the destination of 32 x 32 TMA tensor stores, 64-B
// swizzle (the persistent kernel's staging layout)
bool make_store_map(CUtensorMap *map, const void *ptr, int64_t rows, int64_t cols, int64_t ld_elems) {
    EncodeFn fn = encode_fn();
    if (!fn) return false;
    const cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
    const cuuint64_t strides[1] = {(cuuint64_t)ld_elems * 2};
    const cuuint32_t box[2] = {32, 32};
    const cuuint32_t estr[2] = {1, 1};
    return fn(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void *>(ptr), dims, strides,
              box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B,
              CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace

// X: bf16 [n][ldx] (F used columns), Wt: bf16 [N][ldw] (= W transposed, F used columns);
// B row (row_offset + r) of every dsts[d] (bf16 [.][ldb]) receives row r of X * W.
// Returns cudaErrorNotSupported for shapes the kernel does not cover.
static cudaError_t launch_xw(const void *X, int64_t n, int64_t F, int64_t ldx, const void *Wt,
                             int32_t N, int64_t ldw, void *const *dsts, int nd,
                             int64_t row_offset, int64_t ldb, cudaStream_t s) {
    if (N < 16 || N > 256 || N % 16 || F < 1 || ldx % 8 || ldw % 8 || ldb % 8 ||
        ((uintptr_t)X & 15) || ((uintptr_t)Wt & 15) || nd < 1 || nd > kXwMaxDst)
        return cudaErrorNotSupported;
    XwDst dst{};
    for (int d = 0; d < nd; ++d) {
        if (!dsts[d] || ((uintptr_t)dsts[d] & 15)) return cudaErrorNotSupported;
        dst.p[d] = reinterpret_cast<__nv_bfloat16 *>(dsts[d]);
    }
    dst.nd = nd;
    dst.row_offset = row_offset;
    if (n == 0) return cudaSuccess;
    CUtensorMap mx, mw;
    if (!make_map(&mx, X, n, F, ldx, kXwBM) || !make_map(&mw, Wt, N, F, ldw, N))
        return cudaErrorNotSupported;
    // persistent kernel when W stays resident next to a >= 2-stage X ring (MPS_XW_PERSIST=0:
    // always the one-tile-per-CTA kernel; A/B experiments)
    static const int persist = [] {
        const char *e = getenv("MPS_XW_PERSIST");
        return e ? atoi(e) : 1;
    }();
    static const int max_stages = [] {
        const char *e = getenv("MPS_XW_STAGES");
        return e ? atoi(e) : kXpMaxStages;
    }();
    static const int force_split = [] {
        const char *e = getenv("MPS_XW_SPLIT");
        return e ? atoi(e) : 0;
    }();
    // MPS_XW_WSTREAM: 1 = stream W through the ring even when it fits (A/B), 0 = never
    static const int wstream_env = [] {
        const char *e = getenv("MPS_XW_WSTREAM");
        return e ? atoi(e) : -1;
    }();
    static const int staged = [] {
        const char *e = getenv("MPS_XW_STAGED");
        return e ? atoi(e) : 1;
    }();
    // TMA-store epilogue (one destination, 32-column chunks); MPS_XW_TMA_STORE=0: per-lane
    // global stores from the staging tiles (A/B)
    static const int tma_store = [] {
        const char *e = getenv("MPS_XW_TMA_STORE");
        return e ? atoi(e) : 1;
    }();
    CUtensorMap mb;
    memset(&mb, 0, sizeof(mb));
    const bool can_tma_store = tma_store && staged && nd == 1 &&
                               make_store_map(&mb, reinterpret_cast<const __nv_bfloat16 *>(dsts[0]) + row_offset * ldb,
                                              n, N, ldb);
    auto staged_mode = [&](int nh) { return (can_tma_store && nh % 32 == 0) ? 2 : staged; };
    const size_t xw_budget = 227u << 10, xw_fixed = 1024 + 512 + 8 * 32 * 64;
    auto set_persist_attr = [&]() -> cudaError_t {
        // function attributes are per device: set once for each
        static bool pattr[64] = {false};
        int dev = 0;
        if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) dev = 0;
        if (!pattr[dev]) {
            cudaError_t e = cudaFuncSetAttribute(xw_persistent_kernel,
                                                 cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                 (int)xw_budget);
            if (e != cudaSuccess) return e;
            pattr[dev] = true;
        }
        return cudaSuccess;
    };
    // streamed-W persistent kernel: the whole N per CTA (TMEM 2 x N <= 512 columns), stages
    // of X chunk + W chunk; two CTAs per SM when three stages fit in half the budget
    auto launch_wstream = [&]() -> cudaError_t {
        const size_t stage_bytes = (size_t)kXwBM * kXwBK * 2 + (size_t)N * kXwBK * 2;
        int per_sm = ((113u << 10) - xw_fixed) / stage_bytes >= 3 ? 2 : 1;
        if (2 * 2 * N > 512) per_sm = 1;
        int stages = (int)(((per_sm == 2 ? (113u << 10) : xw_budget) - xw_fixed) / stage_bytes);
        stages = stages > max_stages ? max_stages : stages;
        if (stages < 2) return cudaErrorNotSupported;
        cudaError_t e = set_persist_attr();
        if (e != cudaSuccess) return e;
        const size_t smem = xw_fixed + (size_t)stages * stage_bytes;
        const int64_t ntiles = (n + kXwBM - 1) / kXwBM;
        int64_t grid = (int64_t)num_sms() * per_sm;
        if (grid > ntiles) grid = ntiles;
        xw_persistent_kernel<<<(unsigned)grid, kXpThreads, smem, s>>>(
            mx, mw, mb, n, (int)F, N, stages, dst, ldb, staged_mode(N), 1, 1);
        return cudaGetLastError();
    };
    if (persist && wstream_env == 1) return launch_wstream();
    if (persist) {
        // Choose the column slice width Nh of W / B one CTA owns (nsplit = N / Nh slices
        // on consecutive CTAs; X tiles are then read once per slice, the repeats from L2).
        // Measured (profiles/r01/xw_gemm.md): the whole W (Nh = N) wins whenever it fits,
        // at two CTAs per SM (TMEM 2 x 2N <= 512 columns, W + >= 2 X stages in half the
        // shared memory) or else one; slices only when W does not fit at all.
        const int nkp = (int)((F + kXwBK - 1) / kXwBK);
        const size_t a_bytes = (size_t)kXwBM * kXwBK * 2;
        const size_t fixed = xw_fixed;                      // align, barriers, staging
        const size_t budget = 227u << 10, half_budget = 113u << 10;
        auto wb = [&](int nh) { return (size_t)nkp * nh * kXwBK * 2; };
        int nh = 0, per_sm = 0;
        // slices (d > 1) only when streaming W is switched off (MPS_XW_WSTREAM=0): the
        // streamed-W kernel beat them on Reddit K=256 (0.098 vs 0.139 ms, r02k)
        const int dmax = (wstream_env == 0 || force_split > 1) ? 4 : 1;
        for (int d = 1; d <= dmax && nh == 0; d *= 2)
            for (int pass = 0; pass < 2 && nh == 0; ++pass) {
                const int c = N / d;
                if (N % d || c % 16) continue;
                if (force_split > 0 && d != force_split) continue;
                if (pass == 0 && 4 * c <= 512 && wb(c) + 2 * a_bytes + fixed <= half_budget) {
                    nh = c;
                    per_sm = 2;
                } else if (pass == 1 && wb(c) + 2 * a_bytes + fixed <= budget) {
                    nh = c;
                    per_sm = 1;
                }
            }
        if (nh > 0) {
            const int nsplit = N / nh;
            int stages = (int)(((per_sm == 2 ? half_budget : budget) - fixed - wb(nh)) / a_bytes);
            stages = stages > max_stages ? max_stages : stages;
            // B at least as wide as X (N >= F: as many bytes written as read): a shallow
            // 3-stage X ring measured fastest (big-F 1M x 256 x 256: 3 stages 0.172 ms,
            // 4: 0.177, 5: 0.188; products neutral; profiles/r03/xw_tma_store.md), the
            // wide-F shapes want every stage (Reddit F=602: 8 stages 0.071, 3: 0.083)
            if (N >= F && stages > 3 && max_stages == kXpMaxStages) stages = 3;
            stages = stages < 2 ? 2 : stages;
            const size_t smem = fixed + wb(nh) + (size_t)stages * a_bytes;
            cudaError_t ea = set_persist_attr();
            if (ea != cudaSuccess) return ea;
            CUtensorMap mws;
            if (nh != N && !make_map(&mws, Wt, N, F, ldw, nh)) return cudaErrorNotSupported;
            const int64_t ntiles = (n + kXwBM - 1) / kXwBM;
            int64_t grid = (int64_t)num_sms() * per_sm / nsplit * nsplit;
            if (grid > ntiles * nsplit) grid = ntiles * nsplit;
            if (grid < nsplit) grid = nsplit;
            xw_persistent_kernel<<<(unsigned)grid, kXpThreads, smem, s>>>(
                mx, nh == N ? mw : mws, mb, n, (int)F, nh, stages, dst, ldb, staged_mode(nh),
                nsplit, 0);
            return cudaGetLastError();
        }
        // W does not fit in shared memory: stream it through the ring with X (the
        // one-tile-per-CTA kernel below reached 46% of HBM on Reddit K=256)
        if (wstream_env != 0) {
            const cudaError_t e = launch_wstream();
            if (e != cudaErrorNotSupported) return e;
        }
    }
    // stages: enough to cover the reduction, but small enough that >= 2 CTAs share an SM
    // (one CTA's epilogue overlaps another's TMA loads); TMEM: <= 2 x 256 columns per SM.
    const size_t stage_bytes = (size_t)kXwBM * kXwBK * 2 + (size_t)N * kXwBK * 2;
    const int nk = (int)((F + kXwBK - 1) / kXwBK);
    int stages = (int)((100u << 10) / stage_bytes);
    stages = stages < 2 ? 2 : (stages > kXwMaxStages ? kXwMaxStages : stages);
    if (stages > nk) stages = nk < 2 ? 2 : nk;
    const size_t smem = 1024 + (size_t)stages * stage_bytes + 256;
    static bool attr[64] = {false};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) dev = 0;
    if (!attr[dev]) {
        cudaError_t e = cudaFuncSetAttribute(
            xw_gemm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
            (int)(1024 + kXwMaxStages * (kXwBM * kXwBK * 2 + 256 * kXwBK * 2) + 256));
        if (e != cudaSuccess) return e;
        attr[dev] = true;
    }
    const unsigned grid = (unsigned)((n + kXwBM - 1) / kXwBM);
    xw_gemm_kernel<<<grid, kXwThreads, smem, s>>>(mx, mw, n, (int)F, N, stages, dst, ldb);
    return cudaGetLastError();
}

cudaError_t launch_xw_bf16(const void *X, int64_t n, int64_t F, int64_t ldx, const void *Wt,
                           int32_t N, int64_t ldw, void *Bout, int64_t ldb, cudaStream_t s) {
    void *d[1] = {Bout};
    return launch_xw(X, n, F, ldx, Wt, N, ldw, d, 1, 0, ldb, s);
}

cudaError_t launch_xw_bf16_bcast(const void *X, int64_t n, int64_t F, int64_t ldx,
                                 const void *Wt, int32_t N, int64_t ldw, void *const *dsts,
                                 int32_t nd, int64_t row_offset, int64_t ldb, cudaStream_t s) {
    return launch_xw(X, n, F, ldx, Wt, N, ldw, dsts, nd, row_offset, ldb, s);
}

}  // namespace mps
