// mps_internal.cuh -- device helpers and kernel interfaces of libmpspmm (sm_100a).
//
// Product code.  Shares nothing with oracle/ (the CPU checker): no headers, tables or
// helpers.  Paper citations "P:<line>" refer to PAPER.md (MergePath-SpMM, ISPASS'23).
#pragma once

#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>

#include "../../include/mpspmm.h"

namespace mps {

constexpr int kBlock = 256;  // threads per CTA for every kernel of the library

enum Fix : int { FIX_ATOMIC = 1, FIX_CARRY = 2 };

// a6 tail exchange over peer memory (NEXT: fused collective).  The last CTA of the kernel
// that finalises this rank's tail (segment kernel in atomic mode, carry reduce in carry
// mode; the last column tile) pushes the tail into its owner's mailbox and pulls the tails
// other ranks pushed for this rank's first row.  Mailbox of every rank (device memory,
// peers map it with CUDA IPC), bytes:
//   [0,4)     launch counter (local use)        [64,128)  flags[g]: epoch pushed by rank g
//   [128,192) acks[h]: epoch consumed by owner h [256, ..) inbox f32 [2 slots][16][K]
constexpr int kMailMaxWorld = 16;
constexpr int kMailFlagsOfs = 64, kMailAcksOfs = 128, kMailInboxOfs = 256;
struct TailMail {
    uint32_t *counter;          // this rank's launch counter (zeroed between launches)
    // push (this rank has a tail row owned by another rank)
    const float *tail;          // the finished local tail, K floats
    float *push_dst;            // owner's inbox[slot][rank]
    uint32_t *push_flag;        // owner's flags[rank]
    const uint32_t *push_ack;   // this rank's acks[owner]
    // pull (rows of this rank receive tails)
    float *pull_row;            // this rank's C row that the tails belong to
    const float *pull_src;      // this rank's inbox[slot]
    const uint32_t *pull_flags; // this rank's flags
    uint32_t *ack_dst[kMailMaxWorld];  // sender g's acks[rank]
    uint32_t pull_mask;         // bit g: rank g pushes a tail to this rank
    uint32_t epoch;             // >= 1, +1 per step
    int32_t K;
    int32_t on;                 // 0: no mailbox work in this launch
};

// Per-launch arguments of the segment kernel (a3 + a4).  Indices are global merge-path
// coordinates; col/val are pre-offset so that col[j] is global nnz j (shards hold a
// slice); C row r lives at C + (r - row_base) * ldc; the row `tail_row` (a shard's cut
// last row) is redirected to `tail`.  IT is the type of row_ptr and of the nnz
// coordinate y: int32_t (M = m + nnz < 2^31) or int64_t (NEXT-4: nnz >= 2^31; rows and
// columns stay < 2^31, so coord_x and col_idx stay int32).
template <typename IT>
struct SegArgsT {
    const IT *rp;
    const int32_t *col;
    const float *val;
    const void *B;
    int64_t ldb;
    int32_t K;          // columns of this column tile
    float *C;
    int64_t ldc;
    int64_t row_base;
    int32_t m;          // rows of the global A
    const int32_t *cx;
    const IT *cy;
    int64_t P;
    int32_t tail_row;   // -1: none
    float *tail;
    float *rec;         // carry records [P][2][kpad]
    int32_t kpad;
    int64_t nnz_end;    // one past the last readable (global) nnz index of col/val
    int32_t direct;     // 1: col/val misaligned relative to each other -> no TMA staging
    int32_t l2_hints;   // 1: B evict_last / col,val evict_first; 0: evict_normal everywhere
    const uint32_t *hot; // optional bitmap over B rows: 1 = keep in L2 (evict_last), 0 = stream
    int32_t relu;        // epilogue: 1 = C = max(C, 0) (complete rows at the store; cut rows
                         // by launch_relu_split after the atomics, or in the carry reduce)
    TailMail mail;       // a6 peer-memory tail exchange (mail.on == 0: none)
    unsigned *claim;     // dynamic segment claims: this column tile's counter in the caller's
                         // workspace, zero when the kernel starts (NULL: static assignment)
    int32_t deep;        // 1: deep-gather instantiation (fp32, 64-column tile, DRAM-bound B)
    int32_t pf;          // 1: next-batch B rows into L2 while this batch is in flight
                         // (dynamic bf16 instantiations; 0: off)
    int32_t pf_shift;    // log2 of the 128-B lines per B row slice of this tile
    unsigned long long *wstat;  // Fig. 5 counters of what the kernel wrote (NULL: off):
                                // [0] partial-row updates (atomic / carry record),
                                // [1] empty partial start pieces whose add was elided,
                                // [2] complete-row stores
};
using SegArgs = SegArgsT<int32_t>;
using SegArgs64 = SegArgsT<int64_t>;

// The one-launch online step for small graphs (small.cu): every CTA stages the whole
// row_ptr in shared memory; each warp computes its segment's coordinates, walks it, and
// leaves the cut rows' pieces in the carry records for carry_reduce_kernel.
struct SmallArgs {
    const int32_t *rp;
    const int32_t *col;
    const float *val;
    const void *B;
    int64_t ldb;
    int32_t K;
    float *C;
    int64_t ldc;
    int32_t m, nnz;
    int32_t P, L;
    int32_t *cx, *cy;   // out: coordinates of the P + 1 diagonals
    float *rec;         // carry records [P][2][kpad]
    int32_t kpad;
    int32_t relu;
    int32_t l2_hints;
};
constexpr int kSmallMaxSmem = 112 * 1024;   // row_ptr + col/val staging per CTA (2 CTAs/SM)
constexpr int kSmallMaxL = 512;             // items per segment
size_t small_smem_bytes(int64_t m, int64_t L);
cudaError_t launch_small_online(const SmallArgs &a, int b_dtype, int W, int NR, cudaStream_t s);

// Host launchers (defined in the .cu files).  IT = int32_t or int64_t (row_ptr and the
// nnz coordinate y).
template <typename IT>
cudaError_t launch_partition(const IT *rp, int64_t m, int64_t nnz, int64_t d0,
                             int64_t span, int64_t P, int64_t L, int32_t *cx, IT *cy,
                             float *zero_C, int64_t ldc, int64_t row_base, int32_t K,
                             int32_t tail_row, float *tail, unsigned *claims, int32_t nclaims,
                             cudaStream_t s);
template <typename IT>
cudaError_t launch_zero_split(const IT *rp, int32_t m, const int32_t *cx,
                              const IT *cy, int64_t P, float *C, int64_t ldc,
                              int64_t row_base, int32_t K, int32_t tail_row, float *tail,
                              unsigned *claims, int32_t nclaims, cudaStream_t s);
template <typename IT>
cudaError_t launch_segments(const SegArgsT<IT> &a, int b_dtype, int W, int V, int NR, int fix,
                            cudaStream_t s);
template <typename IT>
cudaError_t launch_carry_reduce(const SegArgsT<IT> &a, cudaStream_t s);
template <typename IT>
cudaError_t launch_relu_split(const SegArgsT<IT> &a, cudaStream_t s);
cudaError_t launch_peer_signal(void *const *bufs, int world, int rank, int slot, uint32_t epoch,
                               cudaStream_t s);
cudaError_t launch_peer_wait(const void *mine, int world, int slot, uint32_t epoch,
                             cudaStream_t s);
cudaError_t launch_relu_to_bf16(const float *C, int64_t rows, int K, int64_t ldc, void *H,
                                int64_t ldh, cudaStream_t s);
cudaError_t launch_apply_tails(const float *tails, int32_t K, const int32_t *idx, int32_t n,
                               float *row, cudaStream_t s);
template <typename IT>
cudaError_t launch_write_stats(const IT *rp, int32_t m, const int32_t *cx,
                               const IT *cy, int64_t P, int64_t *counts, cudaStream_t s);
template <typename IT>
cudaError_t launch_validate(const IT *rp, const int32_t *col, int64_t m, int64_t n,
                            int64_t nnz, unsigned long long *first_bad, cudaStream_t s);

cudaError_t launch_hot_columns(const int32_t *col, int64_t nnz, int64_t n, int64_t budget_rows,
                               int32_t *counts, uint32_t *hist, uint32_t *bitmap,
                               cudaStream_t s);

cudaError_t launch_xw_bf16(const void *X, int64_t n, int64_t F, int64_t ldx, const void *Wt,
                           int32_t N, int64_t ldw, void *Bout, int64_t ldb, cudaStream_t s);
cudaError_t launch_xw_bf16_bcast(const void *X, int64_t n, int64_t F, int64_t ldx,
                                 const void *Wt, int32_t N, int64_t ldw, void *const *dsts,
                                 int32_t nd, int64_t row_offset, int64_t ldb, cudaStream_t s);

int num_sms();

// Dynamic segment claims pay off from ~4 segments per warp; the launcher uses them only
// when the schedule has that many per resident warp and the caller passed a claim
// counter.  Smallest P for which they can be chosen (every instantiation runs >= 2
// CTAs of kBlock threads per SM):
inline int64_t seg_dynamic_min_parts() { return (int64_t)4 * 2 * (kBlock / 32) * num_sms(); }

// ---------------------------------------------------------------------------------
// device helpers
// ---------------------------------------------------------------------------------
// Fig. 5 write statistic counted where the kernel writes; off (NULL) on the
// hot path, where it costs one uniform test per row end.
__device__ __forceinline__ void count_write(unsigned long long *wstat, int lane, int k) {
    if (wstat != nullptr && lane == 0) atomicAdd(wstat + k, 1ull);
}
template <bool ON>
__device__ __forceinline__ void count_write_if(unsigned long long *wstat, int lane, int k) {
    if constexpr (ON) count_write(wstat, lane, k);
}
template <bool ON>
__device__ __forceinline__ void count_write_n_if(unsigned long long *wstat, int lane, int k,
                                                 int n) {
    if constexpr (ON)
        if (wstat != nullptr && lane == 0 && n > 0) atomicAdd(wstat + k, (unsigned long long)n);
}
__device__ __forceinline__ int ld_stream_i32(const int32_t *p) {
    int v;
    asm volatile("ld.global.cs.s32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ float ld_stream_f32(const float *p) {
    float v;
    asm volatile("ld.global.cs.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}

// L2 cache policies: B rows are re-gathered (keep them: evict_last); col/val and C are
// streamed once (evict_first).
__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t policy_evict_normal() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

// W consecutive elements of B (type TB) as one raw vector gather (read-only path, L2
// evict_last), converted to fp32 at use.  MPS_B_L1 selects the L1 policy:
// 0 = no_allocate, 1 = normal allocation, 2 = evict_last (keep hub rows resident).
#ifndef MPS_B_L1
#define MPS_B_L1 0
#endif
#if MPS_B_L1 == 0
#define MPS_LDB "ld.global.nc.L1::no_allocate.L2::cache_hint"
#elif MPS_B_L1 == 1
#define MPS_LDB "ld.global.nc.L2::cache_hint"
#else
#define MPS_LDB "ld.global.nc.L1::evict_last.L2::cache_hint"
#endif
template <typename TB, int W> struct BVec;

template <> struct BVec<float, 4> {
    using raw = float4;
    static __device__ __forceinline__ raw load(const float *p, uint64_t pol) {
        raw r;
        asm volatile(MPS_LDB ".v4.f32 {%0,%1,%2,%3}, [%4], %5;"
                     : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p), "l"(pol));
        return r;
    }
    static __device__ __forceinline__ void cvt(const raw &r, float (&o)[4]) {
        o[0] = r.x; o[1] = r.y; o[2] = r.z; o[3] = r.w;
    }
};
template <> struct BVec<float, 2> {
    using raw = float2;
    static __device__ __forceinline__ raw load(const float *p, uint64_t pol) {
        raw r;
        asm volatile(MPS_LDB ".v2.f32 {%0,%1}, [%2], %3;"
                     : "=f"(r.x), "=f"(r.y) : "l"(p), "l"(pol));
        return r;
    }
    static __device__ __forceinline__ void cvt(const raw &r, float (&o)[2]) {
        o[0] = r.x; o[1] = r.y;
    }
};
template <> struct BVec<float, 1> {
    using raw = float;
    static __device__ __forceinline__ raw load(const float *p, uint64_t pol) {
        raw r;
        asm volatile(MPS_LDB ".f32 %0, [%1], %2;"
                     : "=f"(r) : "l"(p), "l"(pol));
        return r;
    }
    static __device__ __forceinline__ void cvt(const raw &r, float (&o)[1]) { o[0] = r; }
};

__device__ __forceinline__ float bf_lo(uint32_t w) { return __uint_as_float(w << 16); }
__device__ __forceinline__ float bf_hi(uint32_t w) { return __uint_as_float(w & 0xffff0000u); }

template <> struct BVec<__nv_bfloat16, 8> {
    using raw = uint4;
    static __device__ __forceinline__ raw load(const __nv_bfloat16 *p, uint64_t pol) {
        raw r;
        asm volatile(MPS_LDB ".v4.b32 {%0,%1,%2,%3}, [%4], %5;"
                     : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p), "l"(pol));
        return r;
    }
    static __device__ __forceinline__ void cvt(const raw &r, float (&o)[8]) {
        o[0] = bf_lo(r.x); o[1] = bf_hi(r.x); o[2] = bf_lo(r.y); o[3] = bf_hi(r.y);
        o[4] = bf_lo(r.z); o[5] = bf_hi(r.z); o[6] = bf_lo(r.w); o[7] = bf_hi(r.w);
    }
};
template <> struct BVec<__nv_bfloat16, 4> {
    using raw = uint2;
    static __device__ __forceinline__ raw load(const __nv_bfloat16 *p, uint64_t pol) {
        raw r;
        asm volatile(MPS_LDB ".v2.b32 {%0,%1}, [%2], %3;"
                     : "=r"(r.x), "=r"(r.y) : "l"(p), "l"(pol));
        return r;
    }
    static __device__ __forceinline__ void cvt(const raw &r, float (&o)[4]) {
        o[0] = bf_lo(r.x); o[1] = bf_hi(r.x); o[2] = bf_lo(r.y); o[3] = bf_hi(r.y);
    }
};
template <> struct BVec<__nv_bfloat16, 2> {
    using raw = uint32_t;
    static __device__ __forceinline__ raw load(const __nv_bfloat16 *p, uint64_t pol) {
        raw r;
        asm volatile(MPS_LDB ".b32 %0, [%1], %2;"
                     : "=r"(r) : "l"(p), "l"(pol));
        return r;
    }
    static __device__ __forceinline__ void cvt(const raw &r, float (&o)[2]) {
        o[0] = bf_lo(r); o[1] = bf_hi(r);
    }
};
template <> struct BVec<__nv_bfloat16, 1> {
    using raw = unsigned short;
    static __device__ __forceinline__ raw load(const __nv_bfloat16 *p, uint64_t pol) {
        raw r;
        asm volatile(MPS_LDB ".b16 %0, [%1], %2;"
                     : "=h"(r) : "l"(p), "l"(pol));
        return r;
    }
    static __device__ __forceinline__ void cvt(const raw &r, float (&o)[1]) {
        o[0] = __uint_as_float((uint32_t)r << 16);
    }
};

// The 128-B line holding p into L2 (LSU prefetch; no register, no scoreboard).
__device__ __forceinline__ void prefetch_l2_line(const void *p) {
    asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(p));
}
// base + idx * stride as ONE mad.wide.u32 (IMAD.WIDE.U32 with a 64-bit addend).
__device__ __forceinline__ const char *row_addr(const char *base, uint32_t idx, uint32_t stride) {
    uint64_t r;
    asm("mad.wide.u32 %0, %1, %2, %3;" : "=l"(r) : "r"(idx), "r"(stride), "l"(base));
    return reinterpret_cast<const char *>(r);
}

// acc[0..1] += s * b[0..1] as one packed FFMA2 (sm_100: fma.rn.f32x2).
__device__ __forceinline__ void fma2(float &a0, float &a1, float s, float b0, float b1) {
    asm("{\n\t.reg .b64 acc, bb, ss;\n\t"
        "mov.b64 acc, {%0, %1};\n\tmov.b64 bb, {%3, %4};\n\tmov.b64 ss, {%2, %2};\n\t"
        "fma.rn.f32x2 acc, ss, bb, acc;\n\tmov.b64 {%0, %1}, acc;\n\t}"
        : "+f"(a0), "+f"(a1) : "f"(s), "f"(b0), "f"(b1));
}

// ---- mbarrier + 1-D TMA bulk copy (cp.async.bulk) -----------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_fence_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;"
                 :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred P;\n\t"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
        "@!P bra WAIT_%=;\n\t}"
        :: "r"(smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
// Ampere-style asynchronous copies global -> shared (LDGSTS): many in flight per thread
// without a register round trip; cp_async_wait_all() then a barrier makes them visible.
__device__ __forceinline__ void cp_async16(void *dst_smem, const void *src) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(smem_u32(dst_smem)), "l"(src)
                 : "memory");
}
__device__ __forceinline__ void cp_async4(void *dst_smem, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" :: "r"(smem_u32(dst_smem)), "l"(src)
                 : "memory");
}
__device__ __forceinline__ void cp_async8(void *dst_smem, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" :: "r"(smem_u32(dst_smem)), "l"(src)
                 : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() {
    asm volatile("cp.async.wait_all;" ::: "memory");
}
// global -> shared bulk copy of `bytes` (multiple of 16, both addresses 16-B aligned),
// completion counted on `bar`; L2 evict_first (streamed once).
__device__ __forceinline__ void tma_load_1d(void *dst, const void *src, uint32_t bytes,
                                            uint64_t *bar, uint64_t pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1], %2, [%3], %4;"
        :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol) : "memory");
}

// W consecutive fp32 of C: streaming store, or vector reduction (red.global.add.v4.f32).
template <int W> struct CVec;
template <> struct CVec<1> {
    static __device__ __forceinline__ void store(float *p, const float (&v)[1]) { __stcs(p, v[0]); }
    static __device__ __forceinline__ void add(float *p, const float (&v)[1]) { atomicAdd(p, v[0]); }
};
template <> struct CVec<2> {
    static __device__ __forceinline__ void store(float *p, const float (&v)[2]) {
        __stcs(reinterpret_cast<float2 *>(p), make_float2(v[0], v[1]));
    }
    static __device__ __forceinline__ void add(float *p, const float (&v)[2]) {
        atomicAdd(reinterpret_cast<float2 *>(p), make_float2(v[0], v[1]));
    }
};
template <> struct CVec<4> {
    static __device__ __forceinline__ void store(float *p, const float (&v)[4]) {
        __stcs(reinterpret_cast<float4 *>(p), make_float4(v[0], v[1], v[2], v[3]));
    }
    static __device__ __forceinline__ void add(float *p, const float (&v)[4]) {
        atomicAdd(reinterpret_cast<float4 *>(p), make_float4(v[0], v[1], v[2], v[3]));
    }
};
template <> struct CVec<8> {
    static __device__ __forceinline__ void store(float *p, const float (&v)[8]) {
        __stcs(reinterpret_cast<float4 *>(p), make_float4(v[0], v[1], v[2], v[3]));
        __stcs(reinterpret_cast<float4 *>(p + 4), make_float4(v[4], v[5], v[6], v[7]));
    }
    static __device__ __forceinline__ void add(float *p, const float (&v)[8]) {
        atomicAdd(reinterpret_cast<float4 *>(p), make_float4(v[0], v[1], v[2], v[3]));
        atomicAdd(reinterpret_cast<float4 *>(p + 4), make_float4(v[4], v[5], v[6], v[7]));
    }
};

// ---- a6 peer-memory tail exchange, run by the last CTA of the finalising kernel -------
__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(uint32_t *p, uint32_t v) {
    asm volatile("st.release.sys.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}
// bounded wait (about 20 s) so that a peer that never arrives fails loudly, not forever
__device__ __forceinline__ void wait_geq(const uint32_t *p, uint32_t v) {
    for (uint32_t it = 0; ld_acquire_sys(p) < v; ++it) {
        __nanosleep(256);
        if (it > (80u << 20)) __trap();
    }
}

// Every CTA calls this at exit; the last one to arrive does the exchange.
__device__ __forceinline__ void tail_mail_epilogue(const TailMail &m) {
    __shared__ uint32_t s_last;
    __threadfence();                                      // this CTA's tail / row updates
    __syncthreads();
    if (threadIdx.x == 0) {
        const uint32_t t = atomicAdd(m.counter, 1u);
        s_last = (t == gridDim.x - 1) ? 1u : 0u;
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();                                      // see every CTA's updates
    if (m.push_dst) {
        // the owner must have consumed this slot's previous use (epoch - 2)
        if (threadIdx.x == 0 && m.epoch > 2) wait_geq(m.push_ack, m.epoch - 2);
        __syncthreads();
        for (int c = threadIdx.x; c < m.K; c += blockDim.x)
            m.push_dst[c] = __ldcg(m.tail + c);
        __threadfence_system();
        __syncthreads();
        if (threadIdx.x == 0) st_release_sys(m.push_flag, m.epoch);
    }
    if (m.pull_mask) {
        uint32_t mask = m.pull_mask;
        while (mask) {                                    // ascending rank order
            const int g = __ffs(mask) - 1;
            mask &= mask - 1;
            if (threadIdx.x == 0) wait_geq(m.pull_flags + g, m.epoch);
            __syncthreads();
            const float *src = m.pull_src + (size_t)g * m.K;
            for (int c = threadIdx.x; c < m.K; c += blockDim.x)
                m.pull_row[c] = __ldcg(m.pull_row + c) + __ldcg(src + c);
            __syncthreads();
        }
        __threadfence_system();
        __syncthreads();
        if (threadIdx.x == 0) {
            uint32_t done = m.pull_mask;
            while (done) {
                const int g = __ffs(done) - 1;
                done &= done - 1;
                st_release_sys(m.ack_dst[g], m.epoch);
            }
        }
    }
    if (threadIdx.x == 0) *m.counter = 0u;                // ready for the next launch
}

}  // namespace mps
