#pragma once
#include <atomic>
#include <cstdlib>
// segment.cuh -- a3 (+ a4 partial rows): the merge-path segment kernel template (Alg. 2,
// PAPER.md P:100-131, sec. III-B/C P:121-147).  Instantiated per (B dtype, fix-up) in
// seg_*.cu so the build parallelises.
//
// B200 mapping (replaces the paper's thread-to-SIMD-lane mapping of sec. III-C,
// P:137-147, with the same intent: fill every lane with useful dimensions):
//  * one merge-path segment per warp (the paper's "thread");
//  * each lane gathers W consecutive elements of a B row with one vector load
//    (float4 / bf16x8 = 16 B); LR = 32/NR lanes cover a row of K <= 32*W columns, so one
//    warp instruction gathers NR different non-zeros of the segment (K=64 fp32: NR=2;
//    K=16: NR=8; K >= 128: NR=1 and V = K/(32W) slots per lane).  The NR partial sums
//    of a row are combined with a warp-shuffle butterfly only when the row ends;
//  * the segment's contiguous col/val range is staged through shared memory by 1-D TMA
//    bulk copies (cp.async.bulk + mbarrier), double-buffered in chunks of kCH non-zeros
//    per warp, one chunk ahead across the warp's segments;
//  * the nnz stream is flat: U independent gathers are issued before any is consumed,
//    regardless of where rows end; a batch wholly inside the current row takes a
//    check-free fast path (gathers + packed FFMA2);
//  * complete rows: one streaming vector store (Alg. 2 line 15); partial rows (lines 5,
//    9, 13): one vector red.global.add per W floats (atomic mode) or a record in the
//    workspace (carry mode, settled by carry_reduce_kernel).
#include "mps_internal.cuh"

namespace mps {

// non-zeros per staged col/val chunk (per warp; two chunks in flight): 512 = 8 KB per
// warp of dynamic shared memory (192 KB for 3 x 8 fp32 warps per SM).  Measured against
// 256 (profiles/r03/chunk.md): R-MAT -1.3%, Reddit -0.5%, products -0.9%, bf16 Reddit -4%,
// bf16 R-MAT -1.8%; 128 was slower everywhere
#ifndef MPS_CHUNK
#define MPS_CHUNK 512
#endif
constexpr int kCH = MPS_CHUNK;     // non-zeros per staged chunk (per warp)
constexpr int kSegMinBlocks = 3;   // 24 resident warps/SM (<= 80 registers)

struct __align__(16) WarpStage {
    int32_t col[2][kCH];
    float val[2][kCH];
};

// element e (runtime, < 4) of a 4-vector, as selects (no local-memory indexing)
__device__ __forceinline__ int pick4(const int4 &v, int e) {
    const int lo = (e & 1) ? v.y : v.x, hi = (e & 1) ? v.w : v.z;
    return (e & 2) ? hi : lo;
}
__device__ __forceinline__ float pick4f(const float4 &v, int e) {
    const float lo = (e & 1) ? v.y : v.x, hi = (e & 1) ? v.w : v.z;
    return (e & 2) ? hi : lo;
}

// registers: 80 (3 CTAs/SM) unless a lane holds > 8 words of B per gather (K > 256 fp32)
#ifndef MPS_MINB_BF16
#define MPS_MINB_BF16 2   // measured: bf16 variants spill at 80 registers (profiles/r01)
#endif
#ifndef MPS_MINB_F32
#define MPS_MINB_F32 3
#endif
#ifndef MPS_MINB_BF16_NARROW
#define MPS_MINB_BF16_NARROW MPS_MINB_BF16   // bf16 lanes of < 16 B (W <= 4)
#endif
#ifndef MPS_UL_DIV
#define MPS_UL_DIV 1
#endif
#ifndef MPS_UMAX
#define MPS_UMAX 32        // non-zeros per batch (all lane groups) at most
#endif
// Gathers per lane per batch in the static instantiation (graphs with < 4 segments per
// warp: latency-bound kernels of tens of microseconds) when NR >= 2: smaller batches
// cross fewer row ends.  Table-II graphs: fp32 K=32 +16%, K=64 +8%, bf16 K=64 +7%,
// K=128 +5%, others within 1% (profiles/r01/batch_size/).  The dynamic instantiation
// (large graphs) keeps ~4 KB of gathers in flight per warp.
#ifndef MPS_STATIC_ULCAP
#define MPS_STATIC_ULCAP 4
#endif
// column indices / values of a batch: broadcast 16-B LDS of 4 entries + per-lane selects
// when NR <= MPS_BCAST_NR, else one 4-B LDS per entry and lane.  Measured (r02o, same
// box): per-lane LDS for NR >= 2 is 1-4% faster (R-MAT -2.6%, Reddit -0.9%, Pubmed -3%);
// NR = 1 keeps the broadcast (compile-time picks, no selects).
#ifndef MPS_BCAST_NR
#define MPS_BCAST_NR 1
#endif
#ifndef MPS_DYN_ULCAP
#define MPS_DYN_ULCAP 0     // experiment: cap the dynamic instantiation's gathers per lane
#endif
#ifndef MPS_STATIC_ULCAP_MINNR
#define MPS_STATIC_ULCAP_MINNR 2
#endif
// batched zero stores for runs of empty rows: -1 = the measured rule (fp32 B, not the
// deep-gather kernel: R-MAT -2.3%, Reddit neutral; bf16 Reddit +2%, products +1.5%), 0/1
#ifndef MPS_EMPTY_RUNS
#define MPS_EMPTY_RUNS -1
#endif
#ifndef MPS_SLOW_VL_REG
#define MPS_SLOW_VL_REG 1
#endif
#ifndef MPS_SLOW_PARTS
#define MPS_SLOW_PARTS 0     // 0: the measured rule below (2 parts for >= 32-non-zero batches)
#endif
#ifndef MPS_MINB_I64
#define MPS_MINB_I64 3
#endif
// Threads per CTA of an instantiation: kBlock, or MPS_BF16_BLOCK for the 16-B bf16
// gathers with >= 2 rows per warp instruction (int32 indices): 5 CTAs of 4 warps at 96
// registers (slow-path values re-read from shared memory, slow path in two parts, no
// spills) hold 20 warps per SM instead of 16 -- R-MAT bf16 K=64 -3.4%, products bf16
// K=64 -3.0%, Reddit bf16 K=64 -0.3%; two rows per instruction (256-B bf16 rows):
// products K=128 -3.2%, Reddit K=256 -7.6%, R-MAT K=128 -7.4% (profiles/r03/prefetch.md);
// 256 restores 2 x 8 warps at 128 registers
#ifndef MPS_BF16_BLOCK
#define MPS_BF16_BLOCK 128
#endif
#ifndef MPS_BF16_SMALL_MINNR
#define MPS_BF16_SMALL_MINNR 2   // rows per warp instruction from which the small CTAs apply
#endif
#ifndef MPS_BF16_SMALL_MINB
#define MPS_BF16_SMALL_MINB 5
#endif
template <int W, int NR, typename TB, typename IT, bool DEEP = false>
__host__ __device__ constexpr int seg_block() {
    return (sizeof(TB) == 2 && sizeof(IT) == 4 && W >= 8 && NR >= MPS_BF16_SMALL_MINNR && !DEEP)
               ? MPS_BF16_BLOCK : kBlock;
}
template <int W, int V, int NR, typename TB, typename IT, bool DEEP = false>
__host__ __device__ constexpr int seg_min_blocks() {
    if constexpr (DEEP) return 2;
    if constexpr (seg_block<W, NR, TB, IT, DEEP>() != kBlock) return MPS_BF16_SMALL_MINB;
    // int64 indices (NEXT-4): fp32 B measured best at 3 CTAs/SM with a few spills
    // (profiles/r01/next4), bf16 B keeps the int32 choice
    return (V * ((W * (int)sizeof(TB) + 3) / 4) > 8) ? 2
           : (sizeof(TB) == 2 ? (W >= 8 ? MPS_MINB_BF16 : MPS_MINB_BF16_NARROW)
                              : (sizeof(IT) == 8 ? MPS_MINB_I64 : MPS_MINB_F32));
}

// Gathers per lane per batch of a segment-kernel instantiation: ~4 KB of B rows in flight
// per warp (see the MPS_* knobs above).
template <int W, int V, int NR, typename TB, bool DEEP, bool DYN>
__host__ __device__ constexpr int seg_ul() {
    constexpr int kWords = (W * (int)sizeof(TB) + 3) / 4;
    constexpr int UL00 = (V * kWords >= 8) ? 4 : ((V * kWords >= 4) ? 8 : 16);
    constexpr int UL0 = (sizeof(TB) == 2 && UL00 / MPS_UL_DIV >= 2) ? UL00 / MPS_UL_DIV
                                                                    : UL00 * (DEEP ? 2 : 1);
    constexpr int UL1 = (UL0 * NR > MPS_UMAX) ? (MPS_UMAX / NR > 0 ? MPS_UMAX / NR : 1) : UL0;
    constexpr int UL2 = (!DYN && NR >= MPS_STATIC_ULCAP_MINNR && UL1 > MPS_STATIC_ULCAP)
                            ? MPS_STATIC_ULCAP : UL1;
    return (DYN && MPS_DYN_ULCAP > 0 && NR >= 2 && UL2 > MPS_DYN_ULCAP) ? MPS_DYN_ULCAP : UL2;
}
template <int W, int V, int NR, typename TB, int FIX, typename IT, bool DEEP = false,
          bool DYN = false>
__global__ void __launch_bounds__((seg_block<W, NR, TB, IT, DEEP>()),
                                  (seg_min_blocks<W, V, NR, TB, IT, DEEP>()))
segment_kernel(const SegArgsT<IT> a) {
    using BV = BVec<TB, W>;
    using raw_t = typename BV::raw;
    static_assert(NR == 1 || V == 1, "several rows per instruction only for one slot");
    constexpr int LR = 32 / NR;                          // lanes per B row
    constexpr int kWarps = seg_block<W, NR, TB, IT, DEEP>() / 32;
    // slow-path values held in registers, or re-read from shared memory in each pass (the
    // small-CTA bf16 instantiations, to stay within their register budget without spills)
    constexpr bool kVlReg = MPS_SLOW_VL_REG && seg_block<W, NR, TB, IT, DEEP>() == kBlock &&
                            !(MPS_MINB_F32 > 3 && sizeof(TB) == 4);
    constexpr int UL = seg_ul<W, V, NR, TB, DEEP, DYN>();
    constexpr int U = UL * NR;                           // non-zeros per batch
    static_assert(kCH % U == 0, "chunk must hold whole batches");
    constexpr bool kPF = DYN && sizeof(TB) == 2;         // next-batch L2 prefetch (bf16)

    // per-warp col/val staging in dynamic shared memory (kWarps x sizeof(WarpStage), set
    // by the launcher; > 48 KB for large chunks)
    extern __shared__ __align__(16) uint8_t seg_dsmem[];
    WarpStage *stage = reinterpret_cast<WarpStage *>(seg_dsmem);
    __shared__ uint64_t bars[kWarps][2];

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const int grp = NR == 1 ? 0 : lane / LR;  // which of the NR non-zeros of an instruction
    const int lr = lane % LR;      // lane inside the row
    WarpStage &st = stage[warp];
    if (lane == 0) {
        mbar_init(&bars[warp][0], 1);
        mbar_init(&bars[warp][1], 1);
    }
    mbar_fence_init();
    __syncthreads();
    // Programmatic dependent launch: this grid may start while the previous kernel of
    // the stream (the partition / cut-row zeroing) drains; everything above is private
    // set-up, and nothing it wrote is read before this wait (a no-op without PDL).
    asm volatile("griddepcontrol.wait;" ::: "memory");

    const uint64_t pol_last = a.l2_hints ? policy_evict_last() : policy_evict_normal();
    // col/val (and tail B rows with a hot bitmap) stream: evict_first, rebuilt at each use
    // (one createpolicy) rather than held in two registers across the kernel
    auto pol_first = [&]() -> uint64_t {
        return a.l2_hints ? policy_evict_first() : policy_evict_normal();
    };
    // segment indices are 32-bit (the launcher rejects P >= 2^31 - 2^20)
    const int wid = (int)blockIdx.x * kWarps + warp;
    const int wstride = (int)gridDim.x * kWarps;
    const int nseg = (int)a.P;

    const IT *__restrict__ rp = a.rp;
    const int32_t *__restrict__ col = a.col;
    const float *__restrict__ val = a.val;
    const char *__restrict__ Bc = reinterpret_cast<const char *>(a.B);
    const uint32_t ldb_bytes = (uint32_t)(a.ldb * (int64_t)sizeof(TB));
    const int m = a.m;
    const bool direct = a.direct != 0;
    const uint32_t *__restrict__ hot = a.hot;

    int cofs[V];
    bool act[V];
    const char *bl[V];  // this lane's slot inside B row 0 (column 0 if inactive)
#pragma unroll
    for (int s = 0; s < V; ++s) {
        cofs[s] = (s * LR + lr) * W;
        act[s] = cofs[s] < a.K;
        bl[s] = Bc + (act[s] ? cofs[s] * (int)sizeof(TB) : 0);
    }
    const bool writer = grp == 0;  // after the butterfly, group 0 writes the row

    // chunk origin of a segment: nnz index whose col address is 16-B aligned (TMA) or
    // simply ys rounded down to a multiple of 4 (direct mode)
    auto seg_origin = [&](IT ys) -> IT {
        if (direct) return ys & ~(IT)3;
        return ys - (IT)(((uintptr_t)(col + ys) & 15u) >> 2);
    };
    // TMA may not read past the last 16-B boundary inside [.., nnz_end)
    // (recomputed where needed: a.nnz_end lives in the parameter bank, not a register)
    auto lim4 = [&]() -> int64_t {
        return a.nnz_end - (int64_t)(((uintptr_t)(col + a.nnz_end) & 15u) >> 2);
    };

    // ---------------- this warp's sequence of segments ---------------------------------
    // static: wid, wid + wstride, ...; dynamic (a.claim != nullptr): each warp claims its
    // next segment from a grid-wide counter when it starts the current one, so warps
    // that drew cheap segments take more (load balance across SMs and dies).  Claims
    // are issued in increasing order; cur >= P ends the warp's work.
    // (a separate instantiation: the claim code alone costs ~4% on small graphs)
    auto claim_after = [&](int last) -> int {
        if constexpr (!DYN) {
            return last + wstride;
        } else {
            unsigned v = 0;
            if (lane == 0) v = atomicAdd(a.claim, 1u);
            return (int)__shfl_sync(0xffffffffu, v, 0);
        }
    };
    int cur = DYN ? claim_after(0) : wid;
    int nxt = cur < nseg ? claim_after(cur) : nseg;

    // ---------------- producer: one chunk ahead, at most one segment ahead -------------
    int pseg = cur;
    IT psb = 0;                          // chunk origin of the producer's segment
    int pys = 0, pye = 0;                // its non-zero range, relative to psb
    int pk = 0, pnch = 0, pbuf = 0;
    auto prod_load_seg = [&]() {
        if (pseg < nseg) {
            const IT ys_ = __ldg(a.cy + pseg), ye_ = __ldg(a.cy + pseg + 1);
            psb = seg_origin(ys_);
            pys = (int)(ys_ - psb);
            pye = (int)(ye_ - psb);
            pnch = pye > pys ? (pye + kCH - 1) / kCH : 0;
        }
        pk = 0;
    };
    auto produce = [&]() {
        if constexpr (!DYN) {             // static: skip ahead over empty segments
            while (pseg < nseg && pk >= pnch) {
                pseg += wstride;
                prod_load_seg();
            }
        } else if (pk >= pnch) {          // dynamic: move on to the claimed next only
            if (pseg != cur || nxt >= nseg) return;
            pseg = nxt;
            prod_load_seg();
            if (pk >= pnch) return;       // it has no non-zeros: resume when it is cur
        }
        if (pseg >= nseg) return;
        const int cbr = pk * kCH;
        const int hir = min(pye, cbr + kCH);
        const IT cb = psb + cbr;
        const IT hi = psb + hir;
        int32_t *dc = st.col[pbuf];
        float *dv = st.val[pbuf];
        if (!direct) {
            int64_t ce = cb + (((int64_t)hi - cb + 3) & ~3ll);
            const int64_t l4 = lim4();
            if (ce > l4) ce = l4 > cb ? l4 : cb;
            const uint32_t bytes = (uint32_t)(ce - cb) * 4u;
            if (lane == 0) {
                fence_proxy_async_smem();
                mbar_arrive_expect_tx(&bars[warp][pbuf], 2u * bytes);
                if (bytes) {
                    const uint64_t pf = pol_first();
                    tma_load_1d(dc, col + cb, bytes, &bars[warp][pbuf], pf);
                    tma_load_1d(dv, val + cb, bytes, &bars[warp][pbuf], pf);
                }
            }
            const int rem = (int)(hi - (IT)ce);   // < 4 entries at the very end of the array
            if (lane < rem) {
                dc[ce - cb + lane] = col[ce + lane];
                dv[ce - cb + lane] = val[ce + lane];
            }
        } else {
            for (int t = lane; cbr + t < hir; t += 32) {
                if (cbr + t >= pys) {
                    dc[t] = __ldg(col + cb + t);
                    dv[t] = __ldg(val + cb + t);
                }
            }
        }
        ++pk;
        pbuf ^= 1;
    };
    prod_load_seg();
    produce();

    // chunks consumed so far: buffer = bit 0, mbarrier phase of that buffer = bit 1
    uint32_t ccount = 0;

    for (; cur < nseg; cur = nxt, nxt = cur < nseg ? claim_after(cur) : nseg) {
        const int seg = cur;
        // dynamic claims increase, so the producer is at seg, one segment ahead (it moved
        // past an empty seg), or behind (it stopped at an earlier empty one): restart it
        if (DYN && pseg < seg) {
            pseg = seg;
            prod_load_seg();
            produce();
        }
        const int xs = __ldg(a.cx + seg);
        const IT ys64 = __ldg(a.cy + seg);
        const int xe = __ldg(a.cx + seg + 1);
        const IT ye64 = __ldg(a.cy + seg + 1);
        const IT sb64 = seg_origin(ys64);
        const int nch = ye64 > ys64 ? (int)((ye64 - sb64 + kCH - 1) / kCH) : 0;

        // Non-zero positions inside the segment are handled as 32-bit offsets from
        // `base` (0 for int32 indices; the segment's chunk origin for int64 indices,
        // NEXT-4).  Row offsets outside the segment are clamped to [-1, ye + 1], which
        // keeps every comparison the walk makes (all against positions in [ys, ye]).
        const IT base = sizeof(IT) == 8 ? sb64 : (IT)0;
        const IT hic = ye64 - base + 1;
        auto rel = [&](IT v) -> int {
            if constexpr (sizeof(IT) == 8) {
                IT d = v - base;
                d = d < (IT)-1 ? (IT)-1 : (d > hic ? hic : d);
                return (int)d;
            } else {
                return (int)v;
            }
        };
        const int ys = rel(ys64), ye = rel(ye64), sb = rel(sb64);

        // row_ptr window: lane l holds rp[wb + l]
        int wb = xs;
        constexpr IT kInf = sizeof(IT) == 8 ? (IT)0x7fffffffffffffffll : (IT)0x7fffffff;
        int win = rel((wb + lane <= m) ? __ldg(rp + wb + lane) : kInf);
        const int rp_xs = __shfl_sync(0xffffffffu, win, 0);
        int rend = __shfl_sync(0xffffffffu, win, 1);   // rp[r + 1]
        int rbeg = rp_xs;                               // rp[r]
        const bool start_in = xs < m && ys > rp_xs;     // Alg. 2 line 2 (start_nz != 0)
        int r = xs;

        float acc[V][W];
#pragma unroll
        for (int s = 0; s < V; ++s)
#pragma unroll
            for (int w = 0; w < W; ++w) acc[s][w] = 0.f;

        // sum the NR partial accumulators of the row (warp-shuffle butterfly)
        auto combine = [&]() {
            if constexpr (NR > 1) {
#pragma unroll
                for (int off = LR; off < 32; off <<= 1)
#pragma unroll
                    for (int s = 0; s < V; ++s)
#pragma unroll
                        for (int w = 0; w < W; ++w)
                            acc[s][w] += __shfl_xor_sync(0xffffffffu, acc[s][w], off);
            }
        };
        auto write_row = [&](float *dst, bool atomic, bool relu = false) {
            if (writer) {
#pragma unroll
                for (int s = 0; s < V; ++s)
                    if (act[s]) {
                        if (atomic) {
                            CVec<W>::add(dst + cofs[s], acc[s]);
                        } else if (relu) {   // fused epilogue of a complete row
                            float t[W];
#pragma unroll
                            for (int w = 0; w < W; ++w) t[w] = fmaxf(acc[s][w], 0.f);
                            CVec<W>::store(dst + cofs[s], t);
                        } else {
                            CVec<W>::store(dst + cofs[s], acc[s]);
                        }
                    }
            }
        };

        // Row r ends inside this segment: settle it and move to row r + 1.
        auto finish_row = [&]() {
            // an empty row has nothing in any lane group: no butterfly (R-MAT: 48% empty)
            if (rend != rbeg) combine();
            if (r == xs && start_in) {
                // partial start row (Alg. 2 lines 8-9): atomic, or carry record slot 0
                if (FIX == FIX_ATOMIC) {
                    if (ys < rend) {
                        write_row((r == a.tail_row) ? a.tail
                                                    : a.C + ((int64_t)r - a.row_base) * a.ldc,
                                  true);
                        count_write_if<!DYN>(a.wstat, lane, 0);
                    } else {
                        count_write_if<!DYN>(a.wstat, lane, 1);   // empty piece: the add is elided
                    }
                } else {
                    write_row(a.rec + ((int64_t)seg * 2) * a.kpad, false);
                    count_write_if<!DYN>(a.wstat, lane, 0);
                }
            } else {
                // complete row (line 15): plain store, no initialisation of C needed
                write_row(a.C + ((int64_t)r - a.row_base) * a.ldc, false, a.relu != 0);
                count_write_if<!DYN>(a.wstat, lane, 2);
            }
#pragma unroll
            for (int s = 0; s < V; ++s)
#pragma unroll
                for (int w = 0; w < W; ++w) acc[s][w] = 0.f;
            ++r;
            int idx = r + 1 - wb;
            if (idx >= 32) {
                wb = r;
                win = rel((wb + lane <= m) ? __ldg(rp + wb + lane) : kInf);
                idx = 1;
            }
            rbeg = rend;
            rend = __shfl_sync(0xffffffffu, win, idx);
        };

        auto fma_row = [&](float v, const raw_t (&b)[V]) {
#pragma unroll
            for (int s = 0; s < V; ++s) {
                float f[W];
                BV::cvt(b[s], f);
                if constexpr (W == 1) {
                    acc[s][0] = fmaf(v, f[0], acc[s][0]);
                } else {
#pragma unroll
                    for (int w = 0; w < W; w += 2) fma2(acc[s][w], acc[s][w + 1], v, f[w], f[w + 1]);
                }
            }
        };

        constexpr bool kEmptyRuns = MPS_EMPTY_RUNS >= 0 ? (MPS_EMPTY_RUNS != 0)
                                                        : (sizeof(TB) == 4 && !DEEP);
        // A run of empty rows starting at r (rp[r+1] == rbeg ...) is settled with one
        // zero store per NR rows -- no butterfly, no per-row walk (nothing accumulated;
        // R-MAT: 48% of its rows are empty).  Rows stay below xe (their end items lie in
        // this segment); the window lanes give the run length by one ballot.
        auto zero_empty_run = [&]() {
            if constexpr (!kEmptyRuns) return;
            while (r < xe && rend == rbeg) {
                int idx = r + 1 - wb;
                const unsigned eq = __ballot_sync(0xffffffffu, win == rbeg);
                const unsigned run = ~(eq >> idx);
                int k = run ? __ffs(run) - 1 : 32 - idx;
                k = k < xe - r ? k : xe - r;
                {   // every lane group stores its own rows of the run
                    for (int t = grp; t < k; t += NR) {
                        float *dst = a.C + ((int64_t)(r + t) - a.row_base) * a.ldc;
#pragma unroll
                        for (int s = 0; s < V; ++s)
                            if (act[s]) {
                                float z[W];
#pragma unroll
                                for (int w = 0; w < W; ++w) z[w] = 0.f;
                                CVec<W>::store(dst + cofs[s], z);
                            }
                    }
                }
                count_write_n_if<!DYN>(a.wstat, lane, 2, k);
                r += k;
                idx = r + 1 - wb;
                if (idx >= 32) {
                    wb = r;
                    win = rel((wb + lane <= m) ? __ldg(rp + wb + lane) : kInf);
                    idx = 1;
                }
                rend = __shfl_sync(0xffffffffu, win, idx);      // rbeg is unchanged
            }
        };

        for (int k = 0; k < nch; ++k) {
            if (!direct) {
                mbar_wait(&bars[warp][ccount & 1u], (ccount >> 1) & 1u);
            }
            __syncwarp();
            produce();                  // next chunk into the other buffer
            if (direct) __syncwarp();
            const int cb = sb + k * kCH;
            const int32_t *sc = st.col[ccount & 1u];
            const float *sv = st.val[ccount & 1u];
            int q = ys - cb;
            q = q > 0 ? (q / U) * U : 0;
            const int qend = min(kCH, ye - cb);
            // issue(q, bv): the gathers of the batch at chunk offset q into bv;
            // consume(q, bv): its FMAs and the rows it ends
            auto issue = [&](const int q, raw_t (&bv)[UL][V]) {
                const int j0 = cb + q;
                const bool full = j0 >= ys && j0 + U <= ye;
                // my non-zeros of this batch: u = i*NR + grp (i < UL).  Column indices
                // and values are read as broadcast 16-B LDS of 4 consecutive entries
                // (NR <= MPS_BCAST_NR) and each lane selects its own, else per lane;
                // branch-free: outside the segment the column index is clamped to 0 (a
                // harmless in-bounds row).
                uint32_t cid[UL];
                if constexpr (NR <= MPS_BCAST_NR) {
#pragma unroll
                    for (int t = 0; t < U / 4; ++t) {
                        const int4 c4 = *reinterpret_cast<const int4 *>(sc + q + 4 * t);
#pragma unroll
                        for (int k = 0; k < 4 / NR; ++k)
                            cid[t * (4 / NR) + k] =
                                (uint32_t)(NR == 1 ? pick4(c4, k) : pick4(c4, k * NR + grp));
                    }
                } else {
#pragma unroll
                    for (int i = 0; i < UL; ++i) cid[i] = (uint32_t)sc[q + i * NR + grp];
                }
                if (!full) {
#pragma unroll
                    for (int i = 0; i < UL; ++i) {
                        const int j = j0 + i * NR + grp;
                        cid[i] = (j >= ys && j < ye) ? cid[i] : 0u;
                    }
                }
                // (the hot-row bitmap exists in the static instantiation only: the launcher
                // runs that one when a bitmap is passed)
                if (DYN || hot == nullptr) {
#pragma unroll
                    for (int i = 0; i < UL; ++i)
#pragma unroll
                        for (int s = 0; s < V; ++s)
                            bv[i][s] = BV::load(reinterpret_cast<const TB *>(
                                                    row_addr(bl[s], cid[i], ldb_bytes)), pol_last);
                } else {
                    // degree-aware L2 residency: hub rows evict_last, the tail streams
                    uint32_t hw[UL];
#pragma unroll
                    for (int i = 0; i < UL; ++i) hw[i] = __ldg(hot + (cid[i] >> 5));
                    const uint64_t pf = pol_first();
#pragma unroll
                    for (int i = 0; i < UL; ++i) {
                        const uint64_t pol = ((hw[i] >> (cid[i] & 31u)) & 1u) ? pol_last : pf;
#pragma unroll
                        for (int s = 0; s < V; ++s)
                            bv[i][s] = BV::load(reinterpret_cast<const TB *>(
                                                    row_addr(bl[s], cid[i], ldb_bytes)), pol);
                    }
                }
                // bf16 B slices larger than L2: the B rows of the NEXT batch of this chunk
                // go into L2 now (one LSU prefetch per lane, no registers held), so that
                // batch's gathers wait for L2 hits instead of DRAM misses.  The bf16
                // kernels hold only 16 warps per SM (128 registers): products bf16 -10%,
                // R-MAT bf16 -3%; fp32 (24 warps) measured slower with it and does not
                // carry the code (profiles/r03/prefetch.md)
                if constexpr (kPF) {
                    if (a.pf != 0) {
                        const int qn = q + U;
                        const int lines = 1 << a.pf_shift;
                        for (int idx = lane; idx < U * lines; idx += 32) {
                            const int t = idx >> a.pf_shift;
                            if (qn + t < qend)
                                prefetch_l2_line(row_addr(Bc, (uint32_t)sc[qn + t], ldb_bytes) +
                                                 (idx & (lines - 1)) * 128);
                        }
                    }
                }
            };
            auto consume = [&](const int q, const raw_t (&bv)[UL][V]) {
                const int j0 = cb + q;
                const bool full = j0 >= ys && j0 + U <= ye;
                if (full && j0 + U <= rend) {
                    // fast path: U non-zeros of the current row, no checks
                    if constexpr (NR <= MPS_BCAST_NR) {
#pragma unroll
                        for (int t = 0; t < U / 4; ++t) {
                            const float4 v4 = *reinterpret_cast<const float4 *>(sv + q + 4 * t);
#pragma unroll
                            for (int k = 0; k < 4 / NR; ++k)
                                fma_row(NR == 1 ? pick4f(v4, k) : pick4f(v4, k * NR + grp),
                                        bv[t * (4 / NR) + k]);
                        }
                    } else {
#pragma unroll
                        for (int i = 0; i < UL; ++i) fma_row(sv[q + i * NR + grp], bv[i]);
                    }
                } else {
                    // slow path: the batch crosses row ends (or the segment's edges).
                    // One pass per row intersecting the batch: predicated FMAs for the
                    // non-zeros of the current row, then settle the row.
                    // values in registers for the passes (MPS_SLOW_VL_REG=1), or re-read
                    // from shared memory inside each pass (0: fewer live registers)
                    float vl[UL];
                    if constexpr (kVlReg) {
#pragma unroll
                        for (int i = 0; i < UL; ++i) vl[i] = sv[q + i * NR + grp];
                    }
                    // The batch is settled in SP parts of UL/SP entries each; a part's
                    // passes predicate only its own entries, so a row end costs UL/SP
                    // FMA groups instead of UL (MPS_SLOW_PARTS, measured in
                    // profiles/r02/slow_steps.md)
                    // (default: two parts for batches of >= 32 non-zeros -- bf16 K=64 /
                    // fp32 K=32 -- where they measured 4-6% faster; one part otherwise)
                    // (and two parts in the small-CTA bf16 kernels: fewer live registers)
                    constexpr int SP0 = MPS_SLOW_PARTS > 0 ? MPS_SLOW_PARTS
                                        : ((U >= 32 || !kVlReg) ? 2 : 1);
                    constexpr int SP = (UL % SP0 == 0) ? SP0 : 1;
                    constexpr int ULP = UL / SP;
                    int jc = j0 > ys ? j0 : ys;                  // next non-zero to consume
#pragma unroll
                    for (int h = 0; h < SP; ++h) {
                        const int pe = j0 + (h + 1) * ULP * NR;
                        const int jend = pe < ye ? pe : ye;
                        while (jc < jend) {
                            while (jc >= rend) {                  // rows ending before jc
                                finish_row();
                                zero_empty_run();
                            }
                            const int lim = rend < jend ? rend : jend;  // row r's part
#pragma unroll
                            for (int i = h * ULP; i < (h + 1) * ULP; ++i) {
                                const int j = j0 + i * NR + grp;
                                if (j >= jc && j < lim)
                                    fma_row(kVlReg ? vl[i] : sv[q + i * NR + grp], bv[i]);
                            }
                            jc = lim;
                        }
                    }
                }
            };
            for (; q < qend; q += U) {
                raw_t bv[UL][V];
                issue(q, bv);
                consume(q, bv);
            }
            ++ccount;
        }
        // rows whose end item lies in this segment after its last non-zero
        while (r < xe) {
            finish_row();
            zero_empty_run();
        }

        // r == xe: the segment's non-zeros of row xe, if any (lines 3-5 / 11-13)
        if (xe < m && ye > rbeg) {
            combine();
            const bool single = (xs == xe) && start_in;
            if (FIX == FIX_ATOMIC)
                write_row((xe == a.tail_row) ? a.tail : a.C + ((int64_t)xe - a.row_base) * a.ldc,
                          true);
            else
                write_row(a.rec + ((int64_t)seg * 2 + (single ? 0 : 1)) * a.kpad, false);
            count_write_if<!DYN>(a.wstat, lane, 0);
        }
    }
    if (a.mail.on) tail_mail_epilogue(a.mail);   // a6 tail exchange (last CTA, last tile)
}

// MPS_DYN (read per call): 0 = static segment assignment (warp w: w, w + warps, ...)
static bool dynamic_claims() {
    const char *e = getenv("MPS_DYN");
    return e ? atoi(e) != 0 : true;
}

// Occupancy of one instantiation, per device (the carveout / dynamic shared memory are
// per-device function attributes).  `cache` is the calling instantiation's own (a
// static of launch_seg<...>): the kernels share one function-pointer type, so a cache
// keyed on the type alone would hand one kernel's occupancy to all.  Idempotent, so
// concurrent first calls from several host threads only repeat the same query.
template <typename KFn>
static cudaError_t seg_blocks_per_sm(std::atomic<int> (&cache)[64], KFn kstatic, KFn kdyn,
                                     int block, size_t dsmem, int *out) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev >= 0 && dev < 64) {
        const int c = cache[dev].load(std::memory_order_relaxed);
        if (c > 0) { *out = c; return cudaSuccess; }
    }
    // the staging buffers need the large shared-memory carveout for
    // seg_min_blocks() CTAs per SM; MPS_CARVEOUT: carveout hint in percent (-1: none)
    static const int carve = [] {
        const char *ev = getenv("MPS_CARVEOUT");
        return ev ? atoi(ev) : -1;
    }();
    if (carve >= 0) {
        e = cudaFuncSetAttribute(kstatic, cudaFuncAttributePreferredSharedMemoryCarveout, carve);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(kdyn, cudaFuncAttributePreferredSharedMemoryCarveout, carve);
        if (e != cudaSuccess) return e;
    }
    if (dsmem > 0) {   // (the 48-KB default limit counts the static barriers too)
        e = cudaFuncSetAttribute(kstatic, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsmem);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(kdyn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsmem);
        if (e != cudaSuccess) return e;
    }
    int bps = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, kstatic, block, dsmem);
    if (e != cudaSuccess) return e;
    if (bps < 1) bps = 1;
    if (dev >= 0 && dev < 64) cache[dev].store(bps, std::memory_order_relaxed);
    *out = bps;
    return cudaSuccess;
}

template <int W, int V, int NR, typename TB, int FIX, typename IT, bool DEEP = false>
static cudaError_t launch_seg(const SegArgsT<IT> &a, cudaStream_t s) {
    auto kst = segment_kernel<W, V, NR, TB, FIX, IT, DEEP, false>;
    auto kdy = segment_kernel<W, V, NR, TB, FIX, IT, DEEP, true>;
    static std::atomic<int> occ_cache[64];      // per instantiation, per device
    int blocks_per_sm = 0;
    constexpr int block = seg_block<W, NR, TB, IT, DEEP>();
    constexpr size_t dsmem = (size_t)(block / 32) * sizeof(WarpStage);
    cudaError_t e = seg_blocks_per_sm(occ_cache, kst, kdy, block, dsmem, &blocks_per_sm);
    if (e != cudaSuccess) return e;
    const int64_t warps_per_block = block / 32;
    int64_t need = (a.P + warps_per_block - 1) / warps_per_block;
    const int64_t cap = (int64_t)blocks_per_sm * num_sms();
    const int64_t grid = need < cap ? need : cap;
    if (grid <= 0) return cudaSuccess;
    if (a.P >= (int64_t)0x7ff00000) return cudaErrorInvalidValue;   // 32-bit segment ids
    // dynamic claims pay off from ~4 segments per warp (BASELINE graphs: 10-70 per warp,
    // 1-6% faster); at 1-3 per warp the opening burst of claims on one counter costs more
    // than the balance gains (Table-II graphs, profiles/r01/dynamic_claims/).  The counter
    // (a.claim) lives in the caller's workspace and is zero when the kernel starts.
    // (the Fig. 5 write counters exist in the static instantiation only: a counting
    // launch runs it, and the dynamic kernel of the large graphs carries no counting code)
    const bool dyn = a.claim != nullptr && a.wstat == nullptr && a.hot == nullptr &&
                     a.P >= 4 * grid * warps_per_block && dynamic_claims();
    // launched with programmatic stream serialization (PDL): the CTAs may be scheduled
    // as the previous kernel's CTAs retire, hiding the launch gap (tens of percent of a
    // small graph's step); griddepcontrol.wait in the kernel keeps the data dependency.
    // MPS_PDL=0 launches plainly.
    static const int pdl = [] {
        const char *ev = getenv("MPS_PDL");
        return ev ? atoi(ev) : 1;
    }();
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(block);
    cfg.dynamicSmemBytes = dsmem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = pdl ? 1 : 0;
    if (dyn) return cudaLaunchKernelEx(&cfg, kdy, a);
    return cudaLaunchKernelEx(&cfg, kst, a);
}

// (W, V, NR) dispatch.  NR > 1 only with V == 1.
template <typename TB, int FIX, int W, typename IT>
static cudaError_t dispatch_v(const SegArgsT<IT> &a, int V, int NR, cudaStream_t s) {
    if (V == 1) {
        switch (NR) {
        case 1: return launch_seg<W, 1, 1, TB, FIX, IT>(a, s);
        case 2:
            if constexpr (W == 4 && sizeof(TB) == 4)
                if (a.deep) return launch_seg<W, 1, 2, TB, FIX, IT, true>(a, s);
            return launch_seg<W, 1, 2, TB, FIX, IT>(a, s);
        case 4: return launch_seg<W, 1, 4, TB, FIX, IT>(a, s);
        case 8: return launch_seg<W, 1, 8, TB, FIX, IT>(a, s);
        case 16: return launch_seg<W, 1, 16, TB, FIX, IT>(a, s);
        case 32: return launch_seg<W, 1, 32, TB, FIX, IT>(a, s);
        default: return cudaErrorInvalidValue;
        }
    }
    if (NR != 1) return cudaErrorInvalidValue;
    switch (V) {
    case 2: return launch_seg<W, 2, 1, TB, FIX, IT>(a, s);
    case 3: return launch_seg<W, 3, 1, TB, FIX, IT>(a, s);
    case 4: return launch_seg<W, 4, 1, TB, FIX, IT>(a, s);
    default: return cudaErrorInvalidValue;
    }
}

template <typename TB, int FIX, typename IT>
static cudaError_t dispatch_w(const SegArgsT<IT> &a, int W, int V, int NR, cudaStream_t s) {
    switch (W) {
    case 1: return dispatch_v<TB, FIX, 1, IT>(a, V, NR, s);
    case 2: return dispatch_v<TB, FIX, 2, IT>(a, V, NR, s);
    case 4: return dispatch_v<TB, FIX, 4, IT>(a, V, NR, s);
    case 8:
        if constexpr (sizeof(TB) == 2) return dispatch_v<TB, FIX, 8, IT>(a, V, NR, s);
        return cudaErrorInvalidValue;
    default: return cudaErrorInvalidValue;
    }
}

}  // namespace mps
