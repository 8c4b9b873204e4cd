// small.cu -- the online step for small graphs in ONE kernel launch (+ the a4 carry
// reduction, launched behind it with programmatic dependent launch).
//
// For graphs whose row_ptr fits in shared memory (Cora, Pubmed and the small Table-II
// graphs) the online step is a chain of dependent memory round
// trips, not a bandwidth problem: the two-kernel path (partition kernel: 32-ary search
// over a cold row_ptr + window load; segment kernel: coordinates, col/val staging, B
// gathers) pays ~8 of them plus a second launch.  Here every CTA stages the WHOLE
// row_ptr in shared memory with one round of independent 16-B loads, and each warp then
//   a2: finds the coordinates (x, y) of its segment's two diagonals (Alg. 1 lines 6-7,
//       x = max{x : x + RP[x] <= d}, reading R4/R5) by a 32-ary warp search in
//       shared memory and publishes (x_p, y_p);
//   a3: loads its <= L col/val entries, gathers the B rows (16-B vector loads, NR
//       non-zeros per warp instruction) and walks Alg. 2: complete rows are
//       stored (line 15);
//   a4: the partial first / last rows (lines 5, 9, 13) go to the carry records -- the
//       same [P][2][kpad] layout the segment kernel writes in carry mode -- and the
//       existing carry_reduce_kernel sums each cut row's pieces in segment order
//       (deterministic) and stores it.
// Dependent round trips: row_ptr, col/val, B rows (+ the reduction's record reads).
#include <atomic>

#include "mps_internal.cuh"

namespace mps {

// x = max{x in [max(0, d - nnz), min(d, m)] : x + rp[x] <= d} on the staged row_ptr,
// by one warp: each round the lanes probe 32 points of the candidate range, and the
// ballot of the (monotone) predicate shrinks it ~32x.
__device__ __forceinline__ int diag_x_smem(const int32_t *s_rp, int m, int nnz, int d,
                                           int lane) {
    int a = d > nnz ? d - nnz : 0;
    int b = d < m ? d : m;
    while (b > a) {
        const int len = b - a;
        const int q = a + (int)(((int64_t)len * (lane + 1) + 31) / 32);   // in (a, b]
        const bool ok = q + s_rp[q] <= d;
        const unsigned mask = __ballot_sync(0xffffffffu, ok);
        const int k = __popc(mask);
        const int qa = __shfl_sync(0xffffffffu, q, k > 0 ? k - 1 : 0);
        const int qb = __shfl_sync(0xffffffffu, q, k < 32 ? k : 31);
        if (k > 0) a = qa;
        if (k < 32) b = qb - 1;
    }
    return a;
}

template <typename TB, int W, int NR>
__global__ void __launch_bounds__(kBlock) small_online_kernel(const SmallArgs a) {
    using BV = BVec<TB, W>;
    using raw_t = typename BV::raw;
    constexpr int LR = 32 / NR;                 // lanes per B row
    constexpr int UL = NR >= 8 ? 2 : 4;         // gathers per lane per batch
    constexpr int U = UL * NR;                  // non-zeros per batch
    constexpr int kWarps = kBlock / 32;
    extern __shared__ __align__(16) int32_t smem[];
    const int m = a.m, nnz = a.nnz, L = a.L;
    const int rp_words = (m + 1 + 3) & ~3;
    int32_t *s_rp = smem;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    int32_t *s_col = smem + rp_words + warp * 2 * L;
    float *s_val = reinterpret_cast<float *>(s_col + L);

    // the inputs may come from the previous kernel of the stream (PDL: launched early)
    asm volatile("griddepcontrol.wait;" ::: "memory");

    // stage row_ptr[0..m]: asynchronous 16-B copies, all in flight at once (one memory
    // round trip; a load-then-store loop would serialise one round trip per iteration)
    {
        const int n4 = (m + 1) >> 2;
        const int4 *src = reinterpret_cast<const int4 *>(a.rp);
        int4 *dst = reinterpret_cast<int4 *>(s_rp);
        for (int i = threadIdx.x; i < n4; i += blockDim.x) cp_async16(dst + i, src + i);
        for (int i = 4 * n4 + threadIdx.x; i <= m; i += blockDim.x) cp_async4(s_rp + i, a.rp + i);
        cp_async_wait_all();
    }
    __syncthreads();
    const int p = (int)blockIdx.x * kWarps + warp;
    if (p >= a.P) return;

    // a2: this segment's diagonals d_p, d_{p+1} (Alg. 1 lines 4-7, reading R2)
    const int M = m + nnz;
    const int d0 = (int)min((int64_t)p * L, (int64_t)M);
    const int d1 = (int)min((int64_t)(p + 1) * L, (int64_t)M);
    const int xs = diag_x_smem(s_rp, m, nnz, d0, lane);
    const int xe = diag_x_smem(s_rp, m, nnz, d1, lane);
    const int ys = d0 - xs, ye = d1 - xe;
    if (lane == 0) {
        a.cx[p] = xs;
        a.cy[p] = ys;
        if (p == a.P - 1) {
            a.cx[p + 1] = xe;
            a.cy[p + 1] = ye;
        }
    }

    // col/val of the segment's non-zeros [ys, ye) (<= L entries)
    const int nn = ye - ys;
    for (int t = lane; t < nn; t += 32) {
        cp_async4(s_col + t, a.col + ys + t);
        cp_async4(s_val + t, a.val + ys + t);
    }
    cp_async_wait_all();
    __syncwarp();

    // a3: the Alg. 2 walk; NR lane groups each gather one non-zero per instruction
    const int grp = lane / LR, lr = lane % LR;
    const int cofs = lr * W;
    const bool act = cofs < a.K;
    const bool writer = grp == 0 && act;
    const char *bl = reinterpret_cast<const char *>(a.B) + (act ? cofs * (int)sizeof(TB) : 0);
    const uint32_t ldb_bytes = (uint32_t)(a.ldb * (int64_t)sizeof(TB));
    const uint64_t pol = a.l2_hints ? policy_evict_last() : policy_evict_normal();
    constexpr int kInf = 0x7fffffff;
    int r = xs;
    int rbeg = s_rp[xs];
    int rend = xs < m ? s_rp[xs + 1] : kInf;
    const bool start_in = xs < m && ys > rbeg;      // Alg. 2 line 2 (start_nz != 0)
    float acc[W];
#pragma unroll
    for (int w = 0; w < W; ++w) acc[w] = 0.f;

    auto combine = [&]() {
#pragma unroll
        for (int off = LR; off < 32; off <<= 1)
#pragma unroll
            for (int w = 0; w < W; ++w) acc[w] += __shfl_xor_sync(0xffffffffu, acc[w], off);
    };
    auto write_row = [&](float *dst, bool relu) {
        if (!writer) return;
        float t[W];
#pragma unroll
        for (int w = 0; w < W; ++w) t[w] = relu ? fmaxf(acc[w], 0.f) : acc[w];
        CVec<W>::store(dst + cofs, t);
    };
    auto record = [&](int slot) {
        write_row(a.rec + ((int64_t)p * 2 + slot) * a.kpad, false);
    };
    // row r ends inside this segment: a complete row (store), or the partial start row
    // (carry record slot 0); then move to row r + 1
    auto finish_row = [&]() {
        combine();
        if (r == xs && start_in) record(0);
        else write_row(a.C + (int64_t)r * a.ldc, a.relu != 0);
#pragma unroll
        for (int w = 0; w < W; ++w) acc[w] = 0.f;
        ++r;
        rbeg = rend;
        rend = r < m ? s_rp[r + 1] : kInf;
    };
    auto fma_row = [&](float v, const raw_t &b) {
        float f[W];
        BV::cvt(b, f);
        if constexpr (W == 1) {
            acc[0] = fmaf(v, f[0], acc[0]);
        } else {
#pragma unroll
            for (int w = 0; w < W; w += 2) fma2(acc[w], acc[w + 1], v, f[w], f[w + 1]);
        }
    };

    for (int q = 0; q < nn; q += U) {
        raw_t bv[UL];
        float vl[UL];
#pragma unroll
        for (int i = 0; i < UL; ++i) {
            const int j = q + i * NR + grp;
            const bool in = j < nn;
            const uint32_t c = in ? (uint32_t)s_col[j] : 0u;
            vl[i] = in ? s_val[j] : 0.f;
            bv[i] = BV::load(reinterpret_cast<const TB *>(row_addr(bl, c, ldb_bytes)), pol);
        }
        // one pass per row touching the batch: predicated FMAs, then settle the row
        int jc = q;
        const int jend = min(q + U, nn);
        while (jc < jend) {
            while (ys + jc >= rend) finish_row();
            const int lim = min(rend - ys, jend);
#pragma unroll
            for (int i = 0; i < UL; ++i) {
                const int j = q + i * NR + grp;
                if (j >= jc && j < lim) fma_row(vl[i], bv[i]);
            }
            jc = lim;
        }
    }
    while (r < xe) finish_row();                 // rows ending after the last non-zero
    if (xe < m && ye > rbeg) {                   // the segment's piece of row xe
        combine();
        record((xs == xe && start_in) ? 0 : 1);  // single-row segment: slot 0
    }
}

template <typename TB, int W, int NR>
static cudaError_t launch_small_t(const SmallArgs &a, size_t smem, cudaStream_t s) {
    auto k = small_online_kernel<TB, W, NR>;
    static std::atomic<size_t> attr_set[64];
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev < 0 || dev >= 64 || attr_set[dev].load(std::memory_order_relaxed) < smem) {
        e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        if (dev >= 0 && dev < 64) attr_set[dev].store(smem, std::memory_order_relaxed);
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)((a.P + kBlock / 32 - 1) / (kBlock / 32)));
    cfg.blockDim = dim3(kBlock);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k, a);
}

template <typename TB, int W>
static cudaError_t launch_small_nr(const SmallArgs &a, int NR, size_t smem, cudaStream_t s) {
    switch (NR) {
    case 1: return launch_small_t<TB, W, 1>(a, smem, s);
    case 2: return launch_small_t<TB, W, 2>(a, smem, s);
    case 4: return launch_small_t<TB, W, 4>(a, smem, s);
    case 8: return launch_small_t<TB, W, 8>(a, smem, s);
    case 16: return launch_small_t<TB, W, 16>(a, smem, s);
    case 32: return launch_small_t<TB, W, 32>(a, smem, s);
    default: return cudaErrorInvalidValue;
    }
}

size_t small_smem_bytes(int64_t m, int64_t L) {
    return (size_t)(((m + 1 + 3) & ~3ll) * 4) + (size_t)(kBlock / 32) * 2 * (size_t)L * 4;
}

cudaError_t launch_small_online(const SmallArgs &a, int b_dtype, int W, int NR, cudaStream_t s) {
    const size_t smem = small_smem_bytes(a.m, a.L);
    if (smem > (size_t)kSmallMaxSmem || (((uintptr_t)a.rp) & 15u)) return cudaErrorInvalidValue;
    if (a.P <= 0) return cudaSuccess;
    if (b_dtype == MPS_DT_F32) {
        switch (W) {
        case 1: return launch_small_nr<float, 1>(a, NR, smem, s);
        case 2: return launch_small_nr<float, 2>(a, NR, smem, s);
        case 4: return launch_small_nr<float, 4>(a, NR, smem, s);
        default: return cudaErrorInvalidValue;
        }
    }
    switch (W) {
    case 1: return launch_small_nr<__nv_bfloat16, 1>(a, NR, smem, s);
    case 2: return launch_small_nr<__nv_bfloat16, 2>(a, NR, smem, s);
    case 4: return launch_small_nr<__nv_bfloat16, 4>(a, NR, smem, s);
    case 8: return launch_small_nr<__nv_bfloat16, 8>(a, NR, smem, s);
    default: return cudaErrorInvalidValue;
    }
}

}  // namespace mps
