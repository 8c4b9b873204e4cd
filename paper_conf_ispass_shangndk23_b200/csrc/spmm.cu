// spmm.cu -- a3 + a4: the merge-path segment kernel (Alg. 2, PAPER.md P:100-131,
// sec. III-B/C P:121-147), the carry-out reduction and the shard tail application.
//
// B200 mapping (replaces the paper's one-thread-per-SIMD-lane mapping):
//  * one merge-path segment per warp (the paper's "thread"); lanes spread across the K
//    feature columns: lane l covers columns (s*32 + l)*W .. +W-1 for slot s < V, i.e.
//    one B row is read as 32 coalesced W-wide vector loads (float2/float4/bf16x8);
//  * the segment's contiguous col/val range is staged through shared memory by 1-D TMA
//    bulk copies (cp.async.bulk + mbarrier), double-buffered in chunks of kCH non-zeros
//    per warp, and read back with broadcast 16-B LDS;
//  * the nnz stream is flat: U independent B-row gathers are issued before any is
//    consumed, regardless of where rows end; a batch wholly inside the current row takes
//    a check-free fast path (U gathers + U packed FFMA2 groups);
//  * complete rows: one streaming vector store (Alg. 2 line 15); partial rows
//    (lines 5, 9, 13): one vector red.global.add per W floats (atomic mode) or a record
//    in the workspace (carry mode, settled by carry_reduce_kernel).
#include "mps_internal.cuh"

namespace mps {

constexpr int kCH = 256;    // non-zeros per staged chunk (per warp)
constexpr int kSlack = 4;   // room for the 16-B alignment shift of a chunk

struct __align__(16) WarpStage {
    int32_t col[2][kCH + kSlack];
    float val[2][kCH + kSlack];
};

template <int W, int V, typename TB, int FIX>
__global__ void __launch_bounds__(kBlock)
segment_kernel(const SegArgs a) {
    using BV = BVec<TB, W>;
    using raw_t = typename BV::raw;
    constexpr int kWarps = kBlock / 32;
    constexpr int kWords = (W * (int)sizeof(TB) + 3) / 4;
    constexpr int U = (V * kWords >= 8) ? 4 : 8;   // gathers in flight per lane per batch

    __shared__ WarpStage stage[kWarps];
    __shared__ uint64_t bars[kWarps][2];

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    WarpStage &st = stage[warp];
    if (lane == 0) {
        mbar_init(&bars[warp][0], 1);
        mbar_init(&bars[warp][1], 1);
    }
    mbar_fence_init();
    __syncthreads();

    const uint64_t pol_last = policy_evict_last();
    const uint64_t pol_first = policy_evict_first();
    const int64_t wid = (int64_t)blockIdx.x * kWarps + warp;
    const int64_t wstride = (int64_t)gridDim.x * kWarps;

    const int32_t *__restrict__ rp = a.rp;
    const int32_t *__restrict__ col = a.col;
    const float *__restrict__ val = a.val;
    const char *__restrict__ Bc = reinterpret_cast<const char *>(a.B);
    const uint32_t ldb_bytes = (uint32_t)(a.ldb * (int64_t)sizeof(TB));
    const int m = a.m;
    const bool direct = a.direct != 0;

    int cofs[V];
    bool act[V];
    const char *bl[V];  // this lane's slot inside B row 0 (column 0 if inactive)
#pragma unroll
    for (int s = 0; s < V; ++s) {
        cofs[s] = (s * 32 + lane) * W;
        act[s] = cofs[s] < a.K;
        bl[s] = Bc + (act[s] ? cofs[s] * (int)sizeof(TB) : 0);
    }

    // chunk origin of a segment: nnz index whose col address is 16-B aligned (TMA) or
    // simply ys rounded down to a multiple of 4 (direct mode)
    auto seg_origin = [&](int ys) -> int {
        if (direct) return ys & ~3;
        return ys - (int)(((uintptr_t)(col + ys) & 15u) >> 2);
    };
    // TMA may not read past the last 16-B boundary inside [.., nnz_end)
    const int64_t lim4 = a.nnz_end - (int64_t)(((uintptr_t)(col + a.nnz_end) & 15u) >> 2);

    // ---------------- producer: one chunk ahead, across this warp's segments ----------
    int64_t pseg = wid;
    int pys = 0, pye = 0, psb = 0, pk = 0, pnch = 0, pbuf = 0;
    auto prod_load_seg = [&]() {
        if (pseg < a.P) {
            pys = __ldg(a.cy + pseg);
            pye = __ldg(a.cy + pseg + 1);
            psb = seg_origin(pys);
            pnch = pye > pys ? (pye - psb + kCH - 1) / kCH : 0;
        }
        pk = 0;
    };
    auto produce = [&]() {
        while (pseg < a.P && pk >= pnch) {
            pseg += wstride;
            prod_load_seg();
        }
        if (pseg >= a.P) return;
        const int cb = psb + pk * kCH;
        const int hi = min(pye, cb + kCH);
        int32_t *dc = st.col[pbuf];
        float *dv = st.val[pbuf];
        if (!direct) {
            int64_t ce = cb + (((int64_t)hi - cb + 3) & ~3ll);
            if (ce > lim4) ce = lim4 > cb ? lim4 : cb;
            const uint32_t bytes = (uint32_t)(ce - cb) * 4u;
            if (lane == 0) {
                fence_proxy_async_smem();
                mbar_arrive_expect_tx(&bars[warp][pbuf], 2u * bytes);
                if (bytes) {
                    tma_load_1d(dc, col + cb, bytes, &bars[warp][pbuf], pol_first);
                    tma_load_1d(dv, val + cb, bytes, &bars[warp][pbuf], pol_first);
                }
            }
            const int rem = hi - (int)ce;   // < 4 entries at the very end of the array
            if (lane < rem) {
                dc[ce - cb + lane] = col[ce + lane];
                dv[ce - cb + lane] = val[ce + lane];
            }
        } else {
            for (int t = lane; cb + t < hi; t += 32) {
                if (cb + t >= pys) {
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

    uint32_t phase0 = 0, phase1 = 0;
    int cbuf = 0;

    for (int64_t seg = wid; seg < a.P; seg += wstride) {
        const int xs = __ldg(a.cx + seg), ys = __ldg(a.cy + seg);
        const int xe = __ldg(a.cx + seg + 1), ye = __ldg(a.cy + seg + 1);
        const int sb = seg_origin(ys);
        const int nch = ye > ys ? (ye - sb + kCH - 1) / kCH : 0;

        // row_ptr window: lane l holds rp[wb + l]
        int wb = xs;
        int win = (wb + lane <= m) ? __ldg(rp + wb + lane) : 0x7fffffff;
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

        // Row r ends inside this segment: settle it and move to row r + 1.
        auto finish_row = [&]() {
            if (r == xs && start_in) {
                // partial start row (Alg. 2 lines 8-9): atomic, or carry record slot 0
                if (FIX == FIX_ATOMIC) {
                    if (ys < rend) {
                        float *dst = (r == a.tail_row) ? a.tail
                                                       : a.C + ((int64_t)r - a.row_base) * a.ldc;
#pragma unroll
                        for (int s = 0; s < V; ++s)
                            if (act[s]) CVec<W>::add(dst + cofs[s], acc[s]);
                    }
                } else {
                    float *dst = a.rec + (seg * 2) * (int64_t)a.kpad;
#pragma unroll
                    for (int s = 0; s < V; ++s)
                        if (act[s]) CVec<W>::store(dst + cofs[s], acc[s]);
                }
            } else {
                // complete row (line 15): plain store, no initialisation of C needed
                float *dst = a.C + ((int64_t)r - a.row_base) * a.ldc;
#pragma unroll
                for (int s = 0; s < V; ++s)
                    if (act[s]) CVec<W>::store(dst + cofs[s], acc[s]);
            }
#pragma unroll
            for (int s = 0; s < V; ++s)
#pragma unroll
                for (int w = 0; w < W; ++w) acc[s][w] = 0.f;
            ++r;
            int idx = r + 1 - wb;
            if (idx >= 32) {
                wb = r;
                win = (wb + lane <= m) ? __ldg(rp + wb + lane) : 0x7fffffff;
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

        for (int k = 0; k < nch; ++k) {
            if (!direct) {
                mbar_wait(&bars[warp][cbuf], cbuf ? phase1 : phase0);
                if (cbuf) phase1 ^= 1u; else phase0 ^= 1u;
            }
            __syncwarp();
            produce();                  // next chunk into the other buffer
            if (direct) __syncwarp();
            const int cb = sb + k * kCH;
            const int32_t *sc = st.col[cbuf];
            const float *sv = st.val[cbuf];
            int q = ys - cb;
            q = q > 0 ? (q & ~(U - 1)) : 0;
            const int qend = min(kCH, ye - cb);
            for (; q < qend; q += U) {
                const int j0 = cb + q;
                int c[U];
                float v[U];
#pragma unroll
                for (int i = 0; i < U; i += 4) {
                    const int4 c4 = *reinterpret_cast<const int4 *>(sc + q + i);
                    const float4 v4 = *reinterpret_cast<const float4 *>(sv + q + i);
                    c[i] = c4.x; c[i + 1] = c4.y; c[i + 2] = c4.z; c[i + 3] = c4.w;
                    v[i] = v4.x; v[i + 1] = v4.y; v[i + 2] = v4.z; v[i + 3] = v4.w;
                }
                raw_t bv[U][V];
                if (j0 >= ys && j0 + U <= ye && j0 + U <= rend) {
                    // fast path: U non-zeros of the current row, no checks
#pragma unroll
                    for (int u = 0; u < U; ++u) {
#pragma unroll
                        for (int s = 0; s < V; ++s)
                            bv[u][s] = BV::load(reinterpret_cast<const TB *>(
                                                    row_addr(bl[s], (uint32_t)c[u], ldb_bytes)),
                                                pol_last);
                    }
#pragma unroll
                    for (int u = 0; u < U; ++u) fma_row(v[u], bv[u]);
                } else {
#pragma unroll
                    for (int u = 0; u < U; ++u) {
                        const int j = j0 + u;
                        if (j >= ys && j < ye) {
#pragma unroll
                            for (int s = 0; s < V; ++s)
                                bv[u][s] = BV::load(reinterpret_cast<const TB *>(
                                                        row_addr(bl[s], (uint32_t)c[u], ldb_bytes)),
                                                    pol_last);
                        }
                    }
#pragma unroll
                    for (int u = 0; u < U; ++u) {
                        const int j = j0 + u;
                        if (j >= ys && j < ye) {
                            while (j >= rend) finish_row();
                            fma_row(v[u], bv[u]);
                        }
                    }
                }
            }
            cbuf ^= 1;
        }
        // rows whose end item lies in this segment after its last non-zero
        while (r < xe) finish_row();

        // r == xe: the segment's non-zeros of row xe, if any (lines 3-5 / 11-13)
        if (xe < m && ye > rbeg) {
            const bool single = (xs == xe) && start_in;
            if (FIX == FIX_ATOMIC) {
                float *dst = (xe == a.tail_row) ? a.tail : a.C + ((int64_t)xe - a.row_base) * a.ldc;
#pragma unroll
                for (int s = 0; s < V; ++s)
                    if (act[s]) CVec<W>::add(dst + cofs[s], acc[s]);
            } else {
                float *dst = a.rec + (seg * 2 + (single ? 0 : 1)) * (int64_t)a.kpad;
#pragma unroll
                for (int s = 0; s < V; ++s)
                    if (act[s]) CVec<W>::store(dst + cofs[s], acc[s]);
            }
        }
    }
}

template <int W, int V, typename TB, int FIX>
static cudaError_t launch_seg(const SegArgs &a, cudaStream_t s) {
    static int blocks_per_sm = 0;
    if (blocks_per_sm == 0) {
        cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(
            &blocks_per_sm, segment_kernel<W, V, TB, FIX>, kBlock, 0);
        if (e != cudaSuccess) return e;
        if (blocks_per_sm < 1) blocks_per_sm = 1;
    }
    const int64_t warps_per_block = kBlock / 32;
    int64_t need = (a.P + warps_per_block - 1) / warps_per_block;
    const int64_t cap = (int64_t)blocks_per_sm * num_sms();
    const int64_t grid = need < cap ? need : cap;
    if (grid <= 0) return cudaSuccess;
    segment_kernel<W, V, TB, FIX><<<(unsigned)grid, kBlock, 0, s>>>(a);
    return cudaGetLastError();
}

template <typename TB, int FIX>
static cudaError_t dispatch_wv(const SegArgs &a, int W, int V, cudaStream_t s) {
#define MPS_V(WW)                                                       \
    switch (V) {                                                        \
    case 1: return launch_seg<WW, 1, TB, FIX>(a, s);                \
    case 2: return launch_seg<WW, 2, TB, FIX>(a, s);                \
    case 3: return launch_seg<WW, 3, TB, FIX>(a, s);                \
    case 4: return launch_seg<WW, 4, TB, FIX>(a, s);                \
    default: return cudaErrorInvalidValue;                              \
    }
    switch (W) {
    case 1: MPS_V(1)
    case 2: MPS_V(2)
    case 4: MPS_V(4)
    case 8:
        if constexpr (sizeof(TB) == 2) { MPS_V(8) }
        return cudaErrorInvalidValue;
    default: return cudaErrorInvalidValue;
    }
#undef MPS_V
}

cudaError_t launch_segments(const SegArgs &a, int b_dtype, int W, int V, int fix,
                            cudaStream_t s) {
    if (b_dtype == MPS_DT_F32) {
        return fix == FIX_CARRY ? dispatch_wv<float, FIX_CARRY>(a, W, V, s)
                                : dispatch_wv<float, FIX_ATOMIC>(a, W, V, s);
    }
    return fix == FIX_CARRY ? dispatch_wv<__nv_bfloat16, FIX_CARRY>(a, W, V, s)
                            : dispatch_wv<__nv_bfloat16, FIX_ATOMIC>(a, W, V, s);
}

// Carry-out fix-up: one warp per boundary p = 0..P.  For the first boundary p strictly
// inside a row r, the row's pieces are the end piece of segment p-1 (slot 1) and the
// start pieces (slot 0) of segments p, p+1, ... that start inside r.  They are summed
// in segment order (deterministic) and stored -- no zero-initialisation needed.
__global__ void __launch_bounds__(kBlock)
carry_reduce_kernel(const SegArgs a) {
    const int64_t p = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (p > a.P) return;
    const int32_t r = a.cx[p];
    if (r >= a.m) return;
    const int32_t rs = __ldg(a.rp + r);
    if (a.cy[p] <= rs) return;                                 // not inside row r
    if (p > 0 && a.cx[p - 1] == r && a.cy[p - 1] > rs) return; // not the first boundary
    // chain length: segments s = p .. q-1 start inside row r (s < P)
    int64_t q = p;
    for (;;) {
        const int64_t s = q + lane;
        const bool in = s < a.P && a.cx[s] == r && a.cy[s] > rs;
        const unsigned b = __ballot_sync(0xffffffffu, in);
        const int run = (b == 0xffffffffu) ? 32 : __ffs(~b) - 1;
        q += run;
        if (run < 32) break;
    }
    float *dst = (r == a.tail_row) ? a.tail : a.C + ((int64_t)r - a.row_base) * a.ldc;
    for (int c = lane * 4; c < a.K; c += 128) {
        const bool vec = c + 4 <= a.K;
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
        if (p > 0) {
            const float4 v = *reinterpret_cast<const float4 *>(a.rec + ((p - 1) * 2 + 1) * (int64_t)a.kpad + c);
            acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
        }
        int64_t s = p;
        for (; s + 4 <= q; s += 4) {
            float4 v[4];
#pragma unroll
            for (int k = 0; k < 4; ++k)
                v[k] = *reinterpret_cast<const float4 *>(a.rec + ((s + k) * 2) * (int64_t)a.kpad + c);
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                acc.x += v[k].x; acc.y += v[k].y; acc.z += v[k].z; acc.w += v[k].w;
            }
        }
        for (; s < q; ++s) {
            const float4 v = *reinterpret_cast<const float4 *>(a.rec + (s * 2) * (int64_t)a.kpad + c);
            acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
        }
        if (vec) {
            dst[c] = acc.x; dst[c + 1] = acc.y; dst[c + 2] = acc.z; dst[c + 3] = acc.w;
        } else {
            const float t[4] = {acc.x, acc.y, acc.z, acc.w};
            for (int k = 0; c + k < a.K; ++k) dst[c + k] = t[k];
        }
    }
}

cudaError_t launch_carry_reduce(const SegArgs &a, cudaStream_t s) {
    const int64_t threads = (a.P + 1) * 32;
    const int64_t blocks = (threads + kBlock - 1) / kBlock;
    carry_reduce_kernel<<<(unsigned)blocks, kBlock, 0, s>>>(a);
    return cudaGetLastError();
}

struct TailList {
    int32_t idx[128];
};

// Add the gathered tails owned by this rank, in ascending rank order.
__global__ void apply_tails_kernel(const float *__restrict__ tails, int32_t K, TailList t,
                                   int32_t n, float *row) {
    for (int c = threadIdx.x; c < K; c += blockDim.x) {
        float v = row[c];
        for (int i = 0; i < n; ++i) v += tails[(int64_t)t.idx[i] * K + c];
        row[c] = v;
    }
}

cudaError_t launch_apply_tails(const float *tails, int32_t K, const int32_t *idx, int32_t n,
                               float *row, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    if (n > 128) return cudaErrorInvalidValue;
    TailList t;
    for (int i = 0; i < n; ++i) t.idx[i] = idx[i];
    apply_tails_kernel<<<1, kBlock, 0, s>>>(tails, K, t, n, row);
    return cudaGetLastError();
}

}  // namespace mps
