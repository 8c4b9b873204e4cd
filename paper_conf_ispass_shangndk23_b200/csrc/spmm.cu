// spmm.cu -- a3/a4 entry (dispatch to the segment-kernel instantiations), the carry-out
// reduction and the shard tail application (Alg. 2).
#include "mps_internal.cuh"

namespace mps {

// one translation unit per (index type, B dtype, fix-up) so the build parallelises
cudaError_t launch_segments_f32_atomic(const SegArgs &a, int W, int V, int NR, cudaStream_t s);
cudaError_t launch_segments_f32_carry(const SegArgs &a, int W, int V, int NR, cudaStream_t s);
cudaError_t launch_segments_bf16_atomic(const SegArgs &a, int W, int V, int NR, cudaStream_t s);
cudaError_t launch_segments_bf16_carry(const SegArgs &a, int W, int V, int NR, cudaStream_t s);
cudaError_t launch_segments_f32_atomic(const SegArgs64 &a, int W, int V, int NR, cudaStream_t s);
cudaError_t launch_segments_f32_carry(const SegArgs64 &a, int W, int V, int NR, cudaStream_t s);
cudaError_t launch_segments_bf16_atomic(const SegArgs64 &a, int W, int V, int NR, cudaStream_t s);
cudaError_t launch_segments_bf16_carry(const SegArgs64 &a, int W, int V, int NR, cudaStream_t s);

template <typename IT>
cudaError_t launch_segments(const SegArgsT<IT> &a, int b_dtype, int W, int V, int NR, int fix,
                            cudaStream_t s) {
    if (b_dtype == MPS_DT_F32)
        return fix == FIX_CARRY ? launch_segments_f32_carry(a, W, V, NR, s)
                                : launch_segments_f32_atomic(a, W, V, NR, s);
    return fix == FIX_CARRY ? launch_segments_bf16_carry(a, W, V, NR, s)
                            : launch_segments_bf16_atomic(a, W, V, NR, s);
}

// Carry-out fix-up: one warp per boundary p = 0..P.  For the first boundary p strictly
// inside a row r, the row's pieces are the end piece of segment p-1 (slot 1) and the
// start pieces (slot 0) of segments p, p+1, ... that start inside r.  They are summed
// in segment order (deterministic) and stored -- no zero-initialisation needed.
template <typename IT>
__device__ __forceinline__ void carry_one(const SegArgsT<IT> &a) {
    const int64_t p = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (p > a.P) return;
    const int32_t r = a.cx[p];
    if (r >= a.m) return;
    const IT rs = __ldg(a.rp + r);
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
        if (a.relu) {
            acc.x = fmaxf(acc.x, 0.f); acc.y = fmaxf(acc.y, 0.f);
            acc.z = fmaxf(acc.z, 0.f); acc.w = fmaxf(acc.w, 0.f);
        }
        if (vec) {
            dst[c] = acc.x; dst[c + 1] = acc.y; dst[c + 2] = acc.z; dst[c + 3] = acc.w;
        } else {
            const float t[4] = {acc.x, acc.y, acc.z, acc.w};
            for (int k = 0; c + k < a.K; ++k) dst[c + k] = t[k];
        }
    }
}

template <typename IT>
__global__ void __launch_bounds__(kBlock)
carry_reduce_kernel(const SegArgsT<IT> a) {
    // launched with programmatic dependent launch behind the kernel that wrote the
    // records: wait for it before reading them (a no-op without PDL)
    asm volatile("griddepcontrol.wait;" ::: "memory");
    carry_one(a);
    if (a.mail.on) tail_mail_epilogue(a.mail);   // a6 tail exchange (carry mode)
}

template <typename IT>
cudaError_t launch_carry_reduce(const SegArgsT<IT> &a, cudaStream_t s) {
    const int64_t threads = (a.P + 1) * 32;
    const int64_t blocks = (threads + kBlock - 1) / kBlock;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)blocks);
    cfg.blockDim = dim3(kBlock);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, carry_reduce_kernel<IT>, a);
}

// Epilogue for the rows cut by a schedule boundary in atomic mode: they are final only
// after every partial sum has landed, so the ReLU runs here, once per cut row (one warp
// per first boundary inside the row).
template <typename IT>
__global__ void __launch_bounds__(kBlock)
relu_split_kernel(const SegArgsT<IT> a) {
    const int64_t p = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (p > a.P) return;
    const int32_t r = a.cx[p];
    if (r >= a.m || r == a.tail_row) return;
    const IT rs = __ldg(a.rp + r);
    if (a.cy[p] <= rs) return;
    if (p > 0 && a.cx[p - 1] == r && a.cy[p - 1] > rs) return;
    float *dst = a.C + ((int64_t)r - a.row_base) * a.ldc;
    for (int c = lane; c < a.K; c += 32) dst[c] = fmaxf(dst[c], 0.f);
}

template <typename IT>
cudaError_t launch_relu_split(const SegArgsT<IT> &a, cudaStream_t s) {
    const int64_t threads = (a.P + 1) * 32;
    const int64_t blocks = (threads + kBlock - 1) / kBlock;
    relu_split_kernel<IT><<<(unsigned)blocks, kBlock, 0, s>>>(a);
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

// ---- GCN glue: H = bf16(relu(C)), the next layer's combination input ----------------
__global__ void relu_to_bf16_kernel(const float *__restrict__ C, int64_t rows, int K,
                                    int64_t ldc, __nv_bfloat16 *__restrict__ H, int64_t ldh) {
    const int64_t total = rows * (int64_t)K;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = i / K, c = i - r * K;
        H[r * ldh + c] = __float2bfloat16_rn(fmaxf(__ldg(C + r * ldc + c), 0.f));
    }
}

cudaError_t launch_relu_to_bf16(const float *C, int64_t rows, int K, int64_t ldc, void *H,
                                int64_t ldh, cudaStream_t s) {
    if (rows <= 0 || K <= 0) return cudaSuccess;
    int64_t blocks = (rows * K + kBlock - 1) / kBlock;
    const int64_t cap = (int64_t)num_sms() * 8;
    if (blocks > cap) blocks = cap;
    relu_to_bf16_kernel<<<(unsigned)blocks, kBlock, 0, s>>>(
        C, rows, K, ldc, reinterpret_cast<__nv_bfloat16 *>(H), ldh);
    return cudaGetLastError();
}

// ---- cross-GPU signals over peer memory (flags[slot][source rank], epoch values) -------
struct PeerFlags {
    uint32_t *p[kMailMaxWorld];
};

// rank `rank` raises flag[slot][rank] to `epoch` in every rank's signal buffer, after
// everything earlier on this stream (the kernel boundary + a system-scope fence)
__global__ void peer_signal_kernel(PeerFlags f, int world, int rank, int slot, uint32_t epoch) {
    const int g = threadIdx.x;
    __threadfence_system();
    if (g < world) st_release_sys(f.p[g] + slot * kMailMaxWorld + rank, epoch);
}

// wait until every rank raised flag[slot][*] to `epoch` in this rank's signal buffer
__global__ void peer_wait_kernel(const uint32_t *mine, int world, int slot, uint32_t epoch) {
    const int g = threadIdx.x;
    if (g < world) wait_geq(mine + slot * kMailMaxWorld + g, epoch);
    __syncthreads();
    __threadfence_system();
}

cudaError_t launch_peer_signal(void *const *bufs, int world, int rank, int slot, uint32_t epoch,
                               cudaStream_t s) {
    if (world < 1 || world > kMailMaxWorld) return cudaErrorInvalidValue;
    PeerFlags f{};
    for (int g = 0; g < world; ++g) f.p[g] = reinterpret_cast<uint32_t *>(bufs[g]);
    peer_signal_kernel<<<1, 32, 0, s>>>(f, world, rank, slot, epoch);
    return cudaGetLastError();
}

cudaError_t launch_peer_wait(const void *mine, int world, int slot, uint32_t epoch,
                             cudaStream_t s) {
    if (world < 1 || world > kMailMaxWorld) return cudaErrorInvalidValue;
    peer_wait_kernel<<<1, 32, 0, s>>>(reinterpret_cast<const uint32_t *>(mine), world, slot,
                                      epoch);
    return cudaGetLastError();
}

#define MPS_INST_SPMM(IT)                                                                     \
    template cudaError_t launch_segments<IT>(const SegArgsT<IT> &, int, int, int, int, int,     \
                                             cudaStream_t);                                     \
    template cudaError_t launch_carry_reduce<IT>(const SegArgsT<IT> &, cudaStream_t);          \
    template cudaError_t launch_relu_split<IT>(const SegArgsT<IT> &, cudaStream_t);
MPS_INST_SPMM(int32_t)
MPS_INST_SPMM(int64_t)

}  // namespace mps
