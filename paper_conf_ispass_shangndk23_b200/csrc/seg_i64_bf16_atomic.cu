// seg_i64_bf16_atomic.cu -- instantiations of the segment kernel for int64 row_ptr / nnz
// coordinates (NEXT-4), B = __nv_bfloat16, atomic fix-up.
#include "segment.cuh"

namespace mps {
cudaError_t launch_segments_bf16_atomic(const SegArgs64 &a, int W, int V, int NR, cudaStream_t s) {
    return dispatch_w<__nv_bfloat16, FIX_ATOMIC>(a, W, V, NR, s);
}
}  // namespace mps
