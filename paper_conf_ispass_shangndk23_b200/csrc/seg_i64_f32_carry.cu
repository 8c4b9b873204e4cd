// seg_i64_f32_carry.cu -- instantiations of the segment kernel for int64 row_ptr / nnz
// coordinates (NEXT-4), B = float, carry fix-up.
#include "segment.cuh"

namespace mps {
cudaError_t launch_segments_f32_carry(const SegArgs64 &a, int W, int V, int NR, cudaStream_t s) {
    return dispatch_w<float, FIX_CARRY>(a, W, V, NR, s);
}
}  // namespace mps
