// cusparse_ref.cu -- the cuSPARSE reference point of the bench (SURVEY.md
// sec. 8(d)): cusparseSpMM on the same CSR A and row-major B / C, fp32, trying
// CUSPARSE_SPMM_ALG_DEFAULT and CSR_ALG1/2/3 (whichever accept the layout) and reporting
// the best.  Buffer allocation and preprocessing are excluded; each timed call follows
// an L2 flush (a 2 x L2 memset), like the bench's own step.  NOT part of the product:
// libmpspmm never links it; bench.py loads it only to print a reference line.
#include <cuda_runtime.h>
#include <cusparse.h>
#include <stdint.h>
#include <stdio.h>

extern "C" int cusparse_spmm_best(int64_t m, int64_t n, int64_t nnz, const int32_t *rp,
                                  const int32_t *col, const float *val, const float *B,
                                  int64_t ldb, int32_t K, float *C, int64_t ldc, int iters,
                                  float *best_ms, int *best_alg, float *ms_per_alg) {
    cusparseHandle_t h;
    if (cusparseCreate(&h) != CUSPARSE_STATUS_SUCCESS) return 1;
    cusparseSpMatDescr_t A;
    cusparseDnMatDescr_t Bd, Cd;
    cusparseCreateCsr(&A, m, n, nnz, (void *)rp, (void *)col, (void *)val, CUSPARSE_INDEX_32I,
                      CUSPARSE_INDEX_32I, CUSPARSE_INDEX_BASE_ZERO, CUDA_R_32F);
    cusparseCreateDnMat(&Bd, n, K, ldb, (void *)B, CUDA_R_32F, CUSPARSE_ORDER_ROW);
    cusparseCreateDnMat(&Cd, m, K, ldc, (void *)C, CUDA_R_32F, CUSPARSE_ORDER_ROW);
    const float alpha = 1.f, beta = 0.f;
    int dev = 0, l2 = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
    void *flush = nullptr;
    cudaMalloc(&flush, (size_t)l2 * 2);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const cusparseSpMMAlg_t algs[4] = {CUSPARSE_SPMM_ALG_DEFAULT, CUSPARSE_SPMM_CSR_ALG1,
                                       CUSPARSE_SPMM_CSR_ALG2, CUSPARSE_SPMM_CSR_ALG3};
    *best_ms = -1.f;
    *best_alg = -1;
    for (int a = 0; a < 4; ++a) {
        ms_per_alg[a] = -1.f;
        size_t bytes = 0;
        if (cusparseSpMM_bufferSize(h, CUSPARSE_OPERATION_NON_TRANSPOSE,
                                    CUSPARSE_OPERATION_NON_TRANSPOSE, &alpha, A, Bd, &beta, Cd,
                                    CUDA_R_32F, algs[a], &bytes) != CUSPARSE_STATUS_SUCCESS)
            continue;
        void *buf = nullptr;
        if (bytes && cudaMalloc(&buf, bytes) != cudaSuccess) continue;
        if (cusparseSpMM_preprocess(h, CUSPARSE_OPERATION_NON_TRANSPOSE,
                                    CUSPARSE_OPERATION_NON_TRANSPOSE, &alpha, A, Bd, &beta, Cd,
                                    CUDA_R_32F, algs[a], buf) != CUSPARSE_STATUS_SUCCESS) {
            cudaFree(buf);
            continue;
        }
        bool ok = true;
        float best = 1e30f;
        for (int it = 0; it < iters + 1 && ok; ++it) {
            cudaMemsetAsync(flush, it & 1, (size_t)l2 * 2);
            cudaEventRecord(e0);
            ok = cusparseSpMM(h, CUSPARSE_OPERATION_NON_TRANSPOSE,
                              CUSPARSE_OPERATION_NON_TRANSPOSE, &alpha, A, Bd, &beta, Cd,
                              CUDA_R_32F, algs[a], buf) == CUSPARSE_STATUS_SUCCESS;
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms = 0.f;
            cudaEventElapsedTime(&ms, e0, e1);
            if (it > 0 && ms < best) best = ms;       // first call: warm-up
        }
        cudaFree(buf);
        if (!ok) continue;
        ms_per_alg[a] = best;
        if (*best_ms < 0 || best < *best_ms) {
            *best_ms = best;
            *best_alg = a;
        }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(flush);
    cusparseDestroySpMat(A);
    cusparseDestroyDnMat(Bd);
    cusparseDestroyDnMat(Cd);
    cusparseDestroy(h);
    return *best_alg < 0 ? 2 : 0;
}
