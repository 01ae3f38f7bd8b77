// cusparse_ref.cu -- the comparison system on the same box (cuSPARSE
// SpMM, CUSPARSE_SPMM_ALG_DEFAULT, CUSPARSE_FORMAT_CSR).  Bench-only; not part of
// the product library.  Row-major B and C, FP32 compute.
#include <cuda_runtime.h>
#include <cusparse.h>

#include <cstdint>
#include <cstdio>

struct CuspHandle {
    cusparseHandle_t h = nullptr;
    cusparseSpMatDescr_t A = nullptr;
    cusparseDnMatDescr_t B = nullptr, C = nullptr;
    cusparseSpMMAlg_t alg;
    void* buf = nullptr;
    float alpha = 1.f, beta = 0.f;
};

extern "C" void* cusp_create(int64_t M, int64_t K, int64_t nnz, void* rowptr, void* colidx, void* vals, int fp16,
                             void* Bp, int64_t N, void* Cp, int alg, void* stream, int* status) {
    CuspHandle* c = new CuspHandle();
    cudaDataType vt = fp16 ? CUDA_R_16F : CUDA_R_32F;
    cusparseStatus_t st;
    const cusparseSpMMAlg_t algs[4] = {CUSPARSE_SPMM_ALG_DEFAULT, CUSPARSE_SPMM_CSR_ALG1, CUSPARSE_SPMM_CSR_ALG2,
                                       CUSPARSE_SPMM_CSR_ALG3};
    c->alg = algs[alg & 3];
    size_t bytes = 0;
#define CK(x) do { st = (x); if (st != CUSPARSE_STATUS_SUCCESS) goto fail; } while (0)
    CK(cusparseCreate(&c->h));
    CK(cusparseSetStream(c->h, (cudaStream_t)stream));
    CK(cusparseCreateCsr(&c->A, M, K, nnz, rowptr, colidx, vals, CUSPARSE_INDEX_32I, CUSPARSE_INDEX_32I,
                         CUSPARSE_INDEX_BASE_ZERO, vt));
    CK(cusparseCreateDnMat(&c->B, K, N, N, Bp, vt, CUSPARSE_ORDER_ROW));
    CK(cusparseCreateDnMat(&c->C, M, N, N, Cp, CUDA_R_32F, CUSPARSE_ORDER_ROW));
    CK(cusparseSpMM_bufferSize(c->h, CUSPARSE_OPERATION_NON_TRANSPOSE, CUSPARSE_OPERATION_NON_TRANSPOSE, &c->alpha,
                               c->A, c->B, &c->beta, c->C, CUDA_R_32F, c->alg, &bytes));
    if (cudaMalloc(&c->buf, bytes ? bytes : 16) != cudaSuccess) { st = CUSPARSE_STATUS_ALLOC_FAILED; goto fail; }
    CK(cusparseSpMM_preprocess(c->h, CUSPARSE_OPERATION_NON_TRANSPOSE, CUSPARSE_OPERATION_NON_TRANSPOSE, &c->alpha,
                               c->A, c->B, &c->beta, c->C, CUDA_R_32F, c->alg, c->buf));
    *status = 0;
    return c;
fail:
    *status = (int)st;
    if (c->buf) cudaFree(c->buf);
    if (c->A) cusparseDestroySpMat(c->A);
    if (c->B) cusparseDestroyDnMat(c->B);
    if (c->C) cusparseDestroyDnMat(c->C);
    if (c->h) cusparseDestroy(c->h);
    delete c;
    return nullptr;
#undef CK
}

extern "C" int cusp_run(void* p) {
    CuspHandle* c = (CuspHandle*)p;
    return (int)cusparseSpMM(c->h, CUSPARSE_OPERATION_NON_TRANSPOSE, CUSPARSE_OPERATION_NON_TRANSPOSE, &c->alpha, c->A,
                             c->B, &c->beta, c->C, CUDA_R_32F, c->alg, c->buf);
}

extern "C" void cusp_destroy(void* p) {
    CuspHandle* c = (CuspHandle*)p;
    if (!c) return;
    cudaFree(c->buf);
    cusparseDestroySpMat(c->A);
    cusparseDestroyDnMat(c->B);
    cusparseDestroyDnMat(c->C);
    cusparseDestroy(c->h);
    delete c;
}
