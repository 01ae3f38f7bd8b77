// dtc_gcn.cu -- GraphConv layer on top of DTC-SpMM.
//
// PAPER.md:441-443 §5.4, Eq. (2): H_{l+1} = sigma((A x H_l) x w_l + b_l), "A x H
// corresponds to a typical SpMM operation".  Two steps, in the paper's order:
//   1. AH = A * H_l     -- the DTC-SpMM kernel (dtc_spmm, this library's hot path)
//   2. Y  = sigma(AH * W + b) -- a plain dense GEMM: cuBLASLt (TF32 tensor cores, FP32
//      accumulate) with the bias add and ReLU fused into its epilogue, so Y is written once.
// The dense contraction is a library GEMM on purpose (the product here is the sparse step).
#include <cublasLt.h>

#include <mutex>

#include "dtc_internal.h"

namespace dtc {

static cublasLtHandle_t g_lt[64];
static std::mutex g_lt_mu;

static int lt_fail(cublasStatus_t st, const char* what) {
    set_error("%s failed (cublas status %d)", what, (int)st);
    return DTC_ERR_CUDA;
}
#define DTC_LT(call)                                              \
    do {                                                          \
        cublasStatus_t _st = (call);                              \
        if (_st != CUBLAS_STATUS_SUCCESS) return lt_fail(_st, #call); \
    } while (0)

static int lt_handle(int dev, cublasLtHandle_t* out) {
    if (dev < 0 || dev >= 64) { set_error("device index %d", dev); return DTC_ERR_INVALID; }
    std::lock_guard<std::mutex> g(g_lt_mu);
    if (!g_lt[dev]) DTC_LT(cublasLtCreate(&g_lt[dev]));
    *out = g_lt[dev];
    return DTC_OK;
}

struct LtDescs {
    cublasLtMatmulDesc_t op = nullptr;
    cublasLtMatrixLayout_t a = nullptr, b = nullptr, d = nullptr;
    cublasLtMatmulPreference_t pref = nullptr;
    ~LtDescs() {
        if (pref) cublasLtMatmulPreferenceDestroy(pref);
        if (d) cublasLtMatrixLayoutDestroy(d);
        if (b) cublasLtMatrixLayoutDestroy(b);
        if (a) cublasLtMatrixLayoutDestroy(a);
        if (op) cublasLtMatmulDescDestroy(op);
    }
};

constexpr size_t kGemmWs = size_t(32) << 20;

}  // namespace dtc

using namespace dtc;

extern "C" int dtc_graphconv(dtc_handle_t h, const void* H, int64_t F_in, const float* W, int64_t F_out,
                             const float* bias, int32_t act, float* AH, float* Y, void* stream) {
    if (!h || F_in < 1 || F_out < 1 || !W || !AH || !Y || (act != DTC_ACT_NONE && act != DTC_ACT_RELU) ||
        (!H && h->K > 0)) {
        set_error("bad graphconv arguments");
        return DTC_ERR_INVALID;
    }
    cudaStream_t s = (cudaStream_t)stream;
    // 1. AH = A * H (DTC-SpMM)
    int rc = spmm_launch(h, H, F_in, F_in, AH, F_in, s);
    if (rc) return rc;
    if (h->M == 0) return DTC_OK;
    // 2. Y = act(AH * W + b).  Row-major Y (M x F_out) is column-major Y^T (F_out x M):
    //    Y^T = W^T (F_out x F_in, the column-major view of row-major W) * AH^T (F_in x M).
    cublasLtHandle_t lt;
    if ((rc = lt_handle(h->device, &lt))) return rc;
    if (h->gemm_ws_bytes < kGemmWs) {
        dfree(h->gemm_ws, s);
        h->gemm_ws_bytes = 0;
        if ((rc = dalloc(&h->gemm_ws, kGemmWs, s))) return rc;
        h->gemm_ws_bytes = kGemmWs;
    }
    LtDescs L;
    DTC_LT(cublasLtMatmulDescCreate(&L.op, CUBLAS_COMPUTE_32F_FAST_TF32, CUDA_R_32F));
    cublasLtEpilogue_t epi = bias ? (act == DTC_ACT_RELU ? CUBLASLT_EPILOGUE_RELU_BIAS : CUBLASLT_EPILOGUE_BIAS)
                                  : (act == DTC_ACT_RELU ? CUBLASLT_EPILOGUE_RELU : CUBLASLT_EPILOGUE_DEFAULT);
    DTC_LT(cublasLtMatmulDescSetAttribute(L.op, CUBLASLT_MATMUL_DESC_EPILOGUE, &epi, sizeof(epi)));
    if (bias) DTC_LT(cublasLtMatmulDescSetAttribute(L.op, CUBLASLT_MATMUL_DESC_BIAS_POINTER, &bias, sizeof(bias)));
    DTC_LT(cublasLtMatrixLayoutCreate(&L.a, CUDA_R_32F, (uint64_t)F_out, (uint64_t)F_in, F_out));
    DTC_LT(cublasLtMatrixLayoutCreate(&L.b, CUDA_R_32F, (uint64_t)F_in, (uint64_t)h->M, F_in));
    DTC_LT(cublasLtMatrixLayoutCreate(&L.d, CUDA_R_32F, (uint64_t)F_out, (uint64_t)h->M, F_out));
    DTC_LT(cublasLtMatmulPreferenceCreate(&L.pref));
    size_t wsb = h->gemm_ws_bytes;
    DTC_LT(cublasLtMatmulPreferenceSetAttribute(L.pref, CUBLASLT_MATMUL_PREF_MAX_WORKSPACE_BYTES, &wsb, sizeof(wsb)));
    cublasLtMatmulHeuristicResult_t heur;
    int found = 0;
    DTC_LT(cublasLtMatmulAlgoGetHeuristic(lt, L.op, L.a, L.b, L.d, L.d, L.pref, 1, &heur, &found));
    if (found < 1) { set_error("no cuBLASLt algorithm for the GraphConv GEMM"); return DTC_ERR_UNSUPPORTED; }
    const float one = 1.0f, zero = 0.0f;
    DTC_LT(cublasLtMatmul(lt, L.op, &one, W, L.a, AH, L.b, &zero, Y, L.d, Y, L.d, &heur.algo, h->gemm_ws, wsb, s));
    return DTC_OK;
}

extern "C" int dtc_graphconv_launches_per_call(void) { return dtc_spmm_launches_per_call() + 1; }
