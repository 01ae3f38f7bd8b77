// dtc_gcn.cu -- GraphConv layer on top of DTC-SpMM.
//
// PAPER.md:441-443 §5.4, Eq. (2): H_{l+1} = sigma((A x H_l) x w_l + b_l), "A x H
// corresponds to a typical SpMM operation".  Two steps, in the paper's order:
//   1. AH = A * H_l     -- the DTC-SpMM kernel (dtc_spmm, this library's hot path)
//   2. Y  = sigma(AH * W + b) -- a plain dense GEMM: cuBLASLt (TF32 tensor cores, FP32
//      accumulate) with the bias add and ReLU fused into its epilogue, so Y is written once.
// The dense contraction is a library GEMM on purpose (the product here is the sparse step).
#include <cublasLt.h>

#include <algorithm>
#include <cmath>
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

static int ensure_gemm_ws(dtc_format* h, cudaStream_t s) {
    if (h->gemm_ws_bytes >= kGemmWs) return DTC_OK;
    dfree(h->gemm_ws, s);
    h->gemm_ws_bytes = 0;
    int rc = dalloc(&h->gemm_ws, kGemmWs, s);
    if (rc) return rc;
    h->gemm_ws_bytes = kGemmWs;
    return DTC_OK;
}

// Column-major D (m x n, ld m) = op(A) (m x k) * op(B) (k x n) with fp32 storage; lda/ldb are the
// leading dimensions of A and B as stored.  compute: TF32 tensor cores or full FP32.
static int lt_gemm(dtc_format* h, cudaStream_t s, bool ta, bool tb, uint64_t m, uint64_t n, uint64_t k,
                   const float* A, uint64_t lda, const float* B, uint64_t ldb, float* D, bool tf32) {
    cublasLtHandle_t lt;
    int rc = lt_handle(h->device, &lt);
    if (rc) return rc;
    if ((rc = ensure_gemm_ws(h, s))) return rc;
    LtDescs L;
    DTC_LT(cublasLtMatmulDescCreate(&L.op, tf32 ? CUBLAS_COMPUTE_32F_FAST_TF32 : CUBLAS_COMPUTE_32F, CUDA_R_32F));
    const cublasOperation_t opa = ta ? CUBLAS_OP_T : CUBLAS_OP_N, opb = tb ? CUBLAS_OP_T : CUBLAS_OP_N;
    DTC_LT(cublasLtMatmulDescSetAttribute(L.op, CUBLASLT_MATMUL_DESC_TRANSA, &opa, sizeof(opa)));
    DTC_LT(cublasLtMatmulDescSetAttribute(L.op, CUBLASLT_MATMUL_DESC_TRANSB, &opb, sizeof(opb)));
    DTC_LT(cublasLtMatrixLayoutCreate(&L.a, CUDA_R_32F, ta ? k : m, ta ? m : k, lda));
    DTC_LT(cublasLtMatrixLayoutCreate(&L.b, CUDA_R_32F, tb ? n : k, tb ? k : n, ldb));
    DTC_LT(cublasLtMatrixLayoutCreate(&L.d, CUDA_R_32F, m, n, m));
    DTC_LT(cublasLtMatmulPreferenceCreate(&L.pref));
    size_t wsb = h->gemm_ws_bytes;
    DTC_LT(cublasLtMatmulPreferenceSetAttribute(L.pref, CUBLASLT_MATMUL_PREF_MAX_WORKSPACE_BYTES, &wsb, sizeof(wsb)));
    cublasLtMatmulHeuristicResult_t heur;
    int found = 0;
    DTC_LT(cublasLtMatmulAlgoGetHeuristic(lt, L.op, L.a, L.b, L.d, L.d, L.pref, 1, &heur, &found));
    if (found < 1) { set_error("no cuBLASLt algorithm for a GraphConv GEMM"); return DTC_ERR_UNSUPPORTED; }
    const float one = 1.0f, zero = 0.0f;
    DTC_LT(cublasLtMatmul(lt, L.op, &one, A, L.a, B, L.b, &zero, D, L.d, D, L.d, &heur.algo, h->gemm_ws, wsb, s));
    return DTC_OK;
}

// dZ = dY * [Y > 0] (ReLU) or dY (identity); dZ may alias dY
__global__ void k_act_grad(int64_t n, int relu, const float* __restrict__ Y, const float* dY, float* dZ) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        dZ[i] = (!relu || Y[i] > 0.f) ? dY[i] : 0.f;
}

// db[j] = sum_i dZ[i][j], deterministic: fixed 1024-row blocks summed in row order, then the
// block partials summed in block order by one thread per column
constexpr int kColsumRows = 1024;
__global__ void k_colsum_partial(int64_t M, int64_t F, const float* __restrict__ dZ, float* __restrict__ part) {
    const int64_t rb = blockIdx.y;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < F; j += (int64_t)gridDim.x * blockDim.x) {
        float acc = 0.f;
        const int64_t r1 = min(M, (rb + 1) * kColsumRows);
        for (int64_t r = rb * kColsumRows; r < r1; ++r) acc += dZ[r * F + j];
        part[rb * F + j] = acc;
    }
}
__global__ void k_colsum_final(int64_t nb, int64_t F, const float* __restrict__ part, float* __restrict__ db) {
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < F; j += (int64_t)gridDim.x * blockDim.x) {
        float acc = 0.f;
        for (int64_t b = 0; b < nb; ++b) acc += part[b * F + j];
        db[j] = acc;
    }
}

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
    if ((rc = ensure_gemm_ws(h, s))) return rc;
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

extern "C" int dtc_graphconv_backward(dtc_handle_t h, dtc_handle_t ht, const float* AH, const float* W, int64_t F_in,
                                      int64_t F_out, int32_t act, const float* Y, const float* dY, float* dZ,
                                      float* dW, float* db, float* dAH, float* dH, void* stream) {
    if (!h || F_in < 1 || F_out < 1 || !AH || !W || !Y || !dY || !dZ || !dW || !dAH ||
        (act != DTC_ACT_NONE && act != DTC_ACT_RELU)) {
        set_error("bad graphconv_backward arguments");
        return DTC_ERR_INVALID;
    }
    if (dH) {
        if (!ht || ht->M != h->K || ht->K != h->M || ht->nnz != h->nnz) {
            set_error("dH needs the handle of A^T (dtc_build_opts_t.transpose) of this matrix");
            return DTC_ERR_INVALID;
        }
        if (ht->dtype != DTC_TF32) { set_error("dH = A^T dAH needs a TF32 A^T handle (dAH is fp32)"); return DTC_ERR_UNSUPPORTED; }
    }
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t M = h->M;
    int rc;
    if (M > 0) {
        const int64_t n = M * F_out;
        k_act_grad<<<(unsigned)std::min<int64_t>((n + 255) / 256, 148 * 64), 256, 0, s>>>(n, act == DTC_ACT_RELU, Y, dY, dZ);
        DTC_CUDA(cudaGetLastError());
        // dW (F_in x F_out, row-major) = AH^T dZ  -> column-major dW^T (F_out x F_in) = dZ_cm * AH_cm^T
        if ((rc = lt_gemm(h, s, false, true, (uint64_t)F_out, (uint64_t)F_in, (uint64_t)M, dZ, (uint64_t)F_out, AH,
                          (uint64_t)F_in, dW, true)))
            return rc;
        // dAH (M x F_in, row-major) = dZ W^T -> column-major dAH^T (F_in x M) = W_cm^T * dZ_cm
        if ((rc = lt_gemm(h, s, true, false, (uint64_t)F_in, (uint64_t)M, (uint64_t)F_out, W, (uint64_t)F_out, dZ,
                          (uint64_t)F_out, dAH, true)))
            return rc;
    } else {
        DTC_CUDA(cudaMemsetAsync(dW, 0, F_in * F_out * sizeof(float), s));
    }
    if (db) {
        const int64_t nb = std::max<int64_t>(1, (M + kColsumRows - 1) / kColsumRows);
        float* part = nullptr;
        if ((rc = dalloc(&part, (size_t)nb * F_out, s))) return rc;
        const dim3 g1((unsigned)std::min<int64_t>((F_out + 127) / 128, 1024), (unsigned)nb);
        if (M > 0) k_colsum_partial<<<g1, 128, 0, s>>>(M, F_out, dZ, part);
        else cudaMemsetAsync(part, 0, F_out * sizeof(float), s);
        k_colsum_final<<<(unsigned)std::min<int64_t>((F_out + 127) / 128, 1024), 128, 0, s>>>(nb, F_out, part, db);
        dfree(part, s);
        DTC_CUDA(cudaGetLastError());
    }
    // dH (K x F_in) = A^T dAH: the DTC-SpMM kernel on the transposed format
    if (dH) return spmm_launch(ht, dAH, F_in, F_in, dH, F_in, s);
    return DTC_OK;
}

// ---------------------------------------------------------------- loss and update (2-layer training step)
// loss = mean_i [logsumexp(z_i) - z_i[label_i]], dlogits = (softmax(z_i) - onehot(label_i)) / M
__global__ void k_xent_rows(int64_t M, int64_t Cn, const float* __restrict__ z, const int32_t* __restrict__ lab,
                            float* __restrict__ rowloss, float* __restrict__ dz, int* __restrict__ bad) {
    const int lane = threadIdx.x & 31;
    int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = warp; i < M; i += nw) {
        const float* zr = z + i * Cn;
        float mx = -INFINITY;
        for (int64_t c = lane; c < Cn; c += 32) mx = fmaxf(mx, zr[c]);
        for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        float se = 0.f;
        for (int64_t c = lane; c < Cn; c += 32) se += expf(zr[c] - mx);
        for (int o = 16; o > 0; o >>= 1) se += __shfl_xor_sync(0xffffffffu, se, o);
        const int y = lab[i];
        if (y < 0 || y >= Cn) {
            if (lane == 0) atomicOr(bad, 1);
            continue;
        }
        const float inv = 1.f / (float)M;
        for (int64_t c = lane; c < Cn; c += 32) dz[i * Cn + c] = (expf(zr[c] - mx) / se - (c == y ? 1.f : 0.f)) * inv;
        if (lane == 0) rowloss[i] = logf(se) + mx - zr[y];
    }
}
__global__ void k_mean_final(int64_t M, const float* __restrict__ rowloss, float* __restrict__ loss) {
    // one block, fixed order: thread t sums rows t, t+256, ...; then a fixed tree
    __shared__ float red[256];
    float a = 0.f;
    for (int64_t i = threadIdx.x; i < M; i += 256) a += rowloss[i];
    red[threadIdx.x] = a;
    __syncthreads();
    for (int w = 128; w > 0; w >>= 1) {
        if ((int)threadIdx.x < w) red[threadIdx.x] += red[threadIdx.x + w];
        __syncthreads();
    }
    if (threadIdx.x == 0) *loss = M > 0 ? red[0] / (float)M : 0.f;
}
__global__ void k_sgd(int64_t n, float lr, float* __restrict__ p, const float* __restrict__ g) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        p[i] -= lr * g[i];
}

extern "C" int dtc_softmax_xent(const float* logits, const int32_t* labels, int64_t M, int64_t num_classes,
                                float* loss, float* dlogits, void* stream) {
    if (M < 0 || num_classes < 1 || !loss || (M > 0 && (!logits || !labels || !dlogits))) {
        set_error("bad softmax_xent arguments");
        return DTC_ERR_INVALID;
    }
    cudaStream_t s = (cudaStream_t)stream;
    float* rowloss = nullptr;
    int* bad = nullptr;
    int rc;
    if ((rc = dalloc(&rowloss, std::max<int64_t>(M, 1), s))) return rc;
    if ((rc = dalloc(&bad, 1, s))) { dfree(rowloss, s); return rc; }
    cudaMemsetAsync(bad, 0, sizeof(int), s);
    if (M > 0)
        k_xent_rows<<<(unsigned)std::min<int64_t>((M * 32 + 255) / 256, 148 * 32), 256, 0, s>>>(M, num_classes, logits,
                                                                                              labels, rowloss, dlogits, bad);
    k_mean_final<<<1, 256, 0, s>>>(M, rowloss, loss);
    int hbad = 0;
    cudaMemcpyAsync(&hbad, bad, sizeof(int), cudaMemcpyDeviceToHost, s);
    const cudaError_t e = cudaStreamSynchronize(s);
    dfree(rowloss, s);
    dfree(bad, s);
    if (e != cudaSuccess) return cuda_fail(e, "softmax_xent", __FILE__, __LINE__);
    if (hbad) { set_error("label outside [0, num_classes)"); return DTC_ERR_INVALID; }
    return DTC_OK;
}

extern "C" int dtc_sgd_update(float* param, const float* grad, int64_t n, float lr, void* stream) {
    if (n < 0 || (n > 0 && (!param || !grad))) { set_error("bad sgd arguments"); return DTC_ERR_INVALID; }
    if (n == 0) return DTC_OK;
    k_sgd<<<(unsigned)std::min<int64_t>((n + 255) / 256, 148 * 64), 256, 0, (cudaStream_t)stream>>>(n, lr, param, grad);
    DTC_CUDA(cudaGetLastError());
    return DTC_OK;
}
