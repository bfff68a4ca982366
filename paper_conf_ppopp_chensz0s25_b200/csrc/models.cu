// The other GNN aggregations the paper evaluates next to GCN (Table 3's
// "SGC", "SAGE", "Cheb" columns at L546-553), built on the same packed
// sparse-tensor-core SpMM:
//   nm_sgc_propagate : SGC's feature propagation Y = Ahat^K X (K SpMM hops; the operand of
//                      every hop after the first is the previous hop rounded to the pack dtype)
//   nm_sage_layer    : GraphSAGE with the mean aggregator,
//                      Hout = act([H | mean_{j~i} H_j] [W_self; W_neigh] + b)
//                      (the mean is the SpMM of a pack of D^-1 A, row-normalised values)
//   nm_cheb_layer    : Chebyshev convolution, Hout = act(sum_{k<K} T_k(Lhat) H W_k + b),
//                      T_0 = H, T_1 = Lhat H, T_k = 2 Lhat T_{k-1} - T_{k-2}
// The dense products are one cuBLASLt GEMM over the concatenated operands (library GEMM,
// fp32 accumulation); every aggregation runs through nm_spmm (k_spmm_full + k_residual).
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include "nm_internal.h"

namespace nm {
namespace {

inline size_t al256(size_t x) { return (x + 255) & ~(size_t)255; }

inline int grid_ew(int64_t total) {
  int64_t g = (total + 255) / 256;
  if (g > 148 * 16) g = 148 * 16;
  return (int)(g < 1 ? 1 : g);
}

template <int BF>
__device__ __forceinline__ uint16_t to16(float v) {
  if (BF) {
    __nv_bfloat16 h = __float2bfloat16_rn(v);
    return *(uint16_t*)&h;
  }
  __half h = __float2half_rn(v);
  return *(uint16_t*)&h;
}

template <int BF>
__device__ __forceinline__ float from16(uint16_t b) {
  if (BF) return __uint_as_float((uint32_t)b << 16);
  return __half2float(*(const __half*)&b);
}

// dst16[r][f] = 16-bit(src[r][f])   (strided, rows x F)
template <int BF>
__global__ void k_round(const float* __restrict__ src, int64_t lds, uint16_t* __restrict__ dst, int64_t ldd,
                        int64_t rows, int F) {
  const int64_t total = rows * F;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / F;
    const int f = (int)(i - r * F);
    dst[r * ldd + f] = to16<BF>(src[r * lds + f]);
  }
}

// dst16 = 16-bit(2 t - prev16)   (Chebyshev recurrence, strided, rows x F)
template <int BF>
__global__ void k_cheb(const float* __restrict__ t, int64_t ldt, const uint16_t* __restrict__ prev, int64_t ldp,
                       uint16_t* __restrict__ dst, int64_t ldd, int64_t rows, int F) {
  const int64_t total = rows * F;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / F;
    const int f = (int)(i - r * F);
    dst[r * ldd + f] = to16<BF>(2.f * t[r * ldt + f] - from16<BF>(prev[r * ldp + f]));
  }
}

// out16 = act(acc + bias)   (rows x F, contiguous)
template <int BF>
__global__ void k_bias_act16(const float* __restrict__ acc, int64_t rows, int F, const float* __restrict__ bias,
                             int relu, uint16_t* __restrict__ out) {
  const int64_t total = rows * F;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    float v = acc[i] + (bias ? bias[i % F] : 0.f);
    if (relu) v = fmaxf(v, 0.f);
    out[i] = to16<BF>(v);
  }
}

nm_status launch_round(bool bf, const float* src, int64_t lds, void* dst, int64_t ldd, int64_t rows, int F,
                       cudaStream_t s) {
  if (bf) k_round<1><<<grid_ew(rows * F), 256, 0, s>>>(src, lds, (uint16_t*)dst, ldd, rows, F);
  else k_round<0><<<grid_ew(rows * F), 256, 0, s>>>(src, lds, (uint16_t*)dst, ldd, rows, F);
  NM_CUDA(cudaGetLastError());
  return NM_OK;
}

nm_status launch_bias_act(bool bf, const float* acc, int64_t rows, int F, const float* bias, int relu, void* out,
                          cudaStream_t s) {
  if (bf) k_bias_act16<1><<<grid_ew(rows * F), 256, 0, s>>>(acc, rows, F, bias, relu, (uint16_t*)out);
  else k_bias_act16<0><<<grid_ew(rows * F), 256, 0, s>>>(acc, rows, F, bias, relu, (uint16_t*)out);
  NM_CUDA(cudaGetLastError());
  return NM_OK;
}

nm_status check_full_pack(const nm_packed* P, const char* who) {
  if (P->row_begin != 0 || P->row_end != P->n)
    return fail(NM_ERR_UNSUPPORTED, std::string(who) + ": needs a pack of all rows (row-sharded packs chain through "
                                                       "dist.gcn_forward-style all-gathers)");
  return NM_OK;
}

}  // namespace
}  // namespace nm

using namespace nm;

extern "C" size_t nm_sgc_workspace_bytes(int64_t n, int F) {
  const int64_t ld = (F + 7) / 8 * 8;
  return 2 * al256((size_t)n * ld * 2);
}

extern "C" nm_status nm_sgc_propagate(const nm_packed* Ahat, const void* X, int64_t ldx, float* Y, int64_t ldy,
                                      void* Y16, int F, int K, void* ws, size_t ws_bytes, void* stream) {
  if (!Ahat || !X || !Y || !ws) return fail(NM_ERR_INVALID_ARG, "nm_sgc_propagate: NULL argument");
  if (K < 1 || F < 1) return fail(NM_ERR_INVALID_ARG, "nm_sgc_propagate: need K >= 1, F >= 1");
  nm_status st = check_full_pack(Ahat, "nm_sgc_propagate");
  if (st != NM_OK) return st;
  const int64_t n = Ahat->n, ld = (F + 7) / 8 * 8;
  if (ws_bytes < nm_sgc_workspace_bytes(n, F)) return fail(NM_ERR_INVALID_ARG, "nm_sgc_propagate: workspace too small");
  cudaStream_t s = (cudaStream_t)stream;
  const bool bf = Ahat->dtype == NM_BF16;
  uint8_t* w8 = (uint8_t*)ws;
  void* buf[2] = {w8, w8 + al256((size_t)n * ld * 2)};
  const void* cur = X;
  int64_t ldc = ldx;
  for (int k = 0; k < K; ++k) {
    st = nm_spmm(Ahat, cur, ldc, Y, ldy, F, stream);  // hop k + 1 (fp32)
    if (st != NM_OK) return st;
    if (k + 1 < K) {  // the next hop's operand: this hop rounded to the pack dtype
      NM_TRY_STATUS(launch_round(bf, Y, ldy, buf[k & 1], ld, n, F, s));
      cur = buf[k & 1];
      ldc = ld;
    }
  }
  if (Y16) NM_TRY_STATUS(launch_round(bf, Y, ldy, Y16, ldx, n, F, s));
  return NM_OK;
}

extern "C" size_t nm_sage_workspace_bytes(int64_t n, int F_in, int F_out) {
  return al256((size_t)n * 2 * F_in * 2) + al256((size_t)n * F_in * 4) + al256((size_t)n * F_out * 4) +
         al256((size_t)2 * F_in * F_out * 2) + lt_workspace_bytes();
}

extern "C" nm_status nm_sage_layer(const nm_packed* Amean, const void* H, const void* W_self, const void* W_neigh,
                                   const float* bias, void* Hout, int F_in, int F_out, int flags, void* ws,
                                   size_t ws_bytes, void* stream) {
  if (!Amean || !H || !W_self || !W_neigh || !Hout || !ws) return fail(NM_ERR_INVALID_ARG, "nm_sage_layer: NULL argument");
  if (F_in < 1 || F_out < 1 || F_in % 8 || F_out % 8)
    return fail(NM_ERR_UNSUPPORTED, "nm_sage_layer: F_in and F_out must be positive multiples of 8");
  if (flags & ~NM_RELU) return fail(NM_ERR_INVALID_ARG, "nm_sage_layer: unknown flags");
  nm_status st = check_full_pack(Amean, "nm_sage_layer");
  if (st != NM_OK) return st;
  if (Amean->row_map) return fail(NM_ERR_UNSUPPORTED, "nm_sage_layer: needs a pack in permuted order (flags 0)");
  const int64_t n = Amean->n;
  if (ws_bytes < nm_sage_workspace_bytes(n, F_in, F_out)) return fail(NM_ERR_INVALID_ARG, "nm_sage_layer: workspace too small");
  cudaStream_t s = (cudaStream_t)stream;
  const bool bf = Amean->dtype == NM_BF16;
  uint8_t* w8 = (uint8_t*)ws;
  uint8_t* cat = w8;                                                   // n x 2F_in 16-bit: [H | mean]
  float* agg = (float*)(cat + al256((size_t)n * 2 * F_in * 2));        // n x F_in fp32
  float* acc = (float*)((uint8_t*)agg + al256((size_t)n * F_in * 4));  // n x F_out fp32
  uint8_t* wcat = (uint8_t*)acc + al256((size_t)n * F_out * 4);        // 2F_in x F_out 16-bit
  void* lt_ws = wcat + al256((size_t)2 * F_in * F_out * 2);
  NM_CUDA(cudaMemcpy2DAsync(cat, (size_t)2 * F_in * 2, H, (size_t)F_in * 2, (size_t)F_in * 2, (size_t)n,
                            cudaMemcpyDeviceToDevice, s));
  NM_CUDA(cudaMemcpyAsync(wcat, W_self, (size_t)F_in * F_out * 2, cudaMemcpyDeviceToDevice, s));
  NM_CUDA(cudaMemcpyAsync(wcat + (size_t)F_in * F_out * 2, W_neigh, (size_t)F_in * F_out * 2, cudaMemcpyDeviceToDevice, s));
  st = nm_spmm(Amean, H, F_in, agg, F_in, F_in, stream);  // mean over the neighbours (D^-1 A H)
  if (st != NM_OK) return st;
  NM_TRY_STATUS(launch_round(bf, agg, F_in, cat + (size_t)F_in * 2, 2 * F_in, n, F_in, s));
  NM_TRY_STATUS(gemm_rm(cat, 2 * F_in, wcat, F_out, acc, F_out, n, 2 * F_in, F_out, Amean->dtype, true, lt_ws, s));
  return launch_bias_act(bf, acc, n, F_out, bias, flags & NM_RELU, Hout, s);
}

extern "C" size_t nm_cheb_workspace_bytes(int64_t n, int F_in, int F_out, int K) {
  return al256((size_t)n * K * F_in * 2) + al256((size_t)n * F_in * 4) + al256((size_t)n * F_out * 4) +
         lt_workspace_bytes();
}

extern "C" nm_status nm_cheb_layer(const nm_packed* Lhat, const void* H, const void* W, const float* bias, void* Hout,
                                   int F_in, int F_out, int K, int flags, void* ws, size_t ws_bytes, void* stream) {
  if (!Lhat || !H || !W || !Hout || !ws) return fail(NM_ERR_INVALID_ARG, "nm_cheb_layer: NULL argument");
  if (F_in < 1 || F_out < 1 || F_in % 8 || F_out % 8)
    return fail(NM_ERR_UNSUPPORTED, "nm_cheb_layer: F_in and F_out must be positive multiples of 8");
  if (K < 1) return fail(NM_ERR_INVALID_ARG, "nm_cheb_layer: K >= 1");
  if (flags & ~NM_RELU) return fail(NM_ERR_INVALID_ARG, "nm_cheb_layer: unknown flags");
  nm_status st = check_full_pack(Lhat, "nm_cheb_layer");
  if (st != NM_OK) return st;
  if (Lhat->row_map) return fail(NM_ERR_UNSUPPORTED, "nm_cheb_layer: needs a pack in permuted order (flags 0)");
  const int64_t n = Lhat->n, ldc = (int64_t)K * F_in;
  if (ws_bytes < nm_cheb_workspace_bytes(n, F_in, F_out, K)) return fail(NM_ERR_INVALID_ARG, "nm_cheb_layer: workspace too small");
  cudaStream_t s = (cudaStream_t)stream;
  const bool bf = Lhat->dtype == NM_BF16;
  uint8_t* cat = (uint8_t*)ws;                                          // n x K F_in 16-bit: [T_0 | ... | T_{K-1}]
  float* t32 = (float*)(cat + al256((size_t)n * K * F_in * 2));         // n x F_in fp32
  float* acc = (float*)((uint8_t*)t32 + al256((size_t)n * F_in * 4));   // n x F_out fp32
  void* lt_ws = (uint8_t*)acc + al256((size_t)n * F_out * 4);
  auto Tk = [&](int k) { return cat + (size_t)k * F_in * 2; };
  NM_CUDA(cudaMemcpy2DAsync(cat, (size_t)ldc * 2, H, (size_t)F_in * 2, (size_t)F_in * 2, (size_t)n,
                            cudaMemcpyDeviceToDevice, s));  // T_0 = H
  for (int k = 1; k < K; ++k) {
    st = nm_spmm(Lhat, Tk(k - 1), ldc, t32, F_in, F_in, stream);  // Lhat T_{k-1}
    if (st != NM_OK) return st;
    if (k == 1) {
      NM_TRY_STATUS(launch_round(bf, t32, F_in, Tk(1), ldc, n, F_in, s));
    } else {
      if (bf) k_cheb<1><<<grid_ew(n * F_in), 256, 0, s>>>(t32, F_in, (const uint16_t*)Tk(k - 2), ldc, (uint16_t*)Tk(k), ldc, n, F_in);
      else k_cheb<0><<<grid_ew(n * F_in), 256, 0, s>>>(t32, F_in, (const uint16_t*)Tk(k - 2), ldc, (uint16_t*)Tk(k), ldc, n, F_in);
      NM_CUDA(cudaGetLastError());
    }
  }
  NM_TRY_STATUS(gemm_rm(cat, ldc, W, F_out, acc, F_out, n, (int)ldc, F_out, Lhat->dtype, true, lt_ws, s));
  return launch_bias_act(bf, acc, n, F_out, bias, flags & NM_RELU, Hout, s);
}
