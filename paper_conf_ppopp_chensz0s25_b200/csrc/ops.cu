// Residual CSR SpMM (keeps the result lossless), X-row permutation / Y-row unpermutation
// (Fig. 1 caption) and the nm_spmm entry points.
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include "nm_internal.h"

namespace nm {
namespace {

__device__ __forceinline__ float h2f(uint16_t b, int bf) {
  if (bf) return __uint_as_float(((uint32_t)b) << 16);
  __half h;
  *(uint16_t*)&h = b;
  return __half2float(h);
}

// Yp[l][f] += sum_k res_val[k] * PX[res_col[k]][f]  (the residual CSR, lossless remainder).
// One warp per row.  The warp's lanes form SUB = 32 / LPR subgroups of LPR lanes; a subgroup
// covers LPR * 8 features with one 16-byte X load per lane, and the subgroups take alternate
// nonzeros of the row (so F = 128 keeps all 32 lanes busy with 16-byte loads).  The row's
// (col, val) pairs are fetched 32 at a time with one coalesced load and broadcast with
// shuffles; the nonzero loop is unrolled so several X rows are in flight per lane.  Partial
// sums are combined across subgroups with xor-shuffles, then added into Y (fp32).
// F tail: the 16-byte vector at column f0 < F is inside the row (ldx % 8 == 0), only the
// accumulate/store is masked.
template <int BF, int LPR>
__global__ void __launch_bounds__(256) k_residual(const int64_t* __restrict__ rp, const int32_t* __restrict__ rc,
                                                  const uint16_t* __restrict__ rv, int64_t rows,
                                                  const int32_t* __restrict__ row_map,
                                                  const uint16_t* __restrict__ X, int64_t ldx,
                                                  float* __restrict__ Y, int64_t ldy, int F) {
  constexpr int SUB = 32 / LPR;
  constexpr int kUnroll = 4;
  const int lane = threadIdx.x & 31;
  const int sub = lane / LPR, li = lane % LPR;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  const bool vec_y = ((ldy & 3) == 0) && ((((uintptr_t)Y) & 15) == 0);
  for (int64_t l = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; l < rows; l += nw) {
    const int64_t b = rp[l], e = rp[l + 1];
    if (b == e) continue;
    float* yrow = Y + (row_map ? (int64_t)row_map[l] : l) * ldy;
    for (int f0 = li * 8; f0 - li * 8 < F; f0 += LPR * 8) {
      float acc[8];
#pragma unroll
      for (int q = 0; q < 8; ++q) acc[q] = 0.f;
      for (int64_t base = b; base < e; base += 32) {
        const int cnt = (int)min((int64_t)32, e - base);
        int32_t c = 0;
        float v = 0.f;
        if (lane < cnt) {
          c = __ldg(rc + base + lane);
          v = h2f(__ldg(rv + base + lane), BF);
        }
        for (int j = 0; j < cnt; j += SUB * kUnroll) {
          uint4 xv[kUnroll];
          float vv[kUnroll];
#pragma unroll
          for (int u = 0; u < kUnroll; ++u) {
            const int idx = j + u * SUB + sub;
            const int32_t cc = __shfl_sync(0xffffffffu, c, idx & 31);
            vv[u] = __shfl_sync(0xffffffffu, v, idx & 31);
            if (idx < cnt && f0 < F)
              xv[u] = __ldg((const uint4*)(X + (int64_t)cc * ldx + f0));
            else {
              xv[u] = make_uint4(0u, 0u, 0u, 0u);
              vv[u] = 0.f;
            }
          }
#pragma unroll
          for (int u = 0; u < kUnroll; ++u) {
            const uint32_t w[4] = {xv[u].x, xv[u].y, xv[u].z, xv[u].w};
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              acc[2 * q] += vv[u] * h2f((uint16_t)(w[q] & 0xFFFF), BF);
              acc[2 * q + 1] += vv[u] * h2f((uint16_t)(w[q] >> 16), BF);
            }
          }
        }
      }
#pragma unroll
      for (int o = LPR; o < 32; o <<= 1)
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[q] += __shfl_xor_sync(0xffffffffu, acc[q], o);
      if (sub == 0 && f0 < F) {
        float* y = yrow + f0;
        if (vec_y && f0 + 8 <= F) {
          float4 y0 = *(float4*)y, y1 = *(float4*)(y + 4);
          y0.x += acc[0]; y0.y += acc[1]; y0.z += acc[2]; y0.w += acc[3];
          y1.x += acc[4]; y1.y += acc[5]; y1.z += acc[6]; y1.w += acc[7];
          *(float4*)y = y0;
          *(float4*)(y + 4) = y1;
        } else {
#pragma unroll
          for (int q = 0; q < 8; ++q)
            if (f0 + q < F) y[q] += acc[q];
        }
      }
    }
  }
}

// dst[p] = src[idx[p]] (gather) or dst[idx[p]] = src[p] (scatter); row bytes copied with
// 16-byte vectors when aligned.  One warp per row.
template <bool SCATTER>
__global__ void __launch_bounds__(256) k_permute(const uint8_t* __restrict__ src, uint8_t* __restrict__ dst,
                                                 const int32_t* __restrict__ idx, int64_t n,
                                                 int64_t row_bytes, int64_t ld_bytes, int vec16) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t p = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; p < n; p += nw) {
    const int64_t q = idx[p];
    const uint8_t* s = src + (SCATTER ? p : q) * ld_bytes;
    uint8_t* d = dst + (SCATTER ? q : p) * ld_bytes;
    if (vec16) {
      for (int64_t o = lane * 16; o < row_bytes; o += 32 * 16)
        *(uint4*)(d + o) = __ldg((const uint4*)(s + o));
    } else {
      for (int64_t o = lane * 2; o < row_bytes; o += 64) *(uint16_t*)(d + o) = *(const uint16_t*)(s + o);
    }
  }
}

int grid_rows(int64_t rows, int warps_per_block) {
  int64_t g = (rows + warps_per_block - 1) / warps_per_block;
  if (g > 148 * 32) g = 148 * 32;
  return (int)(g < 1 ? 1 : g);
}

nm_status permute_impl(const void* src, void* dst, const int32_t* perm, int64_t n, int F, int64_t ld,
                       nm_dtype dt, cudaStream_t s, bool scatter) {
  if (!src || !dst || !perm) return fail(NM_ERR_INVALID_ARG, "permute: NULL pointer");
  if (src == dst) return fail(NM_ERR_INVALID_ARG, "permute: in-place not supported");
  if (n < 0 || F < 0 || ld < F) return fail(NM_ERR_INVALID_ARG, "permute: bad sizes");
  if (n == 0 || F == 0) return NM_OK;
  const int64_t esz = dt == NM_F32 ? 4 : 2;
  const int64_t row_bytes = F * esz, ld_bytes = ld * esz;
  const int vec16 = (row_bytes % 16 == 0) && (ld_bytes % 16 == 0) && (((uintptr_t)src & 15) == 0) &&
                    (((uintptr_t)dst & 15) == 0);
  if (scatter)
    k_permute<true><<<grid_rows(n, 8), 256, 0, s>>>((const uint8_t*)src, (uint8_t*)dst, perm, n, row_bytes,
                                                    ld_bytes, vec16);
  else
    k_permute<false><<<grid_rows(n, 8), 256, 0, s>>>((const uint8_t*)src, (uint8_t*)dst, perm, n, row_bytes,
                                                     ld_bytes, vec16);
  NM_CUDA(cudaGetLastError());
  return NM_OK;
}

nm_status check_spmm_args(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F) {
  if (!P || !PX || !Yp) return fail(NM_ERR_INVALID_ARG, "nm_spmm: NULL argument");
  if (F < 1 || F > 4096) return fail(NM_ERR_UNSUPPORTED, "nm_spmm: F must be in [1, 4096]");
  if (ldx < F || ldy < F) return fail(NM_ERR_INVALID_ARG, "nm_spmm: leading dimension < F");
  if (ldx % 8 != 0 || ((uintptr_t)PX & 15) != 0)
    return fail(NM_ERR_INVALID_ARG, "nm_spmm: PX rows must be 16-byte aligned (ldx % 8 == 0)");
  return NM_OK;
}

}  // namespace

nm_status launch_spmm_residual(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                               cudaStream_t s) {
  const int64_t rows = P->row_end - P->row_begin;
  if (P->res_nnz == 0 || rows == 0) return NM_OK;
  const int32_t* rcol = P->res_gather ? P->res_gather : P->res_col;
  // lanes per row-slice: 8 features per lane, at most one warp per slice
  const int lpr = F <= 32 ? 4 : F <= 64 ? 8 : F <= 128 ? 16 : 32;
#define NM_RES_LAUNCH(BF, LPR)                                                                       \
  k_residual<BF, LPR><<<grid_rows(rows, 8), 256, 0, s>>>(P->res_rowptr, rcol, P->res_val, rows, P->row_map, \
                                                         (const uint16_t*)PX, ldx, Yp, ldy, F)
  const int bf = P->dtype == NM_BF16;
  switch (lpr * 2 + bf) {
    case 8: NM_RES_LAUNCH(0, 4); break;
    case 9: NM_RES_LAUNCH(1, 4); break;
    case 16: NM_RES_LAUNCH(0, 8); break;
    case 17: NM_RES_LAUNCH(1, 8); break;
    case 32: NM_RES_LAUNCH(0, 16); break;
    case 33: NM_RES_LAUNCH(1, 16); break;
    case 64: NM_RES_LAUNCH(0, 32); break;
    default: NM_RES_LAUNCH(1, 32); break;
  }
#undef NM_RES_LAUNCH
  NM_CUDA(cudaGetLastError());
  return NM_OK;
}

}  // namespace nm

using namespace nm;

extern "C" {

nm_status nm_permute_rows(const void* X, void* PX, const int32_t* perm_dev, int64_t n, int F, int64_t ld,
                          nm_dtype dtype, void* stream) {
  return permute_impl(X, PX, perm_dev, n, F, ld, dtype, (cudaStream_t)stream, false);
}

nm_status nm_unpermute_rows(const void* Yp, void* Y, const int32_t* perm_dev, int64_t n, int F, int64_t ld,
                            nm_dtype dtype, void* stream) {
  return permute_impl(Yp, Y, perm_dev, n, F, ld, dtype, (cudaStream_t)stream, true);
}

nm_status nm_spmm_sptc(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                       void* stream) {
  nm_status st = check_spmm_args(P, PX, ldx, Yp, ldy, F);
  if (st != NM_OK) return st;
  return launch_spmm_sptc(P, PX, ldx, Yp, ldy, F, (cudaStream_t)stream);
}

nm_status nm_spmm_residual(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                           void* stream) {
  nm_status st = check_spmm_args(P, PX, ldx, Yp, ldy, F);
  if (st != NM_OK) return st;
  return launch_spmm_residual(P, PX, ldx, Yp, ldy, F, (cudaStream_t)stream);
}

nm_status nm_spmm(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy, int F,
                  void* stream) {
  nm_status st = check_spmm_args(P, PX, ldx, Yp, ldy, F);
  if (st != NM_OK) return st;
  st = launch_spmm_sptc(P, PX, ldx, Yp, ldy, F, (cudaStream_t)stream);
  if (st != NM_OK) return st;
  return launch_spmm_residual(P, PX, ldx, Yp, ldy, F, (cudaStream_t)stream);
}

}  // extern "C"
