// libnm: status/error plumbing, CSR validation and upload, packed-handle queries and the
// canonical export (decoding the MMA-native image back to the canonical arrays of nm.h).
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "nm_internal.h"

namespace nm {

static thread_local std::string g_last_error;

void set_error(const std::string& msg) { g_last_error = msg; }

nm_status fail(nm_status s, const std::string& msg) {
  g_last_error = msg;
  return s;
}

nm_status cuda_fail(cudaError_t e, const char* what) {
  g_last_error = std::string(what) + ": " + cudaGetErrorString(e);
  return e == cudaErrorMemoryAllocation ? NM_ERR_OOM : NM_ERR_CUDA;
}

uint16_t one_bits(nm_dtype dt) { return dt == NM_BF16 ? (uint16_t)0x3F80 : (uint16_t)0x3C00; }

namespace {
thread_local cudaMemPool_t t_scratch_pool = nullptr;
}

nm_status scratch_alloc(void** p, size_t bytes, cudaStream_t s) {
  if (bytes == 0) bytes = 16;
  if (t_scratch_pool) {
    NM_CUDA(cudaMallocFromPoolAsync(p, bytes, t_scratch_pool, s));
  } else {
    NM_CUDA(cudaMallocAsync(p, bytes, s));
  }
  return NM_OK;
}

nm_status ScopedPool::init(int device) {
  cudaMemPoolProps props = {};
  props.allocType = cudaMemAllocationTypePinned;
  props.handleTypes = cudaMemHandleTypeNone;
  props.location.type = cudaMemLocationTypeDevice;
  props.location.id = device;
  NM_CUDA(cudaMemPoolCreate(&pool, &props));
  uint64_t keep = UINT64_MAX;
  NM_CUDA(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep));
  prev = t_scratch_pool;
  t_scratch_pool = pool;
  return NM_OK;
}

ScopedPool::~ScopedPool() {
  if (!pool) return;
  t_scratch_pool = prev;
  cudaDeviceSynchronize();  // every stream-ordered free into the pool has executed
  cudaMemPoolDestroy(pool);
}

nm_status validate_csr_host(int64_t n, const int64_t* rp, const int32_t* ci, bool check_sym) {
  if (n < 0) return fail(NM_ERR_INVALID_ARG, "n < 0");
  if (rp[0] != 0) return fail(NM_ERR_BAD_CSR, "rowptr[0] != 0");
  for (int64_t i = 0; i < n; ++i) {
    if (rp[i + 1] < rp[i]) return fail(NM_ERR_BAD_CSR, "rowptr not monotone at row " + std::to_string(i));
    for (int64_t k = rp[i]; k < rp[i + 1]; ++k) {
      if (ci[k] < 0 || ci[k] >= n)
        return fail(NM_ERR_BAD_CSR, "column out of range in row " + std::to_string(i));
      if (k > rp[i] && ci[k] <= ci[k - 1])
        return fail(NM_ERR_BAD_CSR, "columns unsorted or duplicated in row " + std::to_string(i));
    }
  }
  if (check_sym) {
    // symmetric pattern: for every (i, j) the entry (j, i) exists.  Count-based check: walk
    // rows in order and keep a cursor per row; each row j must see its entries (j, i) in
    // increasing i as the outer loop advances.
    std::vector<int64_t> cur(rp, rp + n);
    for (int64_t i = 0; i < n; ++i)
      for (int64_t k = rp[i]; k < rp[i + 1]; ++k) {
        int64_t j = ci[k];
        if (cur[j] >= rp[j + 1] || ci[cur[j]] != i)
          return fail(NM_ERR_NOT_SYMMETRIC, "pattern not symmetric at (" + std::to_string(i) +
                                                "," + std::to_string(j) + ")");
        cur[j]++;
      }
    for (int64_t j = 0; j < n; ++j)
      if (cur[j] != rp[j + 1])
        return fail(NM_ERR_NOT_SYMMETRIC, "pattern not symmetric in row " + std::to_string(j));
  }
  return NM_OK;
}

void DevCsr::release() {
  if (rp) cudaFree(rp);
  if (ci) cudaFree(ci);
  if (val) cudaFree(val);
  rp = nullptr;
  ci = nullptr;
  val = nullptr;
}

__global__ void k_convert_vals(const void* __restrict__ src, int src_dt, uint16_t* __restrict__ dst,
                               int dst_dt, int64_t nnz) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  for (; i < nnz; i += (int64_t)gridDim.x * blockDim.x) {
    float v;
    if (src_dt == NM_F32) v = ((const float*)src)[i];
    else if (src_dt == NM_F16) v = __half2float(((const __half*)src)[i]);
    else v = __bfloat162float(((const __nv_bfloat16*)src)[i]);
    uint16_t b;
    if (dst_dt == NM_F16) {
      __half h = __float2half_rn(v);
      memcpy(&b, &h, 2);
    } else {
      __nv_bfloat16 h = __float2bfloat16_rn(v);
      memcpy(&b, &h, 2);
    }
    dst[i] = b;
  }
}

nm_status upload_csr(const nm_csr* A, nm_dtype dtype, DevCsr* out, cudaStream_t s) {
  out->release();
  out->n = A->n;
  out->nnz = A->nnz;
  cudaMemcpyKind kind = A->on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
  NM_CUDA(cudaMalloc(&out->rp, sizeof(int64_t) * (A->n + 1)));
  NM_CUDA(cudaMalloc(&out->ci, sizeof(int32_t) * (A->nnz > 0 ? A->nnz : 1)));
  NM_CUDA(cudaMemcpyAsync(out->rp, A->rowptr, sizeof(int64_t) * (A->n + 1), kind, s));
  if (A->nnz > 0)
    NM_CUDA(cudaMemcpyAsync(out->ci, A->col, sizeof(int32_t) * A->nnz, kind, s));
  if (A->val) {
    NM_CUDA(cudaMalloc(&out->val, sizeof(uint16_t) * (A->nnz > 0 ? A->nnz : 1)));
    if (A->nnz > 0) {
      if (A->val_dtype == dtype) {
        NM_CUDA(cudaMemcpyAsync(out->val, A->val, sizeof(uint16_t) * A->nnz, kind, s));
      } else {
        const void* src = A->val;
        void* tmp = nullptr;
        size_t esz = A->val_dtype == NM_F32 ? 4 : 2;
        if (!A->on_device) {
          NM_CUDA(cudaMalloc(&tmp, esz * A->nnz));
          NM_CUDA(cudaMemcpyAsync(tmp, A->val, esz * A->nnz, cudaMemcpyHostToDevice, s));
          src = tmp;
        }
        k_convert_vals<<<1184, 256, 0, s>>>(src, A->val_dtype, out->val, dtype, A->nnz);
        NM_CUDA(cudaGetLastError());
        if (tmp) {
          NM_CUDA(cudaStreamSynchronize(s));
          cudaFree(tmp);
        }
      }
    }
  }
  return NM_OK;
}

nm_status host_csr(const nm_csr* A, int64_t** rp, int32_t** ci) {
  *rp = (int64_t*)malloc(sizeof(int64_t) * (A->n + 1));
  *ci = (int32_t*)malloc(sizeof(int32_t) * (A->nnz > 0 ? A->nnz : 1));
  if (!*rp || !*ci) return fail(NM_ERR_OOM, "host allocation");
  if (A->on_device) {
    NM_CUDA(cudaMemcpy(*rp, A->rowptr, sizeof(int64_t) * (A->n + 1), cudaMemcpyDeviceToHost));
    if (A->nnz) NM_CUDA(cudaMemcpy(*ci, A->col, sizeof(int32_t) * A->nnz, cudaMemcpyDeviceToHost));
  } else {
    memcpy(*rp, A->rowptr, sizeof(int64_t) * (A->n + 1));
    if (A->nnz) memcpy(*ci, A->col, sizeof(int32_t) * A->nnz);
  }
  return NM_OK;
}

}  // namespace nm

using namespace nm;

extern "C" {

const char* nm_status_string(nm_status s) {
  switch (s) {
    case NM_OK: return "NM_OK";
    case NM_ERR_INVALID_ARG: return "NM_ERR_INVALID_ARG";
    case NM_ERR_UNSUPPORTED: return "NM_ERR_UNSUPPORTED";
    case NM_ERR_BAD_CSR: return "NM_ERR_BAD_CSR";
    case NM_ERR_NOT_SYMMETRIC: return "NM_ERR_NOT_SYMMETRIC";
    case NM_ERR_CUDA: return "NM_ERR_CUDA";
    case NM_ERR_OOM: return "NM_ERR_OOM";
  }
  return "NM_ERR_UNKNOWN";
}

const char* nm_last_error(void) { return g_last_error.c_str(); }

int nm_version(void) { return 1; }

// Hybrid-split threshold from a measured time model (reading #27): a meta-block
// emitted to the tensor-core path costs an eighth of a K = 32 chunk, a residual value one
// gathered X row.  Fitted on B200 (round 2, full-record kernel + cp.async residual, whole-GPU
// times): a chunk costs ~0.28 + 0.0075 F ns (the MMA issue interval, ~242 cycles per
// tcgen05.mma.sp, plus the 4736-B record and the gathers: C3 F = 128 1.24 ns, C4 F = 256
// 2.2 ns); a residual value ~0.16 F ps (C3 21 ps, C4 40 ps).  Blocks keeping fewer values than
// the break-even go to the residual: 8 at F = 128, 7 at F = 256, 10 at F = 64.  Measured tau
// sweeps (profiles/r02_tau_sweep.txt): C4 best at 8, C3 128:2:16 at 6, C3 1:2:4 and C5 flat
// between 4 and 12.
int nm_hybrid_tau(int F) {
  if (F < 1) return 0;
  const double t_chunk = 0.28 + 0.0075 * F;   // ns
  const double t_value = 0.00016 * F;         // ns
  return (int)ceil(t_chunk / (8.0 * t_value));
}

void nm_packed_free(nm_packed* P) {
  if (!P) return;
  int cur = 0;
  cudaGetDevice(&cur);
  cudaSetDevice(P->device);
  void* ptrs[] = {P->panel_mb_ptr, P->panel_chunk_ptr, P->unit_info, P->mb_seg, P->mb_sel,
                  P->image, P->res_rowptr, P->res_col, P->res_val, P->row_map,
                  P->res_gather, P->res_segs, P->rec_len16, P->image_full, P->cta_ptr};
  for (void* p : ptrs)
    if (p) cudaFree(p);
  cudaSetDevice(cur);
  delete P;
}

nm_status nm_packed_info(const nm_packed* P, int64_t* n_mb, int64_t* packed_nnz,
                         int64_t* residual_nnz, int64_t* device_bytes, int64_t* n_chunks) {
  if (!P) return fail(NM_ERR_INVALID_ARG, "nm_packed_info: NULL handle");
  if (n_mb) *n_mb = P->n_mb;
  if (packed_nnz) *packed_nnz = P->packed_nnz;
  if (residual_nnz) *residual_nnz = P->res_nnz;
  if (device_bytes) *device_bytes = (int64_t)P->device_bytes;
  if (n_chunks) *n_chunks = P->n_chunks;
  return NM_OK;
}

nm_status nm_packed_stats(const nm_packed* P, nm_packed_stat* st) {
  if (!P || !st) return fail(NM_ERR_INVALID_ARG, "nm_packed_stats: NULL argument");
  st->n = P->n;
  st->row_begin = P->row_begin;
  st->row_end = P->row_end;
  st->n_panels = P->n_panels;
  st->n_mb = P->n_mb;
  st->n_chunks = P->n_chunks;
  st->packed_nnz = P->packed_nnz;
  st->residual_nnz = P->res_nnz;
  st->image_bytes = P->image_bytes;
  st->device_bytes = (int64_t)P->device_bytes;
  st->residual_items = P->n_res_segs;
  st->residual_split_rows = P->n_res_split;
  st->V = P->V;
  st->M = P->M;
  st->Mp = P->Mp;
  st->Vp = P->Vp;
  st->tau = P->tau;
  st->flags = P->flags;
  st->full_image_bytes = (int64_t)kChunkBytes * P->n_chunks;
  st->gather_rows = P->gather_rows;
  return NM_OK;
}

nm_status nm_export_canonical(const nm_packed* P, int64_t* panel_ptr, int32_t* mb_seg,
                              uint8_t* sel, uint8_t* nib, uint16_t* vals, int64_t* res_rowptr,
                              int32_t* res_col, uint16_t* res_val) {
  if (!P) return fail(NM_ERR_INVALID_ARG, "nm_export_canonical: NULL handle");
  int cur = 0;
  NM_CUDA(cudaGetDevice(&cur));
  NM_CUDA(cudaSetDevice(P->device));
  const int64_t rows = P->row_end - P->row_begin;
  const int64_t Pc = P->n_cpanels, Vp = P->Vp, ratio = kPanelRows / P->Vp;
  std::vector<int64_t> mbp(Pc + 1), chp(P->n_panels + 1);
  NM_CUDA(cudaMemcpy(mbp.data(), P->panel_mb_ptr, sizeof(int64_t) * (Pc + 1), cudaMemcpyDeviceToHost));
  NM_CUDA(cudaMemcpy(chp.data(), P->panel_chunk_ptr, sizeof(int64_t) * (P->n_panels + 1),
                     cudaMemcpyDeviceToHost));
  if (panel_ptr) memcpy(panel_ptr, mbp.data(), sizeof(int64_t) * (Pc + 1));
  if (mb_seg && P->n_mb)
    NM_CUDA(cudaMemcpy(mb_seg, P->mb_seg, sizeof(int32_t) * P->n_mb, cudaMemcpyDeviceToHost));
  if (sel && P->n_mb) {
    std::vector<uint32_t> s(P->n_mb);
    NM_CUDA(cudaMemcpy(s.data(), P->mb_sel, sizeof(uint32_t) * P->n_mb, cudaMemcpyDeviceToHost));
    for (int64_t m = 0; m < P->n_mb; ++m)
      for (int j = 0; j < 4; ++j) sel[m * 4 + j] = (uint8_t)((s[m] >> (8 * j)) & 0xFF);
  }
  if ((nib || vals) && P->n_mb) {
    // expand the compressed HBM records (nm_internal.h kRec* layout) back into full MMA-layout
    // records -- a host decoder independent of the SpMM kernel's shared-memory expansion
    std::vector<uint8_t> cimg((size_t)P->image_bytes);
    std::vector<uint16_t> len16(P->n_chunks);
    NM_CUDA(cudaMemcpy(cimg.data(), P->image, cimg.size(), cudaMemcpyDeviceToHost));
    NM_CUDA(cudaMemcpy(len16.data(), P->rec_len16, sizeof(uint16_t) * P->n_chunks, cudaMemcpyDeviceToHost));
    std::vector<uint8_t> img((size_t)P->n_chunks * kChunkBytes, 0);
    size_t off = 0;
    for (int64_t c = 0; c < P->n_chunks; ++c) {
      const uint8_t* rec = cimg.data() + off;
      off += (size_t)len16[c] * 16;
      uint8_t* fr = img.data() + (size_t)c * kChunkBytes;
      memcpy(fr + kChunkXrowOff, rec, kChunkXrowBytes);
      uint16_t ne, nr;
      memcpy(&ne, rec + kRecTotOff, 2);
      memcpy(&nr, rec + kRecTotOff + 2, 2);
      const uint8_t* pv = rec + kRecHdrBytes;
      const uint8_t* pn = pv + 4 * (size_t)ne;
      uint32_t* meta = (uint32_t*)(fr + kChunkValBytes);
      for (int w = 0; w < 128; ++w) meta[w] = 0;
      for (int r = 0; r < kPanelRows; ++r) {
        const uint8_t mask = rec[kRecMaskOff + r];
        uint32_t W = kMetaNone;
        if (mask) { memcpy(&W, pn, 4); pn += 4; }
        for (int g = 0; g < kChunkMB; ++g) {
          uint32_t v = 0;
          if (mask & (1u << g)) { memcpy(&v, pv, 4); pv += 4; }
          for (int slot = 0; slot < 2; ++slot) {
            const int k = 2 * g + slot;
            const uint16_t h = (uint16_t)(v >> (16 * slot));
            memcpy(fr + (r % 8) * 16 + (r / 8) * 256 + (k / 8) * 128 + (k % 8) * 2, &h, 2);
          }
          const int lane = (r % 8) + 8 * (g / 4) + 16 * (r / 16);
          meta[lane] |= ((W >> (4 * g)) & 0xFu) << (16 * ((r / 8) % 2) + 4 * (g % 4));
        }
      }
    }
    // canonical panel pc (Vp rows) = rows [(pc % ratio) * Vp, +Vp) of kernel panel pc / ratio,
    // whose chunks hold the meta-blocks of its canonical panels in canonical order
    for (int64_t pc = 0; pc < Pc; ++pc) {
      const int64_t p = pc / ratio;
      const int64_t kfirst = mbp[std::min(p * ratio, Pc)];
      const int r0 = (int)(pc % ratio) * (int)Vp;
      for (int64_t m = mbp[pc]; m < mbp[pc + 1]; ++m) {
        int64_t local = m - kfirst;
        int64_t c = chp[p] + local / kChunkMB;
        int g = (int)(local % kChunkMB);
        const uint8_t* cv = img.data() + (size_t)c * kChunkBytes;
        const uint32_t* cm = (const uint32_t*)(cv + kChunkValBytes);
        for (int rc = 0; rc < Vp; ++rc) {
          const int r = r0 + rc;
          int m0 = r % 8, m1 = (r / 8) % 2, m2 = r / 16, k1 = g / 4, q = g % 4;
          int lane = m0 + 8 * k1 + 16 * m2;
          uint32_t w = cm[lane];
          uint8_t nb = (uint8_t)((w >> (16 * m1 + 4 * q)) & 0xF);
          if (nib) nib[m * Vp + rc] = nb;
          if (vals) {
            for (int slot = 0; slot < 2; ++slot) {
              int k = 2 * g + slot;
              size_t off = (size_t)(r % 8) * 16 + (size_t)(r / 8) * 256 + (size_t)(k / 8) * 128 +
                           (size_t)(k % 8) * 2;
              uint16_t v;
              memcpy(&v, cv + off, 2);
              vals[(m * Vp + rc) * 2 + slot] = v;
            }
          }
        }
      }
    }
  }
  if (res_rowptr)
    NM_CUDA(cudaMemcpy(res_rowptr, P->res_rowptr, sizeof(int64_t) * (rows + 1),
                       cudaMemcpyDeviceToHost));
  if (res_col && P->res_nnz)
    NM_CUDA(cudaMemcpy(res_col, P->res_col, sizeof(int32_t) * P->res_nnz, cudaMemcpyDeviceToHost));
  if (res_val && P->res_nnz)
    NM_CUDA(cudaMemcpy(res_val, P->res_val, sizeof(uint16_t) * P->res_nnz, cudaMemcpyDeviceToHost));
  NM_CUDA(cudaSetDevice(cur));
  return NM_OK;
}

}  // extern "C"
