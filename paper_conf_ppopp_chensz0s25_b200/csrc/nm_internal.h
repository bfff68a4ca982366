// Internal declarations of libnm (not part of the ABI).  See include/nm.h for the contract
// and DESIGN.md §4-§5 for the data layouts.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>
#include <string>

#include "../../include/nm.h"

namespace nm {

// ---- packed device image ---------------------------------------------------
// One "chunk" = the operands of one tcgen05.mma.sp (M = 128, K = 32 logical): 8 consecutive
// meta-blocks of one panel.  Its image is
//   values : 128 rows x 16 physical 16-bit elements in the UMMA K-major no-swizzle canonical
//            layout: element (r, k) at (r%8)*16 + (r/8)*256 + (k/8)*128 + (k%8)*2 bytes,
//            physical k = 2*g + slot for meta-block g of the chunk (LBO = 128, SBO = 256);
//   meta   : 128 x 32-bit words in tensor-memory lane order: lane L = m0 + 8*k1 + 16*m2 holds
//            rows r0 = m0 + 16*m2 (bits 0-15) and r0 + 8 (bits 16-31) for K-half k1, the
//            nibble of group 4*k1+q at bit 4*q (layout measured on B200:
//            tools/probes/probe_umma_sp.b200.txt).
constexpr int kPanelRows = 128;   // Vp = MMA M
constexpr int kChunkMB = 8;       // meta-blocks per chunk (K = 32 logical / 4)
//   xrow   : 32 x int32, the row of X gathered for each logical k (meta-block g, selected
//            column j -> k = 4g + j); -1 = zero row (phantom or zero-count column: the TMA
//            gather fills it with zeros without reading memory).
// The record (4736 B) is moved by one cp.async.bulk per chunk.
constexpr int kChunkValBytes = 4096;
constexpr int kChunkMetaBytes = 512;
constexpr int kChunkXrowBytes = 128;
constexpr int kChunkBytes = kChunkValBytes + kChunkMetaBytes + kChunkXrowBytes;
constexpr int kChunkXrowOff = kChunkValBytes + kChunkMetaBytes;
constexpr uint32_t kMetaNone = 0x44444444u;  // every nibble = (0,1): legal code, zero values

}  // namespace nm

struct nm_packed {
  int device = 0;
  int64_t n = 0;                       // number of vertices (columns of B, rows of PX)
  int64_t row_begin = 0, row_end = 0;  // packed rows of B
  int V = 1, N = 2, M = 4, Vp = 128, Mp = 4;
  int tau = 0;                         // hybrid split threshold (0 = plain canonical pack)
  nm_dtype dtype = NM_F16;
  int64_t n_panels = 0, n_mb = 0, n_chunks = 0, packed_nnz = 0, res_nnz = 0;
  // device arrays
  int64_t* panel_mb_ptr = nullptr;     // [n_panels+1]
  int64_t* panel_chunk_ptr = nullptr;  // [n_panels+1]
  int4* unit_info = nullptr;           // [n_panels] schedule: {panel, #chunks, first chunk lo, hi}
  int32_t* mb_seg = nullptr;           // [n_mb]
  uint32_t* mb_sel = nullptr;          // [n_mb] byte j = sel[j]
  uint8_t* image = nullptr;            // [n_chunks * kChunkBytes] chunk records
  int64_t* res_rowptr = nullptr;       // [rows+1]
  int32_t* res_col = nullptr;          // [res_nnz] canonical (permuted) column
  uint16_t* res_val = nullptr;         // [res_nnz]
  // NM_PACK_ORIGINAL_ORDER: xrow holds original vertex ids, plus
  int flags = 0;
  int32_t* row_map = nullptr;          // [rows] output row of Y = perm[row_begin + l]
  int32_t* res_gather = nullptr;       // [res_nnz] X row to gather = perm[res_col]
  size_t device_bytes = 0;
};

namespace nm {

// error plumbing
void set_error(const std::string& msg);
nm_status fail(nm_status s, const std::string& msg);
nm_status cuda_fail(cudaError_t e, const char* what);

#define NM_CUDA(call)                                     \
  do {                                                    \
    cudaError_t e_ = (call);                              \
    if (e_ != cudaSuccess) return nm::cuda_fail(e_, #call); \
  } while (0)

// host-side CSR validation (sorted, in range, no duplicates; optional symmetry check)
nm_status validate_csr_host(int64_t n, const int64_t* rp, const int32_t* ci, bool check_sym);

// A copy of a CSR on the device (owning), uploaded from host or device memory.
struct DevCsr {
  int64_t n = 0, nnz = 0;
  int64_t* rp = nullptr;
  int32_t* ci = nullptr;
  uint16_t* val = nullptr;  // 16-bit bits in the pack dtype (nullptr = all ones)
  void release();
  ~DevCsr() { release(); }
};
nm_status upload_csr(const nm_csr* A, nm_dtype dtype, DevCsr* out, cudaStream_t s);

// host copy of a CSR's structure (for the host reorder)
nm_status host_csr(const nm_csr* A, int64_t** rp, int32_t** ci);

uint16_t one_bits(nm_dtype dt);

// kernels launched from other translation units
nm_status launch_spmm_sptc(const nm_packed* P, const void* PX, int64_t ldx, float* Yp,
                           int64_t ldy, int F, cudaStream_t s);
nm_status launch_spmm_residual(const nm_packed* P, const void* PX, int64_t ldx, float* Yp,
                               int64_t ldy, int F, cudaStream_t s);
nm_status count_violations_dev(const DevCsr& A, const int32_t* perm_dev, int V, int N, int M,
                               int64_t* omega, int64_t* mb, int32_t* pscore_host,
                               cudaStream_t s);

}  // namespace nm
