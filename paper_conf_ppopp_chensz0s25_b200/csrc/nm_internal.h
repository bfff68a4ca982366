// Internal declarations of libnm (not part of the ABI).  See include/nm.h for the contract
// and DESIGN.md §4-§5 for the data layouts.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <exception>
#include <new>
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

// ---- compressed chunk record in HBM (the "SPTC required form on the fly" of L492) ----------
// The MMA operands above are what the tensor core reads from shared memory; in HBM a chunk is
// stored without its empty (row, meta-block) slots and the SpMM's loader warps expand it in
// shared memory.  (row r, group g) is empty iff its nibble is the no-value code 0x4 and both
// value slots are +0 bits.  Layout (variable size, padded to 16 bytes):
//   [  0..128) xrow  int32[32]  gather row per logical k (as in the full record)
//   [128..256) mask  uint8[128] bit g of row r = (r, g) not empty
//   [256..264) qv    uint16[4]  first value entry of each 32-row quarter
//   [264..272) qn    uint16[4]  first nibble word of each 32-row quarter
//   [272..276) ne, nr uint16    #value entries, #non-empty rows
//   [276]      cmask uint8     bit q: gather rows 8q..8q+7 are 8 consecutive rows of X (one
//                               TMA tile load instead of 8 row gathers);  [277..288) zero
//   [288 ..  ) vals  uint32[ne] slot0 | slot1 << 16 per non-empty (r, g), row-major
//   then       nibs  uint32[nr] nibble word of each non-empty row (group g at bits 4g)
constexpr int kRecMaskOff = 128, kRecQvOff = 256, kRecQnOff = 264, kRecTotOff = 272, kRecContOff = 276;
constexpr int kRecHdrBytes = 288;
constexpr int kRecMaxBytes = kRecHdrBytes + 4 * (kPanelRows + kPanelRows * kChunkMB);  // 4896

// Residual work items (DESIGN.md §6 k_residual): each row's residual nonzeros are cut into
// items of at most kResSeg entries, one warp subgroup each, so hub rows of power-law graphs
// spread over many subgroups.  A row cut into several items ("split row") combines their
// partial sums deterministically: each item writes its partial to its workspace slot and the
// last one to finish (per-row arrival counter) adds all partials in item order into Y.  The
// workspace and the counters are allocated per nm_spmm call, stream-ordered (launch time),
// never stored in the handle -- the packed matrix stays immutable, so concurrent calls on one
// handle are safe.
#ifdef __CUDACC__
// The stage sequence of one CTA of the persistent tensor-core kernels: for each panel of its
// range, for each F tile, the panel's chunks CPS at a time (panels without chunks have no
// stages).  The gather groups own every G-th stage; advance(G) steps G stages.
template <int CPS>
struct StageIter {
  int pn, pz, ft, nft, c, nch;
  int64_t c0, c1;
  const int64_t* pcp;
  __device__ __forceinline__ void init(const int64_t* panel_chunk_ptr, int pa, int pz_, int nft_) {
    pcp = panel_chunk_ptr;
    pn = pa;
    pz = pz_;
    ft = 0;
    nft = nft_;
    c = 0;
    nch = 0;
    c0 = c1 = pa < pz_ ? __ldg(pcp + pa) : 0;
    load_panel();
  }
  __device__ __forceinline__ bool valid() const { return pn < pz; }
  __device__ __forceinline__ void load_panel() {
    while (pn < pz) {
      c1 = __ldg(pcp + pn + 1);
      nch = (int)(c1 - c0);
      if (nch > 0) return;
      ++pn;
      c0 = c1;
    }
  }
  __device__ __forceinline__ void next() {
    c += CPS;
    if (c < nch) return;
    c = 0;
    if (++ft < nft) return;
    ft = 0;
    ++pn;
    c0 = c1;
    load_panel();
  }
  __device__ __forceinline__ void advance(int g) {
    for (int k = 0; k < g && pn < pz; ++k) next();
  }
};
#endif

constexpr int kResSeg = 256;   // max residual nonzeros per work item
constexpr int kResSlab = 256;  // features per residual launch (partial-sum slot width)
struct ResSeg {
  int64_t kb;        // first residual entry
  int32_t row, len;  // packed row (local), #entries
  int32_t slot;      // first workspace slot of the row's partials, -1 = single-item row
  int32_t split_id;  // arrival counter of the row (split rows only)
  int32_t nseg, idx; // items of the row, index of this one
  int32_t yrow;      // output row of Y (row_map applied in NM_PACK_ORIGINAL_ORDER)
  int32_t pad;
};
static_assert(sizeof(ResSeg) == 40, "ResSeg layout");

}  // namespace nm

struct nm_packed {
  int device = 0;
  int64_t n = 0;                       // number of vertices (columns of B, rows of PX)
  int64_t row_begin = 0, row_end = 0;  // packed rows of B
  int V = 1, N = 2, M = 4, Vp = 128, Mp = 4;
  int tau = 0;                         // hybrid split threshold (0 = plain canonical pack)
  nm_dtype dtype = NM_F16;
  // n_panels: kernel panels of kPanelRows (= MMA M = 128) rows; n_cpanels: canonical panels of
  // Vp rows (Vp = 64: two per kernel panel, their meta-blocks share its chunks)
  int64_t n_panels = 0, n_cpanels = 0, n_mb = 0, n_chunks = 0, packed_nnz = 0, res_nnz = 0;
  // device arrays
  int64_t* panel_mb_ptr = nullptr;     // [n_cpanels+1] first meta-block of each canonical panel
  int64_t* panel_chunk_ptr = nullptr;  // [n_panels+1] first chunk of each kernel panel
  int4* unit_info = nullptr;           // [2 * n_panels] schedule: {panel, #chunks, first chunk lo, hi},
                                       //   {record byte offset lo, hi, record bytes lo, hi}
  uint16_t* rec_len16 = nullptr;       // [n_chunks] compressed record size / 16
  int64_t image_bytes = 0;             // compressed image size
  int32_t* mb_seg = nullptr;           // [n_mb]
  uint32_t* mb_sel = nullptr;          // [n_mb] byte j = sel[j]
  uint8_t* image = nullptr;            // compressed chunk records (kRec* layout), image_bytes
  uint8_t* image_full = nullptr;       // full chunk records (kChunkBytes each, chunk order)
  int32_t* cta_ptr = nullptr;          // [n_ctas+1] contiguous panel range of each SpMM CTA
  int n_ctas = 0;                      // persistent grid of the full-record kernel (#SMs)
  int sptc_format = 1;                 // tensor-core kernel nm_spmm uses: 1 full, 2 compressed, 3 compressed + A in TMEM
  int64_t gather_rows = 0;             // non-negative gather rows over all chunks
  int64_t* res_rowptr = nullptr;       // [rows+1]
  int32_t* res_col = nullptr;          // [res_nnz] canonical (permuted) column
  uint16_t* res_val = nullptr;         // [res_nnz]
  // NM_PACK_ORIGINAL_ORDER: xrow holds original vertex ids, plus
  int flags = 0;
  int32_t* row_map = nullptr;          // [rows] output row of Y = perm[row_begin + l]
  int32_t* res_gather = nullptr;       // [res_nnz] X row to gather = perm[res_col]
  // residual work list (kResSeg-entry items, longest first); the split rows' partial-sum
  // workspace (n_res_slots x kResSlab floats) and arrival counters (n_res_split) are allocated
  // by each nm_spmm call on its stream
  nm::ResSeg* res_segs = nullptr;      // [n_res_segs]
  int64_t n_res_segs = 0, n_res_slots = 0, n_res_split = 0;
  size_t device_bytes = 0;
};

namespace nm {

// error plumbing
void set_error(const std::string& msg);
nm_status fail(nm_status s, const std::string& msg);
nm_status cuda_fail(cudaError_t e, const char* what);

#define NM_TRY_STATUS(x)             \
  do {                               \
    nm_status st_try_ = (x);         \
    if (st_try_ != NM_OK) return st_try_; \
  } while (0)

#define NM_CUDA(call)                                     \
  do {                                                    \
    cudaError_t e_ = (call);                              \
    if (e_ != cudaSuccess) return nm::cuda_fail(e_, #call); \
  } while (0)

// exception guard for the extern "C" entry points: no C++ exception crosses the ABI
// (std::vector / std::bad_alloc in the host stages, CUB temporaries); nm.h promises status codes
template <typename Fn>
nm_status guarded(const char* what, Fn&& f) {
  try {
    return f();
  } catch (const std::bad_alloc&) {
    return fail(NM_ERR_OOM, std::string(what) + ": host allocation failed");
  } catch (const std::exception& e) {
    return fail(NM_ERR_CUDA, std::string(what) + ": " + e.what());
  } catch (...) {
    return fail(NM_ERR_CUDA, std::string(what) + ": unknown exception");
  }
}

// stream-ordered scratch of the offline stages (reorder Stage-1, counts).  While a ScopedPool
// is alive on this thread the allocations come from its private pool (kept reserved between
// the reorder's iterations and destroyed with it -- the device's default pool, which other
// users such as PyTorch's cudaMallocAsync backend share, is never reconfigured); otherwise
// from the current device's default pool.
nm_status scratch_alloc(void** p, size_t bytes, cudaStream_t s);
struct ScopedPool {
  cudaMemPool_t pool = nullptr, prev = nullptr;
  nm_status init(int device);
  ~ScopedPool();
};

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
nm_status launch_spmm_sptc(const nm_packed* P, const void* PX, int64_t ldx, float* Yp, int64_t ldy,
                           int F, cudaStream_t s, int format);
// fused epilogue of the full-record kernel: out16[row * ldo + col] = 16-bit act(Y + bias)
struct FusedAct {
  void* out16;
  int64_t ldo;
  const float* bias;
  int relu;
};
nm_status launch_spmm_sptc_full(const nm_packed* P, const void* PX, int64_t ldx, float* Yp,
                                int64_t ldy, int F, cudaStream_t s, const FusedAct* fa = nullptr);
nm_status launch_spmm_sptc_compressed(const nm_packed* P, const void* PX, int64_t ldx, float* Yp,
                                      int64_t ldy, int F, cudaStream_t s);
nm_status launch_spmm_sptc_tm(const nm_packed* P, const void* PX, int64_t ldx, float* Yp,
                              int64_t ldy, int F, cudaStream_t s);
nm_status launch_spmm_residual(const nm_packed* P, const void* PX, int64_t ldx, float* Yp,
                               int64_t ldy, int F, cudaStream_t s);
nm_status gemm_rm(const void* A, int64_t lda, const void* W, int64_t ldw, void* C, int64_t ldc, int64_t m, int k,
                  int nc, nm_dtype dt, bool c_f32, void* ws, cudaStream_t s);
size_t lt_workspace_bytes();
nm_status count_violations_dev(const DevCsr& A, const int32_t* perm_dev, int V, int N, int M,
                               int64_t* omega, int64_t* mb, int32_t* pscore_host,
                               cudaStream_t s);
nm_status stage1_sort_dev(const DevCsr& A, int32_t* perm_dev, int N, int M, cudaStream_t s);

// Stage-2 gain tables on the device (reorder_gpu.cu): the tables of a primary segment against a
// batch of targets, entry layout as the host's gain_table (2 int64 per (u, v), u-major).
struct S2DeviceTables;
nm_status s2dev_create(const DevCsr& A, int M, int max_batch, cudaStream_t s, S2DeviceTables** out);
nm_status s2dev_set_perm(S2DeviceTables* t, const int32_t* perm_host);
nm_status s2dev_tables(S2DeviceTables* t, int64_t p, const int64_t* targets, int nb, int N, int64_t* tabs_out);
void s2dev_destroy(S2DeviceTables* t);

}  // namespace nm
