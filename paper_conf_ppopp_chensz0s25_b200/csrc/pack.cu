// nm_pack / nm_pack_rows: the sm_100a V:N:M packer (SPTC form of PAPER.md:L492).
//
//  1. B = P A P^T for the requested row range (row gather + column relabel + radix sort).
//  2. Meta-blocks = distinct (panel, segment) pairs with any nonzero, ascending (radix sort +
//     run-length encode of panel*S + col/Mp keys).
//  3. Column counts per meta-block -> the k = 4 selected columns (vertical constraint,
//     L226-227): largest counts, ties to the smaller offset, ascending.
//  4. Per (row, meta-block): the first <= 2 nonzeros among the selected columns (horizontal
//     constraint, N = 2) go to the two MMA slots with a 4-bit index pair; the rest to the
//     residual CSR.  Values and metadata are written straight into the MMA-native image.
#include <cub/cub.cuh>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>
#include <numeric>
#include <vector>

#include "nm_internal.h"

namespace nm {
namespace {

constexpr int kWarp = 32;

// byte offset of element (r, k) inside a chunk's value block (UMMA K-major no swizzle,
// LBO = 128 B between the two 8-element K chunks, SBO = 256 B between 8-row groups)
__host__ __device__ inline uint32_t val_off(int r, int k) {
  return (uint32_t)((r & 7) * 16 + (r >> 3) * 256 + (k >> 3) * 128 + (k & 7) * 2);
}
// tensor-memory lane word and bit shift of the nibble of row r, meta-block g of a chunk
__host__ __device__ inline void meta_pos(int r, int g, int* word, int* shift) {
  int m0 = r & 7, m1 = (r >> 3) & 1, m2 = r >> 4, k1 = g >> 2, q = g & 3;
  *word = m0 + 8 * k1 + 16 * m2;
  *shift = 16 * m1 + 4 * q;
}

__global__ void k_iperm(const int32_t* __restrict__ perm, int32_t* __restrict__ iperm, int64_t n) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x)
    iperm[perm[p]] = (int32_t)p;
}

__global__ void k_identity(int32_t* __restrict__ perm, int64_t n) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x)
    perm[p] = (int32_t)p;
}

// deg[l] = degree of B row rb + l
__global__ void k_row_deg(const int64_t* __restrict__ rp, const int32_t* __restrict__ perm,
                          int64_t rb, int64_t rows, int64_t* __restrict__ deg) {
  for (int64_t l = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; l < rows;
       l += (int64_t)gridDim.x * blockDim.x) {
    int32_t u = perm[rb + l];
    deg[l] = rp[u + 1] - rp[u];
  }
}

// key = local_row << 32 | new_col, value = 16-bit value bits (warp per row)
__global__ void k_fill_keys(const int64_t* __restrict__ rp, const int32_t* __restrict__ ci,
                            const uint16_t* __restrict__ val, uint16_t one,
                            const int32_t* __restrict__ perm, const int32_t* __restrict__ iperm,
                            int64_t rb, int64_t rows, const int64_t* __restrict__ Brp,
                            uint64_t* __restrict__ key, uint16_t* __restrict__ v16) {
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / kWarp;
  int lane = threadIdx.x % kWarp;
  int64_t nw = (int64_t)gridDim.x * blockDim.x / kWarp;
  for (int64_t l = warp; l < rows; l += nw) {
    int32_t u = perm[rb + l];
    int64_t s = rp[u], d = rp[u + 1] - s, o = Brp[l];
    for (int64_t k = lane; k < d; k += kWarp) {
      key[o + k] = ((uint64_t)l << 32) | (uint32_t)iperm[ci[s + k]];
      v16[o + k] = val ? val[s + k] : one;
    }
  }
}

__global__ void k_split_keys(const uint64_t* __restrict__ key, int32_t* __restrict__ Bci,
                             int64_t nnz) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nnz;
       k += (int64_t)gridDim.x * blockDim.x)
    Bci[k] = (int32_t)(key[k] & 0xFFFFFFFFu);
}

// meta-block key of every entry: (Vp-row panel) * S + col / Mp (warp per row)
__global__ void k_mbkey(const int64_t* __restrict__ Brp, const int32_t* __restrict__ Bci,
                        int64_t rows, int Vp, int Mp, int64_t S, int64_t* __restrict__ key) {
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / kWarp;
  int lane = threadIdx.x % kWarp;
  int64_t nw = (int64_t)gridDim.x * blockDim.x / kWarp;
  for (int64_t l = warp; l < rows; l += nw) {
    int64_t panel = l / Vp;
    for (int64_t k = Brp[l] + lane; k < Brp[l + 1]; k += kWarp)
      key[k] = panel * S + Bci[k] / Mp;
  }
}

__device__ inline int64_t lower_bound64(const int64_t* __restrict__ a, int64_t n, int64_t x) {
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    int64_t mid = (lo + hi) >> 1;
    if (a[mid] < x) lo = mid + 1; else hi = mid;
  }
  return lo;
}

// panel_mb_ptr[r] = first meta-block of panel r; chunk counts per panel
__global__ void k_panel_ptr(const int64_t* __restrict__ mbkey, int64_t n_mb, int64_t P,
                            int64_t S, int64_t* __restrict__ mbp, int64_t* __restrict__ nchunk) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r <= P;
       r += (int64_t)gridDim.x * blockDim.x) {
    mbp[r] = lower_bound64(mbkey, n_mb, r * S);
  }
}

// first meta-block of kernel panel R (kPanelRows rows = `ratio` canonical panels of Vp rows)
__device__ __forceinline__ int64_t kpanel_mb(const int64_t* __restrict__ mbp, int64_t R, int ratio, int64_t Pc) {
  const int64_t c = R * ratio;
  return mbp[c < Pc ? c : Pc];
}

// chunks of every kernel panel: its meta-blocks (those of its `ratio` canonical panels, in
// canonical order), kChunkMB per chunk
__global__ void k_chunk_counts(const int64_t* __restrict__ mbp, int64_t P, int ratio, int64_t Pc,
                               int64_t* __restrict__ nchunk) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < P;
       r += (int64_t)gridDim.x * blockDim.x)
    nchunk[r] = (kpanel_mb(mbp, r + 1, ratio, Pc) - kpanel_mb(mbp, r, ratio, Pc) + kChunkMB - 1) / kChunkMB;
}

__global__ void k_meta_init(uint8_t* __restrict__ image, int64_t n_chunks) {
  int64_t total = n_chunks * (kChunkMetaBytes / 4);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total;
       i += (int64_t)gridDim.x * blockDim.x) {
    int64_t c = i / (kChunkMetaBytes / 4), w = i % (kChunkMetaBytes / 4);
    ((uint32_t*)(image + c * kChunkBytes + kChunkValBytes))[w] = kMetaNone;
  }
}

// perm == nullptr: initialise every record's xrow to -1; else map xrow entries through perm
__global__ void k_count_gather(const uint8_t* __restrict__ image, int64_t n_chunks,
                               unsigned long long* __restrict__ total) {
  unsigned long long c = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n_chunks * 32; i += (int64_t)gridDim.x * blockDim.x)
    c += ((const int32_t*)(image + (i >> 5) * kChunkBytes + kChunkXrowOff))[i & 31] >= 0;
  for (int o = 16; o > 0; o >>= 1) c += __shfl_down_sync(0xffffffffu, c, o);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(total, c);
}

__global__ void k_xrow_map(const int32_t* __restrict__ perm, uint8_t* __restrict__ image, int64_t n_chunks) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n_chunks * 32;
       i += (int64_t)gridDim.x * blockDim.x) {
    int32_t* x = (int32_t*)(image + (i >> 5) * kChunkBytes + kChunkXrowOff) + (i & 31);
    if (!perm) *x = -1;
    else if (*x >= 0) *x = perm[*x];
  }
}

// per-entry meta-block id and column counts (warp per row)
__global__ void k_colcount(const int64_t* __restrict__ Brp, const int32_t* __restrict__ Bci,
                           int64_t rows, int Vp, int Mp, int64_t S, const int64_t* __restrict__ mbkey,
                           int64_t n_mb, int32_t* __restrict__ cnt, int64_t* __restrict__ emb) {
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / kWarp;
  int lane = threadIdx.x % kWarp;
  int64_t nw = (int64_t)gridDim.x * blockDim.x / kWarp;
  for (int64_t l = warp; l < rows; l += nw) {
    int64_t panel = l / Vp;
    for (int64_t k = Brp[l] + lane; k < Brp[l + 1]; k += kWarp) {
      int64_t s = Bci[k] / Mp;
      int64_t m = lower_bound64(mbkey, n_mb, panel * S + s);
      emb[k] = m;
      atomicAdd(&cnt[m * Mp + (Bci[k] - s * Mp)], 1);
    }
  }
}

// selected columns of every candidate meta-block: the 4 largest counts, ties -> smaller
// offset, stored ascending (vertical constraint, L226-227; reading #19)
__global__ void k_select(const int32_t* __restrict__ cnt, int Mp, int64_t n_mb, uint32_t* __restrict__ selc) {
  for (int64_t m = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; m < n_mb;
       m += (int64_t)gridDim.x * blockDim.x) {
    const int32_t* c = cnt + m * Mp;
    int sel[4];
    if (Mp == 4) {
      sel[0] = 0; sel[1] = 1; sel[2] = 2; sel[3] = 3;
    } else {
      uint32_t taken = 0;
      for (int t = 0; t < 4; ++t) {
        int bj = -1;
        for (int j = 0; j < Mp; ++j) {
          if (taken & (1u << j)) continue;
          if (bj < 0 || c[j] > c[bj]) bj = j;
        }
        taken |= 1u << bj;
        sel[t] = bj;
      }
      // ascending
      for (int a = 0; a < 4; ++a)
        for (int b = a + 1; b < 4; ++b)
          if (sel[b] < sel[a]) { int t = sel[a]; sel[a] = sel[b]; sel[b] = t; }
    }
    selc[m] = (uint32_t)sel[0] | ((uint32_t)sel[1] << 8) | ((uint32_t)sel[2] << 16) | ((uint32_t)sel[3] << 24);
  }
}

// index of column `col` (segment s) in the selection, -1 if not selected
__device__ __forceinline__ int sel_index(uint32_t sel, int32_t col, int64_t s, int Mp) {
  const int off = col - (int)(s * Mp);
  for (int j = 0; j < 4; ++j)
    if ((int)((sel >> (8 * j)) & 0xFF) == off) return j;
  return -1;
}

// rank of entry k among the selected entries of its (row, segment) group, the group's
// first two selected entries (ja/ka, jb) -- the group is contiguous and at most Mp long
struct GroupPick {
  int jk, rank, ja, jb;
  int64_t ka;
};
__device__ __forceinline__ GroupPick group_pick(const int32_t* __restrict__ Bci, int64_t b, int64_t e, int64_t k,
                                                int Mp, uint32_t sel) {
  const int32_t col = Bci[k];
  const int64_t s = col / Mp;
  int64_t gs = k;
  while (gs > b && Bci[gs - 1] / Mp == s) --gs;
  int64_t ge = k + 1;
  while (ge < e && Bci[ge] / Mp == s) ++ge;
  GroupPick g{sel_index(sel, col, s, Mp), 0, -1, -1, -1};
  for (int64_t t = gs; t < ge; ++t) {
    const int jt = sel_index(sel, Bci[t], s, Mp);
    if (jt < 0) continue;
    if (t < k) ++g.rank;
    if (g.ja < 0) { g.ja = jt; g.ka = t; }
    else if (g.jb < 0) { g.jb = jt; }
  }
  return g;
}

// hybrid split (reading #27): values each candidate meta-block would keep
// (per row min(2, entries in its selected columns)), one thread per entry
__global__ void k_keep_count(const int64_t* __restrict__ Brp, const int32_t* __restrict__ Bci, int64_t rows,
                             int Mp, const int64_t* __restrict__ emb, const uint32_t* __restrict__ selc,
                             int32_t* __restrict__ keptc) {
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / kWarp;
  int lane = threadIdx.x % kWarp;
  int64_t nw = (int64_t)gridDim.x * blockDim.x / kWarp;
  for (int64_t l = warp; l < rows; l += nw) {
    const int64_t b = Brp[l], e = Brp[l + 1];
    for (int64_t k = b + lane; k < e; k += kWarp) {
      const GroupPick g = group_pick(Bci, b, e, k, Mp, selc[emb[k]]);
      if (g.jk >= 0 && g.rank < 2) atomicAdd(&keptc[emb[k]], 1);
    }
  }
}

__global__ void k_survive(const int32_t* __restrict__ keptc, int64_t n, int tau, int64_t* __restrict__ flag) {
  for (int64_t m = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; m < n; m += (int64_t)gridDim.x * blockDim.x)
    flag[m] = keptc[m] >= tau ? 1 : 0;
}

// compaction of the surviving candidates (newid = exclusive scan of the survive flags)
__global__ void k_compact(const int64_t* __restrict__ flag, const int64_t* __restrict__ newid, int64_t n,
                          const int64_t* __restrict__ key_in, const uint32_t* __restrict__ sel_in,
                          int64_t* __restrict__ key_out, uint32_t* __restrict__ sel_out,
                          int64_t* __restrict__ cand_of) {
  for (int64_t m = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; m < n; m += (int64_t)gridDim.x * blockDim.x) {
    if (!flag[m]) continue;
    const int64_t d = newid[m];
    key_out[d] = key_in[m];
    sel_out[d] = sel_in[m];
    cand_of[d] = m;
  }
}

__global__ void k_remap_emb(const int64_t* __restrict__ flag, const int64_t* __restrict__ newid,
                            int64_t* __restrict__ emb, int64_t nnz) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nnz; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t m = emb[k];
    emb[k] = flag[m] ? newid[m] : -1;
  }
}

// per emitted meta-block: segment id, selection and the X row of each logical k
__global__ void k_write_sel(const int32_t* __restrict__ cnt, const int64_t* __restrict__ cand_of, int Mp,
                            int64_t n_mb, const int64_t* __restrict__ mbkey, int64_t S, int64_t n,
                            const int64_t* __restrict__ mbp, int ratio, int64_t Pc,
                            const int64_t* __restrict__ chp,
                            int32_t* __restrict__ mb_seg, uint32_t* __restrict__ mb_sel,
                            uint8_t* __restrict__ image) {
  for (int64_t m = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; m < n_mb;
       m += (int64_t)gridDim.x * blockDim.x) {
    const int64_t panel = mbkey[m] / S / ratio, s = mbkey[m] % S;  // kernel panel
    mb_seg[m] = (int32_t)s;
    const uint32_t sel = mb_sel[m];
    const int32_t* c = cnt + (cand_of ? cand_of[m] : m) * Mp;
    const int64_t local = m - kpanel_mb(mbp, panel, ratio, Pc);
    const int64_t chunk = chp[panel] + local / kChunkMB;
    const int g = (int)(local % kChunkMB);
    int32_t* xrow = (int32_t*)(image + chunk * kChunkBytes + kChunkXrowOff);
    for (int j = 0; j < 4; ++j) {
      const int off = (int)((sel >> (8 * j)) & 0xFF);
      const int64_t col = s * Mp + off;
      // zero-count or phantom columns gather nothing (zero-filled operand rows)
      xrow[g * 4 + j] = (col < n && c[off] > 0) ? (int32_t)col : -1;
    }
  }
}

// Places every entry: MMA slot (value + nibble) or residual flag.  One thread per entry; the
// entry inspects its (row, segment) group, which is contiguous and at most Mp long.  Entries
// of a meta-block dropped by the hybrid split (emb < 0) all go to the residual.
__global__ void k_place(const int64_t* __restrict__ Brp, const int32_t* __restrict__ Bci,
                        const uint16_t* __restrict__ Bval, int64_t rows, int Mp,
                        const int64_t* __restrict__ emb, const uint32_t* __restrict__ mb_sel,
                        const int64_t* __restrict__ mbp, int ratio, int64_t Pc,
                        const int64_t* __restrict__ chp, uint8_t* __restrict__ image, uint8_t* __restrict__ resflag,
                        unsigned long long* __restrict__ kept_count) {
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / kWarp;
  int lane = threadIdx.x % kWarp;
  int64_t nw = (int64_t)gridDim.x * blockDim.x / kWarp;
  for (int64_t l = warp; l < rows; l += nw) {
    int64_t b = Brp[l], e = Brp[l + 1];
    for (int64_t k = b + lane; k < e; k += kWarp) {
      const int64_t m = emb[k];
      if (m < 0) { resflag[k] = 1; continue; }
      const GroupPick gp = group_pick(Bci, b, e, k, Mp, mb_sel[m]);
      bool kept = gp.jk >= 0 && gp.rank < 2;
      resflag[k] = kept ? 0 : 1;
      if (!kept) continue;
      atomicAdd(kept_count, 1ull);
      // kernel panel (at Vp = 64 its other 64-row half keeps no-value nibbles in this k-group)
      int64_t panel = l / kPanelRows;
      int64_t local = m - kpanel_mb(mbp, panel, ratio, Pc);
      int64_t chunk = chp[panel] + local / kChunkMB;
      int g = (int)(local % kChunkMB);
      int r = (int)(l % kPanelRows);
      uint8_t* cv = image + chunk * kChunkBytes;
      // slot assignment (reading #19): two kept (a<b) -> (a,b) slots 0,1; one kept
      // at j<3 -> (j,3) slot 0; one kept at j=3 -> (0,3) slot 1
      int i0, i1, slot;
      if (gp.jb >= 0) { i0 = gp.ja; i1 = gp.jb; slot = (k == gp.ka) ? 0 : 1; }
      else if (gp.ja < 3) { i0 = gp.ja; i1 = 3; slot = 0; }
      else { i0 = 0; i1 = 3; slot = 1; }
      *(uint16_t*)(cv + val_off(r, 2 * g + slot)) = Bval[k];
      if (k == gp.ka) {
        int w, sh;
        meta_pos(r, g, &w, &sh);
        uint32_t nib = (uint32_t)(i0 | (i1 << 2));
        atomicXor((uint32_t*)(cv + kChunkValBytes) + w, (nib ^ 0x4u) << sh);
      }
    }
  }
}

__global__ void k_res_count(const int64_t* __restrict__ Brp, const uint8_t* __restrict__ resflag,
                            int64_t rows, int64_t* __restrict__ rc) {
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / kWarp;
  int lane = threadIdx.x % kWarp;
  int64_t nw = (int64_t)gridDim.x * blockDim.x / kWarp;
  for (int64_t l = warp; l < rows; l += nw) {
    int64_t c = 0;
    for (int64_t k = Brp[l] + lane; k < Brp[l + 1]; k += kWarp) c += resflag[k];
    for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    if (lane == 0) rc[l] = c;
  }
}

__global__ void k_res_fill(const int64_t* __restrict__ Brp, const int32_t* __restrict__ Bci,
                           const uint16_t* __restrict__ Bval, const uint8_t* __restrict__ resflag,
                           int64_t rows, const int64_t* __restrict__ rrp,
                           int32_t* __restrict__ rci, uint16_t* __restrict__ rval) {
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / kWarp;
  int lane = threadIdx.x % kWarp;
  int64_t nw = (int64_t)gridDim.x * blockDim.x / kWarp;
  for (int64_t l = warp; l < rows; l += nw) {
    int64_t o = rrp[l];
    for (int64_t base = Brp[l]; base < Brp[l + 1]; base += kWarp) {
      int64_t k = base + lane;
      int f = (k < Brp[l + 1]) ? resflag[k] : 0;
      unsigned mask = __ballot_sync(0xffffffffu, f);
      if (f) {
        int pos = __popc(mask & ((1u << lane) - 1));
        rci[o + pos] = Bci[k];
        rval[o + pos] = Bval[k];
      }
      o += __popc(mask);
    }
  }
}

// Compression of the full chunk records into the HBM form (nm_internal.h kRec* layout).
// One 128-thread block per chunk, thread r = row r.  WRITE = false: record sizes only.
template <bool WRITE>
__global__ void __launch_bounds__(128) k_compress(const uint8_t* __restrict__ full, int64_t n_chunks,
                                                  int64_t* __restrict__ size16, const int64_t* __restrict__ off,
                                                  uint8_t* __restrict__ out) {
  __shared__ int s_ne[4], s_nr[4];
  const int r = threadIdx.x, lane = r & 31, q = r >> 5;
  for (int64_t c = blockIdx.x; c < n_chunks; c += gridDim.x) {
    const uint8_t* rec = full + c * kChunkBytes;
    const uint32_t* meta = (const uint32_t*)(rec + kChunkValBytes);
    uint32_t vals[kChunkMB];
    uint32_t W = 0, mask = 0;
#pragma unroll
    for (int g = 0; g < kChunkMB; ++g) {
      const uint32_t v0 = *(const uint16_t*)(rec + val_off(r, 2 * g));
      const uint32_t v1 = *(const uint16_t*)(rec + val_off(r, 2 * g + 1));
      int w, sh;
      meta_pos(r, g, &w, &sh);
      const uint32_t nb = (meta[w] >> sh) & 0xFu;
      W |= nb << (4 * g);
      vals[g] = v0 | (v1 << 16);
      if (!(nb == 0x4u && v0 == 0 && v1 == 0)) mask |= 1u << g;
    }
    const int ne = __popc(mask), nr = mask != 0;
    int ve = ne, vn = nr;  // inclusive warp scans
    for (int o = 1; o < 32; o <<= 1) {
      const int a = __shfl_up_sync(0xffffffffu, ve, o), b = __shfl_up_sync(0xffffffffu, vn, o);
      if (lane >= o) { ve += a; vn += b; }
    }
    if (lane == 31) { s_ne[q] = ve; s_nr[q] = vn; }
    __syncthreads();
    int qv = 0, qn = 0, NE = 0, NR = 0;
    for (int j = 0; j < 4; ++j) {
      if (j < q) { qv += s_ne[j]; qn += s_nr[j]; }
      NE += s_ne[j];
      NR += s_nr[j];
    }
    const int bytes = (kRecHdrBytes + 4 * (NE + NR) + 15) & ~15;
    if (!WRITE) {
      if (r == 0) size16[c] = bytes / 16;
    } else {
      uint8_t* dst = out + off[c];
      if (r < 32) ((int32_t*)dst)[r] = ((const int32_t*)(rec + kChunkXrowOff))[r];
      dst[kRecMaskOff + r] = (uint8_t)mask;
      if (lane == 0) {
        ((uint16_t*)(dst + kRecQvOff))[q] = (uint16_t)qv;
        ((uint16_t*)(dst + kRecQnOff))[q] = (uint16_t)qn;
      }
      if (r < 4) ((uint32_t*)(dst + kRecTotOff))[r] = r == 0 ? ((uint32_t)NE | ((uint32_t)NR << 16)) : 0u;
      __syncthreads();  // the zeroed header word above before the contiguity byte below
      if (r < 4) {  // gather rows 8r..8r+7 consecutive rows of X?
        const int32_t* xr = (const int32_t*)(rec + kChunkXrowOff) + 8 * r;
        bool cont = xr[0] >= 0;
        for (int j = 1; j < 8; ++j) cont = cont && xr[j] == xr[0] + j;
        if (cont) atomicOr((unsigned int*)(dst + kRecTotOff + 4), 1u << r);
      }
      uint32_t* dv = (uint32_t*)(dst + kRecHdrBytes);
      int e = qv + ve - ne;  // exclusive offset of this row's first entry
#pragma unroll
      for (int g = 0; g < kChunkMB; ++g)
        if (mask & (1u << g)) dv[e++] = vals[g];
      if (nr) dv[NE + qn + vn - 1] = W;
      const int used = kRecHdrBytes + 4 * (NE + NR);
      if (r < (bytes - used) / 4) ((uint32_t*)(dst + used))[r] = 0u;  // padding
    }
    __syncthreads();
  }
}

// residual work list: per row #segments, #partial slots (split rows only), split flag
__global__ void k_seg_count(const int64_t* __restrict__ rrp, int64_t rows, int64_t* __restrict__ nseg,
                            int64_t* __restrict__ nslot, int64_t* __restrict__ nsplit) {
  for (int64_t l = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; l < rows; l += (int64_t)gridDim.x * blockDim.x) {
    const int64_t len = rrp[l + 1] - rrp[l];
    const int64_t k = (len + kResSeg - 1) / kResSeg;
    nseg[l] = k;
    nslot[l] = k > 1 ? k : 0;
    nsplit[l] = k > 1 ? 1 : 0;
  }
}

__global__ void k_seg_fill(const int64_t* __restrict__ rrp, int64_t rows, const int64_t* __restrict__ seg_ptr,
                           const int64_t* __restrict__ slot_ptr, const int64_t* __restrict__ split_ptr,
                           ResSeg* __restrict__ segs) {
  for (int64_t l = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; l < rows; l += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = rrp[l], len = rrp[l + 1] - b;
    const int64_t k = seg_ptr[l + 1] - seg_ptr[l];
    for (int64_t i = 0; i < k; ++i) {
      ResSeg g;
      g.kb = b + i * kResSeg;
      g.row = (int32_t)l;
      g.yrow = (int32_t)l;  // NM_PACK_ORIGINAL_ORDER: replaced by row_map[l] (k_seg_yrow)
      g.len = (int32_t)min((int64_t)kResSeg, len - i * kResSeg);
      g.slot = k > 1 ? (int32_t)slot_ptr[l] : -1;
      g.split_id = k > 1 ? (int32_t)split_ptr[l] : -1;
      g.nseg = (int32_t)k;
      g.idx = (int32_t)i;
      g.pad = 0;
      segs[seg_ptr[l] + i] = g;
    }
  }
}

#ifndef NM_RES_ORDER
#define NM_RES_ORDER 0
#endif
__global__ void k_seg_key(const ResSeg* __restrict__ segs, int64_t n, uint32_t* __restrict__ key,
                          int32_t* __restrict__ idx) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
#if NM_RES_ORDER == 0
    key[i] = (uint32_t)(kResSeg - segs[i].len);  // ascending key = longest first
#else
    key[i] = segs[i].slot >= 0 ? 0u : 1u;  // split-row items first, then row order (stable)
#endif
    idx[i] = (int32_t)i;
  }
}

__global__ void k_seg_gather(const ResSeg* __restrict__ in, const int32_t* __restrict__ idx, int64_t n,
                             ResSeg* __restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = in[idx[i]];
}

struct DevBuf {
  void* p = nullptr;
  cudaStream_t s = nullptr;
  DevBuf() = default;
  DevBuf(const DevBuf&) = delete;
  ~DevBuf() {
    if (p) cudaFreeAsync(p, s);
  }
  template <typename T>
  T* as() { return (T*)p; }
};

inline nm_status dalloc(DevBuf& b, size_t bytes, cudaStream_t s) {
  b.s = s;
  NM_CUDA(cudaMallocAsync(&b.p, bytes > 0 ? bytes : 16, s));
  return NM_OK;
}

#define NM_TRY(x)                  \
  do {                             \
    nm_status st_ = (x);           \
    if (st_ != NM_OK) return st_;  \
  } while (0)

inline int grid_for(int64_t work, int block) {
  int64_t g = (work + block - 1) / block;
  if (g < 1) g = 1;
  if (g > 148 * 16) g = 148 * 16;
  return (int)g;
}

nm_status scan_excl(const int64_t* in, int64_t* out, int64_t n, cudaStream_t s) {
  size_t bytes = 0;
  NM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, bytes, in, out, n, s));
  DevBuf tmp;
  NM_TRY(dalloc(tmp, bytes, s));
  NM_CUDA(cub::DeviceScan::ExclusiveSum(tmp.p, bytes, in, out, n, s));
  return NM_OK;
}

// identity == 1: a[i] = perm[i] (perm already offset); else a[i] = a[i] >= 0 ? perm[a[i]] : -1
__global__ void k_seg_yrow(const int32_t* __restrict__ row_map, ResSeg* __restrict__ segs, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    segs[i].yrow = row_map[segs[i].row];
}

__global__ void k_map(const int32_t* __restrict__ perm, int32_t* __restrict__ a, int64_t m, int identity) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x) {
    if (identity) a[i] = perm[i];
    else a[i] = a[i] >= 0 ? perm[a[i]] : -1;
  }
}

// Contiguous split of P panels into G ranges minimising the largest range cost, cost of panel r
// = its chunks + per_panel (linear partition: bisection on the bound, greedy feasibility).
// Returns G+1 boundaries (trailing ranges may be empty).
std::vector<int32_t> balanced_ranges(const std::vector<int64_t>& chp, int64_t P, int G, int64_t per_panel) {
  auto cost = [&](int64_t r) { return chp[r + 1] - chp[r] + per_panel; };
  auto cuts_for = [&](int64_t T, std::vector<int32_t>* out) {
    int used = 1;
    int64_t acc = 0;
    if (out) out->assign(1, 0);
    for (int64_t r = 0; r < P; ++r) {
      const int64_t c = cost(r);
      if (acc + c > T && acc > 0) {
        ++used;
        acc = 0;
        if (out) out->push_back((int32_t)r);
      }
      acc += c;
    }
    return used;
  };
  int64_t lo = 0, hi = 0;
  for (int64_t r = 0; r < P; ++r) {
    lo = std::max(lo, cost(r));
    hi += cost(r);
  }
  while (lo < hi) {
    const int64_t mid = lo + (hi - lo) / 2;
    if (cuts_for(mid, nullptr) <= G) hi = mid; else lo = mid + 1;
  }
  std::vector<int32_t> cuts;
  cuts_for(lo, &cuts);
  while ((int)cuts.size() < G + 1) cuts.push_back((int32_t)P);
  return cuts;
}

nm_status pack_impl(const nm_csr* A, const int32_t* perm_host, int V, int N, int M, int Vp,
                    nm_dtype dtype, int64_t rb, int64_t re, int flags, int tau, cudaStream_t s,
                    nm_packed** out) {
  if (tau < 0) return fail(NM_ERR_INVALID_ARG, "nm_pack: tau < 0");
  if (!A || !out) return fail(NM_ERR_INVALID_ARG, "nm_pack: NULL argument");
  if (N != 2) return fail(NM_ERR_UNSUPPORTED, "nm_pack: N must be 2 (hardware 2:4, L496)");
  if (!(M == 4 || M == 8 || M == 16)) return fail(NM_ERR_UNSUPPORTED, "nm_pack: M must be 4, 8 or 16");
  if (V < 1) return fail(NM_ERR_INVALID_ARG, "nm_pack: V < 1");
  if (Vp == 0) Vp = (V == 16 || V == 32 || V == 64) ? V : kPanelRows;
  if (Vp != 16 && Vp != 32 && Vp != 64 && Vp != kPanelRows)
    return fail(NM_ERR_UNSUPPORTED, "nm_pack: Vp must be 16, 32, 64 or 128");
  const int ratio = kPanelRows / Vp;  // canonical panels per kernel panel
  if (dtype != NM_F16 && dtype != NM_BF16) return fail(NM_ERR_UNSUPPORTED, "nm_pack: dtype must be f16 or bf16");
  const int64_t n = A->n;
  if (n <= 0 || A->nnz < 0) return fail(NM_ERR_INVALID_ARG, "nm_pack: empty graph");
  if (n >= (int64_t)1 << 31) return fail(NM_ERR_UNSUPPORTED, "nm_pack: n >= 2^31");
  if (rb < 0 || re > n || rb > re || (rb % Vp != 0 && rb != re))
    return fail(NM_ERR_INVALID_ARG, "nm_pack_rows: bad row range (row_begin must be a multiple of Vp unless the range is empty)");
  const int Mp = (V == 1) ? 4 : M;
  const int64_t rows = re - rb;
  const int64_t P = (rows + kPanelRows - 1) / kPanelRows;  // kernel panels (MMA M = 128)
  const int64_t Pc = (rows + Vp - 1) / Vp;                 // canonical panels
  const int64_t S = (n + Mp - 1) / Mp;

  if (!A->on_device) {
    nm_status st = validate_csr_host(n, A->rowptr, A->col, false);
    if (st != NM_OK) return st;
  }
  DevCsr dA;
  NM_TRY(upload_csr(A, dtype, &dA, s));

  DevBuf d_perm, d_iperm;
  NM_TRY(dalloc(d_perm, sizeof(int32_t) * n, s));
  NM_TRY(dalloc(d_iperm, sizeof(int32_t) * n, s));
  if (perm_host) {
    // validate the permutation on the host
    std::vector<uint8_t> seen(n, 0);
    for (int64_t p = 0; p < n; ++p) {
      int32_t v = perm_host[p];
      if (v < 0 || v >= n || seen[v]) return fail(NM_ERR_INVALID_ARG, "nm_pack: perm is not a permutation");
      seen[v] = 1;
    }
    NM_CUDA(cudaMemcpyAsync(d_perm.p, perm_host, sizeof(int32_t) * n, cudaMemcpyHostToDevice, s));
  } else {
    k_identity<<<grid_for(n, 256), 256, 0, s>>>(d_perm.as<int32_t>(), n);
  }
  k_iperm<<<grid_for(n, 256), 256, 0, s>>>(d_perm.as<int32_t>(), d_iperm.as<int32_t>(), n);

  // ---- 1. B rows [rb, re) ----
  DevBuf d_deg, d_Brp;
  NM_TRY(dalloc(d_deg, sizeof(int64_t) * (rows + 1), s));
  NM_TRY(dalloc(d_Brp, sizeof(int64_t) * (rows + 1), s));
  NM_CUDA(cudaMemsetAsync(d_deg.p, 0, sizeof(int64_t) * (rows + 1), s));
  k_row_deg<<<grid_for(rows, 256), 256, 0, s>>>(dA.rp, d_perm.as<int32_t>(), rb, rows, d_deg.as<int64_t>());
  NM_TRY(scan_excl(d_deg.as<int64_t>(), d_Brp.as<int64_t>(), rows + 1, s));
  int64_t bnnz = 0;
  NM_CUDA(cudaMemcpyAsync(&bnnz, d_Brp.as<int64_t>() + rows, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  NM_CUDA(cudaStreamSynchronize(s));

  DevBuf d_key, d_key2, d_v, d_v2, d_Bci;
  NM_TRY(dalloc(d_key, sizeof(uint64_t) * bnnz, s));
  NM_TRY(dalloc(d_key2, sizeof(uint64_t) * bnnz, s));
  NM_TRY(dalloc(d_v, sizeof(uint16_t) * bnnz, s));
  NM_TRY(dalloc(d_v2, sizeof(uint16_t) * bnnz, s));
  NM_TRY(dalloc(d_Bci, sizeof(int32_t) * bnnz, s));
  k_fill_keys<<<grid_for(rows * 32, 256), 256, 0, s>>>(
      dA.rp, dA.ci, dA.val, one_bits(dtype), d_perm.as<int32_t>(), d_iperm.as<int32_t>(), rb,
      rows, d_Brp.as<int64_t>(), d_key.as<uint64_t>(), d_v.as<uint16_t>());
  NM_CUDA(cudaGetLastError());
  {
    int end_bit = 32;
    while (end_bit < 64 && (((uint64_t)rows) >> (end_bit - 32)) != 0) ++end_bit;
    size_t bytes = 0;
    NM_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, bytes, d_key.as<uint64_t>(), d_key2.as<uint64_t>(),
                                            d_v.as<uint16_t>(), d_v2.as<uint16_t>(), bnnz, 0, end_bit, s));
    DevBuf tmp;
    NM_TRY(dalloc(tmp, bytes, s));
    NM_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, bytes, d_key.as<uint64_t>(), d_key2.as<uint64_t>(),
                                            d_v.as<uint16_t>(), d_v2.as<uint16_t>(), bnnz, 0, end_bit, s));
  }
  k_split_keys<<<grid_for(bnnz, 256), 256, 0, s>>>(d_key2.as<uint64_t>(), d_Bci.as<int32_t>(), bnnz);
  const int32_t* Bci = d_Bci.as<int32_t>();
  const uint16_t* Bval = d_v2.as<uint16_t>();
  const int64_t* Brp = d_Brp.as<int64_t>();

  // ---- 2. meta-blocks ----
  DevBuf d_mk, d_mk2, d_mbkey, d_runs, d_nruns;
  NM_TRY(dalloc(d_mk, sizeof(int64_t) * bnnz, s));
  NM_TRY(dalloc(d_mk2, sizeof(int64_t) * bnnz, s));
  NM_TRY(dalloc(d_mbkey, sizeof(int64_t) * bnnz, s));
  NM_TRY(dalloc(d_runs, sizeof(int64_t) * bnnz, s));
  NM_TRY(dalloc(d_nruns, sizeof(int64_t), s));
  k_mbkey<<<grid_for(rows * 32, 256), 256, 0, s>>>(Brp, Bci, rows, Vp, Mp, S, d_mk.as<int64_t>());
  {
    size_t bytes = 0;
    NM_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, bytes, d_mk.as<int64_t>(), d_mk2.as<int64_t>(), bnnz, 0, 64, s));
    DevBuf tmp;
    NM_TRY(dalloc(tmp, bytes, s));
    NM_CUDA(cub::DeviceRadixSort::SortKeys(tmp.p, bytes, d_mk.as<int64_t>(), d_mk2.as<int64_t>(), bnnz, 0, 64, s));
  }
  {
    size_t bytes = 0;
    NM_CUDA(cub::DeviceRunLengthEncode::Encode(nullptr, bytes, d_mk2.as<int64_t>(), d_mbkey.as<int64_t>(),
                                               d_runs.as<int64_t>(), d_nruns.as<int64_t>(), bnnz, s));
    DevBuf tmp;
    NM_TRY(dalloc(tmp, bytes, s));
    NM_CUDA(cub::DeviceRunLengthEncode::Encode(tmp.p, bytes, d_mk2.as<int64_t>(), d_mbkey.as<int64_t>(),
                                               d_runs.as<int64_t>(), d_nruns.as<int64_t>(), bnnz, s));
  }
  int64_t n_cand = 0;  // candidate meta-blocks: distinct non-empty (panel, segment) pairs
  if (bnnz > 0) {
    NM_CUDA(cudaMemcpyAsync(&n_cand, d_nruns.p, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    NM_CUDA(cudaStreamSynchronize(s));
  }

  // ---- 3. column counts, selection and (tau > 0) the hybrid split of thin meta-blocks ----
  DevBuf d_cnt, d_emb, d_selc;
  const int64_t nc1 = n_cand > 0 ? n_cand : 1;
  NM_TRY(dalloc(d_cnt, sizeof(int32_t) * Mp * nc1, s));
  NM_TRY(dalloc(d_emb, sizeof(int64_t) * bnnz, s));
  NM_TRY(dalloc(d_selc, sizeof(uint32_t) * nc1, s));
  NM_CUDA(cudaMemsetAsync(d_cnt.p, 0, sizeof(int32_t) * Mp * nc1, s));
  if (bnnz) {
    k_colcount<<<grid_for(rows * 32, 256), 256, 0, s>>>(Brp, Bci, rows, Vp, Mp, S, d_mbkey.as<int64_t>(), n_cand,
                                                       d_cnt.as<int32_t>(), d_emb.as<int64_t>());
    k_select<<<grid_for(n_cand, 256), 256, 0, s>>>(d_cnt.as<int32_t>(), Mp, n_cand, d_selc.as<uint32_t>());
  }
  NM_CUDA(cudaGetLastError());
  int64_t n_mb = n_cand;
  const int64_t* mbkey = d_mbkey.as<int64_t>();
  const uint32_t* selv = d_selc.as<uint32_t>();
  DevBuf d_keptc, d_flag_mb, d_newid, d_key_c, d_sel_c, d_cand_of;
  if (tau > 0 && n_cand > 0) {
    NM_TRY(dalloc(d_keptc, sizeof(int32_t) * n_cand, s));
    NM_TRY(dalloc(d_flag_mb, sizeof(int64_t) * (n_cand + 1), s));
    NM_TRY(dalloc(d_newid, sizeof(int64_t) * (n_cand + 1), s));
    NM_CUDA(cudaMemsetAsync(d_keptc.p, 0, sizeof(int32_t) * n_cand, s));
    NM_CUDA(cudaMemsetAsync(d_flag_mb.p, 0, sizeof(int64_t) * (n_cand + 1), s));
    k_keep_count<<<grid_for(rows * 32, 256), 256, 0, s>>>(Brp, Bci, rows, Mp, d_emb.as<int64_t>(), selv,
                                                         d_keptc.as<int32_t>());
    k_survive<<<grid_for(n_cand, 256), 256, 0, s>>>(d_keptc.as<int32_t>(), n_cand, tau, d_flag_mb.as<int64_t>());
    NM_TRY(scan_excl(d_flag_mb.as<int64_t>(), d_newid.as<int64_t>(), n_cand + 1, s));
    NM_CUDA(cudaMemcpyAsync(&n_mb, d_newid.as<int64_t>() + n_cand, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    NM_CUDA(cudaStreamSynchronize(s));
    NM_TRY(dalloc(d_key_c, sizeof(int64_t) * (n_mb > 0 ? n_mb : 1), s));
    NM_TRY(dalloc(d_sel_c, sizeof(uint32_t) * (n_mb > 0 ? n_mb : 1), s));
    NM_TRY(dalloc(d_cand_of, sizeof(int64_t) * (n_mb > 0 ? n_mb : 1), s));
    k_compact<<<grid_for(n_cand, 256), 256, 0, s>>>(d_flag_mb.as<int64_t>(), d_newid.as<int64_t>(), n_cand, mbkey,
                                                    selv, d_key_c.as<int64_t>(), d_sel_c.as<uint32_t>(),
                                                    d_cand_of.as<int64_t>());
    k_remap_emb<<<grid_for(bnnz, 256), 256, 0, s>>>(d_flag_mb.as<int64_t>(), d_newid.as<int64_t>(),
                                                    d_emb.as<int64_t>(), bnnz);
    NM_CUDA(cudaGetLastError());
    mbkey = d_key_c.as<int64_t>();
    selv = d_sel_c.as<uint32_t>();
  }

  nm_packed* Pk = new nm_packed();
  NM_CUDA(cudaGetDevice(&Pk->device));
  Pk->n = n; Pk->row_begin = rb; Pk->row_end = re;
  Pk->V = V; Pk->N = N; Pk->M = M; Pk->Vp = Vp; Pk->Mp = Mp; Pk->dtype = dtype;
  Pk->n_panels = P; Pk->n_cpanels = Pc; Pk->n_mb = n_mb; Pk->tau = tau;
  struct Guard {
    nm_packed* p;
    bool ok = false;
    ~Guard() { if (!ok) nm_packed_free(p); }
  } guard{Pk};
  auto palloc = [&](void** ptr, size_t bytes) -> nm_status {
    NM_CUDA(cudaMalloc(ptr, bytes > 0 ? bytes : 16));
    Pk->device_bytes += bytes;
    return NM_OK;
  };
  NM_TRY(palloc((void**)&Pk->panel_mb_ptr, sizeof(int64_t) * (Pc + 1)));
  NM_TRY(palloc((void**)&Pk->panel_chunk_ptr, sizeof(int64_t) * (P + 1)));
  k_panel_ptr<<<grid_for(Pc + 1, 256), 256, 0, s>>>(mbkey, n_mb, Pc, S, Pk->panel_mb_ptr, nullptr);
  DevBuf d_nch;
  NM_TRY(dalloc(d_nch, sizeof(int64_t) * (P + 1), s));
  NM_CUDA(cudaMemsetAsync(d_nch.p, 0, sizeof(int64_t) * (P + 1), s));
  k_chunk_counts<<<grid_for(P, 256), 256, 0, s>>>(Pk->panel_mb_ptr, P, ratio, Pc, d_nch.as<int64_t>());
  NM_TRY(scan_excl(d_nch.as<int64_t>(), Pk->panel_chunk_ptr, P + 1, s));
  std::vector<int64_t> chp(P + 1);
  NM_CUDA(cudaMemcpyAsync(chp.data(), Pk->panel_chunk_ptr, sizeof(int64_t) * (P + 1), cudaMemcpyDeviceToHost, s));
  NM_CUDA(cudaStreamSynchronize(s));
  const int64_t n_chunks = chp[P];
  Pk->n_chunks = n_chunks;

  NM_TRY(palloc((void**)&Pk->mb_seg, sizeof(int32_t) * n_mb));
  NM_TRY(palloc((void**)&Pk->mb_sel, sizeof(uint32_t) * n_mb));
  // the full MMA-layout records (the image of the full-record SpMM kernel); step 5 also
  // compresses them into the HBM form of the compressed-record kernel
  NM_TRY(palloc((void**)&Pk->image_full, (size_t)kChunkBytes * n_chunks));
  uint8_t* full = Pk->image_full;
  if (n_chunks) {
    NM_CUDA(cudaMemsetAsync(full, 0, (size_t)kChunkBytes * n_chunks, s));
    k_meta_init<<<grid_for(n_chunks * 128, 256), 256, 0, s>>>(full, n_chunks);
    k_xrow_map<<<grid_for(n_chunks * 32, 256), 256, 0, s>>>(nullptr, full, n_chunks);
  }
  if (n_mb) {
    NM_CUDA(cudaMemcpyAsync(Pk->mb_sel, selv, sizeof(uint32_t) * n_mb, cudaMemcpyDeviceToDevice, s));
    k_write_sel<<<grid_for(n_mb, 256), 256, 0, s>>>(d_cnt.as<int32_t>(), d_cand_of.p ? d_cand_of.as<int64_t>() : nullptr,
                                                    Mp, n_mb, mbkey, S, n, Pk->panel_mb_ptr, ratio, Pc, Pk->panel_chunk_ptr,
                                                    Pk->mb_seg, Pk->mb_sel, full);
  }
  NM_CUDA(cudaGetLastError());

  // ---- 4. placement and residual ----
  DevBuf d_flag, d_kept, d_rc;
  NM_TRY(dalloc(d_flag, bnnz, s));
  NM_TRY(dalloc(d_kept, sizeof(unsigned long long), s));
  NM_TRY(dalloc(d_rc, sizeof(int64_t) * (rows + 1), s));
  NM_CUDA(cudaMemsetAsync(d_kept.p, 0, sizeof(unsigned long long), s));
  NM_CUDA(cudaMemsetAsync(d_rc.p, 0, sizeof(int64_t) * (rows + 1), s));
  if (bnnz) {
    k_place<<<grid_for(rows * 32, 256), 256, 0, s>>>(Brp, Bci, Bval, rows, Mp, d_emb.as<int64_t>(), Pk->mb_sel,
                                                    Pk->panel_mb_ptr, ratio, Pc, Pk->panel_chunk_ptr, full,
                                                    d_flag.as<uint8_t>(), d_kept.as<unsigned long long>());
    k_res_count<<<grid_for(rows * 32, 256), 256, 0, s>>>(Brp, d_flag.as<uint8_t>(), rows, d_rc.as<int64_t>());
  }
  NM_CUDA(cudaGetLastError());
  NM_TRY(palloc((void**)&Pk->res_rowptr, sizeof(int64_t) * (rows + 1)));
  NM_TRY(scan_excl(d_rc.as<int64_t>(), Pk->res_rowptr, rows + 1, s));
  int64_t res_nnz = 0;
  unsigned long long kept = 0;
  NM_CUDA(cudaMemcpyAsync(&res_nnz, Pk->res_rowptr + rows, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  NM_CUDA(cudaMemcpyAsync(&kept, d_kept.p, sizeof(kept), cudaMemcpyDeviceToHost, s));
  NM_CUDA(cudaStreamSynchronize(s));
  Pk->res_nnz = res_nnz;
  Pk->packed_nnz = (int64_t)kept;
  NM_TRY(palloc((void**)&Pk->res_col, sizeof(int32_t) * res_nnz));
  NM_TRY(palloc((void**)&Pk->res_val, sizeof(uint16_t) * res_nnz));
  if (res_nnz)
    k_res_fill<<<grid_for(rows * 32, 256), 256, 0, s>>>(Brp, Bci, Bval, d_flag.as<uint8_t>(), rows,
                                                       Pk->res_rowptr, Pk->res_col, Pk->res_val);
  NM_CUDA(cudaGetLastError());
  if (res_nnz) {
    // residual work list: one item per row, hub rows cut into kResSeg-entry items
    DevBuf d_nseg, d_nslot, d_nsplit, d_segp, d_slotp, d_splitp;
    for (DevBuf* b : {&d_nseg, &d_nslot, &d_nsplit, &d_segp, &d_slotp, &d_splitp})
      NM_TRY(dalloc(*b, sizeof(int64_t) * (rows + 1), s));
    NM_CUDA(cudaMemsetAsync(d_nseg.p, 0, sizeof(int64_t) * (rows + 1), s));
    NM_CUDA(cudaMemsetAsync(d_nslot.p, 0, sizeof(int64_t) * (rows + 1), s));
    NM_CUDA(cudaMemsetAsync(d_nsplit.p, 0, sizeof(int64_t) * (rows + 1), s));
    k_seg_count<<<grid_for(rows, 256), 256, 0, s>>>(Pk->res_rowptr, rows, d_nseg.as<int64_t>(),
                                                    d_nslot.as<int64_t>(), d_nsplit.as<int64_t>());
    NM_TRY(scan_excl(d_nseg.as<int64_t>(), d_segp.as<int64_t>(), rows + 1, s));
    NM_TRY(scan_excl(d_nslot.as<int64_t>(), d_slotp.as<int64_t>(), rows + 1, s));
    NM_TRY(scan_excl(d_nsplit.as<int64_t>(), d_splitp.as<int64_t>(), rows + 1, s));
    int64_t tot[3];
    NM_CUDA(cudaMemcpyAsync(&tot[0], d_segp.as<int64_t>() + rows, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    NM_CUDA(cudaMemcpyAsync(&tot[1], d_slotp.as<int64_t>() + rows, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    NM_CUDA(cudaMemcpyAsync(&tot[2], d_splitp.as<int64_t>() + rows, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    NM_CUDA(cudaStreamSynchronize(s));
    Pk->n_res_segs = tot[0];
    Pk->n_res_slots = tot[1];
    Pk->n_res_split = tot[2];
    NM_TRY(palloc((void**)&Pk->res_segs, sizeof(ResSeg) * tot[0]));
    DevBuf d_segs, d_k1, d_k2, d_i1, d_i2;
    NM_TRY(dalloc(d_segs, sizeof(ResSeg) * tot[0], s));
    k_seg_fill<<<grid_for(rows, 256), 256, 0, s>>>(Pk->res_rowptr, rows, d_segp.as<int64_t>(), d_slotp.as<int64_t>(),
                                                   d_splitp.as<int64_t>(), d_segs.as<ResSeg>());
    // longest work items first (a stable sort by length): the persistent grid's first wave
    // takes the hub rows' items, so they do not form the kernel's tail
    NM_TRY(dalloc(d_k1, sizeof(uint32_t) * tot[0], s));
    NM_TRY(dalloc(d_k2, sizeof(uint32_t) * tot[0], s));
    NM_TRY(dalloc(d_i1, sizeof(int32_t) * tot[0], s));
    NM_TRY(dalloc(d_i2, sizeof(int32_t) * tot[0], s));
    k_seg_key<<<grid_for(tot[0], 256), 256, 0, s>>>(d_segs.as<ResSeg>(), tot[0], d_k1.as<uint32_t>(), d_i1.as<int32_t>());
    {
      size_t bytes = 0;
      NM_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, bytes, d_k1.as<uint32_t>(), d_k2.as<uint32_t>(),
                                              d_i1.as<int32_t>(), d_i2.as<int32_t>(), tot[0], 0, 9, s));
      DevBuf tmp;
      NM_TRY(dalloc(tmp, bytes, s));
      NM_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, bytes, d_k1.as<uint32_t>(), d_k2.as<uint32_t>(),
                                              d_i1.as<int32_t>(), d_i2.as<int32_t>(), tot[0], 0, 9, s));
    }
    k_seg_gather<<<grid_for(tot[0], 256), 256, 0, s>>>(d_segs.as<ResSeg>(), d_i2.as<int32_t>(), tot[0], Pk->res_segs);
    NM_CUDA(cudaGetLastError());
  }
  if (flags & NM_PACK_ORIGINAL_ORDER) {
    // fold P into the operand indices: gather X[perm[q]], write Y[perm[p]]
    Pk->flags = flags;
    NM_TRY(palloc((void**)&Pk->row_map, sizeof(int32_t) * rows));
    NM_TRY(palloc((void**)&Pk->res_gather, sizeof(int32_t) * res_nnz));
    const int32_t* pm = d_perm.as<int32_t>();
    k_map<<<grid_for(rows, 256), 256, 0, s>>>(pm + rb, Pk->row_map, rows, 1);
    if (Pk->n_res_segs)  // residual work items address Y by output row
      k_seg_yrow<<<grid_for(Pk->n_res_segs, 256), 256, 0, s>>>(Pk->row_map, Pk->res_segs, Pk->n_res_segs);
    if (n_chunks) k_xrow_map<<<grid_for(n_chunks * 32, 256), 256, 0, s>>>(pm, full, n_chunks);
    if (res_nnz) {
      NM_CUDA(cudaMemcpyAsync(Pk->res_gather, Pk->res_col, sizeof(int32_t) * res_nnz, cudaMemcpyDeviceToDevice, s));
      k_map<<<grid_for(res_nnz, 256), 256, 0, s>>>(pm, Pk->res_gather, res_nnz, 0);
    }
    NM_CUDA(cudaGetLastError());
  }
  // ---- 5. compression of the records (HBM form) ----
  std::vector<int64_t> coff(n_chunks + 1, 0);
  {
    DevBuf d_sz, d_off;
    NM_TRY(dalloc(d_sz, sizeof(int64_t) * (n_chunks + 1), s));
    NM_TRY(dalloc(d_off, sizeof(int64_t) * (n_chunks + 1), s));
    NM_CUDA(cudaMemsetAsync(d_sz.p, 0, sizeof(int64_t) * (n_chunks + 1), s));
    const int cgrid = (int)std::min<int64_t>(std::max<int64_t>(n_chunks, 1), 148 * 16);
    if (n_chunks)
      k_compress<false><<<cgrid, 128, 0, s>>>(full, n_chunks, d_sz.as<int64_t>(), nullptr, nullptr);
    NM_TRY(scan_excl(d_sz.as<int64_t>(), d_off.as<int64_t>(), n_chunks + 1, s));
    NM_CUDA(cudaMemcpyAsync(coff.data(), d_off.p, sizeof(int64_t) * (n_chunks + 1), cudaMemcpyDeviceToHost, s));
    NM_CUDA(cudaStreamSynchronize(s));
    for (auto& o : coff) o *= 16;  // units of 16 bytes -> bytes
    NM_CUDA(cudaMemcpyAsync(d_off.p, coff.data(), sizeof(int64_t) * (n_chunks + 1), cudaMemcpyHostToDevice, s));
    Pk->image_bytes = coff[n_chunks];
    NM_TRY(palloc((void**)&Pk->image, (size_t)Pk->image_bytes));
    std::vector<uint16_t> len16(n_chunks > 0 ? n_chunks : 1);
    for (int64_t c = 0; c < n_chunks; ++c) len16[c] = (uint16_t)((coff[c + 1] - coff[c]) / 16);
    NM_TRY(palloc((void**)&Pk->rec_len16, sizeof(uint16_t) * len16.size()));
    NM_CUDA(cudaMemcpyAsync(Pk->rec_len16, len16.data(), sizeof(uint16_t) * len16.size(), cudaMemcpyHostToDevice, s));
    if (n_chunks)
      k_compress<true><<<cgrid, 128, 0, s>>>(full, n_chunks, nullptr, d_off.as<int64_t>(), Pk->image);
    NM_CUDA(cudaGetLastError());
    NM_CUDA(cudaStreamSynchronize(s));
  }

  // unit schedule of the compressed-record kernel: natural panel order (consecutive panels run
  // concurrently on the persistent grid, so their X neighbourhoods are shared in L2).
  // Two 16-byte descriptors per panel: {panel, #chunks, first chunk}, {record bytes offset, size}.
  {
    std::vector<int32_t> order(P);
    std::iota(order.begin(), order.end(), 0);
    std::vector<int4> info(2 * P);
    for (int64_t j = 0; j < P; ++j) {
      const int32_t r = order[j];
      const int64_t c0 = chp[r], b0 = coff[c0], b1 = coff[chp[r + 1]];
      info[2 * j] = make_int4(r, (int32_t)(chp[r + 1] - c0), (int32_t)(c0 & 0xFFFFFFFF), (int32_t)(c0 >> 32));
      info[2 * j + 1] = make_int4((int32_t)(b0 & 0xFFFFFFFF), (int32_t)(b0 >> 32), (int32_t)((b1 - b0) & 0xFFFFFFFF),
                                  (int32_t)((b1 - b0) >> 32));
    }
    NM_TRY(palloc((void**)&Pk->unit_info, sizeof(int4) * 2 * P));
    NM_CUDA(cudaMemcpyAsync(Pk->unit_info, info.data(), sizeof(int4) * 2 * P, cudaMemcpyHostToDevice, s));
    NM_CUDA(cudaStreamSynchronize(s));
  }

  if (n_chunks) {  // X rows the tensor-core part gathers (roofline accounting)
    DevBuf d_g;
    NM_TRY(dalloc(d_g, sizeof(unsigned long long), s));
    NM_CUDA(cudaMemsetAsync(d_g.p, 0, sizeof(unsigned long long), s));
    k_count_gather<<<grid_for(n_chunks * 32, 256), 256, 0, s>>>(Pk->image_full, n_chunks, d_g.as<unsigned long long>());
    unsigned long long gr = 0;
    NM_CUDA(cudaMemcpyAsync(&gr, d_g.p, sizeof(gr), cudaMemcpyDeviceToHost, s));
    NM_CUDA(cudaStreamSynchronize(s));
    Pk->gather_rows = (int64_t)gr;
  }
  // persistent-grid work split of the full-record kernel: one contiguous panel range per SM,
  // balanced by chunk count (+ a per-panel term for its epilogue)
  {
    int sms = 148;
    NM_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, Pk->device));
    const int G = (int)std::max<int64_t>(1, std::min<int64_t>(sms, P));
    std::vector<int32_t> cp = balanced_ranges(chp, P, G, /*per_panel=*/4);
    Pk->n_ctas = G;
    NM_TRY(palloc((void**)&Pk->cta_ptr, sizeof(int32_t) * cp.size()));
    NM_CUDA(cudaMemcpyAsync(Pk->cta_ptr, cp.data(), sizeof(int32_t) * cp.size(), cudaMemcpyHostToDevice, s));
  }

  NM_CUDA(cudaStreamSynchronize(s));
  guard.ok = true;
  *out = Pk;
  return NM_OK;
}

// The library's SpMM time model of a pack (fitted to B200 measurements of the two
// kernels): per K = 32 chunk and F, per residual value and F, per residual work item (its Y
// row read-modify-write and item overhead) and F.  ns of whole-GPU time.
double pack_time_model(const nm_packed* P, int F) {
  return (double)P->n_chunks * (0.28 + 0.0075 * F) + (double)P->res_nnz * (0.00016 * F) +
         (double)P->n_res_segs * (0.0024 * F);
}

nm_status pack_auto_impl(const nm_csr* A, const int32_t* perm, int V, int N, int M, int Vp, nm_dtype dtype,
                         int64_t rb, int64_t re, int flags, int F, cudaStream_t s, nm_packed** out, int* tau_out);

// Pattern scoring: reorder + the auto-tau hybrid pack per candidate,
// scored by the library's time model.
nm_status score_patterns_impl(const nm_csr* A, int ncand, const int* Vs, const int* Ms, int F, nm_dtype dtype,
                              const nm_reorder_opts* opts, cudaStream_t s, double* scores, int64_t* chunks_out,
                              int64_t* res_out, int* best, int32_t* perm_out) {
  if (!A || ncand < 1 || !Vs || !Ms || !best || !perm_out)
    return fail(NM_ERR_INVALID_ARG, "nm_score_patterns: NULL argument or no candidate");
  if (F < 1) return fail(NM_ERR_INVALID_ARG, "nm_score_patterns: F < 1");
  const int64_t n = A->n;
  std::vector<int32_t> perm(n > 0 ? n : 1);
  double best_score = 0.0;
  int best_i = -1;
  for (int i = 0; i < ncand; ++i) {
    NM_TRY(nm_reorder_gpu(A, Vs[i], 2, Ms[i], opts, perm.data(), nullptr, s));
    nm_packed* P = nullptr;
    NM_TRY(pack_auto_impl(A, perm.data(), Vs[i], 2, Ms[i], 0, dtype, 0, n, 0, F, s, &P, nullptr));
    const double sc = pack_time_model(P, F);
    if (scores) scores[i] = sc;
    if (chunks_out) chunks_out[i] = P->n_chunks;
    if (res_out) res_out[i] = P->res_nnz;
    nm_packed_free(P);
    if (best_i < 0 || sc < best_score) {  // ties keep the earlier candidate
      best_score = sc;
      best_i = i;
      memcpy(perm_out, perm.data(), sizeof(int32_t) * n);
    }
  }
  *best = best_i;
  return NM_OK;
}

// nm_pack_auto: the hybrid pack whose tau minimises the time model over a candidate set
nm_status pack_auto_impl(const nm_csr* A, const int32_t* perm, int V, int N, int M, int Vp, nm_dtype dtype,
                         int64_t rb, int64_t re, int flags, int F, cudaStream_t s, nm_packed** out, int* tau_out) {
  if (!out) return fail(NM_ERR_INVALID_ARG, "nm_pack_auto: NULL out");
  if (F < 1) return fail(NM_ERR_INVALID_ARG, "nm_pack_auto: F < 1");
  const int tm = nm_hybrid_tau(F);
  const int cands[] = {0, 2, 4, tm / 2, tm, tm + tm / 2, 2 * tm};
  nm_packed* best = nullptr;
  double best_t = 0.0;
  int best_tau = 0;
  std::vector<int> seen;
  for (int tau : cands) {
    if (tau < 0 || std::find(seen.begin(), seen.end(), tau) != seen.end()) continue;
    seen.push_back(tau);
    nm_packed* P = nullptr;
    nm_status st = pack_impl(A, perm, V, N, M, Vp, dtype, rb, re, flags, tau, s, &P);
    if (st != NM_OK) {
      nm_packed_free(best);
      return st;
    }
    const double t = pack_time_model(P, F);
    if (!best || t < best_t) {  // ties keep the smaller tau
      nm_packed_free(best);
      best = P;
      best_t = t;
      best_tau = tau;
    } else {
      nm_packed_free(P);
    }
  }
  *out = best;
  if (tau_out) *tau_out = best_tau;
  return NM_OK;
}

}  // namespace
}  // namespace nm

extern "C" nm_status nm_pack_auto(const nm_csr* A, const int32_t* perm, int V, int N, int M, int Vp, nm_dtype dtype,
                                  int64_t row_begin, int64_t row_end, int flags, int F, void* stream,
                                  nm_packed** out, int* tau_out) {
  if (flags & ~NM_PACK_ORIGINAL_ORDER) return nm::fail(NM_ERR_INVALID_ARG, "nm_pack_auto: unknown flags");
  return nm::guarded("nm_pack_auto", [&] {
    return nm::pack_auto_impl(A, perm, V, N, M, Vp, dtype, row_begin, row_end, flags, F, (cudaStream_t)stream, out,
                              tau_out);
  });
}

extern "C" nm_status nm_score_patterns(const nm_csr* A, int ncand, const int* V, const int* M, int F, nm_dtype dtype,
                                       const nm_reorder_opts* opts, void* stream, double* scores,
                                       int64_t* n_chunks, int64_t* residual_nnz, int* best, int32_t* perm_out) {
  return nm::guarded("nm_score_patterns", [&] {
    return nm::score_patterns_impl(A, ncand, V, M, F, dtype, opts, (cudaStream_t)stream, scores, n_chunks,
                                   residual_nnz, best, perm_out);
  });
}

extern "C" nm_status nm_pack(const nm_csr* A, const int32_t* perm, int V, int N, int M, int Vp,
                             nm_dtype dtype, void* stream, nm_packed** out) {
  if (!A) return nm::fail(NM_ERR_INVALID_ARG, "nm_pack: NULL graph");
  return nm::guarded("nm_pack", [&] { return nm::pack_impl(A, perm, V, N, M, Vp, dtype, 0, A->n, 0, 0, (cudaStream_t)stream, out); });
}

extern "C" nm_status nm_pack_rows(const nm_csr* A, const int32_t* perm, int V, int N, int M,
                                  int Vp, nm_dtype dtype, int64_t row_begin, int64_t row_end,
                                  void* stream, nm_packed** out) {
  return nm::guarded("nm_pack", [&] { return nm::pack_impl(A, perm, V, N, M, Vp, dtype, row_begin, row_end, 0, 0, (cudaStream_t)stream, out); });
}

extern "C" nm_status nm_pack_ex(const nm_csr* A, const int32_t* perm, int V, int N, int M, int Vp,
                                nm_dtype dtype, int64_t row_begin, int64_t row_end, int flags, void* stream,
                                nm_packed** out) {
  if (flags & ~NM_PACK_ORIGINAL_ORDER) return nm::fail(NM_ERR_INVALID_ARG, "nm_pack_ex: unknown flags");
  return nm::guarded("nm_pack", [&] { return nm::pack_impl(A, perm, V, N, M, Vp, dtype, row_begin, row_end, flags, 0, (cudaStream_t)stream, out); });
}

extern "C" nm_status nm_pack_hybrid(const nm_csr* A, const int32_t* perm, int V, int N, int M, int Vp,
                                    nm_dtype dtype, int64_t row_begin, int64_t row_end, int flags, int tau,
                                    void* stream, nm_packed** out) {
  if (flags & ~NM_PACK_ORIGINAL_ORDER) return nm::fail(NM_ERR_INVALID_ARG, "nm_pack_hybrid: unknown flags");
  return nm::guarded("nm_pack", [&] { return nm::pack_impl(A, perm, V, N, M, Vp, dtype, row_begin, row_end, flags, tau, (cudaStream_t)stream, out); });
}
