// GPU Stage-1 of the SGRP heuristic (§4.2, Alg. 2 lines 4-13, L366-384): the
// Hamming position codes of every (row, segment) of B = P A P^T and the stable lexicographic
// row sort, on the device (the paper's SOGRE runs its reordering on the
// GPU, L484).  Bit-identical to the host stage1_sort in reorder.cpp and to the oracle
// (DESIGN.md §3 readings 1-6): the key of row p is the sequence of pairs
// (sgn(c)·(S−s), c) over its non-empty segments s in ascending order, closed by (0, 0), with
// c = invGray(bits) negated when popcount(bits) > N; rows are stably sorted by that key.
//
//   1. entries of B as 64-bit keys (p << 32 | q) -> radix sort: a (row, segment) group is a
//      contiguous run of at most M entries, ascending in segment inside each row;
//   2. one thread per group start folds the run into its mask and count, and emits (x, c);
//   3. per-row group offsets (count + scan);
//   4. merge sort (cub::DeviceMergeSort::StableSortKeys) of the row indices with a comparator that walks two
//      rows' pair sequences — stability gives the "ties keep the current position" rule.
#include <cub/cub.cuh>

#include "nm_internal.h"

namespace nm {
namespace {

inline int grid_for(int64_t work, int block) {
  int64_t g = (work + block - 1) / block;
  return (int)(g < 1 ? 1 : (g > 148 * 32 ? 148 * 32 : g));
}

__global__ void k_s1_inv(const int32_t* __restrict__ perm, int32_t* __restrict__ iperm, int64_t n) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n; p += (int64_t)gridDim.x * blockDim.x)
    iperm[perm[p]] = (int32_t)p;
}

__global__ void k_s1_deg(const int64_t* __restrict__ rp, const int32_t* __restrict__ perm, int64_t n,
                         int64_t* __restrict__ deg) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n; p += (int64_t)gridDim.x * blockDim.x)
    deg[p] = rp[perm[p] + 1] - rp[perm[p]];
}

// entries of row p of B: column q = iperm[c] for every neighbour c of perm[p]
__global__ void k_s1_keys(const int64_t* __restrict__ rp, const int32_t* __restrict__ ci,
                          const int32_t* __restrict__ perm, const int32_t* __restrict__ iperm, int64_t n,
                          const int64_t* __restrict__ Brp, uint64_t* __restrict__ key) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t p = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; p < n; p += nw) {
    const int32_t u = perm[p];
    const int64_t s = rp[u], d = rp[u + 1] - s, o = Brp[p];
    for (int64_t k = lane; k < d; k += 32)
      key[o + k] = ((uint64_t)p << 32) | (uint32_t)iperm[ci[s + k]];
  }
}

__device__ __forceinline__ bool group_start(const uint64_t* key, int64_t k, uint32_t M) {
  if (k == 0) return true;
  const uint64_t a = key[k - 1], b = key[k];
  return (a >> 32) != (b >> 32) || (uint32_t)a / M != (uint32_t)b / M;
}

__global__ void k_s1_flags(const uint64_t* __restrict__ key, int64_t m, uint32_t M, int32_t* __restrict__ flag) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x)
    flag[k] = group_start(key, k, M) ? 1 : 0;
}

// one thread per group start: mask (first column of the segment -> MSB, Listing 1),
// count, code (L339-346) and the key pair; rows count their groups
__global__ void k_s1_codes(const uint64_t* __restrict__ key, int64_t m, uint32_t M, int N, int64_t S,
                           const int64_t* __restrict__ gid, int64_t* __restrict__ gx, int64_t* __restrict__ gc,
                           int32_t* __restrict__ ngroups_row) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x) {
    if (!group_start(key, k, M)) continue;
    const uint32_t p = (uint32_t)(key[k] >> 32);
    const uint32_t s = (uint32_t)key[k] / M;
    uint64_t b = 0;
    int cnt = 0;
    for (int64_t j = k; j < m && (uint32_t)(key[j] >> 32) == p && (uint32_t)key[j] / M == s; ++j) {
      b |= 1ull << (M - 1 - ((uint32_t)key[j] - s * M));
      ++cnt;
    }
    uint64_t h = b;  // rank in the binary reflected Gray order (inverse Gray code)
    for (int sh = 1; sh < 64; sh <<= 1) h ^= h >> sh;
    const int64_t c = (cnt > N) ? -(int64_t)h : (int64_t)h;
    const int64_t g = gid[k];
    gx[g] = (c > 0 ? 1 : -1) * (S - (int64_t)s);
    gc[g] = c;
    atomicAdd(&ngroups_row[p], 1);
  }
}

__global__ void k_s1_apply(const int32_t* __restrict__ perm, const int32_t* __restrict__ order, int64_t n,
                           int32_t* __restrict__ out) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n; p += (int64_t)gridDim.x * blockDim.x)
    out[p] = perm[order[p]];
}

// lexicographic "<" of two rows' pair sequences, each closed by (0, 0)
struct RowKeyLess {
  const int64_t* goff;
  const int64_t* gx;
  const int64_t* gc;
  __device__ bool operator()(int32_t a, int32_t b) const {
    int64_t ia = goff[a], ea = goff[a + 1], ib = goff[b], eb = goff[b + 1];
    for (;;) {
      const int64_t xa = ia < ea ? gx[ia] : 0, ca = ia < ea ? gc[ia] : 0;
      const int64_t xb = ib < eb ? gx[ib] : 0, cb = ib < eb ? gc[ib] : 0;
      if (xa != xb) return xa < xb;
      if (ca != cb) return ca < cb;
      if (ia >= ea) return false;  // both at the terminator: equal keys
      ++ia;
      ++ib;
    }
  }
};

__global__ void k_s1_iota(int32_t* __restrict__ a, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    a[i] = (int32_t)i;
}

template <typename T>
struct DBuf {
  // stream-ordered pool allocations: the reorder calls these once per Stage-1 iteration
  T* p = nullptr;
  cudaStream_t st = 0;
  ~DBuf() { if (p) cudaFreeAsync(p, st); }
  nm_status alloc(size_t n, cudaStream_t s) {
    st = s;
    return scratch_alloc((void**)&p, sizeof(T) * (n > 0 ? n : 1), s);
  }
};

template <typename F>
nm_status with_temp(F&& f, cudaStream_t s) {
  size_t bytes = 0;
  NM_CUDA(f((void*)nullptr, bytes));
  DBuf<uint8_t> tmp;
  nm_status st = tmp.alloc(bytes, s);
  if (st != NM_OK) return st;
  NM_CUDA(f((void*)tmp.p, bytes));
  (void)s;
  return NM_OK;
}

}  // namespace

// One Stage-1 sort of perm_dev (device int32[n], updated in place), stream-ordered.
nm_status stage1_sort_dev(const DevCsr& A, int32_t* perm_dev, int N, int M, cudaStream_t s) {
  const int64_t n = A.n, nnz = A.nnz, S = (n + M - 1) / M;
  const int B = 256;
  DBuf<int32_t> iperm, order, nperm, flag, ngr;
  DBuf<int64_t> deg, Brp, gid, goff, gx, gc;
  DBuf<uint64_t> k1, k2;
  nm_status st;
  if ((st = iperm.alloc(n, s)) || (st = order.alloc(n, s)) || (st = nperm.alloc(n, s)) || (st = ngr.alloc(n + 1, s)) ||
      (st = deg.alloc(n + 1, s)) || (st = Brp.alloc(n + 1, s)) || (st = goff.alloc(n + 1, s)) || (st = k1.alloc(nnz, s)) ||
      (st = k2.alloc(nnz, s)) || (st = flag.alloc(nnz, s)) || (st = gid.alloc(nnz, s)))
    return st;
  k_s1_inv<<<grid_for(n, B), B, 0, s>>>(perm_dev, iperm.p, n);
  NM_CUDA(cudaMemsetAsync(deg.p, 0, sizeof(int64_t) * (n + 1), s));
  k_s1_deg<<<grid_for(n, B), B, 0, s>>>(A.rp, perm_dev, n, deg.p);
  int64_t* dp = deg.p;
  int64_t* bp = Brp.p;
  if ((st = with_temp([&](void* t, size_t& b) { return cub::DeviceScan::ExclusiveSum(t, b, dp, bp, n + 1, s); }, s)))
    return st;
  k_s1_keys<<<grid_for(n * 32, B), B, 0, s>>>(A.rp, A.ci, perm_dev, iperm.p, n, Brp.p, k1.p);
  int hb = 32;  // key bits: 32 column bits + enough row bits for n
  while (hb < 64 && ((int64_t)1 << (hb - 32)) < n) ++hb;
  uint64_t* a1 = k1.p;
  uint64_t* a2 = k2.p;
  if ((st = with_temp([&](void* t, size_t& b) { return cub::DeviceRadixSort::SortKeys(t, b, a1, a2, nnz, 0, hb, s); }, s)))
    return st;
  // group ids = exclusive scan of the group-start flags
  int64_t ngroups = 0;
  if (nnz > 0) {
    k_s1_flags<<<grid_for(nnz, B), B, 0, s>>>(k2.p, nnz, (uint32_t)M, flag.p);
    int32_t* fp = flag.p;
    int64_t* ip = gid.p;
    if ((st = with_temp([&](void* t, size_t& b) { return cub::DeviceScan::ExclusiveSum(t, b, fp, ip, nnz, s); }, s)))
      return st;
    int64_t last = 0;
    int32_t lastf = 0;
    NM_CUDA(cudaMemcpyAsync(&last, gid.p + nnz - 1, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    NM_CUDA(cudaMemcpyAsync(&lastf, flag.p + nnz - 1, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    NM_CUDA(cudaStreamSynchronize(s));
    ngroups = last + lastf;
  }
  if ((st = gx.alloc(ngroups, s)) || (st = gc.alloc(ngroups, s))) return st;
  NM_CUDA(cudaMemsetAsync(ngr.p, 0, sizeof(int32_t) * (n + 1), s));
  if (nnz > 0)
    k_s1_codes<<<grid_for(nnz, B), B, 0, s>>>(k2.p, nnz, (uint32_t)M, N, S, gid.p, gx.p, gc.p, ngr.p);
  int32_t* np_ = ngr.p;
  int64_t* go = goff.p;
  if ((st = with_temp([&](void* t, size_t& b) { return cub::DeviceScan::ExclusiveSum(t, b, np_, go, n + 1, s); }, s)))
    return st;
  NM_CUDA(cudaGetLastError());
  k_s1_iota<<<grid_for(n, B), B, 0, s>>>(order.p, n);
  int32_t* op = order.p;
  const RowKeyLess less{goff.p, gx.p, gc.p};
  if ((st = with_temp([&](void* t, size_t& b) { return cub::DeviceMergeSort::StableSortKeys(t, b, op, n, less, s); }, s)))
    return st;
  k_s1_apply<<<grid_for(n, B), B, 0, s>>>(perm_dev, order.p, n, nperm.p);
  NM_CUDA(cudaMemcpyAsync(perm_dev, nperm.p, sizeof(int32_t) * n, cudaMemcpyDeviceToDevice, s));
  NM_CUDA(cudaGetLastError());
  NM_CUDA(cudaStreamSynchronize(s));
  return NM_OK;
}

}  // namespace nm
