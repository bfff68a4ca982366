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

#include <cstring>

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

namespace nm {

// ---------------------------------------------------------------------------------------------
// Stage-2 gain tables on the device (Alg. 3 lines 11-14 "GetCandidates",
// PAPER.md:L459-462; the paper's SOGRE computes them on the GPU, L484).  For a primary segment p
// and a batch of targets t_1..t_nb, every entry (u, v) of the M x M table of (p, t_b) holds
//   gp = sum_{w in N(x) \ N(y)} [c_p(w) > N] - [c_p(w) - 1 > N] + sum_{w in N(y) \ N(x)} [c_p(w) > N] - [c_p(w) + 1 > N]
//   gt = sum_{w in N(x) \ N(y)} [c_t(w) > N] - [c_t(w) + 1 > N] + sum_{w in N(y) \ N(x)} [c_t(w) > N] - [c_t(w) - 1 > N]
// with x = perm[u], y = perm[v] and c_s(w) = |N(w) ∩ {perm[q] : q in segment s}| -- the same
// integer sums as the host gain_table (reorder.cpp), so the picks made from them are bit-exact.
// c_s lives in one int32 array of n counters per segment of the batch, filled by scattering the
// neighbour lists of the segment's M vertices and emptied the same way after the tables.
// ---------------------------------------------------------------------------------------------
namespace {

__global__ void k_s2_count(const int64_t* __restrict__ rp, const int32_t* __restrict__ ci,
                           const int32_t* __restrict__ perm, int64_t n, int M, const int64_t* __restrict__ segs,
                           int nseg, int32_t* __restrict__ cnt, int delta) {
  // one warp per (segment k, position j)
  const int64_t wid = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (wid >= (int64_t)nseg * M) return;
  const int k = (int)(wid / M), j = (int)(wid % M);
  const int64_t q = segs[k] * M + j;
  if (q >= n) return;
  const int32_t x = perm[q];
  int32_t* c = cnt + (int64_t)k * n;
  for (int64_t e = rp[x] + lane; e < rp[x + 1]; e += 32) atomicAdd(&c[ci[e]], delta);
}

__device__ __forceinline__ bool in_sorted(const int32_t* __restrict__ a, int64_t len, int32_t v) {
  int64_t lo = 0, hi = len;
  while (lo < hi) {
    const int64_t mid = (lo + hi) >> 1;
    if (a[mid] < v) lo = mid + 1; else hi = mid;
  }
  return lo < len && a[lo] == v;
}

__global__ void k_s2_gain(const int64_t* __restrict__ rp, const int32_t* __restrict__ ci,
                          const int32_t* __restrict__ perm, int64_t n, int N, int M, const int64_t* __restrict__ segs,
                          int nb, const int32_t* __restrict__ cnt, int64_t* __restrict__ tabs) {
  // one warp per (target b, u, v) entry
  const int64_t wid = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (wid >= (int64_t)nb * M * M) return;
  const int b = (int)(wid / (M * M)), r = (int)(wid % (M * M)), i = r / M, j = r % M;
  const int64_t u = segs[0] * M + i, v = segs[b + 1] * M + j;
  int64_t* e = tabs + 2 * ((int64_t)b * M * M + r);
  if (u >= n || v >= n) {
    if (lane == 0) e[0] = e[1] = 0;
    return;
  }
  const int32_t x = perm[u], y = perm[v];
  const int32_t* cp = cnt;
  const int32_t* ct = cnt + (int64_t)(b + 1) * n;
  const int32_t* nx = ci + rp[x];
  const int32_t* ny = ci + rp[y];
  const int64_t dx = rp[x + 1] - rp[x], dy = rp[y + 1] - rp[y];
  long long sp = 0, st = 0;
  for (int64_t k = lane; k < dx; k += 32) {  // w in N(x) \ N(y): x's column leaves p (d = -1)
    const int32_t w = nx[k];
    if (in_sorted(ny, dy, w)) continue;
    const int c1 = cp[w], c2 = ct[w];
    sp += (c1 > N) - (c1 - 1 > N);
    st += (c2 > N) - (c2 + 1 > N);
  }
  for (int64_t k = lane; k < dy; k += 32) {  // w in N(y) \ N(x): y's column enters p (d = +1)
    const int32_t w = ny[k];
    if (in_sorted(nx, dx, w)) continue;
    const int c1 = cp[w], c2 = ct[w];
    sp += (c1 > N) - (c1 + 1 > N);
    st += (c2 > N) - (c2 - 1 > N);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    sp += __shfl_down_sync(0xffffffffu, sp, o);
    st += __shfl_down_sync(0xffffffffu, st, o);
  }
  if (lane == 0) {
    e[0] = sp;
    e[1] = st;
  }
}

}  // namespace

struct S2DeviceTables {
  const DevCsr* A = nullptr;
  cudaStream_t s = nullptr;
  int M = 0, max_batch = 0;
  int32_t* perm = nullptr;   // pass-start order
  int32_t* cnt = nullptr;    // (max_batch + 1) x n counters, zero between calls
  int64_t* segs = nullptr;   // [max_batch + 1]
  int64_t* tabs = nullptr;   // [max_batch * M * M * 2]
  int64_t* h_segs = nullptr;  // pinned staging
  int64_t* h_tabs = nullptr;
};

nm_status s2dev_create(const DevCsr& A, int M, int max_batch, cudaStream_t s, S2DeviceTables** out) {
  S2DeviceTables* t = new S2DeviceTables();
  t->A = &A;
  t->s = s;
  t->M = M;
  t->max_batch = max_batch;
  const size_t ntab = (size_t)max_batch * M * M * 2;
  cudaError_t e = cudaMalloc(&t->perm, sizeof(int32_t) * A.n);
  if (e == cudaSuccess) e = cudaMalloc(&t->cnt, sizeof(int32_t) * (size_t)(max_batch + 1) * A.n);
  if (e == cudaSuccess) e = cudaMalloc(&t->segs, sizeof(int64_t) * (max_batch + 1));
  if (e == cudaSuccess) e = cudaMalloc(&t->tabs, sizeof(int64_t) * ntab);
  if (e == cudaSuccess) e = cudaMallocHost(&t->h_segs, sizeof(int64_t) * (max_batch + 1));
  if (e == cudaSuccess) e = cudaMallocHost(&t->h_tabs, sizeof(int64_t) * ntab);
  if (e == cudaSuccess) e = cudaMemsetAsync(t->cnt, 0, sizeof(int32_t) * (size_t)(max_batch + 1) * A.n, s);
  if (e != cudaSuccess) {
    s2dev_destroy(t);
    return cuda_fail(e, "s2dev_create");
  }
  *out = t;
  return NM_OK;
}

void s2dev_destroy(S2DeviceTables* t) {
  if (!t) return;
  if (t->s) cudaStreamSynchronize(t->s);
  cudaFree(t->perm);
  cudaFree(t->cnt);
  cudaFree(t->segs);
  cudaFree(t->tabs);
  cudaFreeHost(t->h_segs);
  cudaFreeHost(t->h_tabs);
  delete t;
}

nm_status s2dev_set_perm(S2DeviceTables* t, const int32_t* perm_host) {
  NM_CUDA(cudaMemcpyAsync(t->perm, perm_host, sizeof(int32_t) * t->A->n, cudaMemcpyHostToDevice, t->s));
  return NM_OK;
}

nm_status s2dev_tables(S2DeviceTables* t, int64_t p, const int64_t* targets, int nb, int N, int64_t* tabs_out) {
  if (nb < 1) return NM_OK;
  if (nb > t->max_batch) return fail(NM_ERR_INVALID_ARG, "s2dev_tables: batch too large");
  const DevCsr& A = *t->A;
  const int M = t->M;
  t->h_segs[0] = p;
  for (int b = 0; b < nb; ++b) t->h_segs[b + 1] = targets[b];
  NM_CUDA(cudaMemcpyAsync(t->segs, t->h_segs, sizeof(int64_t) * (nb + 1), cudaMemcpyHostToDevice, t->s));
  const int B = 256;
  const int64_t wc = (int64_t)(nb + 1) * M, wg = (int64_t)nb * M * M;
  k_s2_count<<<(unsigned)((wc * 32 + B - 1) / B), B, 0, t->s>>>(A.rp, A.ci, t->perm, A.n, M, t->segs, nb + 1, t->cnt, 1);
  k_s2_gain<<<(unsigned)((wg * 32 + B - 1) / B), B, 0, t->s>>>(A.rp, A.ci, t->perm, A.n, N, M, t->segs, nb, t->cnt,
                                                                t->tabs);
  k_s2_count<<<(unsigned)((wc * 32 + B - 1) / B), B, 0, t->s>>>(A.rp, A.ci, t->perm, A.n, M, t->segs, nb + 1, t->cnt, -1);
  NM_CUDA(cudaGetLastError());
  NM_CUDA(cudaMemcpyAsync(t->h_tabs, t->tabs, sizeof(int64_t) * wg * 2, cudaMemcpyDeviceToHost, t->s));
  NM_CUDA(cudaStreamSynchronize(t->s));
  memcpy(tabs_out, t->h_tabs, sizeof(int64_t) * wg * 2);
  return NM_OK;
}

}  // namespace nm
