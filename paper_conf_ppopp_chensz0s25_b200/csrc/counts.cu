// nm_count_violations on the GPU: omega, PScore (L396) and MBscore (L382)
// of B = P A P^T.  Entries of B are produced as sorted 64-bit keys; a (row, segment) group
// or a (panel, segment) group is then a contiguous run, examined by the thread that owns its
// first entry.
#include <cub/cub.cuh>

#include <vector>

#include "nm_internal.h"

namespace nm {
namespace {

__global__ void k_keys(const int64_t* __restrict__ rp, const int32_t* __restrict__ ci,
                       const int32_t* __restrict__ perm, const int32_t* __restrict__ iperm, int64_t n,
                       const int64_t* __restrict__ Brp, int V, uint64_t* __restrict__ krow,
                       uint64_t* __restrict__ kpan) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t p = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; p < n; p += nw) {
    const int32_t u = perm[p];
    const int64_t s = rp[u], d = rp[u + 1] - s, o = Brp[p];
    for (int64_t k = lane; k < d; k += 32) {
      const uint32_t q = (uint32_t)iperm[ci[s + k]];
      krow[o + k] = ((uint64_t)p << 32) | q;
      kpan[o + k] = ((uint64_t)(p / V) << 32) | q;
    }
  }
}

__global__ void k_deg(const int64_t* __restrict__ rp, const int32_t* __restrict__ perm, int64_t n,
                      int64_t* __restrict__ deg) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n; p += (int64_t)gridDim.x * blockDim.x)
    deg[p] = rp[perm[p] + 1] - rp[perm[p]];
}

__global__ void k_inv(const int32_t* __restrict__ perm, int32_t* __restrict__ iperm, int64_t n) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n; p += (int64_t)gridDim.x * blockDim.x)
    iperm[perm[p]] = (int32_t)p;
}

__global__ void k_ident(int32_t* __restrict__ perm, int64_t n) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n; p += (int64_t)gridDim.x * blockDim.x)
    perm[p] = (int32_t)p;
}

// group = same (hi32, lo32 / M); count members; threshold test
__global__ void k_groups(const uint64_t* __restrict__ key, int64_t m, int M, int thresh,
                         unsigned long long* __restrict__ total, int32_t* __restrict__ per_seg) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t hi = key[k] >> 32;
    const uint32_t seg = (uint32_t)(key[k] & 0xFFFFFFFFu) / (uint32_t)M;
    if (k > 0 && (key[k - 1] >> 32) == hi && (uint32_t)(key[k - 1] & 0xFFFFFFFFu) / (uint32_t)M == seg) continue;
    int c = 0;
    for (int64_t j = k; j < m && (key[j] >> 32) == hi && (uint32_t)(key[j] & 0xFFFFFFFFu) / (uint32_t)M == seg; ++j)
      ++c;
    if (c > thresh) {
      atomicAdd(total, 1ull);
      if (per_seg) atomicAdd(&per_seg[seg], 1);
    }
  }
}

template <typename T>
struct Buf {
  // stream-ordered pool allocations: the reorder calls these once per Stage-1 iteration
  T* p = nullptr;
  cudaStream_t st = 0;
  ~Buf() { if (p) cudaFreeAsync(p, st); }
  nm_status alloc(size_t n, cudaStream_t s) {
    st = s;
    return scratch_alloc((void**)&p, sizeof(T) * (n > 0 ? n : 1), s);
  }
};

inline int g256(int64_t w) {
  int64_t g = (w + 255) / 256;
  return (int)(g < 1 ? 1 : (g > 148 * 32 ? 148 * 32 : g));
}

}  // namespace

nm_status count_violations_dev(const DevCsr& A, const int32_t* perm_dev, int V, int N, int M, int64_t* omega,
                               int64_t* mb, int32_t* pscore_host, cudaStream_t s) {
  const int64_t n = A.n, nnz = A.nnz, S = (n + M - 1) / M;
  Buf<int32_t> iperm, pid;
  Buf<int64_t> deg, Brp;
  Buf<uint64_t> k1, k2, k3, k4;
  Buf<int32_t> pscore;
  Buf<unsigned long long> tot;
  nm_status st;
  if ((st = iperm.alloc(n, s)) || (st = pid.alloc(n, s)) || (st = deg.alloc(n + 1, s)) || (st = Brp.alloc(n + 1, s)) ||
      (st = k1.alloc(nnz, s)) || (st = k2.alloc(nnz, s)) || (st = k3.alloc(nnz, s)) || (st = k4.alloc(nnz, s)) ||
      (st = pscore.alloc(S, s)) || (st = tot.alloc(2, s)))
    return st;
  const int32_t* perm = perm_dev;
  if (!perm) {
    k_ident<<<g256(n), 256, 0, s>>>(pid.p, n);
    perm = pid.p;
  }
  k_inv<<<g256(n), 256, 0, s>>>(perm, iperm.p, n);
  NM_CUDA(cudaMemsetAsync(deg.p, 0, sizeof(int64_t) * (n + 1), s));
  k_deg<<<g256(n), 256, 0, s>>>(A.rp, perm, n, deg.p);
  {
    size_t bytes = 0;
    NM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, bytes, deg.p, Brp.p, n + 1, s));
    Buf<uint8_t> tmp;
    if ((st = tmp.alloc(bytes, s))) return st;
    NM_CUDA(cub::DeviceScan::ExclusiveSum(tmp.p, bytes, deg.p, Brp.p, n + 1, s));
  }
  k_keys<<<g256(n * 32), 256, 0, s>>>(A.rp, A.ci, perm, iperm.p, n, Brp.p, V, k1.p, k2.p);
  {
    size_t bytes = 0, b2 = 0;
    NM_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, bytes, k1.p, k3.p, nnz, 0, 64, s));
    NM_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, b2, k2.p, k4.p, nnz, 0, 64, s));
    Buf<uint8_t> tmp;
    if ((st = tmp.alloc(bytes > b2 ? bytes : b2, s))) return st;
    NM_CUDA(cub::DeviceRadixSort::SortKeys(tmp.p, bytes, k1.p, k3.p, nnz, 0, 64, s));
    NM_CUDA(cub::DeviceRadixSort::SortKeys(tmp.p, b2, k2.p, k4.p, nnz, 0, 64, s));
  }
  // distinct (panel, column) keys for the vertical constraint
  Buf<int64_t> nsel;
  if ((st = nsel.alloc(1, s))) return st;
  {
    size_t bytes = 0;
    NM_CUDA(cub::DeviceSelect::Unique(nullptr, bytes, k4.p, k2.p, nsel.p, nnz, s));
    Buf<uint8_t> tmp;
    if ((st = tmp.alloc(bytes, s))) return st;
    NM_CUDA(cub::DeviceSelect::Unique(tmp.p, bytes, k4.p, k2.p, nsel.p, nnz, s));
  }
  int64_t nuniq = 0;
  NM_CUDA(cudaMemcpyAsync(&nuniq, nsel.p, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  NM_CUDA(cudaMemsetAsync(tot.p, 0, 2 * sizeof(unsigned long long), s));
  NM_CUDA(cudaMemsetAsync(pscore.p, 0, sizeof(int32_t) * S, s));
  NM_CUDA(cudaStreamSynchronize(s));
  if (nnz) {
    k_groups<<<g256(nnz), 256, 0, s>>>(k3.p, nnz, M, N, tot.p, pscore.p);
    k_groups<<<g256(nuniq), 256, 0, s>>>(k2.p, nuniq, M, 4, tot.p + 1, nullptr);
  }
  NM_CUDA(cudaGetLastError());
  unsigned long long h[2];
  NM_CUDA(cudaMemcpyAsync(h, tot.p, sizeof(h), cudaMemcpyDeviceToHost, s));
  if (pscore_host) NM_CUDA(cudaMemcpyAsync(pscore_host, pscore.p, sizeof(int32_t) * S, cudaMemcpyDeviceToHost, s));
  NM_CUDA(cudaStreamSynchronize(s));
  *omega = (int64_t)h[0];
  *mb = (int64_t)h[1];
  return NM_OK;
}

}  // namespace nm

static nm_status count_violations_impl(const nm_csr* A, const int32_t* perm, int V, int N, int M,
                                       int64_t* omega, int64_t* mbscore, int32_t* pscore) {
  using namespace nm;
  if (!A || !omega || !mbscore) return fail(NM_ERR_INVALID_ARG, "nm_count_violations: NULL argument");
  if (V < 1 || N < 1 || M <= N || M > 32) return fail(NM_ERR_UNSUPPORTED, "nm_count_violations: bad V/N/M");
  if (A->n <= 0 || A->n >= ((int64_t)1 << 31)) return fail(NM_ERR_INVALID_ARG, "nm_count_violations: bad n");
  if (!A->on_device) {
    nm_status st = validate_csr_host(A->n, A->rowptr, A->col, false);
    if (st != NM_OK) return st;
  }
  if (perm) {  // a bad permutation would index out of bounds on the device (k_inv)
    std::vector<uint8_t> seen((size_t)A->n, 0);
    for (int64_t p = 0; p < A->n; ++p) {
      const int32_t v = perm[p];
      if (v < 0 || v >= A->n || seen[(size_t)v]) return fail(NM_ERR_INVALID_ARG, "nm_count_violations: perm is not a permutation");
      seen[(size_t)v] = 1;
    }
  }
  cudaStream_t s = 0;
  DevCsr d;
  nm_csr pattern = *A;
  pattern.val = nullptr;  // counts need the pattern only
  nm_status st = upload_csr(&pattern, NM_F16, &d, s);
  if (st != NM_OK) return st;
  Buf<int32_t> dperm;
  if (perm) {
    if ((st = dperm.alloc((size_t)A->n, s))) return st;
    NM_CUDA(cudaMemcpyAsync(dperm.p, perm, sizeof(int32_t) * A->n, cudaMemcpyHostToDevice, s));
  }
  int64_t w = 0, m = 0;
  st = count_violations_dev(d, dperm.p, V, N, M, &w, &m, pscore, s);
  if (st != NM_OK) return st;
  *omega = w;
  *mbscore = m;
  return NM_OK;
}

extern "C" nm_status nm_count_violations(const nm_csr* A, const int32_t* perm, int V, int N, int M,
                                         int64_t* omega, int64_t* mbscore, int32_t* pscore) {
  return nm::guarded("nm_count_violations",
                     [&] { return count_violations_impl(A, perm, V, N, M, omega, mbscore, pscore); });
}
