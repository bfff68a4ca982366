// Hardware probe (not product code): random X-row gather throughput into shared memory through
// the TMA bulk-copy path (cp.async.bulk.shared::cta.global, one instruction per row, issued by
// every lane) vs cp.async 16-byte pieces (LDGSTS, the path both SpMM kernels use today).
// X is L2-resident (warmed), rows of RB bytes at random; each warp runs its own ring of S stages
// of 32 rows and waits only on its own mbarriers, like a residual-SpMM warp would.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o probe_bulk_gather probe_bulk_gather.cu
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
  return x;
}

template <int MODE>  // 0 = bulk copy per row (TMA), 1 = cp.async 16-B pieces (LDGSTS)
__global__ void gather_kernel(const uint8_t* __restrict__ X, uint32_t nrows, int RB, int S, int iters,
                              unsigned long long* sink) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ __align__(8) uint64_t bars[32 * 8];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nw = blockDim.x >> 5;
  uint8_t* ring = sm + (size_t)warp * S * 32 * RB;
  uint64_t* wb = bars + warp * 8;
  if (lane < S) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(wb + lane)));
  }
  asm volatile("fence.mbarrier_init.release.cluster;");
  __syncwarp();
  uint32_t seed = (blockIdx.x * nw + warp) * 7919u + lane;
  uint32_t acc = 0;
  for (int it = 0; it < iters + S; ++it) {
    const int s = it % S;
    if (it >= S) {  // consume stage s of iteration it - S
      const uint32_t par = ((it - S) / S) & 1;
      if (MODE == 0) {
        uint32_t done = 0;
        while (!done)
          asm volatile(
              "{\n\t.reg .pred q;\n\tmbarrier.try_wait.parity.shared::cta.b64 q, [%1], %2;\n\tselp.b32 %0, 1, 0, q;\n\t}"
              : "=r"(done)
              : "r"(su32(wb + s)), "r"(par)
              : "memory");
      } else {
        asm volatile("cp.async.wait_group %0;" ::"n"(0) : "memory");
        __syncwarp();
      }
      acc += ring[(size_t)s * 32 * RB + lane * RB];
    }
    if (it < iters) {
      uint8_t* dst = ring + (size_t)s * 32 * RB;
      if (MODE == 0) {
        if (lane == 0)
          asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(wb + s)), "r"(32 * RB)
                       : "memory");
        __syncwarp();
        const uint32_t row = hash32(seed + it * 104729u) % nrows;
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                         su32(dst + lane * RB)),
                     "l"(X + (size_t)row * RB), "r"(RB), "r"(su32(wb + s))
                     : "memory");
      } else {
        const int per = RB / 16;  // pieces per row; 32 rows x per pieces over 32 lanes
        for (int q = 0; q < per; ++q) {
          const int idx = q * 32 + lane, r = idx / per, c = idx % per;
          const uint32_t row = hash32((seed - lane + r) + it * 104729u) % nrows;
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su32(dst + r * RB + c * 16)),
                       "l"(X + (size_t)row * RB + c * 16)
                       : "memory");
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
      }
    }
  }
  if (acc == 0xFFFFFFFFu) sink[0] = acc;
}

int main() {
  setvbuf(stdout, nullptr, _IONBF, 0);
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const size_t xbytes = 60ull << 20;  // C3's X (232,965 x 256 B)
  uint8_t* X;
  cudaMalloc(&X, xbytes);
  cudaMemset(X, 1, xbytes);
  unsigned long long* sink;
  cudaMalloc(&sink, 8);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int mode = 0; mode < 2; ++mode)
    for (int RB : {256, 128})
      for (int warps : {4, 8, 16})
        for (int S : {2, 4}) {
          const size_t smem = (size_t)warps * S * 32 * RB;
          if (smem > 200 * 1024) continue;
          const uint32_t nrows = (uint32_t)(xbytes / RB);
          const int iters = 2000;
          auto k = mode == 0 ? gather_kernel<0> : gather_kernel<1>;
          cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
          k<<<sms, warps * 32, smem>>>(X, nrows, RB, S, 50, sink);  // warm
          cudaEventRecord(a);
          k<<<sms, warps * 32, smem>>>(X, nrows, RB, S, iters, sink);
          cudaEventRecord(b);
          cudaError_t e = cudaEventSynchronize(b);
          if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
          float ms = 0;
          cudaEventElapsedTime(&ms, a, b);
          const double bytes = (double)sms * warps * iters * 32 * RB;
          printf("%s RB=%3d warps=%2d stages=%d: %8.1f GB/s  %.2f B/cycle/SM @1.9GHz\n",
                 mode == 0 ? "bulk(TMA) row/lane" : "cp.async 16B     ", RB, warps, S, bytes / ms / 1e6,
                 bytes / (ms * 1e-3) / sms / 1.9e9);
        }
  printf("PROBE DONE\n");
  return 0;
}
