// Hardware probe (not product code): issue rate of tcgen05.mma (dense kind::f16, K=16) and
// tcgen05.mma.sp (K=32) for M=128 and N in {64,128,256}, with the A operand in K-major
// SWIZZLE_NONE (the packer's current layout) or SWIZZLE_32B, B in MN-major SWIZZLE_128B.
// Values are garbage (timing only).  Prints cycles per MMA measured over 512 back-to-back
// MMAs on one CTA, and for 148 CTAs concurrently.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o probe_mma_rate probe_mma_rate.cu
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo, uint32_t layout) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)layout << 61;
  return d;
}

__global__ void __launch_bounds__(128, 1) rate_kernel(int sparse, int N, int alayout, int iters,
                                                      unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* s = (uint8_t*)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
  __shared__ uint32_t tslot;
  __shared__ __align__(8) uint64_t bar;
  __shared__ __align__(8) uint64_t bars2[8];
  const int warp = threadIdx.x / 32;
  if (threadIdx.x < 8) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bars2[threadIdx.x])));
  for (int i = threadIdx.x; i < 64 * 1024 / 4; i += 128) ((uint32_t*)s)[i] = 0x3c003c00u;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tb = tslot;
  // metadata column 300 (legal 0x4 nibbles)
  {
    uint32_t taddr = tb + ((uint32_t)(warp * 32) << 16) + 300;
    uint32_t w = 0x44444444u;
    asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(w));
    asm volatile("tcgen05.wait::st.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  if (threadIdx.x == 0) {
    const uint32_t A = su32(s), B = su32(s + 16384);
    uint64_t ad = alayout != 1 ? sdesc(A, 128, 256, 0) : sdesc(A, 16, 256, 6);  // none / SW32
    uint64_t bd = sdesc(B, 4096, 1024, 2);
    uint32_t idesc = (1u << 4) | (1u << 16) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    if (sparse) idesc |= 1u << 2;
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      uint32_t acc = i > 0;
      if (sparse)
        asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %5, 0;\n\t"
                     "tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%3], %4, q;\n\t}" ::"r"(tb),
                     "l"(ad), "l"(bd), "r"(tb + 300), "r"(idesc), "r"(acc));
      else
        asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %4, 0;\n\t"
                     "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, q;\n\t}" ::"r"(tb), "l"(ad), "l"(bd),
                     "r"(idesc), "r"(acc));
      if (alayout >= 2) {  // commit after every MMA (to the done barrier's spare slot)
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
            su32(&bars2[i & 7])));
      }
      if (alayout == 3) {  // ... and wait for that MMA to complete before issuing the next
        uint32_t dn = 0;
        const uint32_t ph = (uint32_t)((i >> 3) & 1);
        while (!dn)
          asm volatile("{\n\t.reg .pred q;\n\tmbarrier.try_wait.parity.shared::cta.b64 q, [%1], %2;\n\tselp.b32 %0, 1, 0, q;\n\t}"
                       : "=r"(dn) : "r"(su32(&bars2[i & 7])), "r"(ph));
      }
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)));
    uint32_t done = 0;
    while (!done)
      asm volatile("{\n\t.reg .pred q;\n\tmbarrier.try_wait.parity.shared::cta.b64 q, [%1], 0;\n\tselp.b32 %0, 1, 0, q;\n\t}"
                   : "=r"(done) : "r"(su32(&bar)));
    long long t1 = clock64();
    out[blockIdx.x] = (unsigned long long)(t1 - t0);
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tb));
}

int main() {
  unsigned long long* d;
  cudaMalloc(&d, 148 * 8);
  cudaFuncSetAttribute(rate_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 80 * 1024);
  const int iters = 512;
  for (int sparse = 0; sparse < 2; ++sparse)
    for (int al = 0; al < 4; ++al)
      for (int N : {64, 128, 256})
        for (int grid : {148}) {
          rate_kernel<<<grid, 128, 80 * 1024>>>(sparse, N, al, iters, d);
          cudaError_t e = cudaDeviceSynchronize();
          if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
          unsigned long long h[148];
          cudaMemcpy(h, d, grid * 8, cudaMemcpyDeviceToHost);
          unsigned long long mx = 0;
          for (int i = 0; i < grid; ++i) mx = h[i] > mx ? h[i] : mx;
          printf("%s A=%s N=%3d grid=%3d: %.1f cycles/MMA\n", sparse ? "sparse K=32" : "dense  K=16",
                 al == 1 ? "SW32" : (al == 2 ? "none+commit" : (al == 3 ? "none+commit+wait" : "none")), N, grid,
                 (double)mx / iters);
        }
  printf("PROBE DONE\n");
  return 0;
}
