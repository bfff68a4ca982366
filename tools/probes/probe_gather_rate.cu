// Hardware probe (not product code): throughput of gathering 32 rows x 256 B ("one chunk"
// of the SpMM B operand) from global memory into a 128B-swizzled shared-memory tile, per SM,
// for the mechanisms the SpMM can use:
//   mode 0: cp.async.cg 16 B + commit/wait_group pipelining (depth D groups)
//   mode 1: cp.async.cg 16 B + cp.async.mbarrier.arrive.noinc (asynchronous completion)
//   mode 2: ld.global.v4 into registers (D chunks ahead) + st.shared.v4
// X is either L2-resident (16 MB) or HBM-sized (512 MB).  148 CTAs x T threads.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o probe_gather_rate probe_gather_rate.cu
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

constexpr int kRowBytes = 256;  // F = 128 halves
constexpr int kChunkBytes = 32 * kRowBytes;
constexpr int kStages = 8;

__device__ __forceinline__ int row_of(int64_t chunk, int k, int64_t nrows) {
  // cheap 32-bit hash, nrows is a power of two
  uint32_t h = ((uint32_t)chunk * 32u + (uint32_t)k) * 2654435761u;
  return (int)((h ^ (h >> 15)) & (uint32_t)(nrows - 1));
}

template <int MODE, int T>
__global__ void __launch_bounds__(T, 1) gather_kernel(const uint8_t* __restrict__ X, int64_t nrows, int chunks,
                                                      unsigned long long* out, uint32_t* sink) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* s = (uint8_t*)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
  __shared__ __align__(8) uint64_t bars[kStages];
  const int t = threadIdx.x;
  constexpr int kPer = kChunkBytes / 16 / T;  // 16-byte pieces per thread per chunk
  if (t == 0)
    for (int i = 0; i < kStages; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&bars[i])), "r"(T));
  __syncthreads();
  long long t0 = clock64();
  uint32_t acc = 0;
  if (MODE == 0 || MODE == 1) {
    for (int c = 0; c < chunks; ++c) {
      const int st = c % kStages;
      const uint32_t base = su32(s + st * kChunkBytes);
      if (MODE == 1 && c >= kStages) {
        // wait until this stage's previous gathers landed
        const uint32_t ph = ((c / kStages) - 1) & 1;
        asm volatile("{\n\t.reg .pred P;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t@!P bra W_%=;\n\t}"
                     ::"r"(su32(&bars[st])), "r"(ph) : "memory");
      }
#pragma unroll
      for (int q = 0; q < kPer; ++q) {
        const int idx = t + T * q;
        const int k = idx >> 4, c16 = idx & 15;
        const uint8_t* src = X + (int64_t)row_of((int64_t)blockIdx.x * chunks + c, k, nrows) * kRowBytes + c16 * 16;
        const uint32_t dst = base + (c16 >> 3) * 4096 + (k >> 3) * 1024 + (k & 7) * 128 + (((c16 & 7) ^ (k & 7)) << 4);
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
      }
      if (MODE == 0) {
        asm volatile("cp.async.commit_group;" ::: "memory");
        asm volatile("cp.async.wait_group %0;" ::"n"(kStages - 2) : "memory");
      } else {
        asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(su32(&bars[st])) : "memory");
      }
    }
    asm volatile("cp.async.wait_all;" ::: "memory");
  } else {
    // register pipeline: loads for chunk c + D are in flight while chunk c is stored
    constexpr int D = 4;
    uint4 buf[D][kPer];
#pragma unroll
    for (int d = 0; d < D; ++d)
#pragma unroll
      for (int q = 0; q < kPer; ++q) {
        const int idx = t + T * q;
        const int k = idx >> 4, c16 = idx & 15;
        buf[d][q] = __ldg((const uint4*)(X + (int64_t)row_of((int64_t)blockIdx.x * chunks + d, k, nrows) * kRowBytes + c16 * 16));
      }
    for (int c = 0; c < chunks; c += D) {
#pragma unroll
      for (int d = 0; d < D; ++d) {
        const int cc = c + d;
        const uint32_t base = su32(s + (cc % kStages) * kChunkBytes);
#pragma unroll
        for (int q = 0; q < kPer; ++q) {
          const int idx = t + T * q;
          const int k = idx >> 4, c16 = idx & 15;
          const uint32_t dst = base + (c16 >> 3) * 4096 + (k >> 3) * 1024 + (k & 7) * 128 + (((c16 & 7) ^ (k & 7)) << 4);
          asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(dst), "r"(buf[d][q].x), "r"(buf[d][q].y),
                       "r"(buf[d][q].z), "r"(buf[d][q].w) : "memory");
          if (cc + D < chunks)
            buf[d][q] = __ldg((const uint4*)(X + (int64_t)row_of((int64_t)blockIdx.x * chunks + cc + D, k, nrows) * kRowBytes + c16 * 16));
        }
      }
    }
  }
  __syncthreads();
  long long t1 = clock64();
  acc += ((uint32_t*)s)[t];
  if (acc == 0x12345678u) sink[0] = acc;
  if (t == 0) out[blockIdx.x] = (unsigned long long)(t1 - t0);
}

template <int MODE, int T>
void run(const uint8_t* X, int64_t nrows, const char* name, const char* xs) {
  unsigned long long* d;
  uint32_t* sink;
  cudaMalloc(&d, 148 * 8);
  cudaMalloc(&sink, 4);
  const int smem = kStages * kChunkBytes + 1024;
  cudaFuncSetAttribute(gather_kernel<MODE, T>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int chunks = 2048;
  gather_kernel<MODE, T><<<148, T, smem>>>(X, nrows, chunks, d, sink);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  gather_kernel<MODE, T><<<148, T, smem>>>(X, nrows, chunks, d, sink);
  cudaEventRecord(e1);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); exit(1); }
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long h[148];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  unsigned long long mx = 0;
  for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
  double bytes = 148.0 * chunks * kChunkBytes;
  printf("%-28s T=%3d X=%s: %.1f cycles/chunk/SM, %.0f GB/s\n", name, T, xs, (double)mx / chunks, bytes / (ms * 1e6));
  cudaFree(d);
  cudaFree(sink);
}

int main() {
  uint8_t* X;
  const int64_t big = 512ll << 20, small = 16ll << 20;
  cudaMalloc(&X, big);
  cudaMemset(X, 1, big);
  for (int which = 0; which < 2; ++which) {
    const int64_t nrows = (which ? big : small) / kRowBytes;
    const char* xs = which ? "512MB" : "16MB ";
    run<0, 128>(X, nrows, "cp.async+wait_group", xs);
    run<0, 256>(X, nrows, "cp.async+wait_group", xs);
    run<1, 128>(X, nrows, "cp.async+mbarrier.noinc", xs);
    run<1, 256>(X, nrows, "cp.async+mbarrier.noinc", xs);
    run<2, 128>(X, nrows, "ldg.v4+sts (regs, D=4)", xs);
    run<2, 256>(X, nrows, "ldg.v4+sts (regs, D=4)", xs);
  }
  printf("PROBE DONE\n");
  return 0;
}
