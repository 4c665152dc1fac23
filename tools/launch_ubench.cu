// launch_ubench.cu -- event-timed cost of an (almost) empty kernel after an L2
// flush: no shared memory vs ~200 KB dynamic shared memory vs + TMEM alloc,
// 148 CTAs.  Separates launch / carveout / teardown cost from kernel work.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/launch_ubench tools/launch_ubench.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <algorithm>
#include <vector>

__global__ void k_empty(int* out) { if (out && threadIdx.x == 1023) out[0] = 1; }
__global__ void k_smem(int* out) {
  extern __shared__ uint8_t sm[];
  if (threadIdx.x == 0) sm[0] = 1;
  __syncthreads();
  if (out && sm[0] == 2) out[0] = 1;
}
__global__ void k_tmem(int* out) {
  extern __shared__ uint8_t sm[];
  __shared__ uint32_t slot;
  if ((threadIdx.x >> 5) == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"((uint32_t)__cvta_generic_to_shared(&slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  if ((threadIdx.x >> 5) == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(slot));
  if (out && sm[0] == 2) out[0] = 1;
}

int main() {
  void* flush; cudaMalloc(&flush, 256 << 20);
  int* out; cudaMalloc(&out, 4);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  const int big = 200 * 1024;
  cudaFuncSetAttribute(k_smem, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(k_tmem, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  auto run = [&](const char* name, auto launch, bool fl) {
    std::vector<float> t;
    for (int i = 0; i < 60; ++i) {
      if (fl) cudaMemsetAsync(flush, i, 256 << 20);
      cudaEventRecord(a);
      launch();
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b);
      if (i >= 10) t.push_back(ms * 1e3f);
    }
    std::sort(t.begin(), t.end());
    printf("%-34s flush=%d  median %.2f us  min %.2f us\n", name, (int)fl, t[t.size() / 2], t[0]);
  };
  for (int fl = 0; fl < 2; ++fl) {
    run("empty 148x320, 0 smem", [&] { k_empty<<<148, 320>>>(out); }, fl);
    run("148x320, 200 KB dyn smem", [&] { k_smem<<<148, 320, big>>>(out); }, fl);
    run("148x320, 200 KB + TMEM alloc", [&] { k_tmem<<<148, 320, big>>>(out); }, fl);
    run("1x320, 200 KB + TMEM alloc", [&] { k_tmem<<<1, 320, big>>>(out); }, fl);
  }
  return 0;
}
