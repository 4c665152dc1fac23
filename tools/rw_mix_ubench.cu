// rw_mix_ubench.cu -- HBM ceiling for read:write traffic mixes, measured with a
// plain streaming kernel (16-byte vector loads / stores, grid = 148 x 8 CTAs,
// grid-stride): for each mix R:W the kernel reads R bytes and writes W bytes
// per "unit" so the total is 2 GiB of traffic; also cudaMemsetAsync (write
// only).  Context for the low-rank configs (C-store dominated: 1:16, 1:8,
// 1:4 read:write) -- not a product path.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/rw_mix_ubench tools/rw_mix_ubench.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <vector>

// each thread-iteration: reads r 16-byte vectors, writes w 16-byte vectors
__global__ void k_mix(const uint4* __restrict__ src, uint4* __restrict__ dst, long long n_iter, int r, int w) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n_iter; i += stride) {
    uint4 acc = make_uint4(0, 0, 0, 0);
    for (int j = 0; j < r; ++j) {
      uint4 v = src[i * r + j];
      acc.x ^= v.x;
      acc.y ^= v.y;
      acc.z ^= v.z;
      acc.w ^= v.w;
    }
    // coalesced: consecutive threads write consecutive 16-byte vectors of each of the w streams
    for (int j = 0; j < w; ++j) dst[(long long)j * n_iter + i] = make_uint4(acc.x + j, acc.y, acc.z, acc.w);
  }
}

int main() {
  const size_t total = 2ull << 30;  // traffic per launch
  void *src, *dst;
  cudaMalloc(&src, total);
  cudaMalloc(&dst, total);
  cudaMemset(src, 1, total);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  struct Mix { int r, w; };
  const Mix mixes[] = {{2, 1}, {1, 1}, {1, 2}, {1, 4}, {1, 8}, {1, 16}, {0, 1}};
  printf("{");
  for (const Mix& mx : mixes) {
    const long long n_iter = (long long)(total / 16 / (mx.r + mx.w));
    auto run = [&] {
      k_mix<<<148 * 8, 256>>>((const uint4*)src, (uint4*)dst, n_iter, mx.r, mx.w);
    };
    for (int i = 0; i < 5; ++i) run();
    cudaDeviceSynchronize();
    std::vector<float> ts;
    for (int i = 0; i < 30; ++i) {
      cudaEventRecord(e0);
      run();
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      ts.push_back(ms);
    }
    std::sort(ts.begin(), ts.end());
    const double bytes = (double)n_iter * 16 * (mx.r + mx.w);
    printf("\"kernel_%dr%dw\": %.1f, ", mx.r, mx.w, bytes / (ts[ts.size() / 2] * 1e-3) / 1e9);
  }
  {
    std::vector<float> ts;
    for (int i = 0; i < 30; ++i) {
      cudaEventRecord(e0);
      cudaMemsetAsync(dst, i & 0xff, total);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      ts.push_back(ms);
    }
    std::sort(ts.begin(), ts.end());
    printf("\"memset_0r1w\": %.1f, \"unit\": \"GB/s\"}\n", total / (ts[ts.size() / 2] * 1e-3) / 1e9);
  }
  cudaError_t err = cudaGetLastError();
  if (err != cudaSuccess) printf("error %s\n", cudaGetErrorString(err));
  return 0;
}
