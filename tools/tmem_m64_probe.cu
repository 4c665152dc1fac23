// tmem_m64_probe.cu -- where does tcgen05.mma.cta_group::1 with M = 64 put
// its accumulator rows in tensor memory?  (an m-tail unit of 64
// rows drains through one or four epilogue warps depending on the answer.)
// D[i][j] = 1000 (i + 1) + (j + 1) from integer FP16 inputs (exact in FP32);
// all four warps read their 32 lanes x 64 columns with 32x32b loads and the
// host decodes which (row, column) each (lane, column) holds.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o tools/tmem_m64_probe tools/tmem_m64_probe.cu
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

#include "../paper_conf_sc_wangdltsl25_b200/csrc/ptx.cuh"

using namespace kami;

#define CK(x)                                                                              \
  do {                                                                                     \
    cudaError_t e_ = (x);                                                                  \
    if (e_ != cudaSuccess) {                                                               \
      printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__);      \
      exit(1);                                                                             \
    }                                                                                      \
  } while (0)

constexpr int M = 64, N = 64, K = 16;

__global__ void m64_kernel(const __half* A, const __half* Bt, float* out) {
  __shared__ __align__(1024) uint8_t sA[M * 32];
  __shared__ __align__(1024) uint8_t sB[N * 32];
  __shared__ uint32_t slot;
  __shared__ __align__(8) uint64_t bar;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // K-major rows of 32 bytes, 32-byte swizzle (as a TMA box would write them)
  for (int idx = threadIdx.x; idx < M * 2; idx += blockDim.x) {
    const uint32_t off = idx * 16;
    *reinterpret_cast<uint4*>(sA + ptx::swz(off, 1)) =
        *reinterpret_cast<const uint4*>(reinterpret_cast<const uint8_t*>(A) + off);
    *reinterpret_cast<uint4*>(sB + ptx::swz(off, 1)) =
        *reinterpret_cast<const uint4*>(reinterpret_cast<const uint8_t*>(Bt) + off);
  }
  if (threadIdx.x == 0) {
    ptx::mbar_init(&bar, 1);
    ptx::fence_mbar_init();
  }
  ptx::fence_proxy_async_smem();
  if (warp == 0) ptx::tmem_alloc(&slot, 64);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t t = slot;
  if (warp == 0 && lane == 0) {
    const uint32_t idesc = ptx::make_idesc_f16(0, M, N, 0, 0);
    const uint64_t ad = ptx::make_smem_desc(ptx::smem_u32(sA), 16, 256, ptx::umma_layout_code(32));
    const uint64_t bd = ptx::make_smem_desc(ptx::smem_u32(sB), 16, 256, ptx::umma_layout_code(32));
    ptx::umma_f16_ss(t, ad, bd, idesc, 0);
    ptx::umma_commit(&bar);
  }
  __syncwarp();
  ptx::mbar_wait(&bar, 0);
  ptx::tc_fence_after();
  uint32_t r[32];
  for (int c0 = 0; c0 < 64; c0 += 32) {
    ptx::tmem_ld_32x32b_x32(t + ((uint32_t)(warp * 32) << 16) + c0, r);
    ptx::tmem_wait_ld();
    for (int c = 0; c < 32; ++c) out[(warp * 32 + lane) * 64 + c0 + c] = __uint_as_float(r[c]);
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 0) ptx::tmem_dealloc(t, 64);
}

int main() {
  std::vector<__half> hA(M * K, __float2half(0.f)), hB(N * K, __float2half(0.f));
  for (int i = 0; i < M; ++i) {
    hA[i * K + 0] = __float2half((float)(i + 1));
    hA[i * K + 1] = __float2half(1.f);
  }
  for (int j = 0; j < N; ++j) {
    hB[j * K + 0] = __float2half(1000.f);
    hB[j * K + 1] = __float2half((float)(j + 1));
  }
  __half *dA, *dB;
  float* dO;
  CK(cudaMalloc(&dA, M * K * 2));
  CK(cudaMalloc(&dB, N * K * 2));
  CK(cudaMalloc(&dO, 128 * 64 * 4));
  CK(cudaMemcpy(dA, hA.data(), M * K * 2, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dB, hB.data(), N * K * 2, cudaMemcpyHostToDevice));
  CK(cudaMemset(dO, 0, 128 * 64 * 4));
  m64_kernel<<<1, 128>>>(dA, dB, dO);
  CK(cudaDeviceSynchronize());
  std::vector<float> o(128 * 64);
  CK(cudaMemcpy(o.data(), dO, o.size() * 4, cudaMemcpyDeviceToHost));
  // per lane: the rows / columns it holds (0 = nothing written)
  int found = 0;
  for (int lane = 0; lane < 128; ++lane) {
    int rmin = 1 << 30, rmax = -1, cmin = 1 << 30, cmax = -1, cnt = 0;
    for (int c = 0; c < 64; ++c) {
      const int v = (int)o[lane * 64 + c];
      if (v <= 0) continue;
      const int i = v / 1000 - 1, j = v % 1000 - 1;
      if (i < 0 || i >= M || j < 0 || j >= N) continue;
      ++cnt;
      rmin = i < rmin ? i : rmin;
      rmax = i > rmax ? i : rmax;
      cmin = j < cmin ? j : cmin;
      cmax = j > cmax ? j : cmax;
      if (c < 2 && (lane % 16 == 0 || lane % 16 == 15))
        printf("lane %3d col %2d -> D[%d][%d]\n", lane, c, i, j);
    }
    if (cnt) {
      ++found;
      if (lane % 16 == 0) printf("lane %3d: %d values, rows %d..%d, cols %d..%d\n", lane, cnt, rmin, rmax, cmin, cmax);
    }
  }
  printf("lanes holding D values: %d of 128\n", found);
  return 0;
}
