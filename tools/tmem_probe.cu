// tmem_probe.cu -- measured facts for the TMEM-resident A operand (DESIGN.md
// "tcgen05 TS form").  Two questions, answered on the box:
//  (1) tcgen05.st data layouts: which (lane, column) each thread/register of
//      the .16x64b / .16x128b / .16x256b / .32x32b shapes lands in (read back
//      with the documented .32x32b tcgen05.ld: thread t = lane t).
//  (2) the A-in-TMEM operand layout of tcgen05.mma.cta_group::1.kind::f16
//      with M = 128: A row i in TMEM lane i, K pairs packed per 32-bit column
//      (low half = even k) -- checked by an integer GEMM against the CPU, for
//      K = 16 and K = 32 (second MMA at A column + 8), N = 64.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o tools/tmem_probe tools/tmem_probe.cu
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

#include "../paper_conf_sc_wangdltsl25_b200/csrc/ptx.cuh"

using namespace kami;

#define CK(x)                                                                                \
  do {                                                                                       \
    cudaError_t e_ = (x);                                                                    \
    if (e_ != cudaSuccess) {                                                                 \
      printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__);        \
      exit(1);                                                                               \
    }                                                                                        \
  } while (0)

// ---------------------------------------------------------------- (1) layouts
__global__ void st_layout_kernel(uint32_t* out, int shape) {
  __shared__ uint32_t slot;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == 0) ptx::tmem_alloc(&slot, 32);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t t = slot;
  if (warp == 0) {
    // zero the 32 lanes x 8 columns first
    uint32_t z[16] = {};
    ptx::tmem_st_32x32b_x16(t, z);
    ptx::tmem_wait_st();
    const uint32_t v0 = 1000u + lane * 16 + 0, v1 = 1000u + lane * 16 + 1, v2 = 1000u + lane * 16 + 2,
                   v3 = 1000u + lane * 16 + 3;
    if (shape == 0)
      asm volatile("tcgen05.st.sync.aligned.16x64b.x1.b32 [%0], {%1};" ::"r"(t), "r"(v0) : "memory");
    else if (shape == 1)
      asm volatile("tcgen05.st.sync.aligned.16x128b.x1.b32 [%0], {%1, %2};" ::"r"(t), "r"(v0), "r"(v1) : "memory");
    else if (shape == 2)
      asm volatile("tcgen05.st.sync.aligned.16x256b.x1.b32 [%0], {%1, %2, %3, %4};" ::"r"(t), "r"(v0), "r"(v1),
                   "r"(v2), "r"(v3)
                   : "memory");
    else
      asm volatile("tcgen05.st.sync.aligned.32x32b.x2.b32 [%0], {%1, %2};" ::"r"(t), "r"(v0), "r"(v1) : "memory");
    ptx::tmem_wait_st();
    uint32_t r[16];
    ptx::tmem_ld_32x32b_x16(t, r);
    ptx::tmem_wait_ld();
    for (int c = 0; c < 16; ++c) out[lane * 16 + c] = r[c];
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 0) ptx::tmem_dealloc(t, 32);
}

// --------------------------------------------------------- (2) TS-form MMA
// A: 128 x K (row-major fp16 in global), B: K x 64 given as B^T (64 x K,
// K-major) in global; D = A B (128 x 64 fp32).  B^T goes into SMEM in the
// canonical K-major layout with a 2K-byte swizzle atom (SW32 for K = 16, SW64
// for K = 32): row n at n * 2K bytes, 16-byte chunks XOR-swizzled.
template <int K>
__global__ void ts_mma_kernel(const __half* A, const __half* Bt, float* D) {
  constexpr int N = 64, RB = 2 * K;  // B row bytes
  __shared__ __align__(1024) uint8_t sB[N * RB];
  __shared__ uint32_t slot;
  __shared__ __align__(8) uint64_t bar;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // B^T into smem (generic stores), swizzled like TMA would write it
  const uint32_t bbits = RB == 128 ? 3 : RB == 64 ? 2 : 1;
  for (int idx = threadIdx.x; idx < N * RB / 16; idx += blockDim.x) {
    const uint32_t off = idx * 16;
    const uint4 v = *reinterpret_cast<const uint4*>(reinterpret_cast<const uint8_t*>(Bt) + off);
    *reinterpret_cast<uint4*>(sB + ptx::swz(off, bbits)) = v;
  }
  if (threadIdx.x == 0) {
    ptx::mbar_init(&bar, 1);
    ptx::fence_mbar_init();
  }
  ptx::fence_proxy_async_smem();
  if (warp == 0) ptx::tmem_alloc(&slot, 128);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t t = slot;
  const uint32_t a_tmem = t + 64;  // columns 64..64+K/2 hold A; D at 0..63
  // A: warp w stores lanes 32w.., thread = lane = row, K/2 packed columns
  {
    const int row = warp * 32 + lane;
    uint32_t r[16] = {};
    for (int j = 0; j < K / 2; ++j) {
      const __half lo = A[row * K + 2 * j], hi = A[row * K + 2 * j + 1];
      r[j] = (uint32_t)__half_as_ushort(lo) | ((uint32_t)__half_as_ushort(hi) << 16);
    }
    ptx::tmem_st_32x32b_x16(a_tmem + ((uint32_t)(warp * 32) << 16), r);
    ptx::tmem_wait_st();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 0 && lane == 0) {
    const uint32_t idesc = ptx::make_idesc_f16(0, 128, N, 0, 0);
    const uint64_t bdesc = ptx::make_smem_desc(ptx::smem_u32(sB), 16, 8 * RB, ptx::umma_layout_code(RB));
    for (int ks = 0; ks < K / 16; ++ks)
      ptx::umma_f16_ts(t, a_tmem + 8 * ks, bdesc + 2 * ks, idesc, ks != 0);
    ptx::umma_commit(&bar);
  }
  __syncwarp();
  ptx::mbar_wait(&bar, 0);
  ptx::tc_fence_after();
  {
    uint32_t r[32];
    const int row = warp * 32 + lane;
    for (int c0 = 0; c0 < N; c0 += 32) {
      ptx::tmem_ld_32x32b_x32(t + ((uint32_t)(warp * 32) << 16) + c0, r);
      ptx::tmem_wait_ld();
      for (int c = 0; c < 32; ++c) D[row * N + c0 + c] = __uint_as_float(r[c]);
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 0) ptx::tmem_dealloc(t, 128);
}

template <int K>
int run_ts() {
  const int M = 128, N = 64;
  std::vector<__half> hA(M * K), hBt(N * K);
  std::vector<float> ref(M * N, 0.f), got(M * N);
  srand(7 + K);
  std::vector<int> a(M * K), b(K * N);
  for (int i = 0; i < M * K; ++i) a[i] = rand() % 9 - 4;
  for (int i = 0; i < K * N; ++i) b[i] = rand() % 9 - 4;
  for (int i = 0; i < M; ++i)
    for (int l = 0; l < K; ++l) hA[i * K + l] = __float2half((float)a[i * K + l]);
  for (int l = 0; l < K; ++l)
    for (int j = 0; j < N; ++j) hBt[j * K + l] = __float2half((float)b[l * N + j]);
  for (int i = 0; i < M; ++i)
    for (int j = 0; j < N; ++j) {
      int s = 0;
      for (int l = 0; l < K; ++l) s += a[i * K + l] * b[l * N + j];
      ref[i * N + j] = (float)s;
    }
  __half *dA, *dB;
  float* dD;
  CK(cudaMalloc(&dA, M * K * 2));
  CK(cudaMalloc(&dB, N * K * 2));
  CK(cudaMalloc(&dD, M * N * 4));
  CK(cudaMemcpy(dA, hA.data(), M * K * 2, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dB, hBt.data(), N * K * 2, cudaMemcpyHostToDevice));
  CK(cudaMemset(dD, 0xff, M * N * 4));
  ts_mma_kernel<K><<<1, 128>>>(dA, dB, dD);
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(got.data(), dD, M * N * 4, cudaMemcpyDeviceToHost));
  int bad = 0;
  for (int i = 0; i < M * N; ++i)
    if (got[i] != ref[i]) {
      if (bad < 5) printf("  K=%d mismatch at (%d,%d): got %g want %g\n", K, i / N, i % N, got[i], ref[i]);
      ++bad;
    }
  printf("ts_mma K=%d: %s (%d mismatches of %d)\n", K, bad ? "FAIL" : "OK", bad, M * N);
  cudaFree(dA);
  cudaFree(dB);
  cudaFree(dD);
  return bad;
}

int main() {
  uint32_t* d;
  CK(cudaMalloc(&d, 32 * 16 * 4));
  const char* names[] = {"16x64b.x1", "16x128b.x1", "16x256b.x1", "32x32b.x2"};
  for (int s = 0; s < 4; ++s) {
    CK(cudaMemset(d, 0, 32 * 16 * 4));
    st_layout_kernel<<<1, 32>>>(d, s);
    CK(cudaDeviceSynchronize());
    uint32_t h[32 * 16];
    CK(cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost));
    printf("st %s: (lane,col) <- thread.reg\n", names[s]);
    for (int l = 0; l < 32; ++l) {
      bool any = false;
      for (int c = 0; c < 16; ++c) any |= h[l * 16 + c] != 0;
      if (!any) continue;
      printf("  lane %2d:", l);
      for (int c = 0; c < 8; ++c) {
        const uint32_t v = h[l * 16 + c];
        if (v) printf(" c%d=t%u.r%u", c, (v - 1000) / 16, (v - 1000) % 16);
        else printf(" c%d=-", c);
      }
      printf("\n");
    }
  }
  int bad = run_ts<16>() + run_ts<32>();
  printf("tmem_probe %s\n", bad ? "FAILED" : "PASSED");
  return bad ? 1 : 0;
}
