// ubench_tma.cu -- TMA load throughput vs box row width (microbenchmark, not
// part of the library).  A persistent kernel streams a 1 GiB buffer into an
// S-stage shared-memory ring with cp.async.bulk.tensor (3-D boxes of R rows x
// W bytes) or with 1-D cp.async.bulk of the same bytes; one consumer lane
// releases each stage as soon as it lands.  Prints GB/s per configuration.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I../paper_conf_sc_wangdltsl25_b200/csrc \
//        -o ubench_tma ubench_tma.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>

#include "ptx.cuh"

using namespace kami;

#define CK(x)                                                                      \
  do {                                                                             \
    cudaError_t e = (x);                                                           \
    if (e != cudaSuccess) {                                                        \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e));      \
      exit(1);                                                                     \
    }                                                                              \
  } while (0)

__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   ptx::smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(ptx::smem_u32(bar))
               : "memory");
}

__global__ void __launch_bounds__(64, 1)
    tma_stream(const __grid_constant__ CUtensorMap tm, const uint8_t* src, long long nboxes, int S, uint32_t box_bytes,
               int mode) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* ring = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(ring + (size_t)S * box_bytes);
  uint64_t* empty = full + 16;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    ptx::fence_mbar_init();
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t it = 0;
    for (long long b = blockIdx.x; b < nboxes; b += gridDim.x, ++it) {
      const uint32_t s = it % S, ph = (it / S) & 1;
      ptx::mbar_wait(&empty[s], ph ^ 1);
      ptx::mbar_arrive_expect_tx(&full[s], box_bytes);
      if (mode == 0)
        ptx::tma_load_3d(ring + (size_t)s * box_bytes, &tm, &full[s], 0, 0, (int)b);
      else
        bulk_g2s(ring + (size_t)s * box_bytes, src + b * (long long)box_bytes, box_bytes, &full[s]);
    }
  } else if (threadIdx.x == 32) {
    uint32_t it = 0;
    for (long long b = blockIdx.x; b < nboxes; b += gridDim.x, ++it) {
      const uint32_t s = it % S, ph = (it / S) & 1;
      ptx::mbar_wait(&full[s], ph);
      ptx::mbar_arrive(&empty[s]);
    }
  }
}

typedef CUresult (*PFN_enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                            const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                            CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  PFN_enc enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q));
  const size_t total = 1ull << 30;
  uint8_t* buf;
  CK(cudaMalloc(&buf, total));
  CK(cudaMemset(buf, 1, total));
  int sms = 148;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  printf("[\n");
  bool first = true;
  for (int mode = 0; mode < 2; ++mode)
    for (int W : {32, 64, 128})
      for (uint32_t box_bytes : {8192u, 16384u})
        for (int S : {4, 8, 12}) {
          if (mode == 1 && W != 128) continue;  // 1-D bulk: row width irrelevant
          if ((size_t)S * box_bytes > 200 * 1024) continue;
          const int R = box_bytes / W;
          const long long nboxes = total / box_bytes;
          CUtensorMap tm;
          cuuint64_t dims[3] = {(cuuint64_t)W / 2, (cuuint64_t)R, (cuuint64_t)nboxes};
          cuuint64_t strides[2] = {(cuuint64_t)W, (cuuint64_t)W * R};
          cuuint32_t box[3] = {(cuuint32_t)W / 2, (cuuint32_t)R, 1};
          cuuint32_t es[3] = {1, 1, 1};
          CUtensorMapSwizzle sw = W == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                  : W == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                            : CU_TENSOR_MAP_SWIZZLE_32B;
          if (enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 3, buf, dims, strides, box, es,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
            fprintf(stderr, "encode failed W=%d R=%d\n", W, R);
            continue;
          }
          const size_t smem = (size_t)S * box_bytes + 1024 + 512;
          CK(cudaFuncSetAttribute(tma_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
          float best = 1e30f;
          for (int rep = 0; rep < 8; ++rep) {
            cudaEventRecord(e0);
            tma_stream<<<sms, 64, smem>>>(tm, buf, nboxes, S, box_bytes, mode);
            cudaEventRecord(e1);
            CK(cudaEventSynchronize(e1));
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (rep >= 2 && ms < best) best = ms;
          }
          printf("%s {\"mode\": \"%s\", \"row_bytes\": %d, \"box_bytes\": %u, \"stages\": %d, \"GBs\": %.1f}\n",
                 first ? "" : ",", mode == 0 ? "tensor3d" : "bulk1d", W, box_bytes, S, total / (best * 1e-3) / 1e9);
          first = false;
        }
  printf("]\n");
  return 0;
}
