// ubench.cu -- B200 calibration microbenchmarks for the KAMI planner
// (latency/bandwidth of the intra-SM "network";
// Table 2 constants L_sm, B_sm, O_tc).  Standalone program, not part of the
// library:  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ubench ubench.cu
//
// Prints one JSON object:
//   dmma_m8n8k4_tflops, dmma_m16n8k8_tflops, dmma_m16n8k16_tflops,
//   hmma_m16n8k16_tflops (fp32 acc), lds_latency_cycles, lds_bytes_per_cycle_sm,
//   hbm_copy_gbs, sm_count, clock_mhz
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>

#define CK(x)                                                                 \
  do {                                                                        \
    cudaError_t e = (x);                                                      \
    if (e != cudaSuccess) {                                                   \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); \
      exit(1);                                                                \
    }                                                                         \
  } while (0)

constexpr int kIters = 4096;
constexpr int kAcc = 8;  // independent accumulators per warp (hide MMA latency)

__global__ void dmma_m8n8k4(double* out) {
  double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4;
  double c[kAcc][2] = {};
  for (int i = 0; i < kIters; ++i) {
#pragma unroll
    for (int j = 0; j < kAcc; ++j)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                   : "+d"(c[j][0]), "+d"(c[j][1])
                   : "d"(a), "d"(b));
  }
  double s = 0;
  for (int j = 0; j < kAcc; ++j) s += c[j][0] + c[j][1];
  if (s == 12345.678) out[0] = s;
}

__global__ void dmma_m16n8k8(double* out) {
  double a[4], b[2];
  for (int i = 0; i < 4; ++i) a[i] = threadIdx.x * 1e-3 + i;
  for (int i = 0; i < 2; ++i) b[i] = 1.0 + i;
  double c[kAcc][4] = {};
  for (int i = 0; i < kIters; ++i) {
#pragma unroll
    for (int j = 0; j < kAcc; ++j)
      asm volatile(
          "mma.sync.aligned.m16n8k8.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
          "{%0,%1,%2,%3};"
          : "+d"(c[j][0]), "+d"(c[j][1]), "+d"(c[j][2]), "+d"(c[j][3])
          : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(b[0]), "d"(b[1]));
  }
  double s = 0;
  for (int j = 0; j < kAcc; ++j) s += c[j][0] + c[j][3];
  if (s == 12345.678) out[0] = s;
}

__global__ void dmma_m16n8k16(double* out) {
  double a[8], b[4];
  for (int i = 0; i < 8; ++i) a[i] = threadIdx.x * 1e-3 + i;
  for (int i = 0; i < 4; ++i) b[i] = 1.0 + i;
  double c[4][4] = {};
  for (int i = 0; i < kIters; ++i) {
#pragma unroll
    for (int j = 0; j < 4; ++j)
      asm volatile(
          "mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7,%8,%9,%10,%11}, "
          "{%12,%13,%14,%15}, {%0,%1,%2,%3};"
          : "+d"(c[j][0]), "+d"(c[j][1]), "+d"(c[j][2]), "+d"(c[j][3])
          : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(a[4]), "d"(a[5]), "d"(a[6]), "d"(a[7]), "d"(b[0]),
            "d"(b[1]), "d"(b[2]), "d"(b[3]));
  }
  double s = 0;
  for (int j = 0; j < 4; ++j) s += c[j][0] + c[j][3];
  if (s == 12345.678) out[0] = s;
}

__global__ void hmma_m16n8k16(float* out) {
  unsigned a[4], b[2];
  for (int i = 0; i < 4; ++i) a[i] = 0x3c003c00u + threadIdx.x;
  for (int i = 0; i < 2; ++i) b[i] = 0x3c003c00u;
  float c[kAcc][4] = {};
  for (int i = 0; i < kIters; ++i) {
#pragma unroll
    for (int j = 0; j < kAcc; ++j)
      asm volatile(
          "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
          "{%0,%1,%2,%3};"
          : "+f"(c[j][0]), "+f"(c[j][1]), "+f"(c[j][2]), "+f"(c[j][3])
          : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
  }
  float s = 0;
  for (int j = 0; j < kAcc; ++j) s += c[j][0] + c[j][3];
  if (s == 12345.678f) out[0] = s;
}

// SMEM pointer chase: latency of a dependent LDS (the paper's L_sm, Fig. 4b)
__global__ void lds_latency(long long* cycles, int* sink) {
  __shared__ int buf[1024];
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) buf[i] = (i * 97 + 13) & 1023;
  __syncthreads();
  if (threadIdx.x == 0) {
    int p = 0;
    long long t0 = clock64();
    for (int i = 0; i < 4096; ++i) p = buf[p];
    long long t1 = clock64();
    cycles[0] = (t1 - t0) / 4096;
    sink[0] = p;
  }
}

// SMEM bandwidth: conflict-free LDS.128 from all warps (bytes per cycle per SM, B_sm)
__global__ void lds_bw(long long* cycles, float* sink) {
  __shared__ float4 buf[2048];
  for (int i = threadIdx.x; i < 2048; i += blockDim.x) buf[i] = make_float4(i, i, i, i);
  __syncthreads();
  float4 acc = make_float4(0, 0, 0, 0);
  long long t0 = clock64();
  for (int i = 0; i < 1024; ++i) {
    float4 v = buf[(threadIdx.x + i * 32) & 2047];
    acc.x += v.x;
    acc.y += v.y;
    acc.z += v.z;
    acc.w += v.w;
  }
  __syncthreads();
  long long t1 = clock64();
  if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
  if (acc.x == 1.2345f) sink[0] = acc.y + acc.z + acc.w;
}

__global__ void copy_kernel(const float4* __restrict__ a, float4* __restrict__ b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    b[i] = a[i];
}

template <class F>
float time_ms(F f, int reps = 5) {
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a));
  CK(cudaEventCreate(&b));
  f();
  CK(cudaDeviceSynchronize());
  float best = 1e30f;
  for (int r = 0; r < reps; ++r) {
    CK(cudaEventRecord(a));
    f();
    CK(cudaEventRecord(b));
    CK(cudaEventSynchronize(b));
    float ms;
    CK(cudaEventElapsedTime(&ms, a, b));
    if (ms < best) best = ms;
  }
  return best;
}

int main() {
  int dev = 0, sms = 0, clk = 0;
  CK(cudaGetDevice(&dev));
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  CK(cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev));
  double* dout;
  float* fout;
  long long* cyc;
  int* isink;
  CK(cudaMalloc(&dout, 64));
  CK(cudaMalloc(&fout, 64));
  CK(cudaMalloc(&cyc, 8 * 4096));
  CK(cudaMalloc(&isink, 64));
  const int blocks = sms * 4, threads = 256;
  const double warps = blocks * (threads / 32.0);
  float t = time_ms([&] { dmma_m8n8k4<<<blocks, threads>>>(dout); });
  double m8 = warps * kIters * kAcc * 2.0 * 8 * 8 * 4 / (t * 1e-3) / 1e12;
  t = time_ms([&] { dmma_m16n8k8<<<blocks, threads>>>(dout); });
  double m16k8 = warps * kIters * kAcc * 2.0 * 16 * 8 * 8 / (t * 1e-3) / 1e12;
  t = time_ms([&] { dmma_m16n8k16<<<blocks, threads>>>(dout); });
  double m16k16 = warps * kIters * 4 * 2.0 * 16 * 8 * 16 / (t * 1e-3) / 1e12;
  t = time_ms([&] { hmma_m16n8k16<<<blocks, threads>>>(fout); });
  double h16 = warps * kIters * kAcc * 2.0 * 16 * 8 * 16 / (t * 1e-3) / 1e12;

  lds_latency<<<1, 32>>>(cyc, isink);
  CK(cudaDeviceSynchronize());
  long long lat;
  CK(cudaMemcpy(&lat, cyc, 8, cudaMemcpyDeviceToHost));

  lds_bw<<<sms, 1024>>>(cyc, fout);
  CK(cudaDeviceSynchronize());
  long long* hc = (long long*)malloc(8 * sms);
  CK(cudaMemcpy(hc, cyc, 8 * sms, cudaMemcpyDeviceToHost));
  double cyc_avg = 0;
  for (int i = 0; i < sms; ++i) cyc_avg += hc[i];
  cyc_avg /= sms;
  double bsm = 1024.0 * 1024 * 16 / cyc_avg;  // bytes per cycle per SM

  size_t n = (size_t)1 << 28;  // 4 GiB of float4 = 2^28 * 16 B
  float4 *a, *b;
  CK(cudaMalloc(&a, n * 16));
  CK(cudaMalloc(&b, n * 16));
  CK(cudaMemset(a, 0, n * 16));
  t = time_ms([&] { copy_kernel<<<sms * 8, 512>>>(a, b, n); });
  double hbm = 2.0 * n * 16 / (t * 1e-3) / 1e9;

  printf(
      "{\"sm_count\": %d, \"clock_mhz\": %d, \"dmma_m8n8k4_tflops\": %.3f, \"dmma_m16n8k8_tflops\": %.3f, "
      "\"dmma_m16n8k16_tflops\": %.3f, \"hmma_m16n8k16_tflops\": %.3f, \"lds_latency_cycles\": %lld, "
      "\"lds_bytes_per_cycle_sm\": %.2f, \"hbm_copy_gbs\": %.1f}\n",
      sms, clk / 1000, m8, m16k8, m16k16, h16, lat, bsm, hbm);
  return 0;
}
