// probe.cu -- kami_probe_dmma_peak: the FP64 tensor-core (DMMA) roofline
// denominator measured on the box the library runs on (SURVEY.md 8(d):
// "also measure ... a DMMA loop on the box, and report against both";
// MEASURED_PEAKS.json carries HBM and bf16 figures only).
//
// Every warp of 4 x SM-count CTAs issues chains of independent
// mma.sync.m8n8k4.f64 (8 accumulator pairs per warp hide the DMMA latency),
// the same instruction the FP64 hot path issues (dmma_tma.cu).  Repeated
// launches run for at least `min_ms`: *burst = the best launch (a kernel
// timed alone), *sustained = the median launch of the second half of the run,
// i.e. the rate at the clock the power cap leaves under sustained load
// (bench.py times 50-step graphs of tens to hundreds of ms).
#include <cuda_runtime.h>

#include <algorithm>
#include <vector>

#include "../../include/kami.h"
#include "kernels.h"

namespace kami {
namespace {

constexpr int kIters = 4096;
constexpr int kAcc = 8;

__global__ void __launch_bounds__(256) dmma_probe_kernel(double* out, int iters) {
  double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4;
  double c[kAcc][2] = {};
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < kAcc; ++j)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                   : "+d"(c[j][0]), "+d"(c[j][1])
                   : "d"(a), "d"(b));
  }
  double s = 0;
  for (int j = 0; j < kAcc; ++j) s += c[j][0] + c[j][1];
  if (s == 12345.678) out[0] = s;  // never true; keeps the chains live
}

}  // namespace
}  // namespace kami

extern "C" kami_status_t kami_probe_dmma_peak(double min_ms, double* burst, double* sustained,
                                              kami_stream_t stream_) {
  using namespace kami;
  if (!burst || !sustained || !(min_ms >= 0) || min_ms > 60000) return KAMI_ERROR_INVALID_VALUE;
  cudaStream_t stream = reinterpret_cast<cudaStream_t>(stream_);
  int dev = 0, sms = 148;
  if (cudaGetDevice(&dev) != cudaSuccess) return KAMI_ERROR_CUDA;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  double* sink = nullptr;
  if (cudaMalloc(&sink, 64) != cudaSuccess) return KAMI_ERROR_CUDA;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int blocks = sms * 4, threads = 256;
  const double flops_per_launch = (double)blocks * (threads / 32) * kIters * kAcc * 2.0 * 8 * 8 * 4;
  double best = 0, spent = 0;
  std::vector<std::pair<double, double>> rates;  // (start time ms, TFLOP/s)
  kami_status_t st = KAMI_SUCCESS;
  for (int rep = 0; rep < 100000 && (rep < 3 || spent < min_ms); ++rep) {
    cudaEventRecord(e0, stream);
    dmma_probe_kernel<<<blocks, threads, 0, stream>>>(sink, kIters);
    cudaEventRecord(e1, stream);
    if (cudaEventSynchronize(e1) != cudaSuccess) {
      st = KAMI_ERROR_CUDA;
      break;
    }
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms > 0) {
      const double r = flops_per_launch / (ms * 1e-3) / 1e12;
      rates.emplace_back(spent, r);
      best = std::max(best, r);
    }
    spent += ms;
  }
  set_last_kernel("kami_dmma_probe");
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaFree(sink);
  std::vector<double> late;
  for (const auto& pr : rates)
    if (pr.first >= spent / 2) late.push_back(pr.second);
  if (late.empty())
    for (const auto& pr : rates) late.push_back(pr.second);
  std::sort(late.begin(), late.end());
  *burst = best;
  *sustained = late.empty() ? 0.0 : late[late.size() / 2];
  return st;
}
