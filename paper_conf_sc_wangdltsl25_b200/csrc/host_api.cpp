// host_api.cpp -- kami_gemm_strided_batched_host: end-to-end entry point on
// HOST buffers.  The batch is streamed through a double-buffered device
// workspace in chunks; chunk i's host->device copies, kernel and
// device->host copy are queued on stream i % 2, so the copy engines (H2D and
// D2H are separate engines) overlap the other chunk's kernel and copies.
#include <cuda_runtime.h>

#include <cstdint>
#include <mutex>

#include "../../include/kami.h"

namespace {

struct Workspace {
  int device = -1;
  void* buf[2] = {nullptr, nullptr};
  size_t cap = 0;  // bytes per slot
  cudaStream_t st[2] = {nullptr, nullptr};
};

std::mutex g_mu;
Workspace g_ws;

void release_locked() {
  if (g_ws.device >= 0) {
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(g_ws.device);
    for (int i = 0; i < 2; ++i) {
      if (g_ws.buf[i]) cudaFree(g_ws.buf[i]);
      if (g_ws.st[i]) cudaStreamDestroy(g_ws.st[i]);
      g_ws.buf[i] = nullptr;
      g_ws.st[i] = nullptr;
    }
    cudaSetDevice(cur);
  }
  g_ws.device = -1;
  g_ws.cap = 0;
}

size_t round_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

}  // namespace

extern "C" kami_status_t kami_release_workspace(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  release_locked();
  return KAMI_SUCCESS;
}

extern "C" kami_status_t kami_gemm_strided_batched_host(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                                        kami_layout_t layout, const void* A, const void* B,
                                                        void* C) {
  // argument checks identical to the device entry point (no launch yet)
  kami_plan_t plan;
  kami_status_t st = kami_plan(m > 0 ? m : 0, n > 0 ? n : 0, k > 0 ? k : 0, dtype, layout, KAMI_ALGO_AUTO, 0, &plan);
  if (m <= 0 || n <= 0 || k <= 0 || batch < 0) return KAMI_ERROR_INVALID_VALUE;
  if (st != KAMI_SUCCESS) return st;
  if (batch == 0) return KAMI_SUCCESS;
  if (!A || !B || !C) return KAMI_ERROR_INVALID_VALUE;
  const size_t esi = dtype == KAMI_DTYPE_F64 ? 8 : dtype == KAMI_DTYPE_TF32 ? 4
                    : (dtype == KAMI_DTYPE_E4M3 || dtype == KAMI_DTYPE_E5M2) ? 1 : 2;
  const size_t eso = dtype == KAMI_DTYPE_F64 ? 8 : dtype == KAMI_DTYPE_TF32 ? 4 : 2;
  const size_t ea = (size_t)m * k * esi, eb = (size_t)k * n * esi, ec = (size_t)m * n * eso;
  const size_t per_entry = ea + eb + ec;
  // ~64 MiB per chunk: large enough to amortise launches, small enough to pipeline
  int64_t chunk = (int64_t)((64ull << 20) / per_entry);
  if (chunk < 1) chunk = 1;
  if (chunk > batch) chunk = batch;

  std::lock_guard<std::mutex> lk(g_mu);
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return KAMI_ERROR_CUDA;
  const size_t need = round_up((size_t)chunk * ea, 256) + round_up((size_t)chunk * eb, 256) +
                      round_up((size_t)chunk * ec, 256);
  if (g_ws.device != dev || g_ws.cap < need) {
    release_locked();
    g_ws.device = dev;
    for (int i = 0; i < 2; ++i) {
      if (cudaMalloc(&g_ws.buf[i], need) != cudaSuccess) {
        release_locked();
        return KAMI_ERROR_CUDA;
      }
      if (cudaStreamCreateWithFlags(&g_ws.st[i], cudaStreamNonBlocking) != cudaSuccess) {
        release_locked();
        return KAMI_ERROR_CUDA;
      }
    }
    g_ws.cap = need;
  }
  const char* hA = static_cast<const char*>(A);
  const char* hB = static_cast<const char*>(B);
  char* hC = static_cast<char*>(C);
  // On any error below, earlier chunks' copies may still be running on the
  // workspace streams against the caller's host buffers: drain both streams
  // before returning, so the caller may free or reuse them.
  auto fail = [&](kami_status_t code) {
    for (int j = 0; j < 2; ++j) cudaStreamSynchronize(g_ws.st[j]);
    return code;
  };
  int64_t i = 0;
  for (int64_t e0 = 0; e0 < batch; e0 += chunk, ++i) {
    const int64_t ne = (batch - e0) < chunk ? (batch - e0) : chunk;
    const int slot = (int)(i & 1);
    cudaStream_t s = g_ws.st[slot];
    char* dA = static_cast<char*>(g_ws.buf[slot]);
    char* dB = dA + round_up((size_t)chunk * ea, 256);
    char* dC = dB + round_up((size_t)chunk * eb, 256);
    if (cudaMemcpyAsync(dA, hA + e0 * ea, ne * ea, cudaMemcpyHostToDevice, s) != cudaSuccess)
      return fail(KAMI_ERROR_CUDA);
    if (cudaMemcpyAsync(dB, hB + e0 * eb, ne * eb, cudaMemcpyHostToDevice, s) != cudaSuccess)
      return fail(KAMI_ERROR_CUDA);
    st = kami_gemm_strided_batched(m, n, k, ne, dtype, layout, dA, dB, dC, reinterpret_cast<kami_stream_t>(s));
    if (st != KAMI_SUCCESS) return fail(st);
    if (cudaMemcpyAsync(hC + e0 * ec, dC, ne * ec, cudaMemcpyDeviceToHost, s) != cudaSuccess)
      return fail(KAMI_ERROR_CUDA);
  }
  for (int j = 0; j < 2; ++j)
    if (cudaStreamSynchronize(g_ws.st[j]) != cudaSuccess) return KAMI_ERROR_CUDA;
  return KAMI_SUCCESS;
}
