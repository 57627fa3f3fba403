// abft_runtime.cu — per-stream workspace / counter pools and the inject hook.
#include <mutex>
#include <unordered_map>

#include "abft_common.cuh"

namespace abft {

namespace {
struct Pool {
  void* ws = nullptr;
  size_t ws_bytes = 0;
  int* ctr = nullptr;
  size_t ctr_n = 0;
};
std::mutex g_mu;
std::unordered_map<uint64_t, Pool>& pools() {
  static auto* p = new std::unordered_map<uint64_t, Pool>();
  return *p;
}
uint64_t key_of(cudaStream_t s) {
  int dev = 0;
  cudaGetDevice(&dev);
  return (reinterpret_cast<uint64_t>(s) << 8) ^ (uint64_t)dev;
}
}  // namespace

int workspace_get(cudaStream_t s, size_t bytes, void** out) {
  std::lock_guard<std::mutex> g(g_mu);
  Pool& p = pools()[key_of(s)];
  if (p.ws_bytes < bytes) {
    if (p.ws) {
      // the old buffer may still be in use by queued work on this stream
      ABFT_CUDA_TRY(cudaStreamSynchronize(s));
      ABFT_CUDA_TRY(cudaFree(p.ws));
    }
    size_t nb = bytes + bytes / 4 + (1 << 20);
    if (cudaMalloc(&p.ws, nb) != cudaSuccess) {
      p.ws = nullptr;
      p.ws_bytes = 0;
      return ABFT_E_NOMEM;
    }
    p.ws_bytes = nb;
  }
  *out = p.ws;
  return 0;
}

int counters_get(cudaStream_t s, size_t n, int** out) {
  std::lock_guard<std::mutex> g(g_mu);
  Pool& p = pools()[key_of(s)];
  if (p.ctr_n < n) {
    if (p.ctr) {
      ABFT_CUDA_TRY(cudaStreamSynchronize(s));
      ABFT_CUDA_TRY(cudaFree(p.ctr));
    }
    size_t nn = n + n / 4 + 1024;
    if (cudaMalloc(&p.ctr, nn * sizeof(int)) != cudaSuccess) {
      p.ctr = nullptr;
      p.ctr_n = 0;
      return ABFT_E_NOMEM;
    }
    ABFT_CUDA_TRY(cudaMemset(p.ctr, 0, nn * sizeof(int)));
    ABFT_CUDA_TRY(cudaDeviceSynchronize());
    p.ctr_n = nn;
  }
  *out = p.ctr;
  return 0;
}

__global__ void inject_kernel64(uint64_t* p, int64_t off, uint64_t mask) { p[off] ^= mask; }
__global__ void inject_kernel32(uint32_t* p, int64_t off, uint32_t mask) { p[off] ^= mask; }

}  // namespace abft

extern "C" int abft_inject(void* ptr, int32_t dtype, int64_t offset, uint64_t xor_mask, abft_stream_t stream) {
  if (!ptr) return -1;
  if (dtype != ABFT_F32 && dtype != ABFT_F64) return -2;
  if (offset < 0) return -3;
  cudaStream_t s = (cudaStream_t)stream;
  if (dtype == ABFT_F64)
    abft::inject_kernel64<<<1, 1, 0, s>>>(reinterpret_cast<uint64_t*>(ptr), offset, xor_mask);
  else
    abft::inject_kernel32<<<1, 1, 0, s>>>(reinterpret_cast<uint32_t*>(ptr), offset, (uint32_t)xor_mask);
  ABFT_CUDA_TRY(cudaGetLastError());
  return 0;
}
