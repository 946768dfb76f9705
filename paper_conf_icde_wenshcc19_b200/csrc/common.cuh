// common.cuh -- shared internals of libgmpsvm (CUDA path only; never included by oracle/).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <stdexcept>
#include <string>

#include "gmpsvm.h"

namespace gmpsvm {

// Error carried through the engine and converted to a status code at the ABI boundary.
struct Error : std::runtime_error {
  int code;
  Error(int c, const std::string& m) : std::runtime_error(m), code(c) {}
};

[[noreturn]] void throw_cuda(cudaError_t e, const char* what, const char* file, int line);

// GMPSVM_SLOW_API=<ms> (diagnostics): report every CUDA runtime call of the library that blocks
// the host longer than that
inline double slow_api_ms() {
  static const double v = getenv("GMPSVM_SLOW_API") ? atof(getenv("GMPSVM_SLOW_API")) : 0.0;
  return v;
}

#define GM_CUDA(call)                                                                                     \
  do {                                                                                                    \
    const double thr_ = ::gmpsvm::slow_api_ms();                                                          \
    const auto t0_ = thr_ > 0 ? std::chrono::steady_clock::now() : std::chrono::steady_clock::time_point(); \
    cudaError_t e_ = (call);                                                                              \
    if (thr_ > 0) {                                                                                       \
      const double ms_ = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0_).count(); \
      if (ms_ > thr_) fprintf(stderr, "[gmpsvm slow api] %.2f ms %s (%s:%d)\n", ms_, #call, __FILE__, __LINE__); \
    }                                                                                                     \
    if (e_ != cudaSuccess) ::gmpsvm::throw_cuda(e_, #call, __FILE__, __LINE__);                           \
  } while (0)

#define GM_CHECK_LAUNCH() GM_CUDA(cudaGetLastError())

extern std::atomic<uint64_t> g_launches;  // kernels launched by this library

// Every kernel launch goes through this macro so gmpsvm_launch_count() is exact.
#define GM_LAUNCH(kernel, grid, block, smem, stream, ...)                  \
  do {                                                                     \
    kernel<<<(grid), (block), (smem), (stream)>>>(__VA_ARGS__);            \
    ::gmpsvm::g_launches.fetch_add(1, std::memory_order_relaxed);          \
    GM_CHECK_LAUNCH();                                                     \
  } while (0)

// Stream-ordered device buffer (cudaMallocAsync / cudaFreeAsync on the owning stream).
template <class T>
struct DevBuf {
  T* p = nullptr;
  cudaStream_t st = nullptr;
  DevBuf() = default;
  DevBuf(size_t count, cudaStream_t s) : st(s) {
    if (count) GM_CUDA(cudaMallocAsync((void**)&p, count * sizeof(T), s));
  }
  DevBuf(const DevBuf&) = delete;
  DevBuf& operator=(const DevBuf&) = delete;
  ~DevBuf() {
    if (p) cudaFreeAsync(p, st);
  }
  T* get() const { return p; }
};

inline int64_t round_up(int64_t a, int64_t b) { return (a + b - 1) / b * b; }
inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

constexpr int kTile = 128;  // GEMM tile edge (rows and columns)
constexpr int kBK = 16;     // GEMM k-step; feature dimension is padded to a multiple of it
constexpr double kTau = 1e-12;  // eta floor (reading R3)

// Pair descriptor (device and host): pair p = (s, t), class-sorted layout.
struct PairDesc {
  int32_t s, t;        // classes, s < t; s is the +1 side
  int32_t n_s, n_t;    // class sizes
  int64_t off_s, off_t;  // first sorted position of class s / t
  int64_t a_off;       // offset of this pair in the concatenated alpha/f arrays
  int32_t pid;         // global pair index
  int32_t pad;
  int64_t r_off;       // ROW_CACHE: offset of this pair's B x ldr row buffer (ldr = round_up(n_p, 4))
};

__host__ __device__ inline int pair_index(int s, int t, int k) { return s * k - s * (s + 1) / 2 + (t - s - 1); }

}  // namespace gmpsvm
