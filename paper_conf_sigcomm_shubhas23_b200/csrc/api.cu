#include <atomic>
// C-ABI plumbing: error text, version, device checks.
#include <cstring>
#include <string>

#include "api_common.h"

namespace adainf {

static thread_local std::string t_last_error;

void set_last_error(const std::string& s) { t_last_error = s; }

static std::atomic<int> g_dev_ok[64];  // per device ordinal: 0 unchecked, 1 sm_100 verified

void require_device() {
  int dev = 0;
  if (cudaGetDevice(&dev) == cudaSuccess && dev >= 0 && dev < 64 && g_dev_ok[dev].load(std::memory_order_acquire))
    return;  // verified once per device: one cheap query per ABI call after that
  cudaGetLastError();
  int n = 0;
  cudaError_t e = cudaGetDeviceCount(&n);
  if (e != cudaSuccess || n == 0) {
    cudaGetLastError();
    throw UnsupportedError("no CUDA device: the AdaInf hot path runs only on sm_100 (B200); no CPU fallback");
  }
  int major = 0, minor = 0;
  CK(cudaGetDevice(&dev));
  CK(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev));
  CK(cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev));
  if (major != 10 || minor != 0)
    throw UnsupportedError("device is sm_" + std::to_string(major) + std::to_string(minor) +
                           "; libadainf is built for sm_100a only");
  // stream-ordered workspaces (cudaMallocAsync) stay cached in the device's default pool instead of going back
  // to the driver at every synchronization (the default release threshold of 0 made each eager call allocate)
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
    uint64_t thr = ~0ull;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  cudaGetLastError();
  if (dev < 64) g_dev_ok[dev].store(1, std::memory_order_release);
}

}  // namespace adainf

extern "C" const char* adainf_last_error(void) { return adainf::t_last_error.c_str(); }
extern "C" int32_t adainf_version(void) { return 1; }
