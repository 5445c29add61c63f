// C-ABI plumbing: error text, version, device checks.
#include <cstring>
#include <string>

#include "api_common.h"

namespace adainf {

static thread_local std::string t_last_error;

void set_last_error(const std::string& s) { t_last_error = s; }

void require_device() {
  int n = 0;
  cudaError_t e = cudaGetDeviceCount(&n);
  if (e != cudaSuccess || n == 0) {
    cudaGetLastError();
    throw UnsupportedError("no CUDA device: the AdaInf hot path runs only on sm_100 (B200); no CPU fallback");
  }
  int dev = 0, major = 0, minor = 0;
  CK(cudaGetDevice(&dev));
  CK(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev));
  CK(cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev));
  if (major != 10 || minor != 0)
    throw UnsupportedError("device is sm_" + std::to_string(major) + std::to_string(minor) +
                           "; libadainf is built for sm_100a only");
}

}  // namespace adainf

extern "C" const char* adainf_last_error(void) { return adainf::t_last_error.c_str(); }
extern "C" int32_t adainf_version(void) { return 1; }
