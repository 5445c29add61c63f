// Internal declarations of the AdaInf B200 runtime (host C++ side of libadainf.so).
#pragma once
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <stdexcept>
#include <string>

namespace adainf {

typedef __nv_bfloat16 bf16;

struct CudaError : std::runtime_error {
  using std::runtime_error::runtime_error;
};
struct ShapeError : std::runtime_error {
  using std::runtime_error::runtime_error;
};
struct NcclError : std::runtime_error {  // -> ADAINF_ERR_NCCL
  using std::runtime_error::runtime_error;
};

#define CK(expr)                                                                                         \
  do {                                                                                                   \
    cudaError_t _e = (expr);                                                                             \
    if (_e != cudaSuccess)                                                                               \
      throw ::adainf::CudaError(std::string(#expr) + ": " + cudaGetErrorString(_e) + " @" + __FILE__ + ":" + \
                                std::to_string(__LINE__));                                               \
  } while (0)

int num_sms();
int win_mode();
void set_win_mode(int m);  // 0 off, 1 window kernel (base offset 0), 2 window kernel (base-offset phase)

// conv geometry (Cin = padded input channels as stored, multiple of 8)
struct ConvGeom {
  int Cin, Cout, KH, KW, stride, pad, H, W, Ho, Wo;
};

void conv_fwd(const ConvGeom& g, const bf16* x, const int* x_map, const int* count, int n_static, const bf16* w,
              int ldb, const float* bias, const bf16* res, const int* res_map, int act, void* out, bool out_f32,
              cudaStream_t st);
void conv_dgrad(const ConvGeom& g, const bf16* dz, const bf16* w, int ldb, int n, const float* bcast,
                const bf16* sc, const bf16* yact, int mask_act, bf16* dx, cudaStream_t st);
// stride-2 dgrad as one sub-pixel GEMM (MODE_DGRAD_SP): applicable geometry, packed-weight workspace size
// (bf16 [4*Cin][4*Cout]), and the launch (rebuilds the packed weights from the shadow `w` into `wsp` first).
// sc_compact: the shortcut term is stored on the dZ grid ([n][Ho][Wo][Cin]) and belongs to output phase (0,0)
// only (the compact dgrad of a 1x1 stride-2 projection).
bool dgrad_sp_ok(const ConvGeom& g);
size_t dgrad_sp_ws_bytes(const ConvGeom& g);
void conv_dgrad_sp(const ConvGeom& g, const bf16* dz, const bf16* w, int ldb, bf16* wsp, int n, const float* bcast,
                   const bf16* sc, bool sc_compact, const bf16* yact, int mask_act, bf16* dx, cudaStream_t st);
size_t wgrad_ws_bytes(const ConvGeom& g, int n);
void conv_wgrad(const ConvGeom& g, const bf16* x, const bf16* dz, int n, int cin_real, float* ws, size_t ws_bytes,
                float* dw, float* db, cudaStream_t st);

}  // namespace adainf
