// Status plumbing shared by the C-ABI translation units: no exception crosses the ABI.
#pragma once
#include <cuda_runtime.h>

#include <new>
#include <string>

#include "../../include/adainf.h"
#include "runtime.h"

namespace adainf {

void set_last_error(const std::string& s);
void require_device();  // throws UnsupportedError without an sm_100 device

struct UnsupportedError : std::runtime_error {
  using std::runtime_error::runtime_error;
};
struct InvalidError : std::runtime_error {
  using std::runtime_error::runtime_error;
};
struct CapacityError : std::runtime_error {
  using std::runtime_error::runtime_error;
};

template <class F>
adainf_status guard(F&& f) {
  try {
    f();
    return ADAINF_OK;
  } catch (const ShapeError& e) {
    set_last_error(e.what());
    return ADAINF_ERR_SHAPE;
  } catch (const InvalidError& e) {
    set_last_error(e.what());
    return ADAINF_ERR_INVALID;
  } catch (const CapacityError& e) {
    set_last_error(e.what());
    return ADAINF_ERR_CAPACITY;
  } catch (const UnsupportedError& e) {
    set_last_error(e.what());
    return ADAINF_ERR_UNSUPPORTED;
  } catch (const CudaError& e) {
    set_last_error(e.what());
    return ADAINF_ERR_CUDA;
  } catch (const NcclError& e) {
    set_last_error(e.what());
    return ADAINF_ERR_NCCL;
  } catch (const std::bad_alloc& e) {
    set_last_error("out of host memory");
    return ADAINF_ERR_OOM;
  } catch (const std::exception& e) {
    set_last_error(e.what());
    return ADAINF_ERR_INVALID;
  } catch (...) {
    set_last_error("unknown error");
    return ADAINF_ERR_INVALID;
  }
}

}  // namespace adainf
