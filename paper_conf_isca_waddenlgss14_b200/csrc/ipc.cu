// ipc.cu -- peer device memory for the fused multi-GPU exchange (
// include/rmt.h "rmt_ipc_*"): a rank exports a device buffer as a CUDA IPC
// handle, its partner opens it and passes the resulting pointer straight to a
// kernel (the FWT cross-shard combine reads the partner's shard over NVLink
// peer-to-peer loads instead of receiving a staged copy).  Host plumbing only.
#include <cuda.h>
#include <cuda_runtime.h>
#include <string.h>

#include "rmt_host.cuh"

namespace rmt {
namespace {
typedef CUresult (*GetRangeFn)(CUdeviceptr*, size_t*, CUdeviceptr);

GetRangeFn get_range() {
  static GetRangeFn fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (GetRangeFn)p;
  }
  return fn;
}
}  // namespace
}  // namespace rmt

using namespace rmt;

extern "C" {

int rmt_ipc_export(const void* dev_ptr, void* handle, int64_t* offset) {
  if (!dev_ptr || !handle || !offset) {
    set_error("rmt_ipc_export: NULL argument");
    return RMT_EINVAL;
  }
  GetRangeFn range = get_range();
  if (!range) {
    set_error("rmt_ipc_export: cuMemGetAddressRange unavailable");
    return RMT_ECUDA;
  }
  CUdeviceptr base = 0;
  size_t size = 0;
  if (range(&base, &size, (CUdeviceptr)dev_ptr) != CUDA_SUCCESS) {
    set_error("rmt_ipc_export: not a device allocation");
    return RMT_EINVAL;
  }
  cudaIpcMemHandle_t h;
  int rc = cuda_check(cudaIpcGetMemHandle(&h, (void*)base), "cudaIpcGetMemHandle");
  if (rc) return rc;
  static_assert(sizeof(cudaIpcMemHandle_t) == RMT_IPC_HANDLE_BYTES, "IPC handle size");
  memcpy(handle, &h, sizeof(h));
  *offset = (int64_t)((CUdeviceptr)dev_ptr - base);
  return RMT_OK;
}

int rmt_ipc_open(const void* handle, int64_t offset, void** dev_ptr) {
  if (!handle || !dev_ptr || offset < 0) {
    set_error("rmt_ipc_open: bad argument");
    return RMT_EINVAL;
  }
  cudaIpcMemHandle_t h;
  memcpy(&h, handle, sizeof(h));
  void* base = nullptr;
  // lazily enables peer access when the allocation lives on another GPU
  int rc = cuda_check(cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess), "cudaIpcOpenMemHandle");
  if (rc) return rc;
  *dev_ptr = (char*)base + offset;
  return RMT_OK;
}

int rmt_ipc_close(void* dev_ptr, int64_t offset) {
  if (!dev_ptr) return RMT_OK;
  return cuda_check(cudaIpcCloseMemHandle((char*)dev_ptr - offset), "cudaIpcCloseMemHandle");
}

}  // extern "C"
