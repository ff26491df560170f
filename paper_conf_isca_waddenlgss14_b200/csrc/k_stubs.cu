// k_stubs.cu -- temporary: kernels not yet implemented report RMT_EUNSUPPORTED.
#include "rmt_host.cuh"

namespace rmt {
#define RMT_STUB(name)                                                                   \
  int name##_validate(const rmt_bufs_t*, int64_t) { return RMT_OK; }                     \
  size_t name##_scratch(int64_t, const int64_t*) { return 0; }                           \
  int name##_inter_warps(int64_t, const int64_t*) { return 8; }                          \
  int name##_run(Launch&) {                                                              \
    set_error(#name ": not implemented yet");                                            \
    return RMT_EUNSUPPORTED;                                                             \
  }
}  // namespace rmt
