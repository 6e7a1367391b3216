// tmm_tc.cu -- placeholder until the tcgen05 body lands.
#include "lp_internal.h"
namespace lp {
bool tmm_tc_supported(int64_t, int64_t, int64_t, int, int, int, int64_t, int64_t, int64_t, const void*, const void*,
                      const void*) {
  return false;
}
cudaError_t launch_tmm_tc(const TmmArgs&, cudaStream_t, const char** why) {
  *why = "not built";
  return cudaErrorNotSupported;
}
}  // namespace lp
