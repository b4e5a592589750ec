// pathtrace.cu -- config 4 (path tracer, Loop Merge over bounces).
// Placeholder until the path tracer lands: the ABI rejects the workload.
#include "sr_internal.h"

namespace sr {
std::string check_pathtrace(const sr_pathtrace_params&, uint64_t) {
  return "SR_WL_PATHTRACE is not implemented in this build";
}
size_t pathtrace_perthread_bytes(uint64_t n) { return 12 * n; }
cudaError_t launch_pathtrace(const LaunchCtx&, const sr_workload&, uint64_t, uint32_t, uint64_t,
                             int, uint32_t) {
  return cudaErrorNotSupported;
}
}  // namespace sr

extern "C" int sr_scene_build(const float*, const uint32_t*, uint32_t, const float*, uint32_t,
                              const float*, void*, size_t, size_t* needed) {
  if (needed) *needed = 0;
  return SR_E_INVALID;
}
