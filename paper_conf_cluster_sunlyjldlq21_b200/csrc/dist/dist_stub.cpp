// Placeholder entry points until the distributed layer lands.
#include "../runtime/internal.h"

extern "C" cst_status cst_dist_create(cst_stencil*, int32_t, int32_t, const void*, cst_dist**) {
  return cst::fail(CST_E_UNSUPPORTED, "cst_dist: not built yet");
}
extern "C" cst_status cst_dist_nccl_unique_id(void*) {
  return cst::fail(CST_E_UNSUPPORTED, "cst_dist: not built yet");
}
extern "C" cst_status cst_dist_sweep(cst_dist*, const cst_setting*, const double* const*,
                                     double* const*, int32_t, void*) {
  return cst::fail(CST_E_UNSUPPORTED, "cst_dist: not built yet");
}
extern "C" cst_status cst_dist_sweep_loopback(cst_stencil*, int32_t, const cst_setting*,
                                              double* const*, double* const*, int32_t, void*) {
  return cst::fail(CST_E_UNSUPPORTED, "cst_dist: not built yet");
}
extern "C" void cst_dist_destroy(cst_dist*) {}
