// Placeholder entry points until the tuner and distributed layers land.
#include "../runtime/internal.h"

extern "C" void cst_tune_opts_default(cst_tune_opts* o) {
  if (!o) return;
  o->seed = 1;
  o->dataset_size = 128;
  o->sampling_ratio = 0.10;
  o->n_subpops = 2;
  o->subpop_size = 16;
  o->crossover = 0.8;
  o->mutation = 0.005;
  o->top_n = 10;
  o->cv_threshold = 0.02;
  o->max_generations = 50;
  o->num_collections = 3;
  o->time_budget_s = 100.0;
  o->reps = 5;
  o->warmup = 2;
  o->log_path = nullptr;
}

extern "C" cst_status cst_tune(cst_stencil*, const cst_tune_opts*, const double* const*,
                               double* const*, cst_eval_fn, void*, cst_setting*,
                               cst_tune_report*) {
  return cst::fail(CST_E_UNSUPPORTED, "cst_tune: not built yet");
}

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
