// metrics.cpp — hardware counters of one sweep through the CUPTI range profiler: the
// "GPU metrics" of csTuner's performance dataset, which the paper collects with Nsight
// (SURVEY Q22).  CUPTI is dlopen'ed (absolute path first), so libcst
// loads without it; every failure (library missing, counters not permitted) is reported as
// CST_E_UNSUPPORTED and the tuner then falls back to modelled features.
//
// Flow: host object (chip name + counter availability) -> config image for the metric
// list -> range profiler on the current context, user range + user replay -> push range,
// sweep, pop range, repeated until every pass is submitted -> decode -> evaluate.
#include <cupti_profiler_host.h>
#include <cupti_profiler_target.h>
#include <cupti_range_profiler.h>
#include <cupti_target.h>
#include <dlfcn.h>

#include <cstring>
#include <mutex>

#include "internal.h"

namespace {

struct Cupti {
  decltype(&cuptiProfilerInitialize) init = nullptr;
  decltype(&cuptiDeviceGetChipName) chip = nullptr;
  decltype(&cuptiProfilerGetCounterAvailability) avail = nullptr;
  decltype(&cuptiProfilerHostInitialize) host_init = nullptr;
  decltype(&cuptiProfilerHostDeinitialize) host_deinit = nullptr;
  decltype(&cuptiProfilerHostConfigAddMetrics) add_metrics = nullptr;
  decltype(&cuptiProfilerHostGetConfigImageSize) cfg_size = nullptr;
  decltype(&cuptiProfilerHostGetConfigImage) cfg_image = nullptr;
  decltype(&cuptiProfilerHostEvaluateToGpuValues) evaluate = nullptr;
  decltype(&cuptiRangeProfilerEnable) enable = nullptr;
  decltype(&cuptiRangeProfilerDisable) disable = nullptr;
  decltype(&cuptiRangeProfilerSetConfig) set_config = nullptr;
  decltype(&cuptiRangeProfilerStart) start = nullptr;
  decltype(&cuptiRangeProfilerStop) stop = nullptr;
  decltype(&cuptiRangeProfilerPushRange) push = nullptr;
  decltype(&cuptiRangeProfilerPopRange) pop = nullptr;
  decltype(&cuptiRangeProfilerDecodeData) decode = nullptr;
  decltype(&cuptiRangeProfilerGetCounterDataSize) cd_size = nullptr;
  decltype(&cuptiRangeProfilerCounterDataImageInitialize) cd_init = nullptr;
};

const Cupti* cupti_lib(std::string* err) {
  static Cupti c;
  static bool ok = false;
  static std::string why;
  static std::once_flag once;
  std::call_once(once, [] {
    const char* cands[] = {"/usr/local/cuda/lib64/libcupti.so.12",
                           "/usr/local/cuda/extras/CUPTI/lib64/libcupti.so.12", "libcupti.so.12"};
    void* h = nullptr;
    for (const char* p : cands)
      if ((h = dlopen(p, RTLD_NOW | RTLD_LOCAL))) break;
    if (!h) {
      why = "libcupti.so.12 not found";
      return;
    }
#define CST_SYM(field, name)                          \
  c.field = (decltype(c.field))dlsym(h, #name);       \
  if (!c.field) {                                     \
    why = std::string("libcupti lacks ") + #name;     \
    return;                                           \
  }
    CST_SYM(init, cuptiProfilerInitialize)
    CST_SYM(chip, cuptiDeviceGetChipName)
    CST_SYM(avail, cuptiProfilerGetCounterAvailability)
    CST_SYM(host_init, cuptiProfilerHostInitialize)
    CST_SYM(host_deinit, cuptiProfilerHostDeinitialize)
    CST_SYM(add_metrics, cuptiProfilerHostConfigAddMetrics)
    CST_SYM(cfg_size, cuptiProfilerHostGetConfigImageSize)
    CST_SYM(cfg_image, cuptiProfilerHostGetConfigImage)
    CST_SYM(evaluate, cuptiProfilerHostEvaluateToGpuValues)
    CST_SYM(enable, cuptiRangeProfilerEnable)
    CST_SYM(disable, cuptiRangeProfilerDisable)
    CST_SYM(set_config, cuptiRangeProfilerSetConfig)
    CST_SYM(start, cuptiRangeProfilerStart)
    CST_SYM(stop, cuptiRangeProfilerStop)
    CST_SYM(push, cuptiRangeProfilerPushRange)
    CST_SYM(pop, cuptiRangeProfilerPopRange)
    CST_SYM(decode, cuptiRangeProfilerDecodeData)
    CST_SYM(cd_size, cuptiRangeProfilerGetCounterDataSize)
    CST_SYM(cd_init, cuptiRangeProfilerCounterDataImageInitialize)
#undef CST_SYM
    CUpti_Profiler_Initialize_Params ip = {CUpti_Profiler_Initialize_Params_STRUCT_SIZE};
    if (c.init(&ip) != CUPTI_SUCCESS) {
      why = "cuptiProfilerInitialize failed";
      return;
    }
    ok = true;
  });
  if (!ok && err) *err = why;
  return ok ? &c : nullptr;
}

}  // namespace

using namespace cst;

extern "C" cst_status cst_collect_metrics(cst_stencil* h, const cst_setting* s,
                                          const double* const* in, double* const* out,
                                          const char* const* names, int32_t n, double* values) {
  if (!h || !s || !in || !out || !names || n < 1 || !values)
    return fail(CST_E_INVALID, "null argument");
  std::string why;
  const Cupti* C = cupti_lib(&why);
  if (!C) return fail(CST_E_UNSUPPORTED, "CUPTI range profiler unavailable: " + why);
  // variant first (compile + load outside the profiled range)
  cst_kernel_info info;
  cst_status st = cst_kernel_info_get(h, s, &info);
  if (st != CST_OK) return st;
  CST_CUDA(cudaSetDevice(h->device));
  CST_CUDA(cudaDeviceSynchronize());
  const Driver* d = nullptr;
  st = driver(&d);
  if (st != CST_OK) return st;
  CUcontext ctx = nullptr;
  {
    void* fp = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuCtxGetCurrent", &fp, cudaEnableDefault, &q) != cudaSuccess || !fp)
      return fail(CST_E_CUDA, "cuCtxGetCurrent unavailable");
    if (((CUresult(*)(CUcontext*))fp)(&ctx) != CUDA_SUCCESS || !ctx)
      return fail(CST_E_CUDA, "no current CUDA context");
  }
  auto bad = [&](CUptiResult r, const char* what) {
    return fail(CST_E_UNSUPPORTED, std::string("CUPTI ") + what + " failed (" +
                                       std::to_string((int)r) + ")");
  };
  CUptiResult r;
  // chip + counter availability
  CUpti_Device_GetChipName_Params cp = {CUpti_Device_GetChipName_Params_STRUCT_SIZE};
  cp.deviceIndex = (size_t)h->device;
  if ((r = C->chip(&cp)) != CUPTI_SUCCESS) return bad(r, "GetChipName");
  const std::string chip = cp.pChipName;
  CUpti_Profiler_GetCounterAvailability_Params ap = {
      CUpti_Profiler_GetCounterAvailability_Params_STRUCT_SIZE};
  ap.ctx = ctx;
  if ((r = C->avail(&ap)) != CUPTI_SUCCESS) return bad(r, "GetCounterAvailability(size)");
  std::vector<uint8_t> avail(ap.counterAvailabilityImageSize);
  ap.pCounterAvailabilityImage = avail.data();
  if ((r = C->avail(&ap)) != CUPTI_SUCCESS) return bad(r, "GetCounterAvailability");
  // host object + config image
  CUpti_Profiler_Host_Initialize_Params hp = {CUpti_Profiler_Host_Initialize_Params_STRUCT_SIZE};
  hp.profilerType = CUPTI_PROFILER_TYPE_RANGE_PROFILER;
  hp.pChipName = chip.c_str();
  hp.pCounterAvailabilityImage = avail.data();
  if ((r = C->host_init(&hp)) != CUPTI_SUCCESS) return bad(r, "HostInitialize");
  CUpti_Profiler_Host_Object* host = hp.pHostObject;
  struct HostGuard {
    const Cupti* C;
    CUpti_Profiler_Host_Object* o;
    ~HostGuard() {
      CUpti_Profiler_Host_Deinitialize_Params dp = {
          CUpti_Profiler_Host_Deinitialize_Params_STRUCT_SIZE};
      dp.pHostObject = o;
      C->host_deinit(&dp);
    }
  } hg{C, host};
  std::vector<const char*> mlist(names, names + n);
  CUpti_Profiler_Host_ConfigAddMetrics_Params am = {
      CUpti_Profiler_Host_ConfigAddMetrics_Params_STRUCT_SIZE};
  am.pHostObject = host;
  am.ppMetricNames = mlist.data();
  am.numMetrics = mlist.size();
  if ((r = C->add_metrics(&am)) != CUPTI_SUCCESS) return bad(r, "ConfigAddMetrics");
  CUpti_Profiler_Host_GetConfigImageSize_Params cs = {
      CUpti_Profiler_Host_GetConfigImageSize_Params_STRUCT_SIZE};
  cs.pHostObject = host;
  if ((r = C->cfg_size(&cs)) != CUPTI_SUCCESS) return bad(r, "GetConfigImageSize");
  std::vector<uint8_t> config(cs.configImageSize);
  CUpti_Profiler_Host_GetConfigImage_Params ci = {
      CUpti_Profiler_Host_GetConfigImage_Params_STRUCT_SIZE};
  ci.pHostObject = host;
  ci.pConfigImage = config.data();
  ci.configImageSize = config.size();
  if ((r = C->cfg_image(&ci)) != CUPTI_SUCCESS) return bad(r, "GetConfigImage");
  // range profiler on the context
  CUpti_RangeProfiler_Enable_Params ep = {CUpti_RangeProfiler_Enable_Params_STRUCT_SIZE};
  ep.ctx = ctx;
  if ((r = C->enable(&ep)) != CUPTI_SUCCESS) return bad(r, "RangeProfilerEnable");
  CUpti_RangeProfiler_Object* obj = ep.pRangeProfilerObject;
  struct ObjGuard {
    const Cupti* C;
    CUpti_RangeProfiler_Object* o;
    ~ObjGuard() {
      CUpti_RangeProfiler_Disable_Params dp = {CUpti_RangeProfiler_Disable_Params_STRUCT_SIZE};
      dp.pRangeProfilerObject = o;
      C->disable(&dp);
    }
  } og{C, obj};
  CUpti_RangeProfiler_GetCounterDataSize_Params gs = {
      CUpti_RangeProfiler_GetCounterDataSize_Params_STRUCT_SIZE};
  gs.pRangeProfilerObject = obj;
  gs.pMetricNames = mlist.data();
  gs.numMetrics = mlist.size();
  gs.maxNumOfRanges = 1;
  gs.maxNumRangeTreeNodes = 1;
  if ((r = C->cd_size(&gs)) != CUPTI_SUCCESS) return bad(r, "GetCounterDataSize");
  std::vector<uint8_t> counter(gs.counterDataSize, 0);
  CUpti_RangeProfiler_CounterDataImage_Initialize_Params cdi = {
      CUpti_RangeProfiler_CounterDataImage_Initialize_Params_STRUCT_SIZE};
  cdi.pRangeProfilerObject = obj;
  cdi.pCounterData = counter.data();
  cdi.counterDataSize = counter.size();
  if ((r = C->cd_init(&cdi)) != CUPTI_SUCCESS) return bad(r, "CounterDataImageInitialize");
  CUpti_RangeProfiler_SetConfig_Params sc = {CUpti_RangeProfiler_SetConfig_Params_STRUCT_SIZE};
  sc.pRangeProfilerObject = obj;
  sc.pConfig = config.data();
  sc.configSize = config.size();
  sc.pCounterDataImage = counter.data();
  sc.counterDataImageSize = counter.size();
  sc.range = CUPTI_UserRange;
  sc.replayMode = CUPTI_UserReplay;
  sc.maxRangesPerPass = 1;
  sc.numNestingLevels = 1;
  sc.minNestingLevel = 1;
  sc.passIndex = 0;
  sc.targetNestingLevel = 1;
  if ((r = C->set_config(&sc)) != CUPTI_SUCCESS) return bad(r, "SetConfig");
  bool done = false;
  for (int pass = 0; pass < 64 && !done; ++pass) {
    CUpti_RangeProfiler_Start_Params sp = {CUpti_RangeProfiler_Start_Params_STRUCT_SIZE};
    sp.pRangeProfilerObject = obj;
    if ((r = C->start(&sp)) != CUPTI_SUCCESS) return bad(r, "Start");
    CUpti_RangeProfiler_PushRange_Params pr = {CUpti_RangeProfiler_PushRange_Params_STRUCT_SIZE};
    pr.pRangeProfilerObject = obj;
    pr.pRangeName = "cst_sweep";
    if ((r = C->push(&pr)) != CUPTI_SUCCESS) return bad(r, "PushRange");
    st = cst_sweep(h, s, in, out, 1, nullptr);
    cudaDeviceSynchronize();
    CUpti_RangeProfiler_PopRange_Params pp = {CUpti_RangeProfiler_PopRange_Params_STRUCT_SIZE};
    pp.pRangeProfilerObject = obj;
    C->pop(&pp);
    CUpti_RangeProfiler_Stop_Params so = {CUpti_RangeProfiler_Stop_Params_STRUCT_SIZE};
    so.pRangeProfilerObject = obj;
    if ((r = C->stop(&so)) != CUPTI_SUCCESS) return bad(r, "Stop");
    if (st != CST_OK) return st;
    done = so.isAllPassSubmitted;
  }
  if (!done) return fail(CST_E_INTERNAL, "CUPTI: passes not completed");
  CUpti_RangeProfiler_DecodeData_Params dd = {CUpti_RangeProfiler_DecodeData_Params_STRUCT_SIZE};
  dd.pRangeProfilerObject = obj;
  if ((r = C->decode(&dd)) != CUPTI_SUCCESS) return bad(r, "DecodeData");
  CUpti_Profiler_Host_EvaluateToGpuValues_Params ev = {
      CUpti_Profiler_Host_EvaluateToGpuValues_Params_STRUCT_SIZE};
  ev.pHostObject = host;
  ev.pCounterDataImage = counter.data();
  ev.counterDataImageSize = counter.size();
  ev.ppMetricNames = mlist.data();
  ev.numMetrics = mlist.size();
  ev.rangeIndex = 0;
  std::vector<double> vals(n);
  ev.pMetricValues = vals.data();
  if ((r = C->evaluate(&ev)) != CUPTI_SUCCESS) return bad(r, "EvaluateToGpuValues");
  std::memcpy(values, vals.data(), sizeof(double) * n);
  return CST_OK;
}
