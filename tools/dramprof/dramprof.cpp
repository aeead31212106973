// dramprof.cpp -- measurement helper for bench.py (NOT part of the product path):
// DRAM bytes moved by the GPU during a host-delimited region, read from the
// hardware counters through the CUPTI Range Profiler (user range, one pass, no
// kernel serialisation or replay: the kernels of the region run exactly as they
// do unprofiled, concurrent streams included).
//
//   int  dp_begin(int device);            // enable + start + push the range
//   int  dp_end(double* out, int nout);   // pop + stop + decode; out[i] = metric i
//   const char* dp_error(void);
//
// Metrics (in order): dram__bytes_read.sum, dram__bytes_write.sum,
// lts__t_sectors_srcunit_tex_op_read.sum (L2 read sectors from the SMs),
// gpu__time_duration.sum (the range's GPU time).  dp_begin fails (returns != 0)
// when the counters need more than one pass or another profiler (e.g. ncu) owns
// them; the caller then reports the traffic as unmeasured.
#include <cuda.h>
#include <cupti_profiler_host.h>
#include <cupti_profiler_target.h>
#include <cupti_range_profiler.h>
#include <cupti_target.h>

#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

namespace {

const char* kMetrics[] = {"dram__bytes_read.sum", "dram__bytes_write.sum",
                          "lts__t_sectors_srcunit_tex_op_read.sum", "gpu__time_duration.sum"};
constexpr size_t kNumMetrics = sizeof(kMetrics) / sizeof(kMetrics[0]);

std::string g_err;
CUpti_RangeProfiler_Object* g_obj = nullptr;
CUpti_Profiler_Host_Object* g_host = nullptr;
std::vector<uint8_t> g_config, g_counter;
bool g_inited = false;

int fail(const char* what, CUptiResult r) {
  const char* s = nullptr;
  cuptiGetResultString(r, &s);
  g_err = std::string(what) + ": " + (s ? s : "?");
  return int(r) ? int(r) : -1;
}

#define TRY(call, what)                         \
  do {                                          \
    CUptiResult _r = (call);                    \
    if (_r != CUPTI_SUCCESS) return fail(what, _r); \
  } while (0)

void teardown() {
  if (g_obj) {
    CUpti_RangeProfiler_Disable_Params p{CUpti_RangeProfiler_Disable_Params_STRUCT_SIZE};
    p.pRangeProfilerObject = g_obj;
    cuptiRangeProfilerDisable(&p);
    g_obj = nullptr;
  }
  if (g_host) {
    CUpti_Profiler_Host_Deinitialize_Params p{CUpti_Profiler_Host_Deinitialize_Params_STRUCT_SIZE};
    p.pHostObject = g_host;
    cuptiProfilerHostDeinitialize(&p);
    g_host = nullptr;
  }
}

}  // namespace

extern "C" {

__attribute__((visibility("default"))) const char* dp_error(void) { return g_err.c_str(); }

__attribute__((visibility("default"))) int dp_begin(int device) {
  teardown();
  CUcontext ctx = nullptr;
  if (cuCtxGetCurrent(&ctx) != CUDA_SUCCESS || !ctx) {
    g_err = "no current CUDA context";
    return -1;
  }
  if (!g_inited) {
    CUpti_Profiler_Initialize_Params ip{CUpti_Profiler_Initialize_Params_STRUCT_SIZE};
    TRY(cuptiProfilerInitialize(&ip), "cuptiProfilerInitialize");
    g_inited = true;
  }
  CUpti_Device_GetChipName_Params cp{CUpti_Device_GetChipName_Params_STRUCT_SIZE};
  cp.deviceIndex = size_t(device);
  TRY(cuptiDeviceGetChipName(&cp), "cuptiDeviceGetChipName");
  CUpti_Profiler_GetCounterAvailability_Params ap{CUpti_Profiler_GetCounterAvailability_Params_STRUCT_SIZE};
  ap.ctx = ctx;
  TRY(cuptiProfilerGetCounterAvailability(&ap), "counter availability size");
  std::vector<uint8_t> avail(ap.counterAvailabilityImageSize);
  ap.pCounterAvailabilityImage = avail.data();
  TRY(cuptiProfilerGetCounterAvailability(&ap), "counter availability");

  CUpti_Profiler_Host_Initialize_Params hp{CUpti_Profiler_Host_Initialize_Params_STRUCT_SIZE};
  hp.profilerType = CUPTI_PROFILER_TYPE_RANGE_PROFILER;
  hp.pChipName = cp.pChipName;
  hp.pCounterAvailabilityImage = avail.data();
  TRY(cuptiProfilerHostInitialize(&hp), "cuptiProfilerHostInitialize");
  g_host = hp.pHostObject;
  CUpti_Profiler_Host_ConfigAddMetrics_Params mp{CUpti_Profiler_Host_ConfigAddMetrics_Params_STRUCT_SIZE};
  mp.pHostObject = g_host;
  mp.ppMetricNames = kMetrics;
  mp.numMetrics = kNumMetrics;
  TRY(cuptiProfilerHostConfigAddMetrics(&mp), "ConfigAddMetrics");
  CUpti_Profiler_Host_GetConfigImageSize_Params sp{CUpti_Profiler_Host_GetConfigImageSize_Params_STRUCT_SIZE};
  sp.pHostObject = g_host;
  TRY(cuptiProfilerHostGetConfigImageSize(&sp), "GetConfigImageSize");
  g_config.assign(sp.configImageSize, 0);
  CUpti_Profiler_Host_GetConfigImage_Params gp{CUpti_Profiler_Host_GetConfigImage_Params_STRUCT_SIZE};
  gp.pHostObject = g_host;
  gp.configImageSize = g_config.size();
  gp.pConfigImage = g_config.data();
  TRY(cuptiProfilerHostGetConfigImage(&gp), "GetConfigImage");
  CUpti_Profiler_Host_GetNumOfPasses_Params np{CUpti_Profiler_Host_GetNumOfPasses_Params_STRUCT_SIZE};
  np.configImageSize = g_config.size();
  np.pConfigImage = g_config.data();
  TRY(cuptiProfilerHostGetNumOfPasses(&np), "GetNumOfPasses");
  if (np.numOfPasses != 1) {
    g_err = "metrics need " + std::to_string(np.numOfPasses) + " passes";
    return -2;
  }

  CUpti_RangeProfiler_Enable_Params ep{CUpti_RangeProfiler_Enable_Params_STRUCT_SIZE};
  ep.ctx = ctx;
  TRY(cuptiRangeProfilerEnable(&ep), "cuptiRangeProfilerEnable");
  g_obj = ep.pRangeProfilerObject;
  CUpti_RangeProfiler_GetCounterDataSize_Params dp{CUpti_RangeProfiler_GetCounterDataSize_Params_STRUCT_SIZE};
  dp.pRangeProfilerObject = g_obj;
  dp.pMetricNames = kMetrics;
  dp.numMetrics = kNumMetrics;
  dp.maxNumOfRanges = 1;
  dp.maxNumRangeTreeNodes = 1;
  TRY(cuptiRangeProfilerGetCounterDataSize(&dp), "GetCounterDataSize");
  g_counter.assign(dp.counterDataSize, 0);
  CUpti_RangeProfiler_CounterDataImage_Initialize_Params cip{
      CUpti_RangeProfiler_CounterDataImage_Initialize_Params_STRUCT_SIZE};
  cip.pRangeProfilerObject = g_obj;
  cip.counterDataSize = g_counter.size();
  cip.pCounterData = g_counter.data();
  TRY(cuptiRangeProfilerCounterDataImageInitialize(&cip), "CounterDataImageInitialize");
  CUpti_RangeProfiler_SetConfig_Params scp{CUpti_RangeProfiler_SetConfig_Params_STRUCT_SIZE};
  scp.pRangeProfilerObject = g_obj;
  scp.configSize = g_config.size();
  scp.pConfig = g_config.data();
  scp.counterDataImageSize = g_counter.size();
  scp.pCounterDataImage = g_counter.data();
  scp.range = CUPTI_UserRange;
  scp.replayMode = CUPTI_UserReplay;
  scp.maxRangesPerPass = 1;
  scp.numNestingLevels = 1;
  scp.minNestingLevel = 1;
  scp.passIndex = 0;
  scp.targetNestingLevel = 1;
  TRY(cuptiRangeProfilerSetConfig(&scp), "cuptiRangeProfilerSetConfig");
  CUpti_RangeProfiler_Start_Params stp{CUpti_RangeProfiler_Start_Params_STRUCT_SIZE};
  stp.pRangeProfilerObject = g_obj;
  TRY(cuptiRangeProfilerStart(&stp), "cuptiRangeProfilerStart");
  CUpti_RangeProfiler_PushRange_Params pp{CUpti_RangeProfiler_PushRange_Params_STRUCT_SIZE};
  pp.pRangeProfilerObject = g_obj;
  pp.pRangeName = "region";
  TRY(cuptiRangeProfilerPushRange(&pp), "cuptiRangeProfilerPushRange");
  return 0;
}

__attribute__((visibility("default"))) int dp_end(double* out, int nout) {
  if (!g_obj) {
    g_err = "dp_begin was not successful";
    return -1;
  }
  CUpti_RangeProfiler_PopRange_Params pp{CUpti_RangeProfiler_PopRange_Params_STRUCT_SIZE};
  pp.pRangeProfilerObject = g_obj;
  TRY(cuptiRangeProfilerPopRange(&pp), "cuptiRangeProfilerPopRange");
  CUpti_RangeProfiler_Stop_Params sp{CUpti_RangeProfiler_Stop_Params_STRUCT_SIZE};
  sp.pRangeProfilerObject = g_obj;
  TRY(cuptiRangeProfilerStop(&sp), "cuptiRangeProfilerStop");
  if (!sp.isAllPassSubmitted) {
    teardown();
    g_err = "range needs more than one pass";
    return -2;
  }
  CUpti_RangeProfiler_DecodeData_Params dp{CUpti_RangeProfiler_DecodeData_Params_STRUCT_SIZE};
  dp.pRangeProfilerObject = g_obj;
  TRY(cuptiRangeProfilerDecodeData(&dp), "cuptiRangeProfilerDecodeData");
  std::vector<double> vals(kNumMetrics, -1.0);
  CUpti_Profiler_Host_EvaluateToGpuValues_Params ev{CUpti_Profiler_Host_EvaluateToGpuValues_Params_STRUCT_SIZE};
  ev.pHostObject = g_host;
  ev.pCounterDataImage = g_counter.data();
  ev.counterDataImageSize = g_counter.size();
  ev.rangeIndex = 0;
  ev.ppMetricNames = kMetrics;
  ev.numMetrics = kNumMetrics;
  ev.pMetricValues = vals.data();
  TRY(cuptiProfilerHostEvaluateToGpuValues(&ev), "EvaluateToGpuValues");
  for (int i = 0; i < nout && size_t(i) < kNumMetrics; ++i) out[i] = vals[i];
  teardown();
  return 0;
}

}  // extern "C"
