// trace.hpp — NVTX ranges around the library's build, tune and SpMV entry points
// ("NVTX ranges around build, tune and spmv").  NVTX v3 is header-only: with
// no tool attached a range costs a couple of branches; under Nsight Systems / ncu
// (--nvtx) the calls show as "yaspmv:<entry point>" ranges on the calling thread.
#pragma once

#include <nvtx3/nvToolsExt.h>

namespace yaspmv {

struct TraceRange {
  explicit TraceRange(const char* name) { nvtxRangePushA(name); }
  ~TraceRange() { nvtxRangePop(); }
  TraceRange(const TraceRange&) = delete;
  TraceRange& operator=(const TraceRange&) = delete;
};

}  // namespace yaspmv
