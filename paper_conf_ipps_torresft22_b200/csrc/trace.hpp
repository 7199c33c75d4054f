// trace.hpp -- NVTX ranges around the C-ABI calls (SURVEY.md §5 tracing): the
// host-side phases show up by name in nsys / ncu timelines. NVTX v3 is
// header-only; without an attached tool each range costs a predicted branch.
#pragma once
#include <nvtx3/nvToolsExt.h>

namespace paper {

struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange&) = delete;
    NvtxRange& operator=(const NvtxRange&) = delete;
};

}  // namespace paper

#define PAPER_NVTX(name) ::paper::NvtxRange paper_nvtx_range_(name)
