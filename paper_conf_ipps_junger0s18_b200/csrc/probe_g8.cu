// probe_g8.cu — the probe-kernel dispatch for |g| = 8 (see wd_host.cuh): one
// translation unit per group size so the build compiles them in parallel.
#define WD_PROBE_TU 8
#include "wd_host.cuh"

namespace wdi {
WD_PROBE_COMBOS(WD_PROBE_INST, 8)
}  // namespace wdi
