// probe_g32.cu — the probe-kernel dispatch for |g| = 32 (see wd_host.cuh): one
// translation unit per group size so the build compiles them in parallel.
#define WD_PROBE_TU 32
#include "wd_host.cuh"

namespace wdi {
WD_PROBE_COMBOS(WD_PROBE_INST, 32)
}  // namespace wdi
