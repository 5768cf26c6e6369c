// stubs.cu -- algorithms not yet implemented return GSW_EUNSUPPORTED.
#include "launch.h"

namespace gsw {

gsw_status run_bc(gsw_graph, const int32_t *, int32_t, double *, gsw_run_stats *) { set_error("bc: not built yet"); return GSW_EUNSUPPORTED; }
}  // namespace gsw
