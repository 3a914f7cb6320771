#include "gx_internal.h"
#include "sssp_common.cuh"
namespace gx {
void run_sssp_tpv_iter(gx_graph*, SsspQueues, SsspState*, int&) { GX_THROW(GX_E_UNSUPPORTED, "TPV"); }
}
