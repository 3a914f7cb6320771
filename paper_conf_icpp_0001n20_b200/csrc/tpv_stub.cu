#include "gx_internal.h"
#include "sssp_common.cuh"
namespace gx {
void run_sssp_tpv_iter(gx_graph*, SsspAux, SsspState*, uint32_t*, int&) { GX_THROW(GX_E_UNSUPPORTED, "TPV"); }
}
