// stubs.cpp -- entry points not built yet in this revision (fail loudly).
#include "gx_internal.h"

namespace gx {
void run_scc(gx_graph*, const gx_run_opts&, gx_run_info&) { GX_THROW(GX_E_UNSUPPORTED, "SCC not built yet"); }
void run_mst(gx_graph*, const gx_run_opts&, gx_run_info&) { GX_THROW(GX_E_UNSUPPORTED, "MST not built yet"); }
void run_bc(gx_graph*, const gx_run_opts&, gx_run_info&) { GX_THROW(GX_E_UNSUPPORTED, "BC not built yet"); }
}  // namespace gx
