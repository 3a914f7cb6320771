// sell.cuh -- SELL-32 layout constants and builders (sell.cu).
#pragma once
#include "gx_internal.h"

namespace gx {
constexpr int PRW = 2048;               // rows per exact-mode PR window (CTA)
constexpr uint32_t PR_HEAVY = 256;      // in-degree above which a row is reduced warp-per-row
template <class T>
int64_t build_sell(Ctx* c, const uint32_t* rp, const T* payload, const int32_t* lane_row, int64_t nslices, T sentinel,
                   DBuf& slice_len, DBuf& slice_off, DBuf& slab);
void build_pr_sell(gx_graph* g);
}  // namespace gx
