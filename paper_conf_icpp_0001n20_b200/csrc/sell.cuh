// sell.cuh -- SELL-32 layout constants and builders (sell.cu).
#pragma once
#include "gx_internal.h"

namespace gx {
#ifndef GX_PRW
#define GX_PRW 1024
#endif
constexpr int PRW = GX_PRW;             // rows per window (one CTA per window in the PR pull)
constexpr uint32_t PR_HEAVY = 64;       // degree above which a row is processed warp-per-row (swept: 64 best)
template <class T>
int64_t build_sell(Ctx* c, const uint32_t* rp, const T* payload, const int32_t* lane_row, int64_t nslices, T sentinel,
                   DBuf& slice_len, DBuf& slice_off, DBuf& slab);
// Windowed, degree-sorted SELL-32 of the rows of (rp, payload).
template <class T>
void build_window_sell(Ctx* c, const uint32_t* rp, const T* payload, int64_t n, T sentinel, SellLayout& L);
}  // namespace gx
