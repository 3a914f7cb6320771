// dist.h -- 1-D partitioned execution.
//
// Slot ranges are edge-balanced and aligned to PRW rows (so SSSP bitmap words
// and PR windows never straddle ranks).  Every rank keeps the whole graph and
// full-length attribute vectors but sweeps only its own rows; the exchange
// after each sweep is a collective over the rank copies:
//   SSSP  allreduce(min) of dist + allreduce of the frontier counters
//   PR    allreduce(sum) of the owned contrib slices (zero elsewhere) and of
//         the two scalars (L1 delta, dangling mass)
// `Exch` runs the collective either with NCCL across processes (one GPU per
// rank) or -- for a single device -- across P simulated rank copies with a
// device reduction kernel, which exercises every partitioned code path on
// one GPU.
#pragma once
#include <vector>

#include "gx_internal.h"

namespace gx {

constexpr int64_t PRW_ALIGN = 1024;   // partition alignment = the PR window (sell.cuh PRW)

// edge-balanced bounds [P+1] over rows [0, n) with weights rp, aligned to `align`
std::vector<int64_t> partition_rows(const std::vector<int64_t>& rp, int64_t n, int P, int64_t align);
std::vector<int64_t> partition_rows_dev(Ctx* c, const uint32_t* rp_dev, int64_t n, int P, int64_t align);

struct Exch {
  Ctx* c = nullptr;
  int P = 1;          // ranks (simulated or real)
  bool sim = false;   // true: P copies on this device
  // bufs[p] = rank p's copy (sim) or {local} (NCCL); result replaces every copy
  void min_u32(const std::vector<uint32_t*>& bufs, int64_t n);
  void sum_f32(const std::vector<float*>& bufs, int64_t n);
  void sum_f64(const std::vector<double*>& bufs, int64_t n);
  void sum_u32(const std::vector<uint32_t*>& bufs, int64_t n);
};

}  // namespace gx
