// dist.h -- 1-D partitioned execution (BASELINE north_star:
// "vertices are 1D range-partitioned ... each iteration exchanges boundary
// distances with an NCCL allreduce(min) ..., or allgathers the rank vector
// for PageRank, with a global convergence flag reduced each step").
//
// Slot ranges are edge-balanced and aligned to PRW rows (so SSSP bitmap words
// and PR windows never straddle ranks).  Each rank builds its sweep layouts
// for ITS rows only (rank-local out-CSR for SSSP, rank-local CSC + windowed
// SELL for PageRank; dist.cu build_rank_*), keeps full-length attribute
// vectors (the SURVEY §8(e) design), and exchanges after each sweep:
//   SSSP  reduce-scatter(min) of dist onto the owners' ranges (allreduce(min)
//         when replica groups need every copy's value for the §2.4 merge),
//         plus one sum of the two frontier counters and one min of the far
//         pile's minimum
//   PR    allgather(v) of the owners' contrib slices + ONE fused allreduce of
//         [L1 delta, dangling mass, total mass, replica-group new values]
// `Exch` runs a collective with NCCL across processes (one GPU per rank),
// with a caller-supplied host transport (gx_ctx_create_hosted: staged through
// pinned host memory, e.g. torch.distributed gloo -- two processes can share
// one GPU), or -- for P simulated ranks on ONE device (gx_run_opts.sim_ranks)
// -- across P rank copies with device copies / a reduction kernel.
#pragma once
#include <vector>

#include "gx_internal.h"

namespace gx {

constexpr int64_t PRW_ALIGN = 1024;   // partition alignment = the PR window (sell.cuh PRW)

// edge-balanced bounds [P+1] over rows [0, n) with weights rp, aligned to `align`
std::vector<int64_t> partition_rows(const std::vector<int64_t>& rp, int64_t n, int P, int64_t align);
std::vector<int64_t> partition_rows_dev(Ctx* c, const uint32_t* rp_dev, int64_t n, int P, int64_t align);

enum class Dt { U32 = GX_DT_U32, F32 = GX_DT_F32, F64 = GX_DT_F64 };
enum class Op { SUM = GX_OP_SUM, MIN = GX_OP_MIN };

struct Exch {
  Ctx* c = nullptr;
  int P = 1;          // ranks (simulated or real)
  bool sim = false;   // true: P copies on this device
  // bufs[p] = rank p's copy (sim) or {this rank's buffer}; all in place.
  // allreduce: every copy of [0, n) <- the reduction over the copies
  void allreduce(const std::vector<void*>& bufs, int64_t n, Dt dt, Op op);
  // allgatherv: rank p's slice [off[p], off[p+1]) -> every copy
  void allgatherv(const std::vector<void*>& bufs, const std::vector<int64_t>& off, Dt dt);
  // reduce_scatterv: rank p's copy of its slice [off[p], off[p+1]) <- the
  // reduction over the copies; other slices keep valid (possibly reduced) values
  void reduce_scatterv(const std::vector<void*>& bufs, const std::vector<int64_t>& off, Dt dt, Op op);
};

}  // namespace gx
