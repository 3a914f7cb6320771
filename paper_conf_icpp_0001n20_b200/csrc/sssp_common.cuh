// sssp_common.cuh -- frontier state shared by the SSSP / BC sweep kernels.
#pragma once
#include <cstdint>

namespace gx {

constexpr uint32_t HEAVY_DEG = 256;  // out-degree above which a slot is split into work items
constexpr uint32_t HCHUNK = 1024;    // edges per heavy work item (32 per lane)

// Per-iteration frontier counters, triple-buffered by iteration (t % 3): the
// sweep of iteration t reads ctr[t%3], appends to ctr[(t+1)%3], and the
// advance kernel clears ctr[(t+2)%3], so no host round trip is needed.
struct SsspCtr {
  unsigned int lcount;        // light queue length
  unsigned int lcursor;       // light work cursor (entries handed out)
  unsigned long long hpack;   // heavy queue: (count << 32) | total chunks
  unsigned int hcursor;       // heavy chunk cursor
  unsigned int pad;
};

struct SsspState {
  unsigned int iter;          // current iteration t
  unsigned int stop;          // 0 running, 1 converged (empty frontier), 2 max_iters
  SsspCtr ctr[3];
  unsigned long long edges;   // edges relaxed, all iterations
  unsigned long long active;  // frontier entries, all iterations
  unsigned int raised;        // merges that raised a copy (diagnostic)
  unsigned int pad;
};

struct SsspQueues {
  int32_t* lq[2];             // light frontier (slot ids), by iteration parity
  int32_t* hq[2];             // heavy frontier slots
  uint32_t* hb[2];            // heavy frontier: first chunk index of each entry
};

}  // namespace gx
