// gx_internal.h -- internal types of libgraffix (not part of the C ABI).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <cstring>
#include <stdexcept>
#include <string>
#include <vector>

#include "../../include/graffix.h"

namespace gx {

struct Error : std::runtime_error {
  gx_status st;
  Error(gx_status s, const std::string& m) : std::runtime_error(m), st(s) {}
};

#define GX_THROW(st, msg) throw ::gx::Error((st), (msg))
#define GX_CHECK_ARG(cond, msg) \
  do { if (!(cond)) GX_THROW(GX_E_INVALID, msg); } while (0)
#define CUDA_OK(expr)                                                                  \
  do {                                                                                 \
    cudaError_t e_ = (expr);                                                           \
    if (e_ != cudaSuccess) {                                                           \
      if (e_ == cudaErrorMemoryAllocation)                                             \
        GX_THROW(GX_E_OOM, std::string(#expr ": ") + cudaGetErrorString(e_));          \
      GX_THROW(GX_E_CUDA, std::string(#expr ": ") + cudaGetErrorString(e_));           \
    }                                                                                  \
  } while (0)

constexpr uint32_t INF = 0xFFFFFFFFu;
enum SlotKind : uint8_t { OWNER = 0, REPLICA = 1, HOLE = 2 };
enum AddKind : uint8_t { ADD_NONE = 0, ADD_COALESCE = 1, ADD_SMEM = 2, ADD_DEGNORM = 3 };

struct Ctx;

// Device buffer owned by the library (allocator hook or cudaMallocAsync).
struct DBuf {
  Ctx* ctx = nullptr;
  void* p = nullptr;
  size_t bytes = 0;
  DBuf() = default;
  DBuf(const DBuf&) = delete;
  DBuf& operator=(const DBuf&) = delete;
  DBuf(DBuf&& o) noexcept { *this = std::move(o); }
  DBuf& operator=(DBuf&& o) noexcept;
  ~DBuf() { reset(); }
  void reset();
  void alloc(Ctx* c, size_t b);
  template <class T> T* as() const { return reinterpret_cast<T*>(p); }
};

struct Ctx {
  int device = 0;
  cudaStream_t stream = nullptr;
  cudaStream_t copy_stream = nullptr;   // GX_ASYNC_UPLOAD: weights H2D + {col, w} interleave (lazily created)
  bool own_stream = false;
  gx_alloc_fn alloc = nullptr;
  gx_release_fn release = nullptr;
  void* user = nullptr;
  int rank = 0, world = 1;
  void* nccl = nullptr;  // ncclComm_t
  gx_coll_fn coll = nullptr;   // hosted exchange (gx_ctx_create_hosted): caller's transport
  void* coll_user = nullptr;
  void* hstage = nullptr;      // pinned staging buffer of the hosted exchange
  size_t hstage_bytes = 0;
  int num_sms = 148;
  size_t smem_optin = 0;
  void* dmalloc(size_t b);
  void dfree(void* p, size_t b);
};

// Host canonical graph (original ids).
struct HostCSR {
  int64_t n = 0, m = 0;
  std::vector<int64_t> rp;
  std::vector<int32_t> col;
  std::vector<uint32_t> w;
};

// Host transformed ("slot") graph; rows sorted by destination slot.
struct SlotGraph {
  int64_t n = 0, n_slots = 0, m_slots = 0;
  std::vector<int64_t> rp;
  std::vector<int32_t> col;
  std::vector<uint32_t> w;
  std::vector<uint8_t> added;
  std::vector<int32_t> slot_to_orig;
  std::vector<uint8_t> kind;
  std::vector<int32_t> owner_slot;
  std::vector<int32_t> sched;         // lane -> slot; empty => identity
  std::vector<int64_t> tile_ptr;      // §3 subgraphs
  std::vector<int32_t> tile_members, tile_centre, tile_iters;
  gx_transform_info info{};
};

// Windowed SELL-32 layout (sell.cu): per window of SELL_W rows, the light
// rows sorted by degree into 32-lane slices; heavy rows listed separately.
struct SellLayout {
  int64_t nwin = 0, nslices = 0, nheavy = 0, slab_len = 0;
  DBuf lane_row, heavy_row;   // i32
  DBuf win_slice, win_heavy;  // i64 [nwin+1]
  DBuf slice_len, slice_off;  // u32 [nslices+1], u64 [nslices+1]
  DBuf slab;                  // payload (u32 or uint2), sentinel padding
  bool built() const { return slab.p != nullptr; }
};

// Propagation-blocked PR layout (pagerank.cu k_pr_pb): slots are cut into
// blocks of PB_R rows; the edges u->v are grouped by (sink bin(v), source
// block(u)) into segments, sink-bin major, each edge stored as the two 16-bit
// local indices u%PB_R, v%PB_R; every segment is padded to a multiple of
// PB_PAD entries (source index PB_R = a zero term, sink 0), so all runs are
// 16-byte aligned.  q[s*nb + b] = start of segment (block s -> bin b),
// q[nb*nb + b] = end of bin b: bin b's in-edges are the contiguous range
// [q[b], q[nb*nb + b]); segment (s, b) = [q[s*nb + b], q[(s+1)*nb + b]).
// val f32[m_pad] carries x_u/D_u along every edge (written by the source
// block's scatter, read by the sink bin).
#ifndef GX_PB_R
#define GX_PB_R 16384
#endif
constexpr int PB_R = GX_PB_R;
constexpr int PB_PAD = 8;
struct PbLayout {
  int64_t nb = 0, m_pad = 0;
  DBuf q;                       // u32 [(nb+1)*nb]
  DBuf src_loc, dst_loc;        // u16 [m_pad]
  DBuf val;                     // f32 [m_pad]
  bool built() const { return q.p != nullptr; }
};

// Rank-local sweep layouts of the 1-D partitioned path (dist.h): one rank's
// rows [lo, hi) only.  SSSP: the out-CSR slice (rp rebased to 0, edges
// packed {dst << wbits | w} when they fit 32 bits, else {dst, w}), its static
// heavy-chunk list (hc_row = GLOBAL row, hc_start = local edge index) and
// heavy-row bitmap.  PageRank: the in-CSC slice (crp rebased, csrc = GLOBAL
// source slots, each row sorted by source) and its windowed SELL-32 (rows
// local).  Built once per (kind, P) from the slot graph and cached.
struct RankSlice {
  int64_t lo = 0, hi = 0, m = 0;
  DBuf rp, adj, adjp;          // SSSP
  uint32_t wbits = 0;
  DBuf hc_row, hc_start, heavy;
  int64_t nhc = 0;
  DBuf crp, csrc;              // PageRank
  SellLayout sell;
};
struct RankLayouts {
  int P = 0;                      // 0: not built
  int rank = -1;                  // -1: all P slices (simulated ranks)
  std::vector<int64_t> bounds;    // [P + 1]
  std::vector<RankSlice> r;       // P slices (simulated) or this rank's slice
};

// Device layouts of the current slot graph.
struct DevGraph {
  int64_t n = 0, n_slots = 0, m_slots = 0;
  bool identity = true;        // exact mode: slot == original id, no holes
  uint32_t max_w = 1;
  DBuf rp, adj;                // out-CSR: u32 [n_slots+1], uint2 {col, w} [m_slots]
  DBuf adjp;                   // packed out-edges col << adjp_wbits | w (sssp.cu), when they fit 32 bits
  uint32_t adjp_wbits = 0;
  bool adjp_tried = false;
  DBuf lh_lend;                // sssp.cu light / heavy split of adjp at lh_delta: u32 [n_slots]
  uint32_t lh_delta = 0;
  DBuf crp, csrc;              // in-CSC:  u32 [n_slots+1], i32 [m_slots]
  DBuf D;                      // u32 [n_slots]: logical out-degree (PR divisor)
  DBuf owner;                  // i32 [n]: original id -> owner slot
  DBuf kind;                   // u8 [n_slots] (null in exact mode)
  DBuf gid;                    // i32 [n_slots]: group id or -1 (null if no groups)
  DBuf gptr, gslots;           // groups: ptr [ng+1], slots (owner first)
  int64_t n_groups = 0, n_gslots = 0;   // groups, and their slots (owners + replicas)
  DBuf g_in_ptr, g_in;         // per-group owner in-edges (src slot, w) for SSSP pull
  // windowed SELL-32 layouts (sell.cu): PR pull over in-edges, SSSP dense
  // push over out-edges
  SellLayout pr_sell, sssp_sell;
  PbLayout pr_pb;              // propagation-blocked PR (built on first use)
  DBuf pb_w16;                 // u16 [m_pad]: edge weights in the blocked order (SSSP dense relaxation), built
                               // with the layout when the weights are resident and < 2^16
  RankLayouts rk_sssp, rk_pr;  // partitioned path (dist.h): this rank's rows only
  // LB SSSP: static chunk list of rows with out-degree > HEAVY_DEG, heavy bitmap
  int64_t nhc = 0;
  // SSSP block-local mode (sssp.cu): block size the locality was measured for,
  // fraction of edges inside a block, max out-degree
  int64_t blk_rows = 0, blk_maxdeg = 0;
  double blk_local = 0.0;
  DBuf hc_row, hc_start, heavy_bm;
  // TPV (paper's thread-per-vertex mapping, tpv.cu): lanes = the §4 schedule
  // (or slot order), SELL-32 slabs of out-edges (SSSP) and in-edges (PR)
  bool tpv_ready = false;
  int64_t tpv_nslices = 0;
  DBuf sched;                  // i32 [schedule length] (host sched uploaded)
  DBuf tpv_lane_row;           // i32 [nslices*32 + 32], -1 = idle lane
  DBuf tpv_out_len, tpv_out_off, tpv_out_slab;   // u32, u64, uint2 {dst, w}
  DBuf tpv_in_len, tpv_in_off, tpv_in_slab;      // u32, u64, u32 src
  int64_t tpv_out_slab_len = 0, tpv_in_slab_len = 0;
  // VNS (N4, tpv.cu): virtual nodes of <= vns_k out-edges in TPV lane order;
  // lanes carry their slot (for dist / frontier) and their edge chunk (slabs)
  bool vns_ready = false;
  int64_t vns_nslices = 0, vns_nv = 0;
  int vns_k = 0;
  DBuf vns_lane_slot, vns_len, vns_off, vns_slab;
  // logical graph G_L over original ids (replica rows folded into their
  // owner): SCC / MST / BC (algos.cu); in exact mode it aliases rp / adj
  bool lg_ready = false;
  DBuf lg_rp, lg_adj, lg_esrc;  // u32 [n+1], uint2 {dst, w} [m_L], u32 [m_L]
  int64_t lg_m = 0;
  // §3 tiles
  int64_t n_tiles = 0;
  DBuf t_ptr, t_members, t_eptr, t_edges, t_iters;  // local CSR per tile
  DBuf slot_tile, tile_mark, tile_list;              // slot -> tile (-1), touched-tile bitmap / list (SSSP)
  int64_t t_max_members = 0, t_max_edges = 0;
};

struct RunState {
  // SSSP / BC / SCC scratch (allocated lazily)
  DBuf dist, mark, q[2], hq[2], hbase[2], st, changed;
  // PR
  DBuf x, contrib[2], ysplit, gnew, pst;
  // BC
  DBuf sigma, delta, bc, level;
  // SCC / MST
  DBuf label, label2, mst_best, comp;
  uint64_t mst_weight = 0;
  bool have[6] = {false, false, false, false, false, false};
};

}  // namespace gx

struct gx_ctx : gx::Ctx {};

struct gx_graph {
  gx::Ctx* ctx = nullptr;
  gx::HostCSR host;            // canonical input (host copy, lazily filled)
  bool host_valid = false;
  gx::DBuf in_rp, in_col, in_w;   // canonical input on device (original ids)
  int64_t default_src = -1;       // R36 source (max out-degree of the canonical input), cached
  gx::DBuf in_w8;                 // GX_W_U8: the 8-bit weights as copied (widened into in_w)
  int64_t n = 0, m = 0;
  uint32_t max_w = 1;
  // GX_ASYNC_UPLOAD: the weights' copy, their maximum and the {col, w}
  // interleave run on ctx->copy_stream; pend_ev marks their end and
  // gx::resolve_pending() joins them into the ctx stream (and reads max_w)
  cudaEvent_t pend_ev = nullptr;
  cudaEvent_t dl_ev[8] = {};   // GX_DL_ASYNC: end of the download of result kind k (on ctx->copy_stream)
  gx::DBuf maxw_buf;
  bool maxw_pending = false;
  gx::SlotGraph sg;            // current transform (empty in exact mode)
  bool transformed = false;
  gx_knobs knobs{};
  gx::DevGraph dg;
  gx::RunState rs;
};

// ---- internal entry points across translation units ----
namespace gx {
void canonicalize_host(int64_t n, const int64_t* rp, const int32_t* col, const uint32_t* w,
                       HostCSR& out);
void ensure_host(gx_graph* g);
// dev: the graph's device context (GX_TRANSFORM=mixed), or null (host-only graph, GX_TRANSFORM=host):
// with a device the bulk-parallel steps run there (gtransform.cu, N1)
void transform_host(const HostCSR& g, const gx_knobs& k, SlotGraph& out, Ctx* dev = nullptr);
void gpu_triangles(Ctx* c, int64_t n, const int64_t* np, const int32_t* nc, int64_t* T);
void gpu_bfs_forest(Ctx* c, int64_t n, const int64_t* rp, const int32_t* col, std::vector<int32_t>& sources,
                    std::vector<int32_t>& level);
void gpu_pad_candidates(Ctx* c, int64_t n, const int64_t* lp, const int32_t* ld, const uint32_t* lw, int64_t nq,
                        const int32_t* qu, const int32_t* qtake, int rule, std::vector<int64_t>& rptr,
                        std::vector<uint64_t>& rkeys);
// device pipeline of the transforms (dtransform.cu, driven by transform.cpp's
// transform_device): the slot graph as one edge list in HBM,
// key = src slot << 32 | dst slot, val = weight | AddKind << 32
struct DEdges {
  DBuf key, val;
  int64_t m = 0;
};
struct DtCand { int32_t lv, cnt, s, C; };   // a (slot, chunk) replica candidate of level lv
struct DtAsg { int32_t s, C; int64_t hole; };
// din: the canonical graph resident on the device ({row_ptr i64, col i32, w u32}
// = gx_graph in_rp/in_col/in_w, identical to g), or all null (uploaded from g)
struct DevCSR { const int64_t* rp = nullptr; const int32_t* col = nullptr; const uint32_t* w = nullptr; };
void transform_device(const HostCSR& g, const gx_knobs& k, SlotGraph& out, Ctx* dev, DevCSR din = {});
void dt_from_csr(Ctx* c, const HostCSR& g, const int32_t* nw, DEdges& E, const int64_t* drp = nullptr,
                 const int32_t* dcol = nullptr, const uint32_t* dw = nullptr);
void dt_sort(Ctx* c, DEdges& E, int64_t ns);
void dt_row_ptr(Ctx* c, const DEdges& E, int64_t ns, DBuf& rp);
void dt_replica_candidates(Ctx* c, const DEdges& E, int k, const std::vector<int32_t>& chunk_lv,
                           const std::vector<int32_t>& nonhole, int64_t theta_ppm, std::vector<DtCand>& out);
int64_t dt_replicate(Ctx* c, DEdges& E, int64_t ns, int k, const std::vector<DtAsg>& asg,
                     const std::vector<uint8_t>& kind, int rule);
void dt_append_dev(Ctx* c, DEdges& E, const DBuf& key, const DBuf& val, int64_t na);
void dt_append(Ctx* c, DEdges& E, const std::vector<uint64_t>& key, const std::vector<uint64_t>& val);
void dt_logical(Ctx* c, const DEdges& E, const DBuf& s2o, int64_t n, DBuf& lp, DBuf& ld, DBuf& lw, DBuf* keys);
// (dst, w) pairs of a device CSR as u64 = w << 32 | dst (host layout of std::pair<int32_t, uint32_t>)
void dt_pairs(Ctx* c, const DBuf& ld, const DBuf& lw, int64_t m, DBuf& out);
int64_t dt_undirected(Ctx* c, int64_t n, const DBuf& lkey, int64_t ml, DBuf& np, DBuf& nc);
void dt_degnorm(Ctx* c, DEdges& E, int64_t ns, int64_t n, const std::vector<uint8_t>& kind, const DBuf& s2o,
                const std::vector<int32_t>& owner, int64_t th, int64_t f, bool combined, int rule,
                std::vector<int32_t>& sched, int64_t& added);
void dt_export(Ctx* c, DEdges& E, int64_t ns, SlotGraph& out);
void gpu_triangles_dev(Ctx* c, int64_t n, const int64_t* dnp, const int32_t* dnc, int64_t mm,
                       unsigned long long* dT);
void gpu_pad_candidates_dev(Ctx* c, int64_t n, const int64_t* dlp, const int32_t* dld, const uint32_t* dlw, int64_t nq,
                            const int32_t* dqu, const int32_t* qtake, int rule, std::vector<int64_t>& rptr,
                            std::vector<uint64_t>& rkeys);
void build_device_exact(gx_graph* g);
void resolve_pending(gx_graph* g);
void join_download(gx_graph* g, int kind);   // kind < 0: every kind
void build_device_slots(gx_graph* g);
void ensure_pb(gx_graph* g);
bool ensure_pb_w(gx_graph* g);   // the blocked layout + its 16-bit weights (false: built without them)
void build_tpv(gx_graph* g);
void run_sssp(gx_graph* g, const gx_run_opts& o, gx_run_info& info);
void run_pagerank(gx_graph* g, const gx_run_opts& o, gx_run_info& info);
void run_scc(gx_graph* g, const gx_run_opts& o, gx_run_info& info);
void run_mst(gx_graph* g, const gx_run_opts& o, gx_run_info& info);
void run_bc(gx_graph* g, const gx_run_opts& o, gx_run_info& info);
void download(gx_graph* g, int kind, void* out, int64_t count, uint32_t flags);
}  // namespace gx
