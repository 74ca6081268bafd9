// sigmo_abi.cu -- host side of libsigmo.so: the C ABI of include/sigmo.h,
// batch validation, CSR-GO packing (section 4.1), the query DFS
// planner, device buffer management and the launch sequence of the hot path.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <memory>
#include <string>
#include <thread>
#include <vector>

#include "../../include/sigmo.h"
#include "sigmo_internal.h"

using namespace sigmo;

namespace {

// ---------------------------------------------------------------------------
// device buffers
// ---------------------------------------------------------------------------
struct DBuf {
  void *p = nullptr;
  size_t cap = 0;
};

struct Pinned {
  void *p = nullptr;
  size_t cap = 0;
};

// Per-call CUDA events on the ctx stream (recording never synchronizes).
// Each filter call uses one slot of a ring (events: 0/1 query program if it
// was built by this call, 2/3 filter kernel, 4 end of GMCR scan + chunking);
// each join call one slot of another ring (join kernel).  A slot is
// harvested (its elapsed times added to running sums) when it is reused or
// when sigmo_get_timings is called, which returns averages and resets.
struct Timing {
  static const int RING = 64;
  bool enabled = false;
  cudaEvent_t fev[RING][5] = {};
  bool frec[RING][5] = {};
  bool fpend[RING] = {};
  cudaEvent_t jev[RING][2] = {};
  bool jpend[RING] = {};
  int fi = 0, ji = 0, cur_f = -1, cur_j = -1;
  double s_qprep = 0, s_filter = 0, s_mapping = 0, s_join = 0;
  long long n_qprep = 0, n_filter = 0, n_mapping = 0, n_join = 0;
};

struct ProgCache {
  QueryProg prog;
  DBuf buf, pack;  // device program arrays; packed form for k_filter
  std::vector<uint16_t> qdrow;  // host copy of prog.qdrow
  LaneJitSpec jit;              // the k_filter_lane program (host copy) for the NVRTC-specialised kernel
  bool valid = false;
  int nw = 0;  // the data batch's window words it was packed for (pack_prog's table size)
};

struct HostGraphs {  // validated input view (int64 offsets as given)
  int64_t G = 0, V = 0, E = 0;
  const int64_t *goff = nullptr, *roff = nullptr;
  const int32_t *col = nullptr;
  const uint8_t *nlab = nullptr, *elab = nullptr;
};

int num_host_threads(int64_t work) {
  unsigned hc = std::thread::hardware_concurrency();
  int t = (int)std::min<unsigned>(hc ? hc : 1, 32);
  int64_t by_work = work / 20000 + 1;
  return (int)std::max<int64_t>(1, std::min<int64_t>(t, by_work));
}

template <typename F>
void parallel_for_graphs(int64_t G, int64_t work, F &&fn) {
  const int T = num_host_threads(work);
  if (T <= 1 || G < 2) {
    fn(0, 0, G);
    return;
  }
  std::vector<std::thread> th;
  for (int t = 0; t < T; t++) {
    int64_t a = G * t / T, b = G * (t + 1) / T;
    th.emplace_back([&fn, t, a, b] { fn(t, a, b); });
  }
  for (auto &x : th) x.join();
}

}  // namespace

struct sigmo_ctx {
  int device = 0;
  cudaStream_t stream = nullptr;
  sigmo_allocator alloc{};
  bool has_alloc = false;
  std::string err;
  int state = 0;  // 0 empty, 1 loaded, 2 filtered, 3 joined
  int sm_count = 148;
  size_t max_smem = 227 * 1024;

  // ---- load ----
  Pinned staging;
  cudaEvent_t h2d_done = nullptr;
  cudaStream_t aux = nullptr;                        // the wide-molecule join launch runs beside the narrow one
  cudaEvent_t fork_ev = nullptr, join_ev = nullptr;
  DBuf arena;
  DevGraphs dq, dd;
  int NQ = 0, VQ = 0, EQ = 0, NQW = 0, maxq = 0, NB = 0, NBE = 0, plan_smem = 0;
  int ND = 0, VD = 0, ED = 0, maxn = 0, NW = 1;
  bool has_empty_graph = false;
  int W = 0, Wpad = 0;
  int32_t *qp_row = nullptr, *qp_beoff = nullptr;
  uint16_t *qp_be = nullptr;
  uint32_t *qp_info = nullptr;
  const int4 *qp_ent = nullptr;
  const uint32_t *qp_non = nullptr;
  const uint32_t *qp_qinfo = nullptr;
  int32_t *tile_g0 = nullptr, *tile_g1 = nullptr;
  uint8_t *bclass = nullptr;
  // filter tile geometry per TW (32,16,8,4,2,1)
  int tile_extn[6] = {}, tile_extw[6] = {}, tile_molcap[6] = {};
  bool tile_geom_ok = false;         // dense-tile geometry computed (lazily, first dense-tile filter)
  std::vector<int64_t> goff_host;    // data graph offsets (host copy for the lazy geometry)

  // ---- filter ----
  std::map<int, ProgCache> progs;  // keyed by R = levels-1
  DBuf qcounts;
  DBuf bitmap, gm, mol_cnt, off, scan_tmp, chunk_start, nchunks;
  size_t scan_tmp_bytes = 0;
  int levels = 0;
  uint32_t flags = 0;
  int PC = 512, AC = 512, CMC = 2048, MC = 128;

  // ---- join ----
  DBuf pair_query, pair_rec, pair_cm, pair_result, jcnt, adjb, ent2;
  // jcnt u64 slots: [0] pair cursor / chunk counter, [1] error flag, [2..5] DFS stats, [6..] totals
  int induced = 0;         // sigmo_set_induced (applies to the next sigmo_load_batch)
  int induced_loaded = 0;  // induced mode of the loaded batch (routes it to k_join)
  int wildcard = 0;        // sigmo_set_wildcards (applies to the next sigmo_load_batch)
  int wildcard_loaded = 0; // wildcard mode of the loaded batch (R22)
  int any_bond = 0;        // the loaded queries use '~' bonds: label 0 -> adjacency class NB (all bonds)
  bool lane_join = false;  // per-lane join possible for this batch (<= 64-node graphs, <= 16-node queries)
  bool mol_filter = false; // last sigmo_filter used molecule tiles (candidates in cmol layout)
  bool dense_pad_zero = false;  // padding words >= W of the dense bitmap rows (and the tail) are zero
  size_t bm_bytes = 0;
  // plan entries as loaded (host) and the query node of each plan position;
  // bits 12.. of .x are set to the distinct row of that node for the R whose
  // program last ran (ent_R), re-uploaded when R changes
  std::vector<int4> ent_host;
  std::vector<uint2> ent_up;  // compact entries for k_join_lane (8 B): see JoinParams::qp_ent2
  bool lane_extras = true;     // some entry has > 2 back-edges (the lean lane join does not apply)
  bool count_steps = false;    // sigmo_set_timing bit 1: the join counts its DFS steps (sigmo_timings.dfs_steps)
  std::vector<int32_t> ent_row;
  std::vector<int64_t> qgoff_host;  // query graph offsets (host copy, for the per-query row-word lists)
  int ent_R = -1;
  std::vector<unsigned char> qkey;  // the last successfully loaded query batch (sigmo_load_batch reuse check)
  bool qkey_valid = false;
  int32_t *grp_narrow = nullptr, *grp_wide = nullptr;  // k_filter_lane groups (input arena)
  int NGN = 0, NGW = 0;
  DBuf nb4, mrec;                   // k_filter_lane: packed neighbours [VD], molecule records [ND]
  uint32_t *adj_off = nullptr;      // [ND + 1] 32-bit word offset of each molecule's bond-class adjacency
  uint32_t *cand_units = nullptr;   // [ND + 1] candidate-window units before each molecule (x NDR = its cmol word offset)
  uint32_t cand_total = 0;
  uint32_t adj_words = 0;           // adjacency words (the all-ones entry follows)
  DBuf dense_tmp;          // dense view of cmol for sigmo_get_candidates
  int last_mode = 0;
  DBuf sig_tmp, gstack;

  Timing timing;
  sigmo_timings last{};
  std::string jit_note;  // last lane-filter specialisation outcome ("compiled", "cached" or why not)
  // enumerate mode
  const uint8_t *qp_qn = nullptr;  // [VQ] local query node of each plan position (input arena)
  DBuf eoff, ecur, emaps, esets, ucnt, uoff, uniq, etmp;
  int64_t enum_P = -1, enum_total = 0, enum_uniq = -1;
  int enum_stride = 8;
  // device-side load of large data batches (k_load_data)
  DBuf raw, dpk, ldinfo, lay;
  Pinned ldhost;                    // histogram + error words read back
  // neighbour support on the lane path (k_support_lane)
  bool lane_ns = false;            // the last filter refined per-pair windows (join reads ns_win*)
  bool ns_lane_ok = true;          // every query node has <= 8 neighbours (k_support_lane's lists)
  const uint2 *qp_nbr = nullptr;   // [VQ] query neighbours per plan position (input arena)
  DBuf ns_win32, ns_win64, ns_alive, gm_old, off_old, ent_ns, ns_bitmap, ns_gm, ns_cnt;
  std::vector<uint2> ent_ns_up;    // plan entries whose row field is the plan depth (windows per pair)
};

namespace {

sigmo_status set_err(sigmo_ctx *c, sigmo_status s, const char *fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  if (c) c->err = buf;
  return s;
}

#define CUDA_TRY(ctx, call)                                                                          \
  do {                                                                                               \
    cudaError_t e_ = (call);                                                                         \
    if (e_ != cudaSuccess) {                                                                         \
      return set_err(ctx, e_ == cudaErrorMemoryAllocation ? SIGMO_ERR_OOM : SIGMO_ERR_CUDA,          \
                     "%s: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__);           \
    }                                                                                                \
  } while (0)

void dfree(sigmo_ctx *c, DBuf &b) {
  if (!b.p) return;
  if (c->has_alloc) c->alloc.free(b.p, (void *)c->stream, c->alloc.user);
  else cudaFreeAsync(b.p, c->stream);
  b.p = nullptr;
  b.cap = 0;
}

sigmo_status dreserve(sigmo_ctx *c, DBuf &b, size_t bytes, const char *what) {
  if (bytes == 0) bytes = 16;
  if (b.cap >= bytes) return SIGMO_OK;
  dfree(c, b);
  void *p = nullptr;
  if (c->has_alloc) {
    p = c->alloc.alloc(bytes, (void *)c->stream, c->alloc.user);
    if (!p) return set_err(c, SIGMO_ERR_OOM, "allocator returned NULL for %s (%zu bytes)", what, bytes);
  } else {
    cudaError_t e = cudaMallocAsync(&p, bytes, c->stream);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return set_err(c, SIGMO_ERR_OOM, "cudaMallocAsync %s (%zu bytes): %s", what, bytes, cudaGetErrorString(e));
    }
  }
  b.p = p;
  b.cap = bytes;
  return SIGMO_OK;
}

#define SIGMO_TRY(x)                  \
  do {                                \
    sigmo_status s_ = (x);            \
    if (s_ != SIGMO_OK) return s_;    \
  } while (0)

// ---------------------------------------------------------------------------
// validation (sigmo_load_batch contract)
// ---------------------------------------------------------------------------
sigmo_status validate(const sigmo_graph_batch *b, int is_query, std::string &msg, HostGraphs &out) {
  auto fail = [&](sigmo_status s, const char *fmt, long long x, long long y) {
    char buf[256];
    snprintf(buf, sizeof(buf), fmt, x, y);
    msg = buf;
    return s;
  };
  if (!b) return fail(SIGMO_ERR_INVALID_ARG, "batch pointer is NULL", 0, 0) ;
  if (b->num_graphs < 0 || b->num_nodes < 0) return fail(SIGMO_ERR_INVALID_ARG, "negative num_graphs %lld / num_nodes %lld", b->num_graphs, b->num_nodes);
  if (!b->graph_offsets || !b->row_offsets) return fail(SIGMO_ERR_INVALID_ARG, "graph_offsets/row_offsets NULL", 0, 0);
  if (b->num_nodes >= (1ll << 31) - 1) return fail(SIGMO_ERR_LIMIT, "num_nodes %lld >= 2^31-1", b->num_nodes, 0);
  if (b->num_graphs >= (1ll << 31) - 1) return fail(SIGMO_ERR_LIMIT, "num_graphs %lld >= 2^31-1", b->num_graphs, 0);
  const int64_t G = b->num_graphs, V = b->num_nodes;
  const int64_t *go = b->graph_offsets, *ro = b->row_offsets;
  if (go[0] != 0) return fail(SIGMO_ERR_INVALID_GRAPH, "graph_offsets[0] = %lld, expected 0", go[0], 0);
  for (int64_t g = 0; g < G; g++) {
    if (go[g + 1] < go[g]) return fail(SIGMO_ERR_INVALID_GRAPH, "graph_offsets decreasing at graph %lld (%lld)", g, go[g + 1]);
    const int64_t n = go[g + 1] - go[g];
    if (is_query && n == 0) return fail(SIGMO_ERR_INVALID_GRAPH, "query graph %lld is empty", g, 0);
    if (is_query && n > SIGMO_MAX_QUERY_NODES) return fail(SIGMO_ERR_LIMIT, "query graph %lld has %lld nodes > 32", g, n);
    if (!is_query && n > SIGMO_MAX_DATA_NODES) return fail(SIGMO_ERR_LIMIT, "data graph %lld has %lld nodes > 256", g, n);
  }
  if (go[G] != V) return fail(SIGMO_ERR_INVALID_GRAPH, "graph_offsets[num_graphs] = %lld != num_nodes %lld", go[G], V);
  if (ro[0] != 0) return fail(SIGMO_ERR_INVALID_GRAPH, "row_offsets[0] = %lld, expected 0", ro[0], 0);
  {
    std::vector<int64_t> bad(64, -1);
    parallel_for_graphs(V, V, [&](int th, int64_t a, int64_t b) {
      for (int64_t v = a; v < b; v++)
        if (ro[v + 1] < ro[v]) {
          bad[th] = v;
          return;
        }
    });
    for (int64_t v : bad)
      if (v >= 0) return fail(SIGMO_ERR_INVALID_GRAPH, "row_offsets decreasing at node %lld (%lld)", v, ro[v + 1]);
  }
  const int64_t E = ro[V];
  if (E >= (1ll << 31) - 1) return fail(SIGMO_ERR_LIMIT, "adjacency entries %lld >= 2^31-1", E, 0);
  if (V > 0 && !b->node_labels) return fail(SIGMO_ERR_INVALID_ARG, "node_labels NULL", 0, 0);
  if (E > 0 && (!b->col_indices || !b->edge_labels)) return fail(SIGMO_ERR_INVALID_ARG, "col_indices/edge_labels NULL", 0, 0);
  const int32_t *col = b->col_indices;
  const uint8_t *el = b->edge_labels;
  // per-graph structural checks, parallel over graphs; first error by graph index
  std::vector<int64_t> bad_graph(64, -1);
  std::vector<std::string> bad_msg(64);
  std::vector<sigmo_status> bad_st(64, SIGMO_OK);
  parallel_for_graphs(G, E + V, [&](int t, int64_t ga, int64_t gb) {
    char buf[256];
    // graphs of <= 64 nodes: neighbour bitmasks and a local label matrix
    // replace the per-edge row scans (duplicate / symmetry checks)
    std::vector<uint64_t> nbm(64);
    std::vector<uint8_t> elm(64 * 64);
    auto report = [&](int64_t g, const char *why, long long a1, long long a2) {
      snprintf(buf, sizeof(buf), why, a1, a2);
      bad_graph[t] = g;
      bad_msg[t] = buf;
      bad_st[t] = SIGMO_ERR_INVALID_GRAPH;
    };
    for (int64_t g = ga; g < gb; g++) {
      const int64_t lo = go[g], hi = go[g + 1];
      if (hi - lo <= 64) {
        const int n = (int)(hi - lo);
        for (int i = 0; i < n; i++) nbm[i] = 0ull;
        for (int64_t u = lo; u < hi; u++) {
          const int ul = (int)(u - lo);
          for (int64_t e = ro[u]; e < ro[u + 1]; e++) {
            const int64_t v = col[e];
            if (v < lo || v >= hi) return report(g, "column %lld of node %lld outside its graph", v, u);
            if (v == u) return report(g, "self-loop at node %lld", u, 0);
            const int vl = (int)(v - lo);
            if ((nbm[ul] >> vl) & 1ull) return report(g, "duplicate edge %lld -> %lld", u, v);
            nbm[ul] |= 1ull << vl;
            elm[ul * 64 + vl] = el[e];
          }
        }
        for (int64_t u = lo; u < hi; u++) {
          const int ul = (int)(u - lo);
          for (int64_t e = ro[u]; e < ro[u + 1]; e++) {
            const int vl = (int)(col[e] - lo);
            if (!((nbm[vl] >> ul) & 1ull) || elm[vl * 64 + ul] != el[e])
              return report(g, "asymmetric edge or edge label %lld -> %lld", u, (long long)col[e]);
          }
        }
        continue;
      }
      for (int64_t u = lo; u < hi; u++) {
        for (int64_t e = ro[u]; e < ro[u + 1]; e++) {
          const int64_t v = col[e];
          if (v < lo || v >= hi) return report(g, "column %lld of node %lld outside its graph", v, u);
          if (v == u) return report(g, "self-loop at node %lld", u, 0);
          int dup = 0;
          for (int64_t f = ro[u]; f < ro[u + 1]; f++) dup += (col[f] == v);
          if (dup > 1) return report(g, "duplicate edge %lld -> %lld", u, v);
          bool sym = false;
          for (int64_t f = ro[v]; f < ro[v + 1] && !sym; f++)
            if (col[f] == u && el[f] == el[e]) sym = true;
          if (!sym) return report(g, "asymmetric edge or edge label %lld -> %lld", u, v);
        }
      }
    }
  });
  int64_t first = -1;
  int ft = -1;
  for (int t = 0; t < 64; t++)
    if (bad_graph[t] >= 0 && (first < 0 || bad_graph[t] < first)) {
      first = bad_graph[t];
      ft = t;
    }
  if (ft >= 0) {
    msg = std::string(is_query ? "query" : "data") + " graph " + std::to_string(first) + ": " + bad_msg[ft];
    return bad_st[ft];
  }
  out.G = G;
  out.V = V;
  out.E = E;
  out.goff = go;
  out.roff = ro;
  out.col = col;
  out.nlab = b->node_labels;
  out.elab = el;
  return SIGMO_OK;
}

// O(#graphs) checks of a large data batch; the per-entry checks run on the
// device (k_load_data) with the same error classes
sigmo_status validate_light(const sigmo_graph_batch *b, std::string &msg, HostGraphs &out) {
  auto fail = [&](sigmo_status s, const char *fmt, long long x, long long y) {
    char buf[256];
    snprintf(buf, sizeof(buf), fmt, x, y);
    msg = buf;
    return s;
  };
  if (b->num_graphs < 0 || b->num_nodes < 0) return fail(SIGMO_ERR_INVALID_ARG, "negative num_graphs %lld / num_nodes %lld", b->num_graphs, b->num_nodes);
  if (!b->graph_offsets || !b->row_offsets) return fail(SIGMO_ERR_INVALID_ARG, "graph_offsets/row_offsets NULL", 0, 0);
  if (b->num_nodes >= (1ll << 31) - 1) return fail(SIGMO_ERR_LIMIT, "num_nodes %lld >= 2^31-1", b->num_nodes, 0);
  if (b->num_graphs >= (1ll << 31) - 1) return fail(SIGMO_ERR_LIMIT, "num_graphs %lld >= 2^31-1", b->num_graphs, 0);
  const int64_t G = b->num_graphs, V = b->num_nodes;
  const int64_t *go = b->graph_offsets, *ro = b->row_offsets;
  if (go[0] != 0) return fail(SIGMO_ERR_INVALID_GRAPH, "graph_offsets[0] = %lld, expected 0", go[0], 0);
  for (int64_t g = 0; g < G; g++) {
    if (go[g + 1] < go[g]) return fail(SIGMO_ERR_INVALID_GRAPH, "graph_offsets decreasing at graph %lld (%lld)", g, go[g + 1]);
    if (go[g + 1] - go[g] > SIGMO_MAX_DATA_NODES)
      return fail(SIGMO_ERR_LIMIT, "data graph %lld has %lld nodes > 256", g, go[g + 1] - go[g]);
  }
  if (go[G] != V) return fail(SIGMO_ERR_INVALID_GRAPH, "graph_offsets[num_graphs] = %lld != num_nodes %lld", go[G], V);
  if (ro[0] != 0) return fail(SIGMO_ERR_INVALID_GRAPH, "row_offsets[0] = %lld, expected 0", ro[0], 0);
  const int64_t E = ro[V];
  if (E < 0 || E >= (1ll << 31) - 1) return fail(SIGMO_ERR_LIMIT, "adjacency entries %lld not in [0, 2^31-1)", E, 0);
  if (V > 0 && !b->node_labels) return fail(SIGMO_ERR_INVALID_ARG, "node_labels NULL", 0, 0);
  if (E > 0 && (!b->col_indices || !b->edge_labels)) return fail(SIGMO_ERR_INVALID_ARG, "col_indices/edge_labels NULL", 0, 0);
  out.G = G;
  out.V = V;
  out.E = E;
  out.goff = go;
  out.roff = ro;
  out.col = b->col_indices;
  out.nlab = b->node_labels;
  out.elab = b->edge_labels;
  return SIGMO_OK;
}

// ---------------------------------------------------------------------------
// packing into pinned staging
// ---------------------------------------------------------------------------
struct Layout {
  size_t off = 0;
  size_t take(size_t bytes) {
    size_t o = off;
    off = (off + bytes + 255) & ~(size_t)255;
    return o;
  }
};

struct PackedOffsets {
  size_t goff, label, local, roff, nbr;
};

PackedOffsets plan_graphs(Layout &L, const HostGraphs &h) {
  PackedOffsets p;
  p.goff = L.take(4 * (size_t)(h.G + 1));
  p.label = L.take((size_t)h.V);
  p.local = L.take((size_t)h.V);
  p.roff = L.take(4 * (size_t)(h.V + 1));
  p.nbr = L.take(2 * (size_t)h.E);
  return p;
}

void pack_graphs(unsigned char *base, const PackedOffsets &p, const HostGraphs &h) {
  int32_t *goff = (int32_t *)(base + p.goff);
  uint8_t *label = base + p.label;
  uint8_t *local = base + p.local;
  int32_t *roff = (int32_t *)(base + p.roff);
  uint16_t *nbr = (uint16_t *)(base + p.nbr);
  goff[h.G] = (int32_t)h.V;
  roff[h.V] = (int32_t)h.E;
  parallel_for_graphs(h.G, h.E + h.V, [&](int, int64_t ga, int64_t gb) {
    for (int64_t g = ga; g < gb; g++) {
      const int64_t lo = h.goff[g], hi = h.goff[g + 1];
      goff[g] = (int32_t)lo;
      for (int64_t u = lo; u < hi; u++) {
        label[u] = h.nlab[u];
        local[u] = (uint8_t)(u - lo);
        roff[u] = (int32_t)h.roff[u];
        for (int64_t e = h.roff[u]; e < h.roff[u + 1]; e++) nbr[e] = (uint16_t)(((h.col[e] - lo) << 8) | h.elab[e]);
      }
    }
  });
}

DevGraphs dev_view(unsigned char *dbase, const PackedOffsets &p, const HostGraphs &h) {
  DevGraphs d;
  d.num_graphs = (int)h.G;
  d.num_nodes = (int)h.V;
  d.num_adj = (int)h.E;
  d.max_nodes = 0;
  for (int64_t g = 0; g < h.G; g++) d.max_nodes = std::max<int>(d.max_nodes, (int)(h.goff[g + 1] - h.goff[g]));
  d.goff = (const int32_t *)(dbase + p.goff);
  d.label = dbase + p.label;
  d.local = dbase + p.local;
  d.roff = (const int32_t *)(dbase + p.roff);
  d.nbr = (const uint16_t *)(dbase + p.nbr);
  return d;
}

// ---------------------------------------------------------------------------
// query DFS planner (host, step S1).  Static matching order per query:
// root = rarest label in the data batch (ties: higher degree, lower id); then
// repeatedly the unordered node with most edges into the ordered set (ties:
// rarer label, higher degree, lower id).  Any order yields the same counts
// (reading R12); this one prunes early.
// ---------------------------------------------------------------------------
struct QPlan {
  std::vector<int32_t> row;     // [VQ] global query node of depth e
  std::vector<int32_t> beoff;   // [VQ+1]
  std::vector<uint16_t> be;     // (j << 8) | class
  std::vector<uint32_t> info;   // [VQ] two back-edges inline + #extra + leaf-sum flag (see plan_queries)
  std::vector<uint32_t> qinfo;  // [NQ] nq | last depth n-1 << 8 | first query node << 16 (k_join_lane)
};

void plan_queries(const HostGraphs &q, const std::vector<int64_t> &freq, const uint8_t *bclass, QPlan &out) {
  out.row.assign((size_t)q.V, 0);
  out.beoff.assign((size_t)q.V + 1, 0);
  out.info.assign((size_t)q.V, 0x3fu | (0x3fu << 9));
  out.qinfo.assign((size_t)q.G, 0u);
  out.be.clear();
  for (int64_t g = 0; g < q.G; g++) {
    const int64_t lo = q.goff[g];
    const int n = (int)(q.goff[g + 1] - lo);
    std::vector<int> pos(n, -1), order;
    auto deg = [&](int u) { return (int)(q.roff[lo + u + 1] - q.roff[lo + u]); };
    auto fr = [&](int u) { return freq[q.nlab[lo + u]]; };
    // qinfo: n | (n - 1) << 8 (the last depth, counted by popc) | first query node << 16
    const int t = n <= 1 ? n : n - 1;
    out.qinfo[g] = (uint32_t)n | ((uint32_t)t << 8) | ((uint32_t)lo << 16);
    for (int i = 0; i < n; i++) {
      int best = -1, bc = -1;
      for (int u = 0; u < n; u++) {
        if (pos[u] >= 0) continue;
        int conn = 0;
        for (int64_t e = q.roff[lo + u]; e < q.roff[lo + u + 1]; e++)
          if (pos[q.col[e] - lo] >= 0) conn++;
        bool better = false;
        if (best < 0) better = true;
        else if (conn != bc) better = conn > bc;
        else if (fr(u) != fr(best)) better = fr(u) < fr(best);
        else if (deg(u) != deg(best)) better = deg(u) > deg(best);
        if (better) {
          best = u;
          bc = conn;
        }
      }
      pos[best] = i;
      order.push_back(best);
    }
    for (int e = 0; e < n; e++) {
      const int u = order[e];
      out.row[lo + e] = (int32_t)(lo + u);
      out.beoff[lo + e] = (int32_t)out.be.size();
      for (int64_t k = q.roff[lo + u]; k < q.roff[lo + u + 1]; k++) {
        const int w = (int)(q.col[k] - lo);
        if (pos[w] < e) out.be.push_back((uint16_t)((pos[w] << 8) | bclass[q.elab[k]]));
      }
      // info word: j0 (6 bits, 0x3f none) | b0 << 6 | j1 << 9 (0x3f none) | b1 << 15 |
      // (#back-edges beyond two) << 18 | leaf-sum flag << 24
      const int nbe = (int)out.be.size() - out.beoff[lo + e];
      uint32_t inf = 0x3fu | (0x3fu << 9);
      if (nbe > 0) {
        const uint16_t f = out.be[out.beoff[lo + e]];
        inf = (inf & ~0x1ffu) | (uint32_t)(f >> 8) | ((uint32_t)(f & 7) << 6);
      }
      if (nbe > 1) {
        const uint16_t f = out.be[out.beoff[lo + e] + 1];
        inf = (inf & ~(0x1ffu << 9)) | ((uint32_t)(f >> 8) << 9) | ((uint32_t)(f & 7) << 15);
      }
      if (nbe > 2) inf |= (uint32_t)(nbe - 2) << 18;
      out.info[lo + e] = inf;
      if (e == n - 1 && n >= 3) {
        // bit 24: the last node has no back-edge to depth n-2 (leaf-sum closed form applies)
        bool adj_prev = false;
        for (int k = out.beoff[lo + e]; k < (int)out.be.size(); k++) adj_prev |= (out.be[k] >> 8) == n - 2;
        if (!adj_prev) out.info[lo + e] |= 1u << 24;
      }
    }
  }
  out.beoff[q.V] = (int32_t)out.be.size();
}

int graph_of_host(const int64_t *goff, int64_t G, int64_t n) {
  int64_t lo = 0, hi = G;
  while (lo < hi) {
    int64_t mid = (lo + hi + 1) >> 1;
    if (goff[mid] <= n) lo = mid;
    else hi = mid - 1;
  }
  return (int)lo;
}

float ev_ms(cudaEvent_t a, cudaEvent_t b) {
  float ms = 0.f;
  if (cudaEventElapsedTime(&ms, a, b) != cudaSuccess) {
    cudaGetLastError();
    return 0.f;
  }
  return ms;
}

void harvest_f(Timing &T, int s) {
  if (!T.fpend[s]) return;
  int last = -1;
  for (int k = 0; k < 5; k++)
    if (T.frec[s][k]) last = k;
  if (last >= 0) cudaEventSynchronize(T.fev[s][last]);
  if (T.frec[s][0] && T.frec[s][1]) { T.s_qprep += ev_ms(T.fev[s][0], T.fev[s][1]); T.n_qprep++; }
  if (T.frec[s][2] && T.frec[s][3]) { T.s_filter += ev_ms(T.fev[s][2], T.fev[s][3]); T.n_filter++; }
  if (T.frec[s][3] && T.frec[s][4]) { T.s_mapping += ev_ms(T.fev[s][3], T.fev[s][4]); T.n_mapping++; }
  T.fpend[s] = false;
  for (int k = 0; k < 5; k++) T.frec[s][k] = false;
}

void harvest_j(Timing &T, int s) {
  if (!T.jpend[s]) return;
  cudaEventSynchronize(T.jev[s][1]);
  T.s_join += ev_ms(T.jev[s][0], T.jev[s][1]);
  T.n_join++;
  T.jpend[s] = false;
}

void timing_begin_filter(sigmo_ctx *c) {
  Timing &T = c->timing;
  if (!T.enabled) { T.cur_f = -1; return; }
  const int s = T.fi;
  T.fi = (T.fi + 1) % Timing::RING;
  harvest_f(T, s);
  T.cur_f = s;
}

void timing_mark(sigmo_ctx *c, int k) {
  Timing &T = c->timing;
  if (!T.enabled || T.cur_f < 0) return;
  cudaEventRecord(T.fev[T.cur_f][k], c->stream);
  T.frec[T.cur_f][k] = true;
  T.fpend[T.cur_f] = true;
}

void timing_join(sigmo_ctx *c, int k) {
  Timing &T = c->timing;
  if (!T.enabled) return;
  if (k == 0) {
    const int s = T.ji;
    T.ji = (T.ji + 1) % Timing::RING;
    harvest_j(T, s);
    T.cur_j = s;
  }
  cudaEventRecord(T.jev[T.cur_j][k], c->stream);
  if (k == 1) T.jpend[T.cur_j] = true;
}

// ---------------------------------------------------------------------------
// query plane program (cached per R = levels - 1)
// ---------------------------------------------------------------------------
constexpr int kMaxPlanes = kMaxRadius * kNumFields * 256;  // 49920 keys

// Host packing of the plane program for k_filter (see GroupRec): planes are
// numbered p = 0..P-1 in (radius, field, threshold) order and grouped in
// batches of 32; each (radius, field) group contributes one record per batch
// it touches, whose table maps a count c to the bits of its planes with
// t_p <= c.  Row programs list channel byte offsets, label channel first,
// padded with the all-ones channel to whole 32-bit words.
sigmo_status pack_prog(sigmo_ctx *c, int R, ProgCache &pc) {
  QueryProg &P = pc.prog;
  const QueryProgMeta &m = P.meta;
  const int VQ = c->VQ, NP = m.P, G = m.G, NLAB = m.NLAB;
  const int RE = m.row_entries;
  std::vector<uint8_t> p_t((size_t)NP + 1), grp_f((size_t)G + 1), row_lab((size_t)VQ + 1);
  std::vector<int16_t> grp_poff((size_t)G + 1), rg_off((size_t)R + 1);
  std::vector<int8_t> fslot(kNumFields);
  std::vector<int32_t> row_off((size_t)VQ + 1);
  std::vector<uint16_t> row_ids((size_t)RE + 1);
  cudaStream_t st = c->stream;
  if (NP) CUDA_TRY(c, cudaMemcpyAsync(p_t.data(), P.p_t, NP, cudaMemcpyDeviceToHost, st));
  if (G) CUDA_TRY(c, cudaMemcpyAsync(grp_f.data(), P.grp_f, G, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(c, cudaMemcpyAsync(grp_poff.data(), P.grp_poff, 2 * ((size_t)G + 1), cudaMemcpyDeviceToHost, st));
  CUDA_TRY(c, cudaMemcpyAsync(rg_off.data(), P.rg_off, 2 * ((size_t)R + 1), cudaMemcpyDeviceToHost, st));
  CUDA_TRY(c, cudaMemcpyAsync(fslot.data(), P.fslot, kNumFields, cudaMemcpyDeviceToHost, st));
  if (VQ) CUDA_TRY(c, cudaMemcpyAsync(row_lab.data(), P.row_lab, VQ, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(c, cudaMemcpyAsync(row_off.data(), P.row_off, 4 * ((size_t)VQ + 1), cudaMemcpyDeviceToHost, st));
  if (RE) CUDA_TRY(c, cudaMemcpyAsync(row_ids.data(), P.row_ids, 2 * (size_t)RE, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(c, cudaStreamSynchronize(st));
  const int TS = c->NW == 1 ? 64 : 256;  // counts exclude the node: <= 63 in <= 64-node graphs
  std::vector<GroupRec> rec;
  std::vector<uint32_t> tab;
  std::vector<int32_t> rrec((size_t)R + 1, 0), rcarry((size_t)R + 1, 0);
  const int NBATCH = (NP + 31) / 32;
  std::vector<int32_t> bdone((size_t)NBATCH + 1, 0);
  for (int r0 = 0; r0 < R; r0++) {
    rrec[r0] = (int)rec.size();
    const int g0 = rg_off[r0], g1 = rg_off[r0 + 1];
    if (g0 < g1) rcarry[r0] = (grp_poff[g0] % 32) != 0;
    for (int g = g0; g < g1; g++) {
      for (int p = grp_poff[g]; p < grp_poff[g + 1];) {
        const int b = p / 32;
        const int e = std::min<int>(grp_poff[g + 1], 32 * (b + 1));
        GroupRec r{};
        r.fslot = fslot[grp_f[g]];
        r.toff = (int)tab.size();
        r.batch = b;
        rec.push_back(r);
        for (int cc = 0; cc < TS; cc++) {
          uint32_t bits = 0;
          for (int q = p; q < e; q++)
            if ((int)p_t[q] <= cc) bits |= 1u << (q % 32);
          tab.push_back(bits);
        }
        for (int q = p; q < e; q++) bdone[q / 32] = r0;  // radius of the batch's last plane (planes ascend)
        p = e;
      }
    }
  }
  rrec[R] = (int)rec.size();
  // row programs: every row padded to RW words (the longest row) with
  // all-ones channel pairs, so k_filter's row loop has a fixed trip count
  std::vector<std::vector<int>> chans((size_t)VQ);
  int RW = 1;
  for (int v = 0; v < VQ; v++) {
    std::vector<int> &ch = chans[v];
    ch.push_back(row_lab[v]);
    for (int j = row_off[v]; j < row_off[v + 1]; j++) ch.push_back(NLAB + 1 + row_ids[j]);
    RW = std::max<int>(RW, (int)(ch.size() + 1) / 2);
  }
  if (4 * (NLAB + 1 + NP) > 0xffff) return set_err(c, SIGMO_ERR_LIMIT, "plane program too large (%d planes)", NP);
  std::vector<int32_t> rowp_off((size_t)VQ + 1, 0);
  std::vector<uint32_t> rowp((size_t)VQ * RW, (uint32_t)(4 * NLAB) | ((uint32_t)(4 * NLAB) << 16));
  for (int v = 0; v < VQ; v++) {
    rowp_off[v] = v * RW;
    const std::vector<int> &ch = chans[v];
    for (size_t j = 0; j < ch.size(); j += 2) {
      const int hi = j + 1 < ch.size() ? ch[j + 1] : NLAB;
      rowp[(size_t)v * RW + j / 2] = (uint32_t)(4 * ch[j]) | ((uint32_t)(4 * hi) << 16);
    }
  }
  rowp_off[VQ] = VQ * RW;
  // distinct rows: query nodes with the same channel list (label + the same
  // constraint planes) compute the same candidate row; the lane-path filter
  // computes and stores each distinct row once per molecule.  Distinct rows
  // are numbered by channel count (then content), so a 32-row group of
  // k_filter_lane has nearly uniform program lengths.
  std::map<std::vector<int>, int> dmap;
  for (int v = 0; v < VQ; v++) dmap.emplace(chans[v], 0);
  std::vector<const std::vector<int> *> drows;
  for (auto &kv : dmap) drows.push_back(&kv.first);
  std::stable_sort(drows.begin(), drows.end(),
                   [](const std::vector<int> *a, const std::vector<int> *b) { return a->size() < b->size(); });
  for (size_t i = 0; i < drows.size(); i++) dmap[*drows[i]] = (int)i;
  std::vector<uint16_t> qdrow((size_t)VQ + 1, 0);
  std::vector<uint32_t> drowp((size_t)dmap.size() * RW);
  for (int v = 0; v < VQ; v++) {
    const int d = dmap[chans[v]];
    qdrow[v] = (uint16_t)d;
    std::copy(rowp.begin() + (size_t)v * RW, rowp.begin() + (size_t)(v + 1) * RW, drowp.begin() + (size_t)d * RW);
  }
  const int NDR = (int)dmap.size();
  if (NDR > 0xffff) return set_err(c, SIGMO_ERR_LIMIT, "%d distinct query rows", NDR);
  // GMCR lists of the molecule-tile filter: per query the (word, bits) pairs
  // of its distinct rows in the per-molecule non-empty bit vector
  const int NQ = c->NQ;
  std::vector<int32_t> qw_off((size_t)NQ + 1, 0);
  std::vector<uint32_t> qw;  // word, mask interleaved
  for (int q = 0; q < NQ; q++) {
    qw_off[q] = (int32_t)(qw.size() / 2);
    std::map<int, uint32_t> wm;
    for (int64_t v = c->qgoff_host[q]; v < c->qgoff_host[q + 1]; v++) wm[qdrow[v] >> 5] |= 1u << (qdrow[v] & 31);
    for (const auto &kv : wm) {
      qw.push_back((uint32_t)kv.first);
      qw.push_back(kv.second);
    }
  }
  qw_off[NQ] = (int32_t)(qw.size() / 2);
  // ---- k_filter_lane program (FilterLaneParams) ----
  // plane records: per (radius, field) group, chunks of <= 4 planes; per
  // radius sorted by plane count (k_filter_lane runs the four counts as
  // separate loops): lrrec[4 r0 + k] = first record of radius r0 with k + 1 planes
  std::vector<uint2> lrec;
  std::vector<int32_t> lrrec((size_t)4 * R + 1, 0);
  for (int r0 = 0; r0 < R; r0++) {
    std::vector<uint2> byn[4];
    for (int g = rg_off[r0]; g < rg_off[r0 + 1]; g++)
      for (int p = grp_poff[g]; p < grp_poff[g + 1]; p += 4) {
        const int np = std::min(4, grp_poff[g + 1] - p);
        uint2 e;
        e.x = (uint32_t)(uint8_t)fslot[grp_f[g]] | ((uint32_t)np << 8) | ((uint32_t)(NLAB + 1 + p) << 16);
        e.y = 0;
        for (int j = 0; j < np; j++) e.y |= (uint32_t)p_t[p + j] << (8 * j);
        byn[np - 1].push_back(e);
      }
    for (int k = 0; k < 4; k++) {
      lrrec[4 * r0 + k] = (int)lrec.size();
      lrec.insert(lrec.end(), byn[k].begin(), byn[k].end());
    }
  }
  lrrec[4 * R] = (int)lrec.size();
  // row programs: channel byte offsets (x16: [channel][4 slots] u32), pairs
  // per u32, 4 u32 per uint4, padded with the all-ones channel
  int maxch = 1;
  for (const auto *d : drows) maxch = std::max<int>(maxch, (int)d->size());
  const int LRWV = (maxch + 7) / 8;
  const int NCH = NLAB + 1 + NP;
  if (16 * NCH > 0xffff) return set_err(c, SIGMO_ERR_LIMIT, "plane program too large (%d planes)", NP);
  const uint32_t pad2 = (uint32_t)(16 * NLAB) | ((uint32_t)(16 * NLAB) << 16);
  std::vector<uint32_t> lrowp((size_t)NDR * LRWV * 4, pad2);
  const int NDRW = (NDR + 31) / 32;
  std::vector<int32_t> lrgn((size_t)NDRW + 1, 0);
  for (int d = 0; d < NDR; d++) {
    const std::vector<int> &ch = *drows[d];
    for (size_t j = 0; j < ch.size(); j++) {
      uint32_t &w = lrowp[(size_t)d * LRWV * 4 + j / 2];
      const uint32_t o = (uint32_t)(16 * ch[j]);
      w = (j & 1) ? ((w & 0xffffu) | (o << 16)) : ((w & 0xffff0000u) | o);
    }
    lrgn[d / 32] = std::max<int32_t>(lrgn[d / 32], (int32_t)((ch.size() + 1) / 2));
  }
  // label -> label channel | field slot << 8
  std::vector<uint16_t> llut(256);
  {
    std::vector<uint8_t> lab_val(NLAB > 0 ? NLAB : 1);
    if (NLAB) CUDA_TRY(c, cudaMemcpy(lab_val.data(), P.lab_val, NLAB, cudaMemcpyDeviceToHost));
    for (int l = 0; l < 256; l++) {
      uint32_t lc = 0xff;
      for (int k = 0; k < NLAB; k++)
        if (lab_val[k] == l) lc = (uint32_t)k;
      const int fs = fslot[field_of_label(l)];
      llut[l] = (uint16_t)(lc | ((uint32_t)(fs >= 0 ? fs : 0xff) << 8));
    }
  }
  // GMCR lists per 32-query group: [entry][lane] (word, bits), padded (0, 0)
  const int NQG = (NQ + 31) / 32;
  std::vector<int2> lqwh((size_t)NQG + 1);
  std::vector<uint2> lqwl;
  for (int qg = 0; qg < NQG; qg++) {
    int mx = 0;
    for (int q = 32 * qg; q < std::min(NQ, 32 * qg + 32); q++) mx = std::max(mx, qw_off[q + 1] - qw_off[q]);
    lqwh[qg] = make_int2((int)(lqwl.size() / 32), mx);
    for (int j = 0; j < mx; j++)
      for (int l = 0; l < 32; l++) {
        const int q = 32 * qg + l;
        uint2 e = make_uint2(0u, 0u);
        if (q < NQ && j < qw_off[q + 1] - qw_off[q]) e = make_uint2(qw[2 * (qw_off[q] + j)], qw[2 * (qw_off[q] + j) + 1]);
        lqwl.push_back(e);
      }
  }
  // upload
  Layout L;
  const size_t o_rec = L.take(sizeof(GroupRec) * (rec.size() + 1));
  const size_t o_tab = L.take(4 * (tab.size() + 4));
  const size_t o_rr = L.take(4 * rrec.size());
  const size_t o_rc = L.take(4 * rcarry.size());
  const size_t o_bd = L.take(4 * bdone.size());
  const size_t o_po = L.take(4 * rowp_off.size());
  const size_t o_rp = L.take(4 * (rowp.size() + 1));
  const size_t o_dp = L.take(4 * (drowp.size() + 1));
  const size_t o_qd = L.take(2 * qdrow.size());
  const size_t o_qwo = L.take(4 * qw_off.size());
  const size_t o_qw = L.take(4 * (qw.size() + 2));
  const size_t o_lrec = L.take(8 * (lrec.size() + 1));
  const size_t o_lrr = L.take(4 * lrrec.size());
  const size_t o_lrp = L.take(4 * (lrowp.size() + 4));
  const size_t o_lrg = L.take(4 * lrgn.size());
  const size_t o_lqh = L.take(8 * lqwh.size());
  const size_t o_lql = L.take(8 * (lqwl.size() + 1));
  const size_t o_llu = L.take(2 * llut.size());
  std::vector<unsigned char> hb(L.off, 0);
  auto put = [&](size_t o, const void *src, size_t n) { if (n) memcpy(hb.data() + o, src, n); };
  put(o_rec, rec.data(), sizeof(GroupRec) * rec.size());
  put(o_tab, tab.data(), 4 * tab.size());
  put(o_rr, rrec.data(), 4 * rrec.size());
  put(o_rc, rcarry.data(), 4 * rcarry.size());
  put(o_bd, bdone.data(), 4 * bdone.size());
  put(o_po, rowp_off.data(), 4 * rowp_off.size());
  put(o_rp, rowp.data(), 4 * rowp.size());
  put(o_dp, drowp.data(), 4 * drowp.size());
  put(o_qd, qdrow.data(), 2 * qdrow.size());
  put(o_qwo, qw_off.data(), 4 * qw_off.size());
  put(o_qw, qw.data(), 4 * qw.size());
  put(o_lrec, lrec.data(), 8 * lrec.size());
  put(o_lrr, lrrec.data(), 4 * lrrec.size());
  put(o_lrp, lrowp.data(), 4 * lrowp.size());
  put(o_lrg, lrgn.data(), 4 * lrgn.size());
  put(o_lqh, lqwh.data(), 8 * lqwh.size());
  put(o_lql, lqwl.data(), 8 * lqwl.size());
  put(o_llu, llut.data(), 2 * llut.size());
  SIGMO_TRY(dreserve(c, pc.pack, L.off, "packed query program"));
  unsigned char *db = (unsigned char *)pc.pack.p;
  CUDA_TRY(c, cudaMemcpyAsync(db, hb.data(), L.off, cudaMemcpyHostToDevice, st));
  CUDA_TRY(c, cudaStreamSynchronize(st));  // hb is pageable and goes out of scope
  P.l_grec = (uint2 *)(db + o_lrec);
  P.l_rrec = (int32_t *)(db + o_lrr);
  P.l_rowp = (uint4 *)(db + o_lrp);
  P.l_rgn = (int32_t *)(db + o_lrg);
  P.l_qwh = (int2 *)(db + o_lqh);
  P.l_qwl = (uint2 *)(db + o_lql);
  P.l_lut = (uint16_t *)(db + o_llu);
  pc.jit = LaneJitSpec();
  pc.jit.NLAB = NLAB;
  pc.jit.NFU = m.NFU;
  pc.jit.R = R;
  pc.jit.NDR = NDR;
  pc.jit.RWV = LRWV;
  pc.jit.NQG = NQG;
  pc.jit.NQ = NQ;
  pc.jit.NQW = c->NQW;
  pc.jit.recs.resize((size_t)R);
  for (int r0 = 0; r0 < R; r0++) pc.jit.recs[r0].assign(lrec.begin() + lrrec[4 * r0], lrec.begin() + lrrec[4 * r0 + 4]);
  pc.jit.rgn.assign(lrgn.begin(), lrgn.begin() + NDRW);
  pc.jit.qwh.assign(lqwh.begin(), lqwh.begin() + NQG);
  P.meta.L_NREC = (int)lrec.size();
  P.meta.L_RWV = LRWV;
  P.meta.L_NQWE = (int)lqwl.size();
  P.meta.L_NQG = NQG;
  P.grec = (GroupRec *)(db + o_rec);
  P.tab = (uint32_t *)(db + o_tab);
  P.rrec_off = (int32_t *)(db + o_rr);
  P.rcarry = (int32_t *)(db + o_rc);
  P.bdone = (int32_t *)(db + o_bd);
  P.rowp_off = (int32_t *)(db + o_po);
  P.rowp = (uint32_t *)(db + o_rp);
  P.drowp = (uint32_t *)(db + o_dp);
  P.qdrow = (uint16_t *)(db + o_qd);
  P.meta.NDR = NDR;
  P.qw_off = (int32_t *)(db + o_qwo);
  P.qw = (uint32_t *)(db + o_qw);
  P.meta.NQWL = (int)(qw.size() / 2);
  pc.qdrow.assign(qdrow.begin(), qdrow.begin() + VQ);
  P.meta.NREC = (int)rec.size();
  P.meta.NRP = (int)rowp.size();
  P.meta.RW = RW;
  P.meta.NBATCH = NBATCH;
  P.meta.TS = TS;
  return SIGMO_OK;
}

sigmo_status ensure_prog(sigmo_ctx *c, int R, QueryProg *&out) {
  auto it = c->progs.find(R);
  if (it != c->progs.end() && it->second.valid && it->second.nw == c->NW) {
    out = &it->second.prog;
    return SIGMO_OK;
  }
  ProgCache &pc = c->progs[R];
  const int VQ = c->VQ;
  const size_t rowcap = (size_t)VQ * (R > 0 ? R : 1) * kNumFields + 1;
  Layout L;
  const size_t o_pt = L.take(kMaxPlanes);
  const size_t o_gp = L.take(2 * 256);
  const size_t o_gf = L.take(256);
  const size_t o_rg = L.take(2 * 32);
  const size_t o_fs = L.take(16);
  const size_t o_lv = L.take(256);
  const size_t o_rl = L.take((size_t)VQ + 1);
  const size_t o_ro = L.take(4 * ((size_t)VQ + 1));
  const size_t o_ri = L.take(2 * rowcap);
  const size_t o_me = L.take(sizeof(QueryProgMeta));
  SIGMO_TRY(dreserve(c, pc.buf, L.off, "query program"));
  unsigned char *b = (unsigned char *)pc.buf.p;
  QueryProg &P = pc.prog;
  P.R = R;
  P.p_t = b + o_pt;
  P.grp_poff = (int16_t *)(b + o_gp);
  P.grp_f = b + o_gf;
  P.rg_off = (int16_t *)(b + o_rg);
  P.fslot = (int8_t *)(b + o_fs);
  P.lab_val = b + o_lv;
  P.row_lab = b + o_rl;
  P.row_off = (int32_t *)(b + o_ro);
  P.row_ids = (uint16_t *)(b + o_ri);
  P.d_meta = (QueryProgMeta *)(b + o_me);
  timing_mark(c, 0);
  if (R > 0) {
    SIGMO_TRY(dreserve(c, c->qcounts, (size_t)VQ * R * kNumFields, "query counts"));
    CUDA_TRY(c, launch_sig_counts(c->dq, R, (uint8_t *)c->qcounts.p, c->wildcard_loaded, c->stream));
  }
  CUDA_TRY(c, launch_query_prep(c->dq, R, (const uint8_t *)c->qcounts.p, P, c->wildcard_loaded, c->stream));
  timing_mark(c, 1);
  CUDA_TRY(c, cudaMemcpyAsync(&P.meta, P.d_meta, sizeof(QueryProgMeta), cudaMemcpyDeviceToHost, c->stream));
  CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  if (P.meta.err) return set_err(c, SIGMO_ERR_LIMIT, "query program error %d", P.meta.err);
  SIGMO_TRY(pack_prog(c, R, pc));
  pc.valid = true;
  pc.nw = c->NW;
  out = &P;
  return SIGMO_OK;
}

// per-TW tile geometry (EXTN, EXTW, MOLCAP) of the data batch
void tile_geometry(sigmo_ctx *c, const HostGraphs &d) {
  // one monotone sweep per tile width (the graph of a node only moves forward)
  const int tws[6] = {32, 16, 8, 4, 2, 1};
  for (int k = 0; k < 6; k++) {
    const int TW = tws[k];
    int extn = 1, extw = 1, molcap = 1;
    const int64_t W = c->W;
    int64_t ga = 0, gb = 0;  // graph of the tile's first / last node
    for (int64_t w0 = 0; w0 < W; w0 += TW) {
      const int64_t n0 = w0 * 32, n1 = std::min<int64_t>(n0 + 32ll * TW, d.V);
      while (ga + 1 <= d.G && d.goff[ga + 1] <= n0) ga++;
      if (gb < ga) gb = ga;
      while (gb + 1 <= d.G && d.goff[gb + 1] <= n1 - 1) gb++;
      const int g0 = (int)ga, g1 = (int)gb + 1;
      const int64_t gs = d.goff[g0], ge = d.goff[g1];
      extn = std::max<int>(extn, (int)(ge - gs));
      extw = std::max<int>(extw, (int)(((ge - 1) >> 5) - (gs >> 5) + 1));
      molcap = std::max<int>(molcap, g1 - g0);
    }
    c->tile_extn[k] = extn;
    c->tile_extw[k] = extw;
    c->tile_molcap[k] = molcap;
  }
}

void free_all(sigmo_ctx *c) {
  for (auto &kv : c->progs) {
    dfree(c, kv.second.buf);
    dfree(c, kv.second.pack);
  }
  c->progs.clear();
  DBuf *bufs[] = {&c->arena, &c->qcounts, &c->bitmap, &c->gm, &c->mol_cnt, &c->off, &c->scan_tmp,
                  &c->chunk_start, &c->nchunks, &c->pair_query, &c->pair_rec, &c->pair_cm, &c->pair_result, &c->jcnt,
                  &c->sig_tmp, &c->gstack, &c->adjb, &c->dense_tmp, &c->ent2, &c->nb4, &c->mrec,
                  &c->eoff, &c->ecur, &c->emaps, &c->esets, &c->ucnt, &c->uoff, &c->uniq, &c->etmp,
                  &c->ns_win32, &c->ns_win64, &c->ns_alive, &c->gm_old, &c->off_old, &c->ent_ns, &c->ns_bitmap,
                  &c->ns_gm, &c->ns_cnt, &c->raw, &c->dpk, &c->ldinfo, &c->lay};
  for (DBuf *b : bufs) dfree(c, *b);
}

// chunk/stack/slice capacities of the join for the loaded batch
void fill_join_caps(sigmo_ctx *c, JoinParams &jp) {
  jp.NQ = c->NQ;
  jp.NQW = c->NQW;
  jp.VQ = c->VQ;
  jp.NB = c->NB;
  jp.induced = c->induced_loaded;
  jp.any_bond = c->any_bond;
  jp.qp_non = c->qp_non;
  jp.maxq = std::max(c->maxq, 2);
  jp.PCAP = c->PC;
  jp.ACAP = c->AC + c->maxn;
  jp.CMCAP = std::max(c->CMC, jp.maxq);
  jp.MCAP = c->MC;
  jp.NBE = c->NBE;
  jp.plan_smem = c->plan_smem;
  const int scg = 32 * (jp.maxq + 1) + 64;
  jp.SCS = std::min(scg, 128);
  if (const char *e = getenv("SIGMO_JOIN_SCS")) jp.SCS = std::max(128, atoi(e));  // test knob (spill path)
  jp.SW = 0;
  jp.slice_rows = 0;
}

// join internal-capacity flag and DFS step counter (synchronizes)
sigmo_status read_join_flags(sigmo_ctx *c) {
  unsigned long long f[6] = {0, 0, 0, 0, 0, 0};
  CUDA_TRY(c, cudaMemcpyAsync(f, c->jcnt.p, sizeof(f), cudaMemcpyDeviceToHost, c->stream));
  c->last.dfs_iters = (int64_t)f[3];
  c->last.dfs_tail_iters = (int64_t)f[4];
  c->last.dfs_max_stack = (int64_t)f[5];
  CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  c->last.dfs_steps = (int64_t)f[2];
  if ((int)f[1] != 0) return set_err(c, SIGMO_ERR_LIMIT, "join DFS stack capacity exceeded (internal limit)");
  return SIGMO_OK;
}

// Dense-tile filter (general path: > 64-atom graphs or > 11-node queries)
// into `bitmap` [VQ][Wpad] with its GMCR bits and counts, plus the
// neighbour-support pass on it (flag).  Also the dense view of the
// neighbour-support bitmap for sigmo_get_candidates on the lane path.
sigmo_status launch_dense(sigmo_ctx *c, int R, const QueryProg &P, uint32_t *bitmap, uint32_t *gm, I64x2 *mol_cnt,
                          bool ns, int &launches) {
  const QueryProgMeta &m = P.meta;
  if (!c->tile_geom_ok) {
    if ((int64_t)c->goff_host.size() != (int64_t)c->ND + 1) {  // device-loaded batch: read the offsets back
      std::vector<int32_t> g32((size_t)c->ND + 1);
      CUDA_TRY(c, cudaMemcpyAsync(g32.data(), c->dd.goff, 4 * g32.size(), cudaMemcpyDeviceToHost, c->stream));
      CUDA_TRY(c, cudaStreamSynchronize(c->stream));
      c->goff_host.assign(g32.begin(), g32.end());
    }
    HostGraphs hg;
    hg.G = c->ND;
    hg.V = c->VD;
    hg.goff = c->goff_host.data();
    tile_geometry(c, hg);
    c->tile_geom_ok = true;
  }
  const int tws[6] = {32, 16, 8, 4, 2, 1};
  int k = 0, rows_smem = 1;
  size_t smem = 0;
  for (k = 0; k < 12; k++) {
    rows_smem = k < 6 ? 1 : 0;
    const int kk = k % 6;
    smem = filter_smem_bytes(c->NW, c->tile_extn[kk], c->tile_extw[kk], c->tile_molcap[kk], m.NFU, m.NLAB, m.P, m.NREC,
                             c->VQ, m.NRP, rows_smem, c->NQW, m.TS, 0);
    // prefer >= 2 CTAs per SM with row programs in shared memory
    if (smem <= (rows_smem ? c->max_smem / 2 : c->max_smem)) break;
  }
  if (k == 12) return set_err(c, SIGMO_ERR_LIMIT, "filter shared memory %zu exceeds %zu (P=%d)", smem, c->max_smem, m.P);
  k = k % 6;
  if (c->has_empty_graph) {
    CUDA_TRY(c, cudaMemsetAsync(gm, 0, 4 * (size_t)c->ND * c->NQW, c->stream));
    CUDA_TRY(c, cudaMemsetAsync(mol_cnt, 0, sizeof(I64x2) * ((size_t)c->ND + 1), c->stream));
  }
    FilterParams fp{};
    fp.D = c->dd;
    fp.TW = tws[k];
    fp.W = c->W;
    fp.Wpad = c->Wpad;
    fp.VQ = c->VQ;
    fp.NQ = c->NQ;
    fp.NQW = c->NQW;
    fp.R = R;
    fp.P = m.P;
    fp.NFU = m.NFU;
    fp.NLAB = m.NLAB;
    fp.NREC = m.NREC;
    fp.NRP = m.NRP;
    fp.NBATCH = m.NBATCH;
    fp.RW = m.RW;
    fp.TS = m.TS;
    fp.grec = P.grec;
    fp.rrec_off = P.rrec_off;
    fp.rcarry = P.rcarry;
    fp.bdone = P.bdone;
    fp.tab = P.tab;
    fp.fslot = P.fslot;
    fp.lab_val = P.lab_val;
    fp.rowp_off = P.rowp_off;
    fp.rowp = P.rowp;
    fp.qgoff = c->dq.goff;
    fp.bitmap = bitmap;
    fp.gm = gm;
    fp.mol_cnt = mol_cnt;
    fp.EXTN = c->tile_extn[k];
    fp.EXTW = c->tile_extw[k];
    fp.MOLCAP = c->tile_molcap[k];
    fp.tile_g0 = tws[k] == 32 ? c->tile_g0 : nullptr;
    fp.tile_g1 = tws[k] == 32 ? c->tile_g1 : nullptr;
    fp.cmol = nullptr;
    fp.rows_smem = rows_smem;
    fp.smem_bytes = smem;
    const int tiles = (c->W + fp.TW - 1) / fp.TW;
    if (getenv("SIGMO_DEBUG_FILTER"))
      fprintf(stderr, "sigmo filter (dense): smem=%zu EXTN=%d EXTW=%d NFU=%d NLAB=%d P=%d NREC=%d TS=%d RW=%d tiles=%d\n",
              smem, fp.EXTN, fp.EXTW, m.NFU, m.NLAB, m.P, m.NREC, m.TS, m.RW, tiles);
    timing_mark(c, 2);
    CUDA_TRY(c, launch_filter(c->NW, fp, tiles, c->stream));
    launches++;
    if (ns) {
      SupportParams sp{};
      sp.ND = c->ND;
      sp.NQ = c->NQ;
      sp.NQW = c->NQW;
      sp.NB = c->NB;
      sp.any_bond = c->any_bond;
      sp.maxq = std::max(c->maxq, 1);
      sp.Wpad = c->Wpad;
      sp.goff = c->dd.goff;
      sp.roff = c->dd.roff;
      sp.nbr = c->dd.nbr;
      sp.bclass = c->bclass;
      sp.qgoff = c->dq.goff;
      sp.qroff = c->dq.roff;
      sp.qnbr = c->dq.nbr;
      sp.bitmap = bitmap;
      sp.gm = gm;
      sp.mol_cnt = mol_cnt;
      if (support_smem_bytes(c->NW, c->NB, sp.maxq, c->NQW) > c->max_smem)
        return set_err(c, SIGMO_ERR_LIMIT, "neighbour-support shared memory exceeds the device limit");
      CUDA_TRY(c, launch_support(c->NW, sp, c->stream));
      launches++;
    }
  return SIGMO_OK;
}

}  // namespace

// ===========================================================================
// C ABI
// ===========================================================================
extern "C" {

const char *sigmo_version(void) { return "sigmo-b200 0.1 (sm_100a)"; }

const char *sigmo_last_error(const sigmo_ctx *ctx) { return ctx ? ctx->err.c_str() : "NULL context"; }

sigmo_status sigmo_validate_batch(const sigmo_graph_batch *batch, int is_query, char *msg, size_t msg_len) {
  std::string m;
  HostGraphs h;
  sigmo_status s;
  try {
    s = validate(batch, is_query, m, h);
  } catch (...) {
    s = SIGMO_ERR_INVALID_ARG;
    m = "exception during validation";
  }
  if (msg && msg_len) {
    snprintf(msg, msg_len, "%s", m.c_str());
  }
  return s;
}

sigmo_status sigmo_create(int device, void *cuda_stream, const sigmo_allocator *alloc, sigmo_ctx **out) {
  if (!out) return SIGMO_ERR_INVALID_ARG;
  *out = nullptr;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
    cudaGetLastError();
    return SIGMO_ERR_CUDA;
  }
  if (alloc && (!alloc->alloc || !alloc->free)) return SIGMO_ERR_INVALID_ARG;
  sigmo_ctx *c = new (std::nothrow) sigmo_ctx();
  if (!c) return SIGMO_ERR_OOM;
  c->device = device;
  c->stream = (cudaStream_t)cuda_stream;
  if (alloc) {
    c->alloc = *alloc;
    c->has_alloc = true;
  }
  if (cudaSetDevice(device) != cudaSuccess) {
    delete c;
    return SIGMO_ERR_CUDA;
  }
  cudaDeviceGetAttribute(&c->sm_count, cudaDevAttrMultiProcessorCount, device);
  int smem = 0;
  cudaDeviceGetAttribute(&smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, device);
  if (smem > 0) c->max_smem = (size_t)smem;
  if (cudaEventCreateWithFlags(&c->h2d_done, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->fork_ev, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->join_ev, cudaEventDisableTiming) != cudaSuccess ||
      cudaStreamCreateWithFlags(&c->aux, cudaStreamNonBlocking) != cudaSuccess) {
    delete c;
    return SIGMO_ERR_CUDA;
  }
  for (int r = 0; r < Timing::RING; r++) {
    for (int k = 0; k < 5; k++) cudaEventCreate(&c->timing.fev[r][k]);
    for (int k = 0; k < 2; k++) cudaEventCreate(&c->timing.jev[r][k]);
  }
  *out = c;
  return SIGMO_OK;
}

sigmo_status sigmo_destroy(sigmo_ctx *c) {
  if (!c) return SIGMO_ERR_INVALID_ARG;
  cudaSetDevice(c->device);
  cudaStreamSynchronize(c->stream);
  free_all(c);
  cudaStreamSynchronize(c->stream);
  if (c->staging.p) cudaFreeHost(c->staging.p);
  if (c->ldhost.p) cudaFreeHost(c->ldhost.p);
  if (c->h2d_done) cudaEventDestroy(c->h2d_done);
  if (c->aux) {
    cudaStreamSynchronize(c->aux);
    cudaStreamDestroy(c->aux);
  }
  if (c->fork_ev) cudaEventDestroy(c->fork_ev);
  if (c->join_ev) cudaEventDestroy(c->join_ev);
  for (int r = 0; r < Timing::RING; r++) {
    for (int k = 0; k < 5; k++) cudaEventDestroy(c->timing.fev[r][k]);
    for (int k = 0; k < 2; k++) cudaEventDestroy(c->timing.jev[r][k]);
  }
  delete c;
  return SIGMO_OK;
}

sigmo_status sigmo_set_induced(sigmo_ctx *c, int enable) {
  if (!c) return SIGMO_ERR_INVALID_ARG;
  c->induced = enable != 0;
  return SIGMO_OK;
}

sigmo_status sigmo_set_wildcards(sigmo_ctx *c, int enable) {
  if (!c) return SIGMO_ERR_INVALID_ARG;
  c->wildcard = enable != 0;
  return SIGMO_OK;
}

sigmo_status sigmo_set_timing(sigmo_ctx *c, int enable) {
  if (!c) return SIGMO_ERR_INVALID_ARG;
  c->timing.enabled = (enable & 1) != 0;
  c->count_steps = (enable & 2) != 0;
  return SIGMO_OK;
}

sigmo_status sigmo_get_timings(sigmo_ctx *c, sigmo_timings *out) {
  if (!c || !out) return SIGMO_ERR_INVALID_ARG;
  CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  Timing &T = c->timing;
  for (int s = 0; s < Timing::RING; s++) {
    harvest_f(T, s);
    harvest_j(T, s);
  }
  c->last.query_prep_ms = T.n_qprep ? (float)(T.s_qprep / T.n_qprep) : 0.f;
  c->last.filter_ms = T.n_filter ? (float)(T.s_filter / T.n_filter) : 0.f;
  c->last.support_ms = 0.f;
  c->last.mapping_ms = T.n_mapping ? (float)(T.s_mapping / T.n_mapping) : 0.f;
  c->last.join_ms = T.n_join ? (float)(T.s_join / T.n_join) : 0.f;
  if (c->state >= 3) SIGMO_TRY(read_join_flags(c));
  c->last.filter_calls = T.n_filter;
  c->last.join_calls = T.n_join;
  T.s_qprep = T.s_filter = T.s_mapping = T.s_join = 0;
  T.n_qprep = T.n_filter = T.n_mapping = T.n_join = 0;
  *out = c->last;
  return SIGMO_OK;
}

sigmo_status sigmo_load_batch(sigmo_ctx *c, const sigmo_graph_batch *queries, const sigmo_graph_batch *data) {
  if (!c) return SIGMO_ERR_INVALID_ARG;
  if (!queries || !data) return set_err(c, SIGMO_ERR_INVALID_ARG, "queries/data batch is NULL");
  CUDA_TRY(c, cudaSetDevice(c->device));
  HostGraphs hq, hd;
  std::string msg;
  const auto t0 = std::chrono::steady_clock::now();
  sigmo_status s = validate(queries, 1, msg, hq);
  if (s != SIGMO_OK) return set_err(c, s, "query batch: %s", msg.c_str());
  // the same query batch as the previous load (byte for byte, same wildcard mode): the query programs
  // and the join's plan entries built for it are reused
  bool same_q = false;
  {
    std::vector<unsigned char> key;
    auto add = [&](const void *p, size_t n) {
      const unsigned char *b = (const unsigned char *)p;
      key.insert(key.end(), b, b + n);
    };
    const int64_t dims[4] = {hq.G, hq.V, hq.E, c->wildcard ? 1 : 0};
    add(dims, sizeof(dims));
    add(hq.goff, 8 * (size_t)(hq.G + 1));
    add(hq.roff, 8 * (size_t)(hq.V + 1));
    if (hq.E) add(hq.col, 4 * (size_t)hq.E);
    if (hq.V) add(hq.nlab, (size_t)hq.V);
    if (hq.E) add(hq.elab, (size_t)hq.E);
    same_q = c->qkey_valid && key == c->qkey;
    c->qkey.swap(key);
    c->qkey_valid = false;  // valid again once this load succeeded
  }
  // large data batches: O(#graphs) checks here, the per-entry checks and the
  // packing on the device (k_load_data) from the raw arrays
  const char *hl = getenv("SIGMO_HOST_LOAD");  // test knob: host validation + packing at any size
  const bool dev_load = data->num_nodes >= kDeviceLoadMinNodes && !(hl && atoi(hl));
  s = dev_load ? validate_light(data, msg, hd) : validate(data, 0, msg, hd);
  if (s != SIGMO_OK) return set_err(c, s, "data batch: %s", msg.c_str());
  // bond classes = distinct query bond labels; in wildcard mode (R22) the
  // '~' label 0 is no class of its own: it reads class NB, the union of all
  // bonds (the all-bonds adjacency every kernel builds)
  c->wildcard_loaded = c->wildcard;
  uint8_t bclass[256];
  memset(bclass, 255, sizeof(bclass));
  {
    bool seen[256] = {};
    for (int64_t e = 0; e < hq.E; e++) seen[hq.elab[e]] = true;
    c->any_bond = c->wildcard_loaded && seen[0];
    if (c->any_bond) seen[0] = false;
    int nb = 0;
    for (int l = 0; l < 256; l++)
      if (seen[l]) {
        if (nb >= SIGMO_MAX_BOND_CLASSES - (c->any_bond ? 1 : 0))
          return set_err(c, SIGMO_ERR_LIMIT, "more than %d distinct query bond labels",
                         SIGMO_MAX_BOND_CLASSES - (c->any_bond ? 1 : 0));
        bclass[l] = (uint8_t)nb++;
      }
    c->NB = nb;
    if (c->any_bond) bclass[0] = (uint8_t)nb;
  }
  size_t raw_bytes = 0;
  PackedOffsets pdd{};
  struct {
    long long an, aw;
    int cn, cw, maxn, nempty;
  } lay{};
  if (dev_load) {
    CUDA_TRY(c, cudaEventSynchronize(c->h2d_done));  // the previous load's copies no longer read our buffers
    Layout R;
    const size_t r_go = R.take(8 * (size_t)(hd.G + 1)), r_ro = R.take(8 * (size_t)(hd.V + 1));
    const size_t r_co = R.take(4 * (size_t)hd.E + 4), r_nl = R.take((size_t)hd.V + 1), r_el = R.take((size_t)hd.E + 1);
    SIGMO_TRY(dreserve(c, c->raw, R.off, "raw data batch"));
    unsigned char *rb = (unsigned char *)c->raw.p;
    // from the caller's buffers: DMA when they are pinned, else the driver stages them
    CUDA_TRY(c, cudaMemcpyAsync(rb + r_go, hd.goff, 8 * (size_t)(hd.G + 1), cudaMemcpyHostToDevice, c->stream));
    CUDA_TRY(c, cudaMemcpyAsync(rb + r_ro, hd.roff, 8 * (size_t)(hd.V + 1), cudaMemcpyHostToDevice, c->stream));
    if (hd.E) CUDA_TRY(c, cudaMemcpyAsync(rb + r_co, hd.col, 4 * (size_t)hd.E, cudaMemcpyHostToDevice, c->stream));
    if (hd.V) CUDA_TRY(c, cudaMemcpyAsync(rb + r_nl, hd.nlab, (size_t)hd.V, cudaMemcpyHostToDevice, c->stream));
    if (hd.E) CUDA_TRY(c, cudaMemcpyAsync(rb + r_el, hd.elab, (size_t)hd.E, cudaMemcpyHostToDevice, c->stream));
    raw_bytes = 8 * (size_t)(hd.G + 1) + 8 * (size_t)(hd.V + 1) + 5 * (size_t)hd.E + (size_t)hd.V;
    Layout Ld;
    pdd = plan_graphs(Ld, hd);
    SIGMO_TRY(dreserve(c, c->dpk, Ld.off, "packed data batch"));
    SIGMO_TRY(dreserve(c, c->ldinfo, 8 * 272, "load info"));
    CUDA_TRY(c, cudaMemsetAsync(c->ldinfo.p, 0, 8 * 256, c->stream));
    CUDA_TRY(c, cudaMemsetAsync((char *)c->ldinfo.p + 8 * 256, 0x7f, 8 * 8, c->stream));
    unsigned char *pk = (unsigned char *)c->dpk.p;
    DataLoadParams lp;
    lp.G = hd.G;
    lp.goff = (const int64_t *)(rb + r_go);
    lp.roff = (const int64_t *)(rb + r_ro);
    lp.col = (const int32_t *)(rb + r_co);
    lp.nlab = rb + r_nl;
    lp.elab = rb + r_el;
    lp.goff32 = (int32_t *)(pk + pdd.goff);
    lp.roff32 = (int32_t *)(pk + pdd.roff);
    lp.label = pk + pdd.label;
    lp.local = pk + pdd.local;
    lp.nbr = (uint16_t *)(pk + pdd.nbr);
    lp.hist = (unsigned long long *)c->ldinfo.p;
    lp.err_graph = (long long *)((char *)c->ldinfo.p + 8 * 256);
    if (hd.G == 0) CUDA_TRY(c, cudaMemsetAsync(pk + pdd.goff, 0, 4, c->stream));
    if (hd.G == 0) CUDA_TRY(c, cudaMemsetAsync(pk + pdd.roff, 0, 4, c->stream));
    CUDA_TRY(c, launch_load_data(lp, c->stream));
    // per-molecule layout (adjacency blocks, candidate units, group lists,
    // molecule records) from the packed offsets, on the device
    {
      const size_t G1 = (size_t)hd.G + 1;
      Layout LL;
      const size_t l_ao = LL.take(4 * G1), l_cu = LL.take(4 * G1), l_gn = LL.take(4 * (G1 + 8)),
                   l_gw = LL.take(4 * (G1 + 8)), l_sc = LL.take(layout_scan_bytes((int)hd.G));
      SIGMO_TRY(dreserve(c, c->lay, LL.off, "molecule layout"));
      SIGMO_TRY(dreserve(c, c->mrec, 16 * std::max<size_t>(G1, 2), "molecule records"));
      unsigned char *lb = (unsigned char *)c->lay.p;
      CUDA_TRY(c, cudaMemsetAsync(lb + l_gn, 0xff, 4 * (G1 + 8), c->stream));  // -1: empty group slots
      CUDA_TRY(c, cudaMemsetAsync(lb + l_gw, 0xff, 4 * (G1 + 8), c->stream));
      CUDA_TRY(c, launch_layout((const int32_t *)(pk + pdd.goff), (int)hd.G, std::max(c->NB, 0), lb + l_sc,
                                (uint32_t *)(lb + l_ao), (uint32_t *)(lb + l_cu), (int32_t *)(lb + l_gn),
                                (int32_t *)(lb + l_gw), (uint4 *)c->mrec.p,
                                (long long *)((char *)c->ldinfo.p + 8 * 264), c->stream));
      c->adj_off = (uint32_t *)(lb + l_ao);
      c->cand_units = (uint32_t *)(lb + l_cu);
      c->grp_narrow = (int32_t *)(lb + l_gn);
      c->grp_wide = (int32_t *)(lb + l_gw);
    }
    if (c->ldhost.cap < 8 * 272) {
      if (c->ldhost.p) cudaFreeHost(c->ldhost.p);
      c->ldhost.p = nullptr;
      CUDA_TRY(c, cudaHostAlloc(&c->ldhost.p, 8 * 272, cudaHostAllocDefault));
      c->ldhost.cap = 8 * 272;
    }
    CUDA_TRY(c, cudaMemcpyAsync(c->ldhost.p, c->ldinfo.p, 8 * 272, cudaMemcpyDeviceToHost, c->stream));
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    memcpy(&lay, (const char *)c->ldhost.p + 8 * 264, sizeof(lay));
    const long long *eg = (const long long *)c->ldhost.p + 256;
    const char *why[5] = {"row_offsets decreasing", "column outside its graph", "self-loop", "duplicate edge",
                          "asymmetric edge or edge label"};
    long long first = -1;
    int cls = -1;
    for (int k = 0; k < 5; k++)
      if (eg[k] < (long long)hd.G && (first < 0 || eg[k] < first)) {
        first = eg[k];
        cls = k;
      }
    if (cls >= 0) return set_err(c, SIGMO_ERR_INVALID_GRAPH, "data batch: data graph %lld: %s", first, why[cls]);
  }
  const auto t1 = std::chrono::steady_clock::now();
  c->state = 0;
  // label frequencies of the data batch (planner heuristic)
  std::vector<int64_t> freq(256, 0);
  if (dev_load) {
    const unsigned long long *h = (const unsigned long long *)c->ldhost.p;
    for (int l = 0; l < 256; l++) freq[l] = (int64_t)h[l];
  } else {
    std::vector<std::vector<int64_t>> part(64, std::vector<int64_t>(256, 0));
    parallel_for_graphs(hd.V, hd.V, [&](int th, int64_t a, int64_t b) {
      int64_t *f = part[th].data();
      for (int64_t v = a; v < b; v++) f[hd.nlab[v]]++;
    });
    for (const auto &p : part)
      for (int l = 0; l < 256; l++) freq[l] += p[l];
  }
  if (c->wildcard_loaded) freq[0] = std::max<int64_t>(hd.V, 1);  // '*' matches every atom: the least selective
  QPlan plan;
  plan_queries(hq, freq, bclass, plan);

  // per-tile graph ranges of the filter for TW = 32 (1,024 nodes per tile)
  std::vector<int32_t> tg0, tg1;
  if (!dev_load) {  // device-loaded batches: the dense filter finds its tiles' graphs by binary search
    const int64_t W = (hd.V + 31) / 32, tiles = (W + 31) / 32;
    tg0.resize((size_t)tiles + 1);
    tg1.resize((size_t)tiles + 1);
    for (int64_t t = 0; t < tiles; t++) {
      const int64_t n0 = t * 1024, n1 = std::min<int64_t>(n0 + 1024, hd.V);
      tg0[t] = graph_of_host(hd.goff, hd.G, n0);
      tg1[t] = graph_of_host(hd.goff, hd.G, n1 - 1) + 1;
    }
  }
  // per-lane join + molecule-tile filter possible for this batch?
  bool lane_ok = false;
  c->induced_loaded = c->induced;
  {
    int64_t maxn_h = 0, maxq_h = 0;
    if (dev_load) maxn_h = lay.maxn;
    else
      for (int64_t g = 0; g < hd.G; g++) maxn_h = std::max<int64_t>(maxn_h, hd.goff[g + 1] - hd.goff[g]);
    for (int64_t g = 0; g < hq.G; g++) maxq_h = std::max<int64_t>(maxq_h, hq.goff[g + 1] - hq.goff[g]);
    const char *legacy = getenv("SIGMO_JOIN_LEGACY");
    lane_ok = maxn_h <= 64 && (c->NB > 0 || c->any_bond) && maxq_h <= kJoinLaneMaxQ && !(legacy && atoi(legacy)) && hq.V < 65536 &&
              (unsigned long long)std::max<int64_t>(hq.V, 1) * (unsigned long long)std::max<int64_t>(hd.G, 1) <
                  (1ull << 32) &&
              (unsigned long long)(c->NB + 2) * hd.V + 1 < (1ull << 31) &&
              plan.be.size() + 2 < 0xffff;  // compact plan entries: 16-bit extra back-edge offsets
  }
  const auto t2 = std::chrono::steady_clock::now();
  // ---- staging layout ----
  Layout L;
  const PackedOffsets pq = plan_graphs(L, hq);
  const size_t o_row = L.take(4 * (size_t)hq.V);
  const size_t o_beoff = L.take(4 * ((size_t)hq.V + 1));
  const size_t o_be = L.take(2 * plan.be.size() + 2);
  const size_t o_bc = L.take(256);
  const size_t o_info = L.take(4 * (size_t)hq.V + 4);
  const size_t o_ent = L.take(16 * (size_t)hq.V + 16);
  const size_t o_non = L.take(4 * (size_t)hq.V + 4);  // induced mode: non-adjacent earlier depths per plan position
  const size_t o_qinfo = L.take(4 * (size_t)hq.G + 4);
  const size_t o_qn = L.take((size_t)hq.V + 16);  // enumerate mode: local query node of each plan position
  const size_t o_qnb = L.take(8 * (size_t)hq.V + 16);  // lane neighbour support: query neighbours per plan position
  HostGraphs hd_arena = hd;  // the data batch's packed arrays travel in the arena only when packed on the host
  if (dev_load) hd_arena.G = hd_arena.V = hd_arena.E = 0;
  const PackedOffsets pd = plan_graphs(L, hd_arena);
  const size_t o_tg0 = L.take(4 * tg0.size());
  const size_t o_tg1 = L.take(4 * tg1.size());
  // bond-class adjacency layout (k_join_lane): per molecule class-major,
  // 32-bit masks for <= 32-node molecules, 64-bit (even word offset) otherwise
  std::vector<uint32_t> aoff(dev_load ? 1 : (size_t)hd.G + 1, 0), cu(dev_load ? 1 : (size_t)hd.G + 1, 0);
  std::vector<int32_t> grpn, grpw;
  uint64_t adj_words_total = 0, cand_units_total = 0;
  if (dev_load) {
    // computed on the device (launch_layout): narrow molecules first, wide ones from an even offset
    adj_words_total = (((uint64_t)lay.an + 1) & ~1ull) + (uint64_t)lay.aw;
    cand_units_total = (((uint64_t)lay.cn + 1) & ~1ull) + 2ull * (uint64_t)lay.cw;
    if (adj_words_total + 4 >= (1ull << 32)) lane_ok = false;
    if ((unsigned long long)std::max<int64_t>(hq.V, 1) * (cand_units_total + 2) >= (1ull << 32)) lane_ok = false;
  } else {
    uint64_t w = 0;
    for (int64_t g = 0; g < hd.G; g++) {
      const int64_t n = hd.goff[g + 1] - hd.goff[g];
      if (n > 32) w = (w + 1) & ~1ull;
      aoff[g] = (uint32_t)std::min<uint64_t>(w, 0xffffffffull);
      w += (uint64_t)n * (uint64_t)(c->NB + 1) * (n > 32 ? 2 : 1);  // + the all-bonds class (index NB)
    }
    w = (w + 1) & ~1ull;
    aoff[hd.G] = (uint32_t)std::min<uint64_t>(w, 0xffffffffull);
    adj_words_total = w;
    if (w + 4 >= (1ull << 32)) lane_ok = false;  // + the all-ones and all-zeros sentinel entries
    // molecule-padded candidate windows (filter output, join input): per
    // molecule NDR windows of one 32-bit word (<= 32 nodes) or two (64-bit,
    // even unit offset); molecule g starts at word NDR * cu[g]
    uint64_t u = 0;
    for (int64_t g = 0; g < hd.G; g++) {
      const int64_t n = hd.goff[g + 1] - hd.goff[g];
      if (n > 32) u = (u + 1) & ~1ull;
      cu[g] = (uint32_t)std::min<uint64_t>(u, 0xffffffffull);
      u += n > 32 ? 2 : 1;
    }
    cu[hd.G] = (uint32_t)std::min<uint64_t>(u, 0xffffffffull);
    cand_units_total = u;
    if ((unsigned long long)std::max<int64_t>(hq.V, 1) * (u + 2) >= (1ull << 32)) lane_ok = false;
    // k_filter_lane groups: 4 molecules of <= 32 atoms / 2 of 33-64 atoms (-1 = empty slot)
    for (int64_t g = 0; g < hd.G; g++) {
      const int64_t n = hd.goff[g + 1] - hd.goff[g];
      (n > 32 ? grpw : grpn).push_back((int32_t)g);
    }
    while (grpn.size() % 4) grpn.push_back(-1);
    while (grpw.size() % 2) grpw.push_back(-1);
  }
  const size_t o_ao = L.take(4 * aoff.size());
  const size_t o_cu = L.take(4 * cu.size());
  const size_t o_grpn = L.take(4 * grpn.size() + 16);
  const size_t o_grpw = L.take(4 * grpw.size() + 16);
  const size_t total = L.off;
  const auto t3 = std::chrono::steady_clock::now();
  // wait until the previous upload no longer reads the staging buffer
  CUDA_TRY(c, cudaEventSynchronize(c->h2d_done));
  if (c->staging.cap < total) {
    if (c->staging.p) cudaFreeHost(c->staging.p);
    c->staging.p = nullptr;
    c->staging.cap = 0;
    size_t cap = std::max<size_t>(total, c->staging.cap * 3 / 2);
    CUDA_TRY(c, cudaHostAlloc(&c->staging.p, cap, cudaHostAllocDefault));
    c->staging.cap = cap;
  }
  unsigned char *hb = (unsigned char *)c->staging.p;
  pack_graphs(hb, pq, hq);
  memcpy(hb + o_row, plan.row.data(), 4 * plan.row.size());
  memcpy(hb + o_beoff, plan.beoff.data(), 4 * plan.beoff.size());
  if (!plan.be.empty()) memcpy(hb + o_be, plan.be.data(), 2 * plan.be.size());
  memcpy(hb + o_bc, bclass, 256);
  if (!plan.info.empty()) memcpy(hb + o_info, plan.info.data(), 4 * plan.info.size());
  {
    // per plan position: back-edge depths, bond-class offsets into adjb
    // (class * VD) and the extra back-edge start, for k_join_lane
    int4 *ent = (int4 *)(hb + o_ent);
    int64_t qg = 0;
    for (int64_t i = 0; i < hq.V; i++) {
      while (hq.goff[qg + 1] <= i) qg++;
      const uint32_t inf = plan.info[i];
      const uint32_t j0 = inf & 0x3f, j1 = (inf >> 9) & 0x3f;
      // x: j0 | j1 << 4 (15 = none; map slot 15 reads 0) | #extra << 8 | query node << 12
      // y, z: bond class of back-edge 0 / 1 (adjb[v * NB + class])
      // w: first extra back-edge in qp_be
      // (fields are only meaningful for queries of <= kJoinLaneMaxQ nodes)
      int4 e4;
      e4.x = (int)((j0 == 0x3f ? 15u : (j0 & 15u)) | ((j1 == 0x3f ? 15u : (j1 & 15u)) << 4) |
                   (((inf >> 18) & 15u) << 8) | ((uint32_t)((plan.row[i] - hq.goff[qg]) & 15) << 12));
      e4.y = j0 == 0x3f ? 0 : (int)((inf >> 6) & 7u);
      e4.z = j1 == 0x3f ? 0 : (int)((inf >> 15) & 7u);
      e4.w = plan.beoff[i] + 2;
      ent[i] = e4;
    }
    if (hq.G) memcpy(hb + o_qinfo, plan.qinfo.data(), 4 * (size_t)hq.G);
    {
      // neighbours (plan depth | bond class << 4 | 0x80) of each plan position, <= 8
      uint2 *qnb = (uint2 *)(hb + o_qnb);
      std::vector<uint8_t> cnt((size_t)hq.V, 0);
      c->ns_lane_ok = true;
      for (int64_t i = 0; i < hq.V; i++) qnb[i] = make_uint2(0u, 0u);
      auto put = [&](int64_t pos, uint32_t depth, uint32_t cls) {
        const int k = cnt[(size_t)pos]++;
        if (k >= 8) {
          c->ns_lane_ok = false;
          return;
        }
        const uint32_t b = (depth & 15u) | ((cls & 7u) << 4) | 0x80u;
        if (k < 4) qnb[pos].x |= b << (8 * k);
        else qnb[pos].y |= b << (8 * (k - 4));
      };
      int64_t qq = 0;
      for (int64_t i = 0; i < hq.V; i++) {
        while (hq.goff[qq + 1] <= i) qq++;
        const int64_t lo = hq.goff[qq];
        for (int k = plan.beoff[i]; k < plan.beoff[i + 1]; k++) {
          const uint32_t j = plan.be[k] >> 8, cls = plan.be[k] & 255u;
          put(i, j, cls);                                        // i's back-edge to depth j
          put(lo + j, (uint32_t)(i - lo), cls);                  // and the forward edge of depth j
        }
      }
    }
    {
      uint8_t *qn = hb + o_qn;
      int64_t qq = 0;
      for (int64_t i = 0; i < hq.V; i++) {
        while (hq.goff[qq + 1] <= i) qq++;
        qn[i] = (uint8_t)(plan.row[i] - hq.goff[qq]);
      }
    }
    // induced mode (R21): bit j of non[i] = earlier depth j < e not adjacent to depth e
    uint32_t *non = (uint32_t *)(hb + o_non);
    int64_t qn = 0;
    for (int64_t i = 0; i < hq.V; i++) {
      while (hq.goff[qn + 1] <= i) qn++;
      const int e = (int)(i - hq.goff[qn]);
      uint64_t m = e >= 32 ? 0xffffffffull : ((1ull << e) - 1ull);
      for (int k = plan.beoff[i]; k < plan.beoff[i + 1]; k++) m &= ~(1ull << (plan.be[k] >> 8));
      non[i] = (uint32_t)m;
    }
    // the join's plan entries stay valid when the query batch and its matching order did not change
    // (a stream of data batches against the same queries: no re-upload and no host sync per batch)
    const bool same_plan = same_q && c->ent_host.size() == (size_t)hq.V &&
                           (hq.V == 0 || !memcmp(c->ent_host.data(), ent, sizeof(int4) * (size_t)hq.V)) &&
                           c->ent_row == plan.row;
    c->ent_host.assign(ent, ent + hq.V);
    c->ent_row.assign(plan.row.begin(), plan.row.end());
    c->qgoff_host.assign(hq.goff, hq.goff + hq.G + 1);
    if (!same_plan) c->ent_R = -1;
  }
  if (!dev_load) pack_graphs(hb, pd, hd);
  memcpy(hb + o_tg0, tg0.data(), 4 * tg0.size());
  memcpy(hb + o_tg1, tg1.data(), 4 * tg1.size());
  memcpy(hb + o_ao, aoff.data(), 4 * aoff.size());
  memcpy(hb + o_cu, cu.data(), 4 * cu.size());
  if (!grpn.empty()) memcpy(hb + o_grpn, grpn.data(), 4 * grpn.size());
  if (!grpw.empty()) memcpy(hb + o_grpw, grpw.data(), 4 * grpw.size());

  const auto t4 = std::chrono::steady_clock::now();
  // ---- device arena + one H2D copy ----
  SIGMO_TRY(dreserve(c, c->arena, total, "input arena"));
  unsigned char *db = (unsigned char *)c->arena.p;
  CUDA_TRY(c, cudaMemcpyAsync(db, hb, total, cudaMemcpyHostToDevice, c->stream));
  c->last.h2d_bytes = (int64_t)(total + raw_bytes);
  CUDA_TRY(c, cudaEventRecord(c->h2d_done, c->stream));
  c->dq = dev_view(db, pq, hq);
  if (dev_load) {
    HostGraphs hd0 = hd;
    hd0.G = 0;  // dev_view's O(#graphs) maximum: known from the device layout pass
    c->dd = dev_view((unsigned char *)c->dpk.p, pdd, hd0);
    c->dd.num_graphs = (int)hd.G;
    c->dd.max_nodes = lay.maxn;
  } else {
    c->dd = dev_view(db, pd, hd);
  }
  c->qp_row = (int32_t *)(db + o_row);
  c->qp_beoff = (int32_t *)(db + o_beoff);
  c->qp_be = (uint16_t *)(db + o_be);
  c->bclass = db + o_bc;
  c->tile_g0 = dev_load ? nullptr : (int32_t *)(db + o_tg0);
  if (!dev_load) {
    c->adj_off = (uint32_t *)(db + o_ao);
    c->cand_units = (uint32_t *)(db + o_cu);
    c->grp_narrow = (int32_t *)(db + o_grpn);
    c->grp_wide = (int32_t *)(db + o_grpw);
    c->NGN = (int)(grpn.size() / 4);
    c->NGW = (int)(grpw.size() / 2);
  } else {
    c->NGN = (lay.cn + 3) / 4;
    c->NGW = (lay.cw + 1) / 2;
  }
  c->adj_words = (uint32_t)std::min<uint64_t>(adj_words_total, 0xffffffffull);
  c->cand_total = (uint32_t)std::min<uint64_t>(cand_units_total, 0xffffffffull);

  c->tile_g1 = dev_load ? nullptr : (int32_t *)(db + o_tg1);
  c->qp_info = (uint32_t *)(db + o_info);
  c->qp_ent = (const int4 *)(db + o_ent);
  c->qp_non = (const uint32_t *)(db + o_non);
  c->qp_qinfo = (const uint32_t *)(db + o_qinfo);
  c->qp_qn = (const uint8_t *)(db + o_qn);
  c->qp_nbr = (const uint2 *)(db + o_qnb);
  c->enum_P = -1;
  c->NQ = (int)hq.G;
  c->VQ = (int)hq.V;
  c->EQ = (int)hq.E;
  c->NQW = (c->NQ + 31) / 32;
  c->maxq = c->dq.max_nodes;
  c->ND = (int)hd.G;
  c->VD = (int)hd.V;
  c->ED = (int)hd.E;
  c->maxn = c->dd.max_nodes;
  c->NW = c->maxn <= 64 ? 1 : (c->maxn <= 128 ? 2 : 4);
  c->has_empty_graph = false;
  if (dev_load) c->has_empty_graph = lay.nempty > 0;
  else
    for (int64_t g = 0; g < hd.G && !c->has_empty_graph; g++) c->has_empty_graph = hd.goff[g + 1] == hd.goff[g];
  c->W = (c->VD + 31) / 32;
  c->Wpad = ((c->W + 31) / 32) * 32;
  if (c->Wpad == 0) c->Wpad = 32;
  // dense-tile geometry: now if the dense path is the only one, else lazily
  if (dev_load) c->goff_host.clear();  // read back from the device if the dense path ever needs it
  else c->goff_host.assign(hd.goff, hd.goff + hd.G + 1);
  c->tile_geom_ok = false;
  if (!lane_ok) {
    tile_geometry(c, hd);
    c->tile_geom_ok = true;
  }
  c->NBE = (int)plan.be.size();
  c->plan_smem = 0;  // plans are read through the read-only cache
  // join chunk capacities (pairs, atoms, candidate masks, graphs per warp
  // chunk): shrink until the join's shared memory allows >= 2 CTAs per SM
  {
    c->PC = 80;
    c->AC = 48;
    c->CMC = 320;
    c->MC = 8;
    for (int tries = 0; tries < 12; tries++) {
      JoinParams jp{};
      fill_join_caps(c, jp);
      if (join_smem_bytes(c->NW, jp) <= c->max_smem / 2 || c->PC <= 8) break;
      c->PC = std::max(c->PC / 2, 8);
      c->AC = std::max(c->AC / 2, 8);
      c->CMC = std::max(c->CMC / 2, 32);
      c->MC = std::max(c->MC / 2, 1);
    }
  }
  // query programs depend on the query batch (and the wildcard mode) only
  if (!same_q)
    for (auto &kv : c->progs) kv.second.valid = false;

  // ---- per-batch device buffers ----
  // (+64 B: the join reads up to two words past a molecule window)
  size_t bm_bytes = 4 * (size_t)std::max(c->VQ, 1) * c->Wpad + 64;
  if (lane_ok) bm_bytes = std::max(bm_bytes, 4 * (size_t)std::max(c->VQ, 1) * (c->cand_total + 2));  // cmol layout
  SIGMO_TRY(dreserve(c, c->bitmap, bm_bytes, "candidate bitmap"));
  c->dense_pad_zero = false;  // zeroed before the first dense-tile filter (sigmo_filter)
  c->bm_bytes = bm_bytes;
  SIGMO_TRY(dreserve(c, c->gm, 4 * (size_t)std::max(c->ND, 1) * std::max(c->NQW, 1), "gmcr bits"));
  SIGMO_TRY(dreserve(c, c->mol_cnt, sizeof(I64x2) * ((size_t)c->ND + 1), "gmcr counts"));
  CUDA_TRY(c, cudaMemsetAsync(c->mol_cnt.p, 0, sizeof(I64x2) * ((size_t)c->ND + 1), c->stream));
  SIGMO_TRY(dreserve(c, c->off, sizeof(I64x2) * ((size_t)c->ND + 1), "gmcr offsets"));
  size_t tb = 0;
  CUDA_TRY(c, launch_scan(nullptr, nullptr, c->ND + 1, nullptr, &tb, c->stream));
  SIGMO_TRY(dreserve(c, c->scan_tmp, tb, "scan temp"));
  c->scan_tmp_bytes = std::max(tb, (size_t)16);
  const long long pair_cap = (long long)c->NQ * c->ND;
  const long long max_chunks = (long long)c->VD / c->AC + (long long)c->ND / c->MC + 4;
  SIGMO_TRY(dreserve(c, c->chunk_start, 4 * (size_t)max_chunks, "chunk starts"));
  SIGMO_TRY(dreserve(c, c->nchunks, 16, "chunk count"));
  SIGMO_TRY(dreserve(c, c->pair_query, 4 * (size_t)std::max(pair_cap, 1ll), "pair queries"));
  // per-lane join: pair records, per-pair candidate masks, bond-class adjacency
  c->lane_join = lane_ok;
  c->mol_filter = false;
  if (c->lane_join) {
    SIGMO_TRY(dreserve(c, c->pair_rec, 16 * (size_t)std::max(pair_cap, 1ll), "pair records"));
    SIGMO_TRY(dreserve(c, c->adjb, 4 * ((size_t)c->adj_words + 4), "bond-class adjacency"));
    // words adj_words, adj_words + 1 = all ones: the target of absent back-edges;
    // adj_words + 2, + 3 = all zeros (absent non-edge in the induced lane join)
    CUDA_TRY(c, cudaMemsetAsync((uint32_t *)c->adjb.p + c->adj_words, 0xff, 8, c->stream));
    CUDA_TRY(c, cudaMemsetAsync((uint32_t *)c->adjb.p + c->adj_words + 2, 0, 8, c->stream));
    SIGMO_TRY(dreserve(c, c->nb4, 4 * (size_t)std::max(c->VD, 1), "packed neighbours"));
    if (!dev_load) SIGMO_TRY(dreserve(c, c->mrec, 16 * (size_t)std::max(c->ND, 1), "molecule records"));
    CUDA_TRY(c, launch_adjb(c->dd, c->bclass, c->NB, c->adj_off, (uint32_t *)c->adjb.p, (uint32_t *)c->nb4.p, c->stream));
    if (!dev_load) CUDA_TRY(c, launch_mrec(c->dd.goff, c->adj_off, c->cand_units, c->ND, (uint4 *)c->mrec.p, c->stream));
  }
  SIGMO_TRY(dreserve(c, c->pair_result, 8 * (size_t)std::max(pair_cap, 1ll), "pair results"));
  SIGMO_TRY(dreserve(c, c->jcnt, 8 * ((size_t)c->NQ + 8), "join counters"));  // + the second claim counter
  if (getenv("SIGMO_DEBUG_LOAD")) {
    const auto t5 = std::chrono::steady_clock::now();
    auto ms = [](std::chrono::steady_clock::time_point a, std::chrono::steady_clock::time_point b) {
      return std::chrono::duration<double, std::milli>(b - a).count();
    };
    cudaStreamSynchronize(c->stream);
    const auto t6 = std::chrono::steady_clock::now();
    fprintf(stderr, "sigmo load: validate(+device pass) %.1f  plan %.1f  layout %.1f  pack %.1f  h2d+device enqueue %.1f  "
            "drain %.1f ms\n", ms(t0, t1), ms(t1, t2), ms(t2, t3), ms(t3, t4), ms(t4, t5), ms(t5, t6));
  }
  c->state = 1;
  c->qkey_valid = true;
  c->err.clear();
  return SIGMO_OK;
}

sigmo_status sigmo_filter(sigmo_ctx *c, int levels, uint32_t flags) {
  if (!c) return SIGMO_ERR_INVALID_ARG;
  if (c->state < 1) return set_err(c, SIGMO_ERR_STATE, "sigmo_filter before sigmo_load_batch");
  if (levels < 1 || levels > SIGMO_MAX_LEVELS) return set_err(c, SIGMO_ERR_INVALID_ARG, "levels %d not in 1..16", levels);
  if (flags & ~(uint32_t)SIGMO_FILTER_NEIGHBOR_SUPPORT) return set_err(c, SIGMO_ERR_INVALID_ARG, "unknown flags 0x%x", flags);
  CUDA_TRY(c, cudaSetDevice(c->device));
  const int R = levels - 1;
  timing_begin_filter(c);
  QueryProg *prog = nullptr;
  SIGMO_TRY(ensure_prog(c, R, prog));
  int launches = 0;
  if (c->ND > 0 && c->VD > 0) {
    const QueryProgMeta &m = prog->meta;
    // lane path (cmol layout for the per-lane join, k_filter_lane; the
    // neighbour-support pass on it refines per-pair windows, k_support_lane)
    // or the dense tiles of the general path
    const bool mol = c->lane_join;
    const bool lane_ns = mol && (flags & SIGMO_FILTER_NEIGHBOR_SUPPORT) != 0;
    c->lane_ns = false;
    if (lane_ns && !c->ns_lane_ok)
      return set_err(c, SIGMO_ERR_LIMIT, "neighbour support on the lane path: a query node has more than 8 neighbours");
    c->mol_filter = mol;
    if (mol) {
      c->dense_pad_zero = false;  // the molecule-padded layout overwrites the dense padding
    } else if (!c->dense_pad_zero) {
      // the dense filter writes words [0, W) of every row; the padding words
      // (read past molecule windows by the general join) and the tail are zero
      if (c->Wpad > c->W)
        CUDA_TRY(c, cudaMemset2DAsync((uint32_t *)c->bitmap.p + c->W, 4 * (size_t)c->Wpad, 0, 4 * (size_t)(c->Wpad - c->W),
                                      (size_t)std::max(c->VQ, 1), c->stream));
      const size_t used = 4 * (size_t)std::max(c->VQ, 1) * c->Wpad;
      if (c->bm_bytes > used) CUDA_TRY(c, cudaMemsetAsync((char *)c->bitmap.p + used, 0, c->bm_bytes - used, c->stream));
      c->dense_pad_zero = true;
    }
    if (mol && c->ent_R != R) {
      // distinct-row index of each plan position's query node into the plan entries
      const std::vector<uint16_t> &qd = c->progs[R].qdrow;
      c->ent_up.resize(c->ent_host.size());
      // k_join_lane entry of plan position i (JoinParams::qp_ent2): byte offsets of the two
      // back-edge map slots (slot maxq - 1 = absent), leaf flag, #extra back-edges;
      // bond classes and the distinct row
      int64_t q = 0;
      for (size_t i = 0; i < c->ent_up.size(); i++) {
        while (c->qgoff_host[q + 1] <= (int64_t)i) q++;
        const int4 e = c->ent_host[i];
        const unsigned j0 = (unsigned)e.x & 15u, j1 = ((unsigned)e.x >> 4) & 15u, nex = ((unsigned)e.x >> 8) & 15u;
        const unsigned absent = (unsigned)std::max(c->maxq, 2) - 1u;  // = JoinParams::maxq - 1
        const unsigned s0 = j0 == 15u ? absent : j0, s1 = j1 == 15u ? absent : j1;
        const unsigned leaf = (int64_t)i == c->qgoff_host[q + 1] - 1 ? 1u : 0u;
        c->ent_up[i].x = (s0 << 7) | (leaf << 11) | (nex << 12) | ((s1 << 7) << 16);
        c->ent_up[i].y = ((unsigned)e.y & 7u) | (((unsigned)e.z & 7u) << 3) | ((unsigned)qd[(size_t)c->ent_row[i]] << 12);
      }
      c->lane_extras = false;  // some plan position has > 2 back-edges (fused rings): the join keeps its extra loop
      for (const uint2 &u : c->ent_up) c->lane_extras = c->lane_extras || (u.x & 0xf000u);
      SIGMO_TRY(dreserve(c, c->ent2, sizeof(uint2) * (c->ent_up.size() + 1), "plan entries"));
      if (!c->ent_up.empty())
        CUDA_TRY(c, cudaMemcpyAsync(c->ent2.p, c->ent_up.data(), sizeof(uint2) * c->ent_up.size(),
                                    cudaMemcpyHostToDevice, c->stream));
      // neighbour-support mode: the join reads per-pair windows in plan-depth order
      c->ent_ns_up = c->ent_up;
      {
        int64_t q = 0;
        for (size_t i = 0; i < c->ent_ns_up.size(); i++) {
          while (c->qgoff_host[q + 1] <= (int64_t)i) q++;
          c->ent_ns_up[i].y = (c->ent_ns_up[i].y & 0xfffu) | ((unsigned)(i - c->qgoff_host[q]) << 12);
        }
      }
      SIGMO_TRY(dreserve(c, c->ent_ns, sizeof(uint2) * (c->ent_ns_up.size() + 1), "plan entries (support)"));
      if (!c->ent_ns_up.empty())
        CUDA_TRY(c, cudaMemcpyAsync(c->ent_ns.p, c->ent_ns_up.data(), sizeof(uint2) * c->ent_ns_up.size(),
                                    cudaMemcpyHostToDevice, c->stream));
      CUDA_TRY(c, cudaStreamSynchronize(c->stream));  // the host vectors may change before the copies ran
      c->ent_R = R;
    }
    if (c->has_empty_graph) {
      CUDA_TRY(c, cudaMemsetAsync(c->gm.p, 0, 4 * (size_t)c->ND * c->NQW, c->stream));
      CUDA_TRY(c, cudaMemsetAsync(c->mol_cnt.p, 0, sizeof(I64x2) * ((size_t)c->ND + 1), c->stream));
    }
    if (mol) {
      FilterLaneParams lp{};
      lp.NGN = c->NGN;
      lp.NGW = c->NGW;
      lp.grp_narrow = c->grp_narrow;
      lp.grp_wide = c->grp_wide;
      lp.mrec = (const uint4 *)c->mrec.p;
      lp.label = c->dd.label;
      lp.nb4 = (const uint32_t *)c->nb4.p;
      lp.adjw = (const uint32_t *)c->adjb.p;
      lp.NB = c->NB;
      lp.R = R;
      lp.NLAB = m.NLAB;
      lp.NFU = m.NFU;
      lp.NCH = m.NLAB + 1 + m.P;
      lp.lut = prog->l_lut;
      lp.grec = prog->l_grec;
      lp.NREC = m.L_NREC;
      lp.rrec = prog->l_rrec;
      lp.rowp = prog->l_rowp;
      lp.rgn = prog->l_rgn;
      lp.NDR = m.NDR;
      lp.RWV = m.L_RWV;
      lp.qwl = prog->l_qwl;
      lp.NQWE = m.L_NQWE;
      lp.qwh = prog->l_qwh;
      lp.NQG = m.L_NQG;
      lp.NQ = c->NQ;
      lp.NQW = c->NQW;
      lp.cmol = (uint32_t *)c->bitmap.p;
      lp.gm = (uint32_t *)c->gm.p;
      lp.mol_cnt = (I64x2 *)c->mol_cnt.p;
      lp.tables_global = 0;
      lp.smem_bytes = filter_lane_smem_bytes(lp);
      const char *tg = getenv("SIGMO_FILTER_TABLES_GLOBAL");  // test knob: tables from global memory
      if (lp.smem_bytes > c->max_smem / 3 || (tg && atoi(tg))) {
        lp.tables_global = 1;
        lp.smem_bytes = filter_lane_smem_bytes(lp);
      }
      if (lp.smem_bytes > c->max_smem)
        return set_err(c, SIGMO_ERR_LIMIT, "lane filter shared memory %zu exceeds %zu", lp.smem_bytes, c->max_smem);
      // the program-specialised kernel (NVRTC, cached per process) unless
      // disabled (SIGMO_FILTER_JIT=0) or unavailable; the generic one otherwise
      cudaKernel_t jk = nullptr;
      const char *je = getenv("SIGMO_FILTER_JIT");
      if (!(je && atoi(je) == 0)) {
        LaneJitSpec &js = c->progs[R].jit;
        js.GL = lp.tables_global != 0;
        js.min_blocks = 3;  // 80 registers, 24 warps/SM (configs[2]: 0.93 ms at the unbounded 110 registers)
        if (const char *mb = getenv("SIGMO_FILTER_JIT_MINB")) js.min_blocks = std::max(1, std::min(8, atoi(mb)));
        std::string why;
        double cms = 0.0;
        jk = lane_jit_kernel(js, &why, &cms);
        c->jit_note = jk ? (cms > 0.0 ? "compiled" : "cached") : why;
        if (cms > 0.0) c->last.jit_compile_ms = cms;
        if (!jk && getenv("SIGMO_DEBUG_FILTER")) fprintf(stderr, "sigmo filter: JIT unavailable: %s\n", why.c_str());
      }
      c->last.filter_jit = jk ? 1 : 0;
      const int bps = jk ? filter_lane_jit_blocks_per_sm(jk, lp) : filter_lane_blocks_per_sm(lp);
      const int ngroups = c->NGN + c->NGW;
      const int grid = std::max(1, std::min(bps * c->sm_count, (ngroups + kFilterLaneThreads / 32 - 1) / (kFilterLaneThreads / 32)));
      if (getenv("SIGMO_DEBUG_FILTER"))
        fprintf(stderr, "sigmo filter (lane%s): smem=%zu global=%d NCH=%d NFU=%d NREC=%d NDR=%d RWV=%d NQG=%d NQWE=%d groups=%d+%d grid=%d\n",
                jk ? ", specialised" : "", lp.smem_bytes, lp.tables_global, lp.NCH, lp.NFU, lp.NREC, lp.NDR, lp.RWV, lp.NQG,
                lp.NQWE, c->NGN, c->NGW, grid);
      timing_mark(c, 2);
      if (jk) CUDA_TRY(c, launch_filter_lane_jit(jk, lp, grid, c->stream));
      else CUDA_TRY(c, launch_filter_lane(lp, grid, c->stream));
      launches++;
    } else {
      SIGMO_TRY(launch_dense(c, R, *prog, (uint32_t *)c->bitmap.p, (uint32_t *)c->gm.p, (I64x2 *)c->mol_cnt.p,
                             (flags & SIGMO_FILTER_NEIGHBOR_SUPPORT) != 0, launches));
    }
    timing_mark(c, 3);
    size_t tb = c->scan_tmp_bytes;
    CUDA_TRY(c, launch_scan((const I64x2 *)c->mol_cnt.p, (I64x2 *)c->off.p, c->ND + 1, c->scan_tmp.p, &tb, c->stream));
    launches += 2;
    ChunkParams cp;
    cp.ND = c->ND;
    cp.goff = c->dd.goff;
    cp.off = (const I64x2 *)c->off.p;
    cp.PC = c->PC;
    cp.AC = c->AC;
    cp.CMC = c->CMC;
    cp.MC = c->MC;
    cp.chunk_start = (int32_t *)c->chunk_start.p;
    cp.nchunks = (int32_t *)c->nchunks.p;
    CUDA_TRY(c, launch_chunks(cp, c->stream));
    launches++;
    PairsParams pp{};
    pp.ND = c->ND;
    pp.NQ = c->NQ;
    pp.VQ = c->VQ;
    pp.NQW = c->NQW;
    pp.MQ = std::max(c->maxq, 2);
    pp.Wpad = c->Wpad;
    pp.gm = (const uint32_t *)c->gm.p;
    pp.off = (const I64x2 *)c->off.p;
    pp.goff = c->dd.goff;
    pp.adj_off = c->adj_off;
    pp.cand_units = c->cand_units;
    pp.qgoff = c->dq.goff;
    pp.qp_row = c->qp_row;
    pp.bitmap = (const uint32_t *)c->bitmap.p;
    pp.pair_query = (int32_t *)c->pair_query.p;
    pp.prec = mol ? (int4 *)c->pair_rec.p : nullptr;
    pp.rowstride = m.NDR;
    pp.qinfo = c->qp_qinfo;
    CUDA_TRY(c, launch_pairs(pp, c->stream));
    launches++;
    if (lane_ns) {
      // neighbour support on the pre-support pair list: refined windows per
      // pair + alive flags, then the GMCR bits, counts and records again
      const size_t gmb = 4 * (size_t)c->ND * c->NQW, offb = sizeof(I64x2) * ((size_t)c->ND + 1);
      SIGMO_TRY(dreserve(c, c->gm_old, gmb, "pre-support gmcr bits"));
      SIGMO_TRY(dreserve(c, c->off_old, offb, "pre-support offsets"));
      CUDA_TRY(c, cudaMemcpyAsync(c->gm_old.p, c->gm.p, gmb, cudaMemcpyDeviceToDevice, c->stream));
      CUDA_TRY(c, cudaMemcpyAsync(c->off_old.p, c->off.p, offb, cudaMemcpyDeviceToDevice, c->stream));
      I64x2 pt{};
      CUDA_TRY(c, cudaMemcpyAsync(&pt, (const I64x2 *)c->off.p + c->ND, sizeof(I64x2), cudaMemcpyDeviceToHost, c->stream));
      CUDA_TRY(c, cudaStreamSynchronize(c->stream));
      const int MQ = std::max(c->maxq, 1);
      SIGMO_TRY(dreserve(c, c->ns_win32, 4 * (size_t)std::max<long long>(pt.a, 1) * MQ, "support windows"));
      SIGMO_TRY(dreserve(c, c->ns_win64, 8 * (size_t)std::max<long long>(pt.b, 1) * MQ, "support windows (wide)"));
      SIGMO_TRY(dreserve(c, c->ns_alive, (size_t)(pt.a + pt.b + 1), "support flags"));
      SupportLaneParams sl{};
      sl.Pn = pt.a;
      sl.Pw = pt.b;
      sl.prec = (const int4 *)c->pair_rec.p;
      sl.cmol = (const uint32_t *)c->bitmap.p;
      sl.adjw = (const uint32_t *)c->adjb.p;
      sl.qp_ent2 = (const uint2 *)c->ent2.p;
      sl.qp_be = c->qp_be;
      sl.qp_nbr = c->qp_nbr;
      sl.MQ = MQ;
      sl.win32 = (uint32_t *)c->ns_win32.p;
      sl.win64 = (unsigned long long *)c->ns_win64.p;
      sl.alive = (uint8_t *)c->ns_alive.p;
      CUDA_TRY(c, launch_support_lane(sl, c->stream));
      CUDA_TRY(c, launch_gmcr_update(c->ND, c->NQW, (const uint32_t *)c->gm_old.p, (const I64x2 *)c->off_old.p,
                                     c->dd.goff, (const uint8_t *)c->ns_alive.p, (uint32_t *)c->gm.p,
                                     (I64x2 *)c->mol_cnt.p, c->stream));
      size_t tb2 = c->scan_tmp_bytes;
      CUDA_TRY(c, launch_scan((const I64x2 *)c->mol_cnt.p, (I64x2 *)c->off.p, c->ND + 1, c->scan_tmp.p, &tb2, c->stream));
      pp.gm_old = (const uint32_t *)c->gm_old.p;
      pp.off_old = (const I64x2 *)c->off_old.p;
      pp.ns_mq = MQ;
      CUDA_TRY(c, launch_pairs(pp, c->stream));
      launches += 4;
      c->lane_ns = true;
    }
    timing_mark(c, 4);
  }
  c->last.filter_launches = launches;
  c->enum_P = -1;
  c->levels = levels;
  c->flags = flags;
  c->state = 2;
  return SIGMO_OK;
}

namespace {
// enumerate-mode outputs of the lane join; all null: counting
struct EnumOut {
  unsigned char *emaps = nullptr;
  int estride = 8;
  unsigned long long *esets = nullptr, *ecur = nullptr;
};
sigmo_status join_impl(sigmo_ctx *c, sigmo_mode mode, uint64_t *total_matches_out, const EnumOut &eo);
}  // namespace

sigmo_status sigmo_join(sigmo_ctx *c, sigmo_mode mode, uint64_t *total_matches_out) {
  if (!c) return SIGMO_ERR_INVALID_ARG;
  if (c->state < 2) return set_err(c, SIGMO_ERR_STATE, "sigmo_join before sigmo_filter");
  if (mode != SIGMO_FIND_ALL && mode != SIGMO_FIND_FIRST) return set_err(c, SIGMO_ERR_INVALID_ARG, "bad mode %d", (int)mode);
  return join_impl(c, mode, total_matches_out, EnumOut());
}

namespace {
sigmo_status join_impl(sigmo_ctx *c, sigmo_mode mode, uint64_t *total_matches_out, const EnumOut &eo) {
  CUDA_TRY(c, cudaSetDevice(c->device));
  CUDA_TRY(c, cudaMemsetAsync(c->jcnt.p, 0, 8 * ((size_t)c->NQ + 8), c->stream));
  int launches = 0;
  if (c->ND > 0 && c->VD > 0 && c->NQ > 0) {
    JoinParams jp{};
    jp.ND = c->ND;
    jp.NQ = c->NQ;
    jp.NQW = c->NQW;
    jp.VQ = c->VQ;
    jp.Wpad = c->Wpad;
    jp.NB = c->NB;
    jp.goff = c->dd.goff;
    jp.roff = c->dd.roff;
    jp.nbr = c->dd.nbr;
    jp.bclass = c->bclass;
    jp.bitmap = (const uint32_t *)c->bitmap.p;
    jp.gm = (const uint32_t *)c->gm.p;
    jp.off = (const I64x2 *)c->off.p;
    jp.chunk_start = (const int32_t *)c->chunk_start.p;
    jp.nchunks = (const int32_t *)c->nchunks.p;
    jp.chunk_counter = (int *)c->jcnt.p;
    jp.qgoff = c->dq.goff;
    jp.qp_row = c->qp_row;
    jp.qp_beoff = c->qp_beoff;
    jp.qp_be = c->qp_be;
    jp.qp_info = c->qp_info;
    jp.pair_query = (int32_t *)c->pair_query.p;
    jp.pair_result = (unsigned long long *)c->pair_result.p;
    jp.totals = (unsigned long long *)c->jcnt.p + 6;
    jp.error = (int *)((unsigned long long *)c->jcnt.p + 1);
    jp.stats = (unsigned long long *)c->jcnt.p + 2;
    fill_join_caps(c, jp);
    if (c->mol_filter) {
      // one GMCR pair per lane (k_join_lane) over the molecule-padded candidates
      jp.maxq = std::max(c->maxq, 2);
      jp.VD = c->VD;
      jp.prec = (const int4 *)c->pair_rec.p;
      jp.adjw = (const uint32_t *)c->adjb.p;
      jp.adj_ones = c->adj_words;
      jp.adj_limit = (unsigned long long)c->adj_words + 4;
      jp.cmol_limit = c->bm_bytes / 4;
      jp.qp_ent = c->qp_ent;
      jp.qp_ent2 = (const uint2 *)(c->lane_ns ? c->ent_ns.p : c->ent2.p);
      jp.cmol = (const uint32_t *)c->bitmap.p;
      // refill batch (lanes that must be free before a warp refills): swept on
      // configs[2] (r2 kernel with registers-only pair hand-out), FA 4/6/8/10/12
      // -> 5.91/5.58/5.42/5.35/5.34 ms join
      jp.batchK = 12;
      jp.emaps = eo.emaps;
      jp.estride = eo.estride;
      jp.esets = eo.esets;
      jp.ecur = eo.ecur;
      jp.qp_qn = c->qp_qn;
      if (const char *e = getenv("SIGMO_JOIN_BATCH")) jp.batchK = std::max(1, std::min(32, atoi(e)));
      jp.plan_smem_max = kJoinLanePlanSmemMax;
      jp.lean = (!c->lane_extras && !c->count_steps) ? 1 : 0;
      if (const char *e = getenv("SIGMO_JOIN_PLAN_SMEM")) jp.plan_smem_max = atoi(e);  // test knob: 0 = plan through L1
      // preferred shared-memory carveout: the driver default for Find All; 75 % for Find First (configs[2]
      // sweep, r2: FA default/75/50 -> 5.04/5.06/5.12 ms, FF 3.75/3.61/3.83 ms; less shares the L1 that
      // caches the adjacency and windows)
      jp.carveout = mode == SIGMO_FIND_FIRST ? 75 : -1;
      if (const char *e = getenv("SIGMO_JOIN_CARVEOUT")) jp.carveout = atoi(e);  // test knob (percent)
      // two launches: pairs of <= 32-node molecules with 32-bit masks, and
      // the others with 64-bit masks (each finds its range in off[ND]); the
      // wide one on the auxiliary stream, so its CTAs fill the SMs the narrow
      // launch frees at its tail
      timing_join(c, 0);
      const bool two = c->maxn > 32;
      if (two) {
        CUDA_TRY(c, cudaEventRecord(c->fork_ev, c->stream));
        CUDA_TRY(c, cudaStreamWaitEvent(c->aux, c->fork_ev, 0));
      }
      for (int w = 0; w < 2; w++) {
        const bool w64 = w == 1;
        if (w64 && !two) break;
        jp.lane_threads = jl_threads(w64);
        if (const char *e = getenv(w64 ? "SIGMO_JOIN_WARPS_WIDE" : "SIGMO_JOIN_WARPS"))  // test knob: warps per CTA
          jp.lane_threads = 32 * std::max(1, std::min(jl_threads(w64) / 32, atoi(e)));
        const size_t smem = join_lane_smem_bytes(jp, w64);
        if (smem > c->max_smem)
          return set_err(c, SIGMO_ERR_LIMIT, "join shared memory %zu exceeds %zu", smem, c->max_smem);
        jp.smem_bytes = smem;
        jp.chunk_counter = (int *)((unsigned long long *)c->jcnt.p + (w64 ? 6 + (size_t)c->NQ : 0));
        // neighbour-support mode: the refined windows of each pair (plan-depth order)
        if (c->lane_ns) {
          jp.cmol = (const uint32_t *)(w64 ? c->ns_win64.p : c->ns_win32.p);
          jp.cmol_limit = (w64 ? c->ns_win64.cap : c->ns_win32.cap) / 4;
        }
        int bps = join_lane_blocks_per_sm((int)mode, w64, jp, smem);
        if (const char *e = getenv("SIGMO_JOIN_BPS")) bps = std::max(1, std::min(bps, atoi(e)));
        if (const char *e = getenv(w64 ? "SIGMO_JOIN_BPS_FORCE_WIDE" : "SIGMO_JOIN_BPS_FORCE"))  // experiment knob
          bps = std::max(1, std::min(32, atoi(e)));
        const int grid = bps * c->sm_count;
        if (getenv("SIGMO_DEBUG_JOIN"))
          fprintf(stderr, "sigmo join: lane %s mode %d threads %d smem %zu blocks/SM %d grid %d\n", w64 ? "wide" : "narrow",
                  (int)mode, jp.lane_threads, smem, bps, grid);
        CUDA_TRY(c, launch_join_lane((int)mode, w64, jp, grid, w64 ? c->aux : c->stream));
        launches++;
      }
      if (two) {
        CUDA_TRY(c, cudaEventRecord(c->join_ev, c->aux));
        CUDA_TRY(c, cudaStreamWaitEvent(c->stream, c->join_ev, 0));
      }
      // S7: per-query totals from the pair results
      CUDA_TRY(c, launch_lane_totals(c->ND, c->NQ, c->NQW, (const uint32_t *)c->gm.p, (const I64x2 *)c->off.p,
                                     jp.pair_result, jp.totals, c->sm_count, c->stream));
      launches++;
      timing_join(c, 1);
    } else {
      const size_t smem = join_smem_bytes(c->NW, jp);
      if (smem > c->max_smem) return set_err(c, SIGMO_ERR_LIMIT, "join shared memory %zu exceeds %zu", smem, c->max_smem);
      jp.smem_bytes = smem;
      const int bps = join_blocks_per_sm(c->NW, (int)mode, jp, smem);
      const int grid = bps * c->sm_count;
      SIGMO_TRY(dreserve(c, c->gstack, join_gstack_bytes(c->NW, jp, grid), "join stack"));
      jp.gstack = (unsigned char *)c->gstack.p;
      timing_join(c, 0);
      CUDA_TRY(c, launch_join(c->NW, (int)mode, jp, grid, c->stream));
      launches++;
      timing_join(c, 1);
    }
  }
  c->last.join_launches = launches;
  c->last_mode = (int)mode;
  c->state = 3;
  if (total_matches_out) {
    SIGMO_TRY(read_join_flags(c));
    std::vector<uint64_t> t((size_t)c->NQ + 1);
    if (c->NQ > 0)
      CUDA_TRY(c, cudaMemcpyAsync(t.data(), (uint64_t *)c->jcnt.p + 6, 8 * (size_t)c->NQ, cudaMemcpyDeviceToHost,
                                  c->stream));
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    uint64_t s = 0;
    for (int q = 0; q < c->NQ; q++) s += t[q];
    *total_matches_out = s;
  }
  return SIGMO_OK;
}
}  // namespace

sigmo_status sigmo_enumerate(sigmo_ctx *c, uint32_t flags, int64_t *num_embeddings) {
  if (!c) return SIGMO_ERR_INVALID_ARG;
  if (c->state < 2) return set_err(c, SIGMO_ERR_STATE, "sigmo_enumerate before sigmo_filter");
  if (flags & ~(uint32_t)SIGMO_ENUM_NODE_SETS) return set_err(c, SIGMO_ERR_INVALID_ARG, "unknown flags 0x%x", flags);
  if (c->ND > 0 && c->VD > 0 && c->NQ > 0 && !c->mol_filter)
    return set_err(c, SIGMO_ERR_LIMIT,
                   "embedding enumeration runs on the lane path: data graphs <= 64 atoms, queries <= %d nodes",
                   kJoinLaneMaxQ);
  CUDA_TRY(c, cudaSetDevice(c->device));
  // count pass (Find All) -> per-pair counts -> scan -> first slot per pair
  SIGMO_TRY(join_impl(c, SIGMO_FIND_ALL, nullptr, EnumOut()));
  SIGMO_TRY(read_join_flags(c));
  int64_t P = 0;
  SIGMO_TRY(sigmo_num_pairs(c, &P));
  SIGMO_TRY(dreserve(c, c->eoff, 8 * ((size_t)P + 1), "embedding offsets"));
  CUDA_TRY(c, cudaMemsetAsync(c->eoff.p, 0, 8, c->stream));
  unsigned long long total = 0;
  if (P > 0) {
    size_t tb = 0;
    CUDA_TRY(c, launch_u64_inclusive_sum(nullptr, nullptr, P, nullptr, &tb, c->stream));
    SIGMO_TRY(dreserve(c, c->etmp, tb, "scan temp"));
    CUDA_TRY(c, launch_u64_inclusive_sum((const unsigned long long *)c->pair_result.p,
                                         (unsigned long long *)c->eoff.p + 1, P, c->etmp.p, &tb, c->stream));
    CUDA_TRY(c, cudaMemcpyAsync(&total, (unsigned long long *)c->eoff.p + P, 8, cudaMemcpyDeviceToHost, c->stream));
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  }
  const int stride = c->maxq <= 8 ? 8 : 16;
  const bool sets = (flags & SIGMO_ENUM_NODE_SETS) != 0;
  if (total > 0) {
    SIGMO_TRY(dreserve(c, c->emaps, (size_t)stride * total, "embeddings"));
    SIGMO_TRY(dreserve(c, c->ecur, 8 * (size_t)P, "embedding cursors"));
    if (sets) SIGMO_TRY(dreserve(c, c->esets, 8 * (size_t)total, "embedding node sets"));
    CUDA_TRY(c, cudaMemcpyAsync(c->ecur.p, c->eoff.p, 8 * (size_t)P, cudaMemcpyDeviceToDevice, c->stream));
    // write pass
    EnumOut eo;
    eo.emaps = (unsigned char *)c->emaps.p;
    eo.estride = stride;
    eo.esets = sets ? (unsigned long long *)c->esets.p : nullptr;
    eo.ecur = (unsigned long long *)c->ecur.p;
    SIGMO_TRY(join_impl(c, SIGMO_FIND_ALL, nullptr, eo));
    SIGMO_TRY(read_join_flags(c));
  }
  c->enum_uniq = -1;
  if (sets && P > 0) {
    // distinct node sets per pair (NLSM's X)
    SIGMO_TRY(dreserve(c, c->ucnt, 8 * (size_t)P, "node-set counts"));
    SIGMO_TRY(dreserve(c, c->uoff, 8 * ((size_t)P + 1), "node-set offsets"));
    CUDA_TRY(c, launch_nodesets((const unsigned long long *)c->eoff.p, P, (unsigned long long *)c->esets.p,
                                (unsigned long long *)c->ucnt.p, nullptr, nullptr, c->stream));
    size_t tb = 0;
    CUDA_TRY(c, launch_u64_inclusive_sum(nullptr, nullptr, P, nullptr, &tb, c->stream));
    SIGMO_TRY(dreserve(c, c->etmp, tb, "scan temp"));
    CUDA_TRY(c, cudaMemsetAsync(c->uoff.p, 0, 8, c->stream));
    CUDA_TRY(c, launch_u64_inclusive_sum((const unsigned long long *)c->ucnt.p, (unsigned long long *)c->uoff.p + 1,
                                         P, c->etmp.p, &tb, c->stream));
    unsigned long long nu = 0;
    CUDA_TRY(c, cudaMemcpyAsync(&nu, (unsigned long long *)c->uoff.p + P, 8, cudaMemcpyDeviceToHost, c->stream));
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    SIGMO_TRY(dreserve(c, c->uniq, 8 * (size_t)std::max<unsigned long long>(nu, 1), "distinct node sets"));
    CUDA_TRY(c, launch_nodesets((const unsigned long long *)c->eoff.p, P, (unsigned long long *)c->esets.p, nullptr,
                                (const unsigned long long *)c->uoff.p, (unsigned long long *)c->uniq.p, c->stream));
    c->enum_uniq = (int64_t)nu;
  } else if (sets) {
    c->enum_uniq = 0;
  }
  CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  c->enum_P = P;
  c->enum_total = (int64_t)total;
  c->enum_stride = stride;
  if (num_embeddings) *num_embeddings = (int64_t)total;
  return SIGMO_OK;
}

namespace {
// pairs of the lane path in getter order (graph, then query): the internal
// position of each, as in sigmo_get_pair_results
sigmo_status lane_pair_order(sigmo_ctx *c, int64_t P, std::vector<int64_t> &pos, std::vector<int64_t> &gidx,
                             std::vector<int32_t> &qidx) {
  std::vector<I64x2> off((size_t)c->ND + 1);
  CUDA_TRY(c, cudaMemcpyAsync(off.data(), c->off.p, sizeof(I64x2) * off.size(), cudaMemcpyDeviceToHost, c->stream));
  std::vector<int32_t> q((size_t)P + 1);
  if (P)
    CUDA_TRY(c, cudaMemcpy2DAsync(q.data(), 4, (const char *)c->pair_rec.p + 4, 16, 4, (size_t)P, cudaMemcpyDeviceToHost,
                                  c->stream));
  CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  pos.clear();
  gidx.clear();
  qidx.clear();
  const long long Pn = off[c->ND].a;
  for (int g = 0; g < c->ND; g++) {
    long long s0, s1;
    if (off[g + 1].a > off[g].a) {
      s0 = off[g].a;
      s1 = off[g + 1].a;
    } else {
      s0 = Pn + off[g].b;
      s1 = Pn + off[g + 1].b;
    }
    for (long long p = s0; p < s1; p++) {
      pos.push_back(p);
      gidx.push_back(g);
      qidx.push_back(q[(size_t)p]);
    }
  }
  return SIGMO_OK;
}

// copy per-pair segments [seg[p], seg[p+1]) of a device array of `esize`-byte
// elements to the host in getter order
sigmo_status copy_segments(sigmo_ctx *c, const DBuf &segs, const DBuf &data, size_t esize, int64_t P,
                           const std::vector<int64_t> &pos, int64_t cap, int64_t *offsets, void *out,
                           int64_t *n_out) {
  std::vector<unsigned long long> seg((size_t)P + 1, 0);
  if (P) CUDA_TRY(c, cudaMemcpyAsync(seg.data(), segs.p, 8 * ((size_t)P + 1), cudaMemcpyDeviceToHost, c->stream));
  CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  const int64_t total = P ? (int64_t)seg[(size_t)P] : 0;
  if (n_out) *n_out = total;
  if (!out) return SIGMO_OK;
  if (cap < total) return set_err(c, SIGMO_ERR_INVALID_ARG, "capacity %lld < %lld", (long long)cap, (long long)total);
  std::vector<unsigned char> h(esize * (size_t)total + 1);
  if (total) CUDA_TRY(c, cudaMemcpyAsync(h.data(), data.p, esize * (size_t)total, cudaMemcpyDeviceToHost, c->stream));
  CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  int64_t o = 0;
  for (size_t k = 0; k < pos.size(); k++) {
    const unsigned long long a = seg[(size_t)pos[k]], b = seg[(size_t)pos[k] + 1];
    if (offsets) offsets[k] = o;
    memcpy((unsigned char *)out + esize * (size_t)o, h.data() + esize * a, esize * (size_t)(b - a));
    o += (int64_t)(b - a);
  }
  if (offsets) offsets[pos.size()] = o;
  return SIGMO_OK;
}
}  // namespace

sigmo_status sigmo_get_embeddings(sigmo_ctx *c, int64_t pair_cap, int64_t *num_pairs, int64_t *data_idx,
                                  int32_t *query_idx, int64_t *emb_offsets, int64_t emb_cap, uint8_t *maps,
                                  int64_t *num_embeddings, int32_t *stride) {
  if (!c) return SIGMO_ERR_INVALID_ARG;
  if (c->enum_P < 0 || c->state < 3) return set_err(c, SIGMO_ERR_STATE, "sigmo_get_embeddings before sigmo_enumerate");
  CUDA_TRY(c, cudaSetDevice(c->device));
  const int64_t P = c->enum_P;
  if (num_pairs) *num_pairs = P;
  if (stride) *stride = c->enum_stride;
  if (num_embeddings) *num_embeddings = c->enum_total;
  if (!data_idx && !query_idx && !emb_offsets && !maps) return SIGMO_OK;
  if (pair_cap < P) return set_err(c, SIGMO_ERR_INVALID_ARG, "pair capacity %lld < %lld", (long long)pair_cap, (long long)P);
  std::vector<int64_t> pos, gi;
  std::vector<int32_t> qi;
  SIGMO_TRY(lane_pair_order(c, P, pos, gi, qi));
  for (size_t k = 0; k < pos.size(); k++) {
    if (data_idx) data_idx[k] = gi[k];
    if (query_idx) query_idx[k] = qi[k];
  }
  return copy_segments(c, c->eoff, c->emaps, (size_t)c->enum_stride, P, pos, emb_cap, emb_offsets, maps, nullptr);
}

sigmo_status sigmo_get_node_sets(sigmo_ctx *c, int64_t pair_cap, int64_t *num_pairs, int64_t *set_offsets,
                                 int64_t set_cap, uint64_t *sets, int64_t *num_sets) {
  if (!c) return SIGMO_ERR_INVALID_ARG;
  if (c->enum_P < 0 || c->state < 3 || c->enum_uniq < 0)
    return set_err(c, SIGMO_ERR_STATE, "sigmo_get_node_sets before sigmo_enumerate(SIGMO_ENUM_NODE_SETS)");
  CUDA_TRY(c, cudaSetDevice(c->device));
  const int64_t P = c->enum_P;
  if (num_pairs) *num_pairs = P;
  if (num_sets) *num_sets = c->enum_uniq;
  if (!set_offsets && !sets) return SIGMO_OK;
  if (pair_cap < P) return set_err(c, SIGMO_ERR_INVALID_ARG, "pair capacity %lld < %lld", (long long)pair_cap, (long long)P);
  std::vector<int64_t> pos, gi;
  std::vector<int32_t> qi;
  SIGMO_TRY(lane_pair_order(c, P, pos, gi, qi));
  return copy_segments(c, c->uoff, c->uniq, 8, P, pos, set_cap, set_offsets, sets, nullptr);
}

sigmo_status sigmo_num_pairs(sigmo_ctx *c, int64_t *n) {
  if (!c || !n) return SIGMO_ERR_INVALID_ARG;
  if (c->state < 2) return set_err(c, SIGMO_ERR_STATE, "sigmo_num_pairs before sigmo_filter");
  if (c->ND == 0 || c->VD == 0) {
    *n = 0;
    return SIGMO_OK;
  }
  I64x2 t;
  CUDA_TRY(c, cudaMemcpyAsync(&t, (I64x2 *)c->off.p + c->ND, sizeof(I64x2), cudaMemcpyDeviceToHost, c->stream));
  CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  *n = t.a + t.b;  // .b: pairs of > 32-node molecules on the lane-join path (else 0)
  return SIGMO_OK;
}

sigmo_status sigmo_get_pair_results(sigmo_ctx *c, int64_t cap, int64_t *n, int64_t *data_idx, int32_t *query_idx,
                                    uint64_t *result) {
  if (!c || !n) return SIGMO_ERR_INVALID_ARG;
  if (c->state < 3) return set_err(c, SIGMO_ERR_STATE, "sigmo_get_pair_results before sigmo_join");
  SIGMO_TRY(read_join_flags(c));
  int64_t P = 0;
  SIGMO_TRY(sigmo_num_pairs(c, &P));
  *n = P;
  if (cap < P) return set_err(c, SIGMO_ERR_INVALID_ARG, "capacity %lld < %lld pairs", (long long)cap, (long long)P);
  if (P == 0) return SIGMO_OK;
  std::vector<I64x2> off((size_t)c->ND + 1);
  CUDA_TRY(c, cudaMemcpyAsync(off.data(), c->off.p, sizeof(I64x2) * off.size(), cudaMemcpyDeviceToHost, c->stream));
  if (!c->mol_filter) {
    if (query_idx)
      CUDA_TRY(c, cudaMemcpyAsync(query_idx, c->pair_query.p, 4 * (size_t)P, cudaMemcpyDeviceToHost, c->stream));
    if (result)
      CUDA_TRY(c, cudaMemcpyAsync(result, c->pair_result.p, 8 * (size_t)P, cudaMemcpyDeviceToHost, c->stream));
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    if (data_idx)
      for (int g = 0; g < c->ND; g++)
        for (long long p = off[g].a; p < off[g + 1].a; p++) data_idx[p] = g;
    return SIGMO_OK;
  }
  // lane-join path: records of <= 32-node molecules first, then the others;
  // the query is field .y of the int4 records.  Merge back to graph order.
  std::vector<int32_t> q((size_t)P);
  std::vector<uint64_t> r((size_t)P);
  CUDA_TRY(c, cudaMemcpy2DAsync(q.data(), 4, (const char *)c->pair_rec.p + 4, 16, 4, (size_t)P, cudaMemcpyDeviceToHost,
                                c->stream));
  CUDA_TRY(c, cudaMemcpyAsync(r.data(), c->pair_result.p, 8 * (size_t)P, cudaMemcpyDeviceToHost, c->stream));
  CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  const long long Pn = off[c->ND].a;
  long long o = 0;
  for (int g = 0; g < c->ND; g++) {
    long long s0, s1;
    if (off[g + 1].a > off[g].a) {
      s0 = off[g].a;
      s1 = off[g + 1].a;
    } else {
      s0 = Pn + off[g].b;
      s1 = Pn + off[g + 1].b;
    }
    for (long long p = s0; p < s1; p++, o++) {
      if (data_idx) data_idx[o] = g;
      if (query_idx) query_idx[o] = q[(size_t)p];
      if (result) result[o] = r[(size_t)p];
    }
  }
  return SIGMO_OK;
}

sigmo_status sigmo_get_dense_results(sigmo_ctx *c, uint64_t *out) {
  if (!c || !out) return SIGMO_ERR_INVALID_ARG;
  if (c->state < 3) return set_err(c, SIGMO_ERR_STATE, "sigmo_get_dense_results before sigmo_join");
  int64_t P = 0;
  SIGMO_TRY(sigmo_num_pairs(c, &P));
  std::vector<int64_t> di((size_t)P);
  std::vector<int32_t> qi((size_t)P);
  std::vector<uint64_t> r((size_t)P);
  int64_t n = 0;
  SIGMO_TRY(sigmo_get_pair_results(c, P, &n, di.data(), qi.data(), r.data()));
  memset(out, 0, 8 * (size_t)c->NQ * c->ND);
  for (int64_t p = 0; p < n; p++) out[(size_t)qi[p] * c->ND + di[p]] = r[p];
  return SIGMO_OK;
}

sigmo_status sigmo_get_query_totals(sigmo_ctx *c, uint64_t *out, int device_ptr) {
  if (!c || !out) return SIGMO_ERR_INVALID_ARG;
  if (c->state < 3) return set_err(c, SIGMO_ERR_STATE, "sigmo_get_query_totals before sigmo_join");
  if (c->NQ == 0) return SIGMO_OK;
  if (!device_ptr) SIGMO_TRY(read_join_flags(c));
  if (device_ptr) {
    CUDA_TRY(c, cudaMemcpyAsync(out, (uint64_t *)c->jcnt.p + 6, 8 * (size_t)c->NQ, cudaMemcpyDeviceToDevice, c->stream));
  } else {
    CUDA_TRY(c, cudaMemcpyAsync(out, (uint64_t *)c->jcnt.p + 6, 8 * (size_t)c->NQ, cudaMemcpyDeviceToHost, c->stream));
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  }
  return SIGMO_OK;
}

sigmo_status sigmo_get_candidates(sigmo_ctx *c, uint32_t *out) {
  if (!c || !out) return SIGMO_ERR_INVALID_ARG;
  if (c->state < 2) return set_err(c, SIGMO_ERR_STATE, "sigmo_get_candidates before sigmo_filter");
  if (c->VQ == 0 || c->W == 0) return SIGMO_OK;
  const void *src = c->bitmap.p;
  if (c->lane_ns) {
    // the neighbour-support fixed point over the whole bitmap (pairs the GMCR
    // pruned included), by the dense-tile filter + k_support into scratch
    const size_t bytes = 4 * (size_t)c->VQ * c->Wpad + 64;
    SIGMO_TRY(dreserve(c, c->ns_bitmap, bytes, "candidate view (support)"));
    SIGMO_TRY(dreserve(c, c->ns_gm, 4 * (size_t)c->ND * std::max(c->NQW, 1), "scratch gmcr bits"));
    SIGMO_TRY(dreserve(c, c->ns_cnt, sizeof(I64x2) * ((size_t)c->ND + 1), "scratch gmcr counts"));
    CUDA_TRY(c, cudaMemsetAsync(c->ns_bitmap.p, 0, bytes, c->stream));
    int nl = 0;
    SIGMO_TRY(launch_dense(c, c->levels - 1, c->progs[c->levels - 1].prog, (uint32_t *)c->ns_bitmap.p,
                           (uint32_t *)c->ns_gm.p, (I64x2 *)c->ns_cnt.p, true, nl));
    src = c->ns_bitmap.p;
  } else if (c->mol_filter) {  // dense view of the molecule-padded layout
    const size_t bytes = 4 * (size_t)c->VQ * c->Wpad;
    SIGMO_TRY(dreserve(c, c->dense_tmp, bytes, "dense candidate view"));
    CUDA_TRY(c, cudaMemsetAsync(c->dense_tmp.p, 0, bytes, c->stream));
    const QueryProg &pg = c->progs[c->levels - 1].prog;  // the program of the last filter
    CUDA_TRY(c, launch_unpad((const uint32_t *)c->bitmap.p, c->cand_units, pg.qdrow, pg.meta.NDR, c->dd.goff, c->ND,
                             c->VQ, c->Wpad, (uint32_t *)c->dense_tmp.p, c->stream));
    src = c->dense_tmp.p;
  }
  CUDA_TRY(c, cudaMemcpy2DAsync(out, 4 * (size_t)c->W, src, 4 * (size_t)c->Wpad, 4 * (size_t)c->W,
                                (size_t)c->VQ, cudaMemcpyDeviceToHost, c->stream));
  CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  return SIGMO_OK;
}

sigmo_status sigmo_get_packed_batch(sigmo_ctx *c, int which, int64_t *num_graphs, int64_t *num_nodes, int64_t *num_adj,
                                    int64_t *graph_offsets, int64_t *row_offsets, int32_t *col_indices,
                                    uint8_t *node_labels, uint8_t *edge_labels) {
  if (!c || (which != 0 && which != 1)) return SIGMO_ERR_INVALID_ARG;
  if (c->state < 1) return set_err(c, SIGMO_ERR_STATE, "sigmo_get_packed_batch before sigmo_load_batch");
  const DevGraphs &d = which ? c->dd : c->dq;
  if (num_graphs) *num_graphs = d.num_graphs;
  if (num_nodes) *num_nodes = d.num_nodes;
  if (num_adj) *num_adj = d.num_adj;
  if (!graph_offsets && !row_offsets && !col_indices && !node_labels && !edge_labels) return SIGMO_OK;
  if (!graph_offsets || !row_offsets || !col_indices || !node_labels || !edge_labels)
    return set_err(c, SIGMO_ERR_INVALID_ARG, "sigmo_get_packed_batch: NULL output array");
  CUDA_TRY(c, cudaSetDevice(c->device));
  std::vector<int32_t> goff((size_t)d.num_graphs + 1), roff((size_t)d.num_nodes + 1);
  std::vector<uint16_t> nbr((size_t)d.num_adj + 1);
  std::vector<uint8_t> lab((size_t)d.num_nodes + 1);
  CUDA_TRY(c, cudaMemcpyAsync(goff.data(), d.goff, 4 * goff.size(), cudaMemcpyDeviceToHost, c->stream));
  CUDA_TRY(c, cudaMemcpyAsync(roff.data(), d.roff, 4 * roff.size(), cudaMemcpyDeviceToHost, c->stream));
  if (d.num_adj) CUDA_TRY(c, cudaMemcpyAsync(nbr.data(), d.nbr, 2 * (size_t)d.num_adj, cudaMemcpyDeviceToHost, c->stream));
  if (d.num_nodes) CUDA_TRY(c, cudaMemcpyAsync(lab.data(), d.label, (size_t)d.num_nodes, cudaMemcpyDeviceToHost, c->stream));
  CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  for (int g = 0; g <= d.num_graphs; g++) graph_offsets[g] = goff[g];
  for (int v = 0; v <= d.num_nodes; v++) row_offsets[v] = roff[v];
  for (int v = 0; v < d.num_nodes; v++) node_labels[v] = lab[v];
  // packed neighbour = molecule-local index << 8 | bond label -> global id
  for (int g = 0; g < d.num_graphs; g++)
    for (int v = goff[g]; v < goff[g + 1]; v++)
      for (int e = roff[v]; e < roff[v + 1]; e++) {
        col_indices[e] = goff[g] + (nbr[e] >> 8);
        edge_labels[e] = (uint8_t)(nbr[e] & 0xffu);
      }
  return SIGMO_OK;
}

sigmo_status sigmo_check_join(sigmo_ctx *c) {
  if (!c) return SIGMO_ERR_INVALID_ARG;
  if (c->state < 3) return set_err(c, SIGMO_ERR_STATE, "sigmo_check_join before sigmo_join");
  CUDA_TRY(c, cudaSetDevice(c->device));
  return read_join_flags(c);
}

sigmo_status sigmo_get_signatures(sigmo_ctx *c, int which, int radius, uint64_t *out) {
  if (!c || !out || (which != 0 && which != 1)) return SIGMO_ERR_INVALID_ARG;
  if (radius < 1 || radius > 255) return set_err(c, SIGMO_ERR_INVALID_ARG, "radius %d not in 1..255", radius);
  if (c->state < 1) return set_err(c, SIGMO_ERR_STATE, "sigmo_get_signatures before sigmo_load_batch");
  CUDA_TRY(c, cudaSetDevice(c->device));
  const DevGraphs &g = which == 0 ? c->dq : c->dd;
  if (g.num_nodes == 0) return SIGMO_OK;
  SIGMO_TRY(dreserve(c, c->sig_tmp, 8 * (size_t)g.num_nodes, "signature export"));
  CUDA_TRY(c, launch_sig_pack(g, radius, (unsigned long long *)c->sig_tmp.p, which == 0 ? c->wildcard_loaded : 0,
                              c->stream));
  CUDA_TRY(c, cudaMemcpyAsync(out, c->sig_tmp.p, 8 * (size_t)g.num_nodes, cudaMemcpyDeviceToHost, c->stream));
  CUDA_TRY(c, cudaStreamSynchronize(c->stream));
  return SIGMO_OK;
}

}  // extern "C"
