// sigmo_internal.h -- internal (non-ABI) structures shared by the host side
// (sigmo_abi.cu) and the device side (sigmo_kernels.cu) of libsigmo.so.
// Nothing here is visible to the oracle (oracle/ shares no code with this).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "lane_filter_types.h"

namespace sigmo {

constexpr int kNumFields = 13;   // R7 field table (see sigmo_kernels.cu kFieldWidth)
constexpr int kFilterThreads = 256;
constexpr int kJoinThreads = 128;
constexpr int kQueryPrepThreads = 1024;


// R7 field of an atom label (atomic number): C N O S F Cl Br I P H B Si, other
__host__ __device__ inline int field_of_label(int lab) {
  switch (lab) {
    case 6: return 0;
    case 7: return 1;
    case 8: return 2;
    case 16: return 3;
    case 9: return 4;
    case 17: return 5;
    case 35: return 6;
    case 53: return 7;
    case 15: return 8;
    case 1: return 9;
    case 5: return 10;
    case 14: return 11;
    default: return 12;
  }
}

// Packed CSR-GO batch on the device (produced by sigmo_load_batch).
//   nbr[e] = (molecule-local index of the neighbour << 8) | bond label
struct DevGraphs {
  int num_graphs = 0, num_nodes = 0, num_adj = 0, max_nodes = 0;
  const int32_t *goff = nullptr;   // [G+1]
  const uint8_t *label = nullptr;  // [V]
  const uint8_t *local = nullptr;  // [V] index of the node inside its graph
  const int32_t *roff = nullptr;   // [V+1]
  const uint16_t *nbr = nullptr;   // [E2]
};

// Query-side plane program, built on the device by k_query_prep from the
// query signatures (one per `levels`); see DESIGN.md "Filter".
struct QueryProgMeta {
  int P;       // distinct (radius, field, threshold) planes
  int G;       // distinct (radius, field) count groups
  int NFU;     // fields used by any plane
  int NLAB;    // distinct query labels (label planes)
  int row_entries;
  int err;
  int NREC;    // group records (one per group part per 32-plane batch)
  int NRP;     // packed row-program words (two 16-bit channels each)
  int NBATCH;  // 32-plane batches
  int TS;      // threshold-table entries per record (64, or 256 for > 64-node graphs)
  int RW;      // row-program words per query node (padded)
  int NDR;     // distinct rows (query nodes with the same label and constraint list share one)
  int NQWL;    // (word, bits) entries of the per-query GMCR lists over distinct rows
  // k_filter_lane program (FilterLaneParams)
  int L_NREC;  // plane records (<= 4 planes each)
  int L_RWV;   // uint4 words per distinct row program
  int L_NQWE;  // GMCR list entries x 32
  int L_NQG;   // 32-query groups
};

// One part of a (radius, field) count group inside one 32-plane batch of the
// plane program, used by k_filter: with c = |ball_r(v) \ {v}| restricted to
// field `fslot`, tab[toff + min(c, TS-1)] holds the bits (plane % 32) of the
// batch's planes [c >= t] of this group (a thermometer code).
struct __align__(16) GroupRec {
  int fslot, toff, batch, pad;
};

struct QueryProg {
  QueryProgMeta meta{};
  int R = 0;                   // levels - 1
  // device arrays
  uint8_t *p_t = nullptr;      // [P]   threshold t of plane p
  int16_t *grp_poff = nullptr; // [G+1] plane range of group
  uint8_t *grp_f = nullptr;    // [G]   field of group
  int16_t *rg_off = nullptr;   // [R+1] group range per radius
  int8_t *fslot = nullptr;     // [13]  used-field slot or -1
  uint8_t *lab_val = nullptr;  // [NLAB]
  uint8_t *row_lab = nullptr;  // [VQ]  label-plane index of query node
  int32_t *row_off = nullptr;  // [VQ+1]
  uint16_t *row_ids = nullptr; // plane ids per query node
  // packed form used by k_filter (built on the host from the arrays above).
  // Channels: 0..NLAB-1 label planes, NLAB all ones, NLAB+1+p constraint plane p.
  GroupRec *grec = nullptr;    // [NREC] sorted by (radius, batch)
  int32_t *rrec_off = nullptr; // [R+1] record range per radius
  int32_t *rcarry = nullptr;   // [R] 1 if the radius' first plane continues a batch of the previous radius
  int32_t *bdone = nullptr;    // [NBATCH] radius index (r-1) of the batch's last plane
  uint32_t *tab = nullptr;     // [NREC * TS] thermometer tables
  int32_t *rowp_off = nullptr; // [VQ+1] row-program word range per query node
  uint32_t *rowp = nullptr;    // [NRP] channel byte offsets (lo | hi << 16), label channel first
  uint32_t *drowp = nullptr;   // [NDR * RW] row programs of the distinct rows (molecule tiles)
  uint16_t *qdrow = nullptr;   // [VQ] distinct row of each query node
  int32_t *qw_off = nullptr;   // [NQ+1] per-query range of (word, bits) entries
  uint32_t *qw = nullptr;      // [NQWL][2] word of the distinct-row bit vector, bits of the query's rows in it
  QueryProgMeta *d_meta = nullptr;
  // k_filter_lane program (see FilterLaneParams)
  uint2 *l_grec = nullptr;
  int32_t *l_rrec = nullptr;
  uint4 *l_rowp = nullptr;
  int32_t *l_rgn = nullptr;
  uint2 *l_qwl = nullptr;
  int2 *l_qwh = nullptr;
  uint16_t *l_lut = nullptr;
};

struct FilterParams {
  DevGraphs D;
  int TW, W, Wpad;
  int VQ, NQ, NQW;
  int R;
  int P, NFU, NLAB, NREC, NRP, NBATCH, TS, RW;
  const GroupRec *grec;
  const int32_t *rrec_off;
  const int32_t *rcarry;
  const int32_t *bdone;
  const uint32_t *tab;
  const int8_t *fslot;
  const uint8_t *lab_val;
  const int32_t *rowp_off;
  const uint32_t *rowp;
  const int32_t *qgoff;        // [NQ+1] query node offsets (rows)
  uint32_t *bitmap;            // [VQ][Wpad] (dense tiles)
  uint32_t *cmol;              // molecule-padded windows of the distinct rows (molecule tiles), else null: molecule g
                               // at word NDR * cand_units[g], NDR u32 windows (<= 32 nodes) or u64 (> 32 nodes)
  const uint32_t *cand_units;
  const uint16_t *qdrow;       // [VQ] distinct row of each query node (molecule tiles)
  const int32_t *qw_off;       // [NQ+1] GMCR (word, bits) lists per query (molecule tiles)
  const uint32_t *qw;
  int NDR, NQWL;
  const int32_t *mtile;        // [tiles+1] first graph of each molecule tile (<= 32 graphs, <= 1,024 nodes)
  uint32_t *gm;                // [ND][NQW] surviving-query bits per data graph
  I64x2 *mol_cnt;              // [ND+1] (surviving pairs, candidate-mask entries)
  int EXTN, EXTW, MOLCAP;
  int rows_smem;               // 1 = copy row programs to smem
  const int32_t *tile_g0, *tile_g1;  // per-tile graph range for TW = 32 (null: binary search)
  size_t smem_bytes;
};

struct JoinParams {
  int ND, NQ, NQW, VQ, Wpad, NB;
  const int32_t *goff;
  const int32_t *roff;
  const uint16_t *nbr;
  const uint8_t *bclass;       // [256] bond label -> class (255 = not in any query)
  const uint32_t *bitmap;
  const uint32_t *gm;
  const I64x2 *off;            // [ND+1] exclusive scan of mol_cnt
  const int32_t *chunk_start;  // [nchunks+1]
  const int32_t *nchunks;      // device scalar
  int *chunk_counter;          // device scalar (zeroed before launch)
  const int32_t *qgoff;        // [NQ+1]
  const int32_t *qp_row;       // [VQ] plan order: global query node of depth e
  const int32_t *qp_beoff;     // [VQ+1] back-edge list per (query, depth)
  const uint16_t *qp_be;       // (depth j << 8) | bond class
  const uint32_t *qp_info;     // [VQ] first back-edge j | class << 8 | (#back-edges - 1) << 16 (j = 0xff: none)
  int32_t *pair_query;
  unsigned long long *pair_result;
  unsigned long long *totals;  // [NQ]
  int PCAP, ACAP, CMCAP, MCAP, maxq;
  int NBE, plan_smem;          // back-edge entries; 1 = copy the query plans to smem
  int SCS;                     // per-warp DFS stack entries kept in shared memory
  int slice_rows, SW;          // bitmap slice copy: rows (0 = read windows from global), words per row
  unsigned char *gstack;       // per-warp global DFS stack area (promotion target)
  int *error;                  // device flag, nonzero = internal capacity exceeded
  unsigned long long *stats;   // optional: DFS iterator steps (nullable)
  size_t smem_bytes;
  // per-lane DFS kernel (k_join_lane)
  int VD;                      // data nodes
  const int4 *prec;            // [P] pair records {adjacency word offset, query, cmol word base, qinfo | size << 8}
  const uint32_t *cmol;        // molecule-padded candidate windows (filter output, see FilterParams::cmol)
  const uint32_t *adjw;        // bond-class adjacency masks (molecule-local bits), per molecule at word adj_off[g]:
                               // class-major [NB][n], u32 masks (n <= 32) or u64 (n > 32); all ones at word adj_ones
  unsigned adj_ones;
  unsigned long long adj_limit;   // words of adjw / of the candidate-window array (SIGMO_BOUNDS_CHECK builds)
  unsigned long long cmol_limit;
  const int4 *qp_ent;          // [VQ] per plan position {j0 | j1 << 4 (15 none) | #extra << 8 | node << 12, class0, class1, extra back-edge start}
  const uint2 *qp_ent2;        // [VQ] compact, k_join_lane: x = slot0 * 128 | leaf << 11 | #extra back-edges << 12 |
                               // slot1 * 128 << 16 (slot = back-edge depth, maxq - 1 = none: the map slot
                               // holding the all-ones index); y = class0 | class1 << 3 | distinct row << 12
  int batchK;                  // finish/assign pairs when >= batchK lanes are free
  int induced;                 // 1 = induced-subgraph embeddings (k_join only, R21):
                               // the union of all bonds is staged as adjacency class NB
  const uint32_t *qp_non;      // [VQ] induced mode: mask of the earlier plan depths NOT adjacent to depth e
  int any_bond;                // wildcard query bonds ('~', label 0; R22) map to adjacency class NB (all bonds)
  // enumerate mode (k_join_lane); emaps == nullptr: counting
  unsigned char *emaps;        // [embeddings][estride] molecule-local data node per query node (query node order)
  int estride;                 // 8 (queries <= 8 nodes) or 16 bytes per embedding
  unsigned long long *esets;   // [embeddings] node set f(V_q) as a molecule-local bit mask (nullable)
  unsigned long long *ecur;    // [P] write cursor per pair (= its first embedding slot after the scan)
  const uint8_t *qp_qn;        // [VQ] local query node of each plan position
  int plan_smem_max;           // k_join_lane: plan entries copied to shared memory when VQ <= this
  int carveout;                // k_join_lane: preferred shared-memory carveout in percent (-1: driver default)
  int lane_threads;            // k_join_lane: threads per CTA of this launch (<= jl_threads(w64))
  int lean;                    // k_join_lane: no plan position has > 2 back-edges and DFS steps are not counted
                               // (the lean instantiation: no extra back-edge loop, no step counter)
};

// k_pairs: GMCR pair list + per-pair candidate masks
struct PairsParams {
  int ND, NQ, NQW, MQ, Wpad, VQ;
  int rowstride;               // cmol row stride per graph (distinct rows)
  const uint32_t *adj_off;     // [ND+1] adjacency word offset per graph (pair record .x)
  const uint32_t *cand_units;  // [ND+1] candidate-window units per graph (pair record .z = rowstride * units)
  const uint32_t *gm;
  const I64x2 *off;
  const int32_t *goff, *qgoff, *qp_row;
  const uint32_t *bitmap;
  int32_t *pair_query;
  int4 *prec;                  // null: pair_query only
  const uint32_t *qinfo;       // [NQ] nq | tail start << 8 | first query node << 16
  // neighbour-support mode of the lane path: records of the surviving pairs point
  // (.z) at the refined windows k_support_lane wrote for the pre-support pair list
  const uint32_t *gm_old;      // pre-support GMCR bits (null: normal mode)
  const I64x2 *off_old;        // pre-support pair offsets
  int ns_mq;                   // windows per pair in the refined arrays
};

// k_support_lane: neighbour support (R9) on the lane path, one thread per
// pre-support GMCR pair
struct SupportLaneParams {
  long long Pn, Pw;            // pre-support pairs on <= 32-node / larger molecules
  const int4 *prec;            // pre-support pair records
  const uint32_t *cmol;        // filter windows (distinct rows)
  const uint32_t *adjw;        // bond-class adjacency (as JoinParams::adjw)
  const uint2 *qp_ent2;        // plan entries with distinct rows (JoinParams::qp_ent2)
  const uint16_t *qp_be;       // back-edge lists
  const uint2 *qp_nbr;         // [VQ] query neighbours of each plan position (depth | class << 4 | 0x80, 8 bytes)
  int MQ;                      // max query nodes (window slots per pair)
  uint32_t *win32;             // [Pn][MQ] refined windows (<= 32-node molecules)
  unsigned long long *win64;   // [Pw][MQ] refined windows (larger molecules)
  uint8_t *alive;              // [Pn + Pw] 0 = the fixed point emptied a node of the pair
};

struct SupportParams {
  int ND, NQ, NQW, NB, maxq, Wpad;
  int any_bond;                  // wildcard query bonds map to class NB (all bonds)
  const int32_t *goff, *roff;
  const uint16_t *nbr;
  const uint8_t *bclass;
  const int32_t *qgoff, *qroff;  // query CSR (global query node ids; qnbr local index << 8 | bond)
  const uint16_t *qnbr;
  uint32_t *bitmap;
  uint32_t *gm;
  I64x2 *mol_cnt;
};

struct ChunkParams {
  int ND;
  const int32_t *goff;
  const I64x2 *off;
  long long PC, AC, CMC, MC;
  int32_t *chunk_start;
  int32_t *nchunks;
};


// k_load_data (sigmo_load.cu): device-side validation + packing of a large data batch
struct DataLoadParams {
  long long G;
  const int64_t *goff, *roff;  // raw CSR-GO (caller's layout, on the device)
  const int32_t *col;
  const uint8_t *nlab, *elab;
  int32_t *goff32, *roff32;    // packed (DevGraphs)
  uint8_t *label, *local;
  uint16_t *nbr;
  unsigned long long *hist;    // [256] node label histogram (query planner)
  long long *err_graph;        // [5] first offending graph per error class (LLONG_MAX-ish = none):
                               //     row offsets decreasing, column outside graph, self-loop, duplicate, asymmetric
};
constexpr long long kDeviceLoadMinNodes = 65536;  // smaller data batches are validated and packed on the host
cudaError_t launch_load_data(const DataLoadParams &p, cudaStream_t st);
// per-molecule adjacency / candidate layout of a device-loaded batch (sigmo_load.cu)
size_t layout_scan_bytes(int G);
cudaError_t launch_layout(const int32_t *goff, int G, int NB, void *scratch, uint32_t *aoff, uint32_t *cu,
                          int32_t *grpn, int32_t *grpw, uint4 *mrec, long long *info_out, cudaStream_t st);

// ---- launchers (sigmo_kernels.cu); all enqueue on `st` ----
cudaError_t launch_sig_counts(const DevGraphs &g, int R, uint8_t *counts, int skip0, cudaStream_t st);
cudaError_t launch_sig_pack(const DevGraphs &g, int radius, unsigned long long *out, int skip0, cudaStream_t st);
cudaError_t launch_query_prep(const DevGraphs &q, int R, const uint8_t *qcounts, QueryProg &prog, int wild,
                              cudaStream_t st);
cudaError_t launch_filter(int NW, const FilterParams &p, int num_tiles, cudaStream_t st);
size_t filter_smem_bytes(int NW, int EXTN, int EXTW, int MOLCAP, int NFU, int NLAB, int P, int NREC, int VQ,
                         int NRP, int rows_smem, int NQW, int TS, int mol, int NDR = 0, int NQ = 0, int NQWL = 0);
cudaError_t launch_support(int NW, const SupportParams &p, cudaStream_t st);
size_t support_smem_bytes(int NW, int NB, int maxq, int NQW);
cudaError_t launch_scan(const I64x2 *in, I64x2 *out, int n, void *temp, size_t *temp_bytes, cudaStream_t st);
cudaError_t launch_chunks(const ChunkParams &p, cudaStream_t st);
cudaError_t launch_u64_inclusive_sum(const unsigned long long *in, unsigned long long *out, long long n, void *temp,
                                     size_t *temp_bytes, cudaStream_t st);
// enumerate mode: uoff == nullptr -> sort each pair's node masks and count the distinct ones (ucnt);
// else write them at uoff
cudaError_t launch_nodesets(const unsigned long long *eoff, long long P, unsigned long long *sets,
                            unsigned long long *ucnt, const unsigned long long *uoff, unsigned long long *uniq,
                            cudaStream_t st);
cudaError_t launch_join(int NW, int mode, const JoinParams &p, int grid, cudaStream_t st);
cudaError_t launch_pairs(const PairsParams &p, cudaStream_t st);
cudaError_t launch_support_lane(const SupportLaneParams &p, cudaStream_t st);
cudaError_t launch_gmcr_update(int ND, int NQW, const uint32_t *gm_old, const I64x2 *off_old, const int32_t *goff,
                               const uint8_t *alive, uint32_t *gm, I64x2 *mol_cnt, cudaStream_t st);
cudaError_t launch_unpad(const uint32_t *cmol, const uint32_t *cand_units, const uint16_t *qdrow, int NDR, const int32_t *goff, int ND,
                         int VQ, int Wpad, uint32_t *dense,
                         cudaStream_t st);
cudaError_t launch_adjb(const DevGraphs &d, const uint8_t *bclass, int NB, const uint32_t *adj_off, uint32_t *adjw,
                        uint32_t *nb4, cudaStream_t st);
cudaError_t launch_filter_lane(const FilterLaneParams &p, int grid, cudaStream_t st);
// run-time specialised lane filter (sigmo_jit.cu)
struct LaneJitSpec {
  int NLAB = 0, NFU = 0, R = 0, NDR = 0, RWV = 1, NQG = 0, NQ = 0, NQW = 0;
  bool GL = false;
  int min_blocks = 3;                    // __launch_bounds__ min CTAs per SM (register cap)
  std::vector<std::vector<uint2>> recs;  // [R] plane records of each radius (FilterLaneParams::grec format)
  std::vector<int> rgn;                  // channel-pair words per 32-row group
  std::vector<int2> qwh;                 // {first entry, entries} per 32-query group
};
std::string lane_jit_header(const LaneJitSpec &s);
cudaKernel_t lane_jit_kernel(const LaneJitSpec &s, std::string *why, double *compile_ms);
cudaError_t launch_filter_lane_jit(cudaKernel_t k, const FilterLaneParams &p, int grid, cudaStream_t st);
int filter_lane_jit_blocks_per_sm(cudaKernel_t k, const FilterLaneParams &p);
size_t filter_lane_smem_bytes(const FilterLaneParams &p);
int filter_lane_blocks_per_sm(const FilterLaneParams &p);
cudaError_t launch_mrec(const int32_t *goff, const uint32_t *adj_off, const uint32_t *cand_units, int ND, uint4 *mrec,
                        cudaStream_t st);
cudaError_t launch_join_lane(int mode, bool w64, const JoinParams &p, int grid, cudaStream_t st);
cudaError_t launch_lane_totals(int ND, int NQ, int NQW, const uint32_t *gm, const I64x2 *off,
                               const unsigned long long *presult, unsigned long long *totals, int sm_count, cudaStream_t st);
size_t join_lane_smem_bytes(const JoinParams &p, bool w64);
int join_lane_blocks_per_sm(int mode, bool w64, const JoinParams &p, size_t smem);
constexpr int kJoinLaneThreads = 128;
constexpr int kJoinLanePlanSmemMax = 2048;  // k_join_lane: plan positions copied to shared memory (16 KB)
// k_join_lane CTA size (the launch-bounds maximum; JoinParams::lane_threads is the launched size): 6 warps for
// 32-bit masks (7 CTAs x 6 warps at <= 48 registers and ~30 KB of shared memory; the plan copy and the per-query
// totals are per CTA), 4 for 64-bit masks
#ifndef SIGMO_JL_THREADS_NARROW
#define SIGMO_JL_THREADS_NARROW 192
#endif
__host__ __device__ constexpr int jl_threads(bool w64) { return w64 ? 128 : SIGMO_JL_THREADS_NARROW; }
// SIGMO_BOUNDS_CHECK builds (tools/bounds_check.sh): index and address bounds of the lane join and the
// totals reduction checked on the device (trap on violation); compiled out otherwise
#ifdef SIGMO_BOUNDS_CHECK
#define SIGMO_BOUND(cond) \
  do {                    \
    if (!(cond)) __trap(); \
  } while (0)
#else
#define SIGMO_BOUND(cond) \
  do {                    \
  } while (0)
#endif
constexpr int kJoinLaneMaxQ = 11;  // k_join_lane handles queries <= 11 nodes in <= 64-node graphs (map: 6 bits x 10 depths)
size_t join_smem_bytes(int NW, const JoinParams &p);
size_t join_gstack_bytes(int NW, const JoinParams &p, int grid);
int join_blocks_per_sm(int NW, int mode, const JoinParams &p, size_t smem);

}  // namespace sigmo
