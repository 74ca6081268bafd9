// lane_filter_types.h -- types shared by the host side and the lane-path
// filter kernel (lane_filter_body.cuh).  Self-contained: it is also handed to
// NVRTC as an in-memory header when sigmo_jit.cu specialises the kernel for
// one query program (no CUDA runtime or C library headers there).
#pragma once
#ifdef __CUDACC_RTC__
typedef unsigned int uint32_t;
typedef int int32_t;
typedef unsigned short uint16_t;
typedef unsigned char uint8_t;
typedef unsigned long size_t;
#else
#include <cuda_runtime.h>
#include <stdint.h>
#include <stddef.h>
#endif

namespace sigmo {

constexpr int kMaxRadius = 15;   // levels <= 16

struct I64x2 {
  long long a, b;
};

// k_filter_lane (sigmo_filter_lane.cu): the filter of the lane-join path.
// Groups of 4 slots of 32 nodes: narrow groups = 4 molecules of <= 32 atoms,
// wide groups = 2 molecules of 33-64 atoms.  Channels of the per-warp plane
// array: 0..NLAB-1 label planes, NLAB all ones, NLAB+1+p constraint plane p.
constexpr int kFilterLaneThreads = 256;
struct FilterLaneParams {
  int NGN, NGW;                 // narrow / wide groups
  const int32_t *grp_narrow;    // [4 NGN] molecule ids (-1 = empty slot)
  const int32_t *grp_wide;      // [2 NGW]
  const uint4 *mrec;            // [ND] {first node, atoms, adjacency word offset, candidate units}
  const uint8_t *label;         // [VD]
  const uint32_t *nb4;          // [VD] first <= 4 neighbours (molecule-local ids, filler = self; bit 7: degree > 4)
  const uint32_t *adjw;         // bond-class adjacency, class NB = all bonds (slow path of degree > 4 nodes)
  int NB, R, NLAB, NFU, NCH;
  const uint16_t *lut;          // [256] label -> label channel (0xff none) | field slot << 8 (0xff unused)
  const uint2 *grec;            // [NREC] plane records: x = field slot | #planes (<= 4) << 8 | first channel << 16,
  int NREC;                     //        y = thresholds (bytes), sorted by radius
  const int32_t *rrec;          // [4R+1] record ranges: radius r, k+1 planes at [rrec[4(r-1)+k], rrec[4(r-1)+k+1])
  const uint4 *rowp;            // [NDR][RWV] row programs: pairs of 16-bit channel byte offsets (x16), all-ones padded
  const int32_t *rgn;           // [ceil(NDR/32)] channel-pair words needed by each 32-row group (rows sorted by length)
  int NDR, RWV;
  const uint2 *qwl;             // GMCR lists [entries][32 lanes] (word, bits), (0, 0) padded
  int NQWE;                     // entries x 32
  const int2 *qwh;              // [NQG] {first entry, entries} per 32-query group
  int NQG, NQ, NQW;
  uint32_t *cmol;               // molecule-padded windows (FilterParams::cmol)
  uint32_t *gm;                 // [ND][NQW]
  I64x2 *mol_cnt;               // [ND+1]
  int tables_global;            // 1: row programs and GMCR lists read from global memory (too large for smem)
  size_t smem_bytes;
};


}  // namespace sigmo
