// sigmo_filter_lane.cu -- the generic (table-driven) build of the lane-path
// filter kernel (device code in lane_filter_body.cuh) and its launchers.  The
// NVRTC-specialised build of the same body is in sigmo_jit.cu.
#include "sigmo_internal.h"
#include "lane_filter_body.cuh"

namespace sigmo {

size_t filter_lane_smem_bytes(const FilterLaneParams &p) { return lane_filter_layout(p).total; }

cudaError_t launch_filter_lane(const FilterLaneParams &p, int grid, cudaStream_t st) {
  if (grid <= 0 || p.NGN + p.NGW <= 0) return cudaSuccess;
  cudaError_t e;
  if (p.tables_global) {
    e = cudaFuncSetAttribute(k_filter_lane<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p.smem_bytes);
    if (e != cudaSuccess) return e;
    k_filter_lane<true><<<grid, kFilterLaneThreads, p.smem_bytes, st>>>(p);
  } else {
    e = cudaFuncSetAttribute(k_filter_lane<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p.smem_bytes);
    if (e != cudaSuccess) return e;
    k_filter_lane<false><<<grid, kFilterLaneThreads, p.smem_bytes, st>>>(p);
  }
  return cudaGetLastError();
}

int filter_lane_blocks_per_sm(const FilterLaneParams &p) {
  int n = 0;
  cudaError_t e;
  if (p.tables_global) {
    cudaFuncSetAttribute(k_filter_lane<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p.smem_bytes);
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_filter_lane<true>, kFilterLaneThreads, p.smem_bytes);
  } else {
    cudaFuncSetAttribute(k_filter_lane<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p.smem_bytes);
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_filter_lane<false>, kFilterLaneThreads, p.smem_bytes);
  }
  if (e != cudaSuccess) {
    cudaGetLastError();
    return 1;
  }
  return n < 1 ? 1 : n;
}

// per-molecule records {first node, atoms, adjacency word offset, candidate units}
__global__ void k_mrec(const int32_t *goff, const uint32_t *adj_off, const uint32_t *cand_units, int ND, uint4 *mrec) {
  const int g = blockIdx.x * blockDim.x + threadIdx.x;
  if (g >= ND) return;
  const int a = goff[g];
  mrec[g] = make_uint4((unsigned)a, (unsigned)(goff[g + 1] - a), adj_off[g], cand_units[g]);
}

cudaError_t launch_mrec(const int32_t *goff, const uint32_t *adj_off, const uint32_t *cand_units, int ND, uint4 *mrec,
                        cudaStream_t st) {
  if (ND <= 0) return cudaSuccess;
  k_mrec<<<(ND + 255) / 256, 256, 0, st>>>(goff, adj_off, cand_units, ND, mrec);
  return cudaGetLastError();
}

}  // namespace sigmo
