// sigmo_load.cu -- device-side validation and CSR-GO packing of a large data
// batch (section 4.1; the sigmo_load_batch contract of
// include/sigmo.h).  The host checks what is O(#graphs) -- offsets, sizes,
// limits -- and ships the raw arrays (one H2D copy per array, directly from
// the caller's pinned buffers when they are pinned); this kernel checks every
// adjacency entry (inside its graph, no self-loop, no duplicate, the reverse
// entry present with the same bond label, row offsets non-decreasing), writes
// the packed device form (int32 offsets, molecule-local neighbour | bond
// label, local index) and the label histogram the query planner uses.
// One thread per graph (graphs are <= 256 atoms and sparse).
#include "sigmo_internal.h"

namespace sigmo {

__global__ void __launch_bounds__(256) k_load_data(DataLoadParams p) {
  __shared__ unsigned int s_hist[256];
  for (int i = threadIdx.x; i < 256; i += blockDim.x) s_hist[i] = 0u;
  __syncthreads();
  const long long g = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (g < p.G) {
    const long long a = p.goff[g], b = p.goff[g + 1];
    p.goff32[g] = (int32_t)a;
    if (g == p.G - 1) {
      p.goff32[p.G] = (int32_t)b;
      p.roff32[b] = (int32_t)p.roff[b];
    }
    int bad = 0;  // first error class of this graph (0 none)
    for (long long v = a; v < b; v++) {
      p.local[v] = (uint8_t)(v - a);
      const uint8_t lab = p.nlab[v];
      p.label[v] = lab;
      atomicAdd(&s_hist[lab], 1u);
      const long long r0 = p.roff[v], r1 = p.roff[v + 1];
      p.roff32[v] = (int32_t)r0;
      if (r1 < r0) {
        bad = bad ? bad : 1;
        continue;
      }
      for (long long e = r0; e < r1; e++) {
        const long long u = p.col[e];
        if (u < a || u >= b) {
          bad = bad ? bad : 2;
          continue;
        }
        if (u == v) {
          bad = bad ? bad : 3;
          continue;
        }
        const uint8_t el = p.elab[e];
        p.nbr[e] = (uint16_t)(((u - a) << 8) | el);
        int dup = 0;
        for (long long f = r0; f < r1; f++) dup += p.col[f] == u;
        if (dup > 1) bad = bad ? bad : 4;
        bool sym = false;
        const long long s0 = p.roff[u], s1 = p.roff[u + 1];
        for (long long f = s0; f < s1 && !sym; f++) sym = p.col[f] == v && p.elab[f] == el;
        if (!sym) bad = bad ? bad : 5;
      }
    }
    if (bad) atomicMin(&p.err_graph[bad - 1], (long long)g);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < 256; i += blockDim.x)
    if (s_hist[i]) atomicAdd(&p.hist[i], (unsigned long long)s_hist[i]);
}

cudaError_t launch_load_data(const DataLoadParams &p, cudaStream_t st) {
  if (p.G <= 0) return cudaSuccess;
  k_load_data<<<(unsigned)((p.G + 255) / 256), 256, 0, st>>>(p);
  return cudaGetLastError();
}

}  // namespace sigmo
