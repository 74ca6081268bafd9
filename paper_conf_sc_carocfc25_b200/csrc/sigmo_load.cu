// sigmo_load.cu -- device-side validation and CSR-GO packing of a large data
// batch (section 4.1; the sigmo_load_batch contract of
// include/sigmo.h).  The host checks what is O(#graphs) -- offsets, sizes,
// limits -- and ships the raw arrays (one H2D copy per array, directly from
// the caller's pinned buffers when they are pinned); this kernel checks every
// adjacency entry (inside its graph, no self-loop, no duplicate, the reverse
// entry present with the same bond label, row offsets non-decreasing), writes
// the packed device form (int32 offsets, molecule-local neighbour | bond
// label, local index) and the label histogram the query planner uses.
// One warp per graph, lane = node (graphs are <= 256 atoms and sparse); a
// graph with several invalid classes reports the lowest.
#include <cub/cub.cuh>

#include "sigmo_internal.h"

namespace sigmo {

__global__ void __launch_bounds__(256) k_load_data(DataLoadParams p) {
  __shared__ unsigned int s_hist[256];
  for (int i = threadIdx.x; i < 256; i += blockDim.x) s_hist[i] = 0u;
  __syncthreads();
  // one warp per graph, lane = node (strided for graphs of > 32 nodes)
  const long long g = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (g < p.G) {
    const long long a = p.goff[g], b = p.goff[g + 1];
    if (lane == 0) {
      p.goff32[g] = (int32_t)a;
      if (g == p.G - 1) {
        p.goff32[p.G] = (int32_t)b;
        p.roff32[b] = (int32_t)p.roff[b];
      }
    }
    unsigned bad = 0u;  // error classes found in this graph (bit k: class k + 1)
    for (long long v = a + lane; v < b; v += 32) {
      p.local[v] = (uint8_t)(v - a);
      const uint8_t lab = p.nlab[v];
      p.label[v] = lab;
      {  // label histogram: one shared atomic per distinct label of the warp
        const unsigned act = __activemask();
        const unsigned same = __match_any_sync(act, (unsigned)lab);
        if ((__ffs(same) - 1) == lane) atomicAdd(&s_hist[lab], (unsigned)__popc(same));
      }
      const long long r0 = p.roff[v], r1 = p.roff[v + 1];
      p.roff32[v] = (int32_t)r0;
      if (r1 < r0) {
        bad |= 1u;
        continue;
      }
      for (long long e = r0; e < r1; e++) {
        const long long u = p.col[e];
        if (u < a || u >= b) {
          bad |= 2u;
          continue;
        }
        if (u == v) {
          bad |= 4u;
          continue;
        }
        const uint8_t el = p.elab[e];
        p.nbr[e] = (uint16_t)(((u - a) << 8) | el);
        int dup = 0;
        for (long long f = r0; f < r1; f++) dup += p.col[f] == u;
        if (dup > 1) bad |= 8u;
        bool sym = false;
        const long long s0 = p.roff[u], s1 = p.roff[u + 1];
        for (long long f = s0; f < s1 && !sym; f++) sym = p.col[f] == v && p.elab[f] == el;
        if (!sym) bad |= 16u;
      }
    }
    bad = __reduce_or_sync(0xffffffffu, bad);
    if (lane < 5 && ((bad >> lane) & 1u)) atomicMin(&p.err_graph[lane], (long long)g);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < 256; i += blockDim.x)
    if (s_hist[i]) atomicAdd(&p.hist[i], (unsigned long long)s_hist[i]);
}

cudaError_t launch_load_data(const DataLoadParams &p, cudaStream_t st) {
  if (p.G <= 0) return cudaSuccess;
  k_load_data<<<(unsigned)((p.G + 7) / 8), 256, 0, st>>>(p);  // 8 graphs (warps) per block
  return cudaGetLastError();
}

}  // namespace sigmo

// ---------------------------------------------------------------------------
// Per-molecule layout of a device-loaded batch, from the packed offsets:
// bond-class adjacency blocks ([NB+1][n] words, u64 for > 32 atoms) and
// candidate-window units (NDR x 1 word, or 2 for > 32 atoms), narrow
// molecules first, then the wide ones from an even word / unit offset; the
// k_filter_lane group lists (narrow / wide molecule ids); the molecule records
// of the lane filter; the batch maxima.  One exclusive scan of per-molecule
// sizes, then a scatter.
// ---------------------------------------------------------------------------
namespace sigmo {
namespace {
struct LayAcc {
  long long an, aw;  // adjacency words of narrow / wide molecules
  int cn, cw;        // narrow / wide molecules
  int maxn, nempty;  // largest molecule, empty molecules
};
struct LayOp {
  __host__ __device__ __forceinline__ LayAcc operator()(const LayAcc &x, const LayAcc &y) const {
    LayAcc r;
    r.an = x.an + y.an;
    r.aw = x.aw + y.aw;
    r.cn = x.cn + y.cn;
    r.cw = x.cw + y.cw;
    r.maxn = x.maxn > y.maxn ? x.maxn : y.maxn;
    r.nempty = x.nempty + y.nempty;
    return r;
  }
};

__global__ void k_layout_sizes(const int32_t *goff, int G, int NB, LayAcc *acc) {
  const int g = blockIdx.x * blockDim.x + threadIdx.x;
  if (g > G) return;
  LayAcc a{0, 0, 0, 0, 0, 0};
  if (g < G) {
    const int n = goff[g + 1] - goff[g];
    const bool wide = n > 32;
    a.an = wide ? 0 : (long long)n * (NB + 1);
    a.aw = wide ? 2ll * n * (NB + 1) : 0;
    a.cn = wide ? 0 : 1;
    a.cw = wide ? 1 : 0;
    a.maxn = n;
    a.nempty = n == 0;
  }
  acc[g] = a;
}

__global__ void k_layout_scatter(const int32_t *goff, int G, const LayAcc *pre, uint32_t *aoff, uint32_t *cu,
                                 int32_t *grpn, int32_t *grpw, uint4 *mrec) {
  const int g = blockIdx.x * blockDim.x + threadIdx.x;
  if (g > G) return;
  const LayAcc tot = pre[G];
  const unsigned long long an_even = ((unsigned long long)tot.an + 1ull) & ~1ull;
  const unsigned long long cn_even = ((unsigned long long)tot.cn + 1ull) & ~1ull;
  if (g == G) {
    aoff[G] = (uint32_t)(an_even + (unsigned long long)tot.aw);
    cu[G] = (uint32_t)(cn_even + 2ull * (unsigned long long)tot.cw);
    return;
  }
  const LayAcc p = pre[g];
  const int a = goff[g], n = goff[g + 1] - a;
  uint32_t ao, c;
  if (n > 32) {
    ao = (uint32_t)(an_even + (unsigned long long)p.aw);
    c = (uint32_t)(cn_even + 2ull * (unsigned long long)p.cw);
    grpw[p.cw] = g;
  } else {
    ao = (uint32_t)p.an;
    c = (uint32_t)p.cn;
    grpn[p.cn] = g;
  }
  aoff[g] = ao;
  cu[g] = c;
  mrec[g] = make_uint4((unsigned)a, (unsigned)n, ao, c);
}
}  // namespace

size_t layout_scan_bytes(int G) {
  size_t tb = 0;
  cub::DeviceScan::ExclusiveScan(nullptr, tb, (const LayAcc *)nullptr, (LayAcc *)nullptr, LayOp(),
                                 LayAcc{0, 0, 0, 0, 0, 0}, G + 1, (cudaStream_t)0);
  return tb + 2 * sizeof(LayAcc) * ((size_t)G + 1) + 256;
}

// scratch: layout_scan_bytes(G) bytes; info_out (device, 32 B): {int64 an, aw; int32 cn, cw, maxn, nempty} totals
cudaError_t launch_layout(const int32_t *goff, int G, int NB, void *scratch, uint32_t *aoff, uint32_t *cu,
                          int32_t *grpn, int32_t *grpw, uint4 *mrec, long long *info_out, cudaStream_t st) {
  LayAcc *acc = (LayAcc *)scratch;
  LayAcc *pre = acc + (G + 1);
  void *tmp = (void *)(pre + (G + 1));
  size_t tb = 0;
  cudaError_t e = cub::DeviceScan::ExclusiveScan(nullptr, tb, acc, pre, LayOp(), LayAcc{0, 0, 0, 0, 0, 0}, G + 1, st);
  if (e != cudaSuccess) return e;
  const unsigned blocks = (unsigned)((G + 1 + 255) / 256);
  k_layout_sizes<<<blocks, 256, 0, st>>>(goff, G, NB, acc);
  e = cub::DeviceScan::ExclusiveScan(tmp, tb, acc, pre, LayOp(), LayAcc{0, 0, 0, 0, 0, 0}, G + 1, st);
  if (e != cudaSuccess) return e;
  k_layout_scatter<<<blocks, 256, 0, st>>>(goff, G, pre, aoff, cu, grpn, grpw, mrec);
  e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  // the totals pre[G] for the host: {int64 an, aw; int32 cn, cw, maxn, nempty}
  return cudaMemcpyAsync(info_out, pre + G, sizeof(LayAcc), cudaMemcpyDeviceToDevice, st);
}

}  // namespace sigmo
