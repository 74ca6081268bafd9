// sigmo_kernels.cu -- sm_100a kernels of the SIGMo hot path.
//
// Stages (Fig. 2) and the B200 design:
//   k_sig_counts   GenerateSignatures (Alg. 1 l.11-18, section 4.4)
//                  per graph with molecule-local bitset BFS; used for the
//                  query side and for the signature export.
//   k_query_prep   turns query signatures into a "plane program": the
//                  distinct (radius, field, threshold) constraints of all
//                  query nodes (RefineCandidates l.19-28 restated as
//                  per-field >= tests, reading R5) and one AND-list per
//                  query node.
//   k_filter       InitializeCandidates + every refinement level fused in one
//                  pass over 32-word bitmap tiles: data signatures by bitset
//                  BFS in shared memory, bit-sliced threshold planes via warp
//                  ballots, each bitmap word written ONCE (the paper rewrites
//                  the bitmap every level), and the GMCR test of
//                  section 4.5 in the epilogue.
//   (CUB scan)     GMCR offsets on the device (no host round trip)
//   k_chunks       cuts the molecule range into smem-sized join chunks
//   k_join         stack-based DFS (section 4.6) over bitset
//                  candidate masks; lanes pull (pair, root) work items from a
//                  per-CTA queue, per-query totals reduced in smem.
#include <cub/cub.cuh>

#include "sigmo_internal.h"

namespace sigmo {

#define FULL_MASK 0xffffffffu

// ---------------------------------------------------------------------------
// R7 field table (LSB-first): C 8, N 6, O 6, S 5, F 5, Cl 5, Br 4, I 4, P 4,
// H 7, B 3, Si 3, other 4 = 64 bits.  (section 4.2)
// ---------------------------------------------------------------------------
__constant__ int c_field_width[kNumFields] = {8, 6, 6, 5, 5, 5, 4, 4, 4, 7, 3, 3, 4};
__constant__ int c_field_off[kNumFields] = {0, 8, 14, 20, 25, 30, 35, 39, 43, 47, 54, 57, 60};

__device__ __forceinline__ int field_of(int lab) {
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

// ---------------------------------------------------------------------------
// Molecule-local bitset (NW x 64 bits)
// ---------------------------------------------------------------------------
template <int NW>
struct Mask {
  unsigned long long w[NW];
  __device__ __forceinline__ void clear() {
#pragma unroll
    for (int k = 0; k < NW; k++) w[k] = 0ull;
  }
  __device__ __forceinline__ static Mask bit(int i) {
    Mask m;
#pragma unroll
    for (int k = 0; k < NW; k++) m.w[k] = ((i >> 6) == k) ? (1ull << (i & 63)) : 0ull;
    return m;
  }
  __device__ __forceinline__ void set(int i) {
#pragma unroll
    for (int k = 0; k < NW; k++)
      if ((i >> 6) == k) w[k] |= 1ull << (i & 63);
  }
  __device__ __forceinline__ void reset(int i) {
#pragma unroll
    for (int k = 0; k < NW; k++)
      if ((i >> 6) == k) w[k] &= ~(1ull << (i & 63));
  }
  __device__ __forceinline__ bool any() const {
    unsigned long long x = 0;
#pragma unroll
    for (int k = 0; k < NW; k++) x |= w[k];
    return x != 0ull;
  }
  __device__ __forceinline__ int popc() const {
    int c = 0;
#pragma unroll
    for (int k = 0; k < NW; k++) c += __popcll(w[k]);
    return c;
  }
  __device__ __forceinline__ int lowest() const {
    int r = -1;
#pragma unroll
    for (int k = NW - 1; k >= 0; k--)
      if (w[k]) r = k * 64 + __ffsll((long long)w[k]) - 1;
    return r;
  }
  __device__ __forceinline__ void clear_lowest() {
    bool done = false;
#pragma unroll
    for (int k = 0; k < NW; k++)
      if (!done && w[k]) {
        w[k] &= w[k] - 1ull;
        done = true;
      }
  }
  __device__ __forceinline__ Mask operator&(const Mask &o) const {
    Mask m;
#pragma unroll
    for (int k = 0; k < NW; k++) m.w[k] = w[k] & o.w[k];
    return m;
  }
  __device__ __forceinline__ Mask operator|(const Mask &o) const {
    Mask m;
#pragma unroll
    for (int k = 0; k < NW; k++) m.w[k] = w[k] | o.w[k];
    return m;
  }
  __device__ __forceinline__ Mask andnot(const Mask &o) const {
    Mask m;
#pragma unroll
    for (int k = 0; k < NW; k++) m.w[k] = w[k] & ~o.w[k];
    return m;
  }
  __device__ __forceinline__ void operator&=(const Mask &o) {
#pragma unroll
    for (int k = 0; k < NW; k++) w[k] &= o.w[k];
  }
  __device__ __forceinline__ void operator|=(const Mask &o) {
#pragma unroll
    for (int k = 0; k < NW; k++) w[k] |= o.w[k];
  }
};

// Extract `n` bits starting at bit `s` of a u32 word array of `nw` words
// (bits beyond the array read as 0) into a molecule-local mask.
template <int NW>
__device__ __forceinline__ Mask<NW> extract_window(const uint32_t *words, long long nw, long long s, int n) {
  Mask<NW> m;
#pragma unroll
  for (int k = 0; k < NW; k++) {
    long long b = s + 64ll * k;
    long long wi = b >> 5;
    int sh = (int)(b & 31);
    unsigned long long w0 = (wi < nw) ? words[wi] : 0u;
    unsigned long long w1 = (wi + 1 < nw) ? words[wi + 1] : 0u;
    unsigned long long w2 = (wi + 2 < nw) ? words[wi + 2] : 0u;
    unsigned long long lo = w0 | (w1 << 32);
    unsigned long long x = lo >> sh;
    if (sh) x |= w2 << (64 - sh);
    int rem = n - 64 * k;
    if (rem <= 0) x = 0ull;
    else if (rem < 64) x &= (1ull << rem) - 1ull;
    m.w[k] = x;
  }
  return m;
}

// Largest g in [0, G] with goff[g] <= n (goff[G] = V > n): the graph of node n.
__device__ __forceinline__ int graph_of(const int32_t *goff, int G, int n) {
  int lo = 0, hi = G;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (__ldg(&goff[mid]) <= n) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

// Exclusive block scan of n ints in place (any memory space visible to the
// block); returns the total.  Must be called by all NT threads.
template <int NT, typename T>
__device__ int block_exclusive_scan(T *data, int n, int *s_warp) {
  const int per = (n + NT - 1) / NT;
  const int b = threadIdx.x * per;
  const int e = min(b + per, n);
  int sum = 0;
  for (int i = b; i < e; i++) sum += (int)data[i];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int x = sum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int y = __shfl_up_sync(FULL_MASK, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_warp[wid] = x;
  __syncthreads();
  if (wid == 0) {
    int v = (lane < NT / 32) ? s_warp[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int y = __shfl_up_sync(FULL_MASK, v, o);
      if (lane >= o) v += y;
    }
    s_warp[lane] = v;
  }
  __syncthreads();
  int run = x - sum + (wid > 0 ? s_warp[wid - 1] : 0);
  const int total = s_warp[NT / 32 - 1];
  for (int i = b; i < e; i++) {
    int t = (int)data[i];
    data[i] = (T)run;
    run += t;
  }
  __syncthreads();
  return total;
}

// ===========================================================================
// k_sig_counts: per graph, cumulative radius-r label counts (R4) for
// r = 1..R, saturated per field (R8), optionally packed at one radius.
// One CTA per graph (<= 256 nodes, NW = 4); not on the data hot path.
// ===========================================================================
__global__ void __launch_bounds__(128) k_sig_counts(DevGraphs g, int R, uint8_t *counts,
                                                    unsigned long long *packed, int pack_radius) {
  using M = Mask<4>;
  __shared__ M s_ballA[256], s_ballB[256], s_adj[256], s_fm[kNumFields];
  __shared__ uint8_t s_fid[256];
  const int gi = blockIdx.x;
  const int base = g.goff[gi];
  const int n = g.goff[gi + 1] - base;
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    M a;
    a.clear();
    for (int e = g.roff[base + i]; e < g.roff[base + i + 1]; e++) a.set(g.nbr[e] >> 8);
    s_adj[i] = a;
    s_ballA[i] = M::bit(i);
    s_fid[i] = (uint8_t)field_of(g.label[base + i]);
  }
  for (int f = threadIdx.x; f < kNumFields; f += blockDim.x) s_fm[f].clear();
  __syncthreads();
  for (int i = threadIdx.x; i < n; i += blockDim.x)
    atomicOr(&s_fm[s_fid[i]].w[i >> 6], 1ull << (i & 63));
  __syncthreads();
  M *cur = s_ballA, *nxt = s_ballB;
  for (int r = 1; r <= R; r++) {
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
      M x = cur[i];
      M a = s_adj[i];
      for (int u = a.lowest(); u >= 0; a.clear_lowest(), u = a.lowest()) x |= cur[u];
      nxt[i] = x;
    }
    __syncthreads();
    M *t = cur;
    cur = nxt;
    nxt = t;
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
      unsigned long long pk = 0;
      for (int f = 0; f < kNumFields; f++) {
        int c = (cur[i] & s_fm[f]).popc() - (s_fid[i] == f ? 1 : 0);
        int mx = (1 << c_field_width[f]) - 1;
        if (c > mx) c = mx;  // R8: saturate, never wrap
        if (counts) counts[((size_t)(base + i) * R + (r - 1)) * kNumFields + f] = (uint8_t)c;
        pk |= (unsigned long long)c << c_field_off[f];
      }
      if (packed && r == pack_radius) packed[base + i] = pk;
    }
    __syncthreads();
  }
}

cudaError_t launch_sig_counts(const DevGraphs &g, int R, uint8_t *counts, cudaStream_t st) {
  if (g.num_graphs == 0 || R <= 0) return cudaSuccess;
  k_sig_counts<<<g.num_graphs, 128, 0, st>>>(g, R, counts, nullptr, 0);
  return cudaGetLastError();
}

cudaError_t launch_sig_pack(const DevGraphs &g, int radius, unsigned long long *out, cudaStream_t st) {
  if (g.num_graphs == 0) return cudaSuccess;
  k_sig_counts<<<g.num_graphs, 128, 0, st>>>(g, radius, nullptr, out, radius);
  return cudaGetLastError();
}

// ===========================================================================
// k_query_prep: one CTA.  From saturated query counts t_r(v_q, f) build
//   * planes  = distinct constraints (r, f, t) with t > t_{r-1}(v_q, f)
//     (a constraint whose threshold did not grow since radius r-1 is implied
//     by the radius r-1 one because data counts are monotone in r; t = 0 is
//     always true), sorted by (r, f, t);
//   * groups  = distinct (r, f) with their plane range;
//   * label planes = distinct query labels;
//   * per query node: its label plane and the list of its plane ids.
// Dominance of saturated values (R8) is equivalent to count_d >= t because
// t <= 2^w - 1.
// ===========================================================================
constexpr int kKeyWords = (kMaxRadius * kNumFields * 256) / 32;  // 1560
constexpr int kRF = kMaxRadius * kNumFields;                     // 195

__global__ void __launch_bounds__(kQueryPrepThreads) k_query_prep(int VQ, int R, const uint8_t *qlabel,
                                                                   const uint8_t *qc, QueryProg prog) {
  constexpr int NT = kQueryPrepThreads;
  __shared__ uint32_t s_key[kKeyWords];
  __shared__ int s_rank[kKeyWords];
  __shared__ int s_g[kRF + 1];
  __shared__ uint32_t s_lab[8];
  __shared__ int s_labrank[8];
  __shared__ int s_warp[32];
  __shared__ int s_fslot[kNumFields];
  const int tid = threadIdx.x;
  for (int i = tid; i < kKeyWords; i += NT) s_key[i] = 0u;
  if (tid < 8) s_lab[tid] = 0u;
  __syncthreads();
  const int RF = R * kNumFields;
  const long long total = (long long)VQ * RF;
  for (long long idx = tid; idx < total; idx += NT) {
    int vq = (int)(idx / RF), rem = (int)(idx % RF);
    int r0 = rem / kNumFields, f = rem % kNumFields;
    int t = qc[((size_t)vq * R + r0) * kNumFields + f];
    int prev = r0 > 0 ? qc[((size_t)vq * R + r0 - 1) * kNumFields + f] : 0;
    if (t > prev) {
      int key = (r0 * kNumFields + f) * 256 + t;
      atomicOr(&s_key[key >> 5], 1u << (key & 31));
    }
  }
  for (int v = tid; v < VQ; v += NT) atomicOr(&s_lab[qlabel[v] >> 5], 1u << (qlabel[v] & 31));
  __syncthreads();
  for (int i = tid; i < kKeyWords; i += NT) s_rank[i] = __popc(s_key[i]);
  __syncthreads();
  const int P = block_exclusive_scan<NT>(s_rank, kKeyWords, s_warp);
  // planes
  for (int i = tid; i < kKeyWords; i += NT) {
    uint32_t m = s_key[i];
    while (m) {
      int b = __ffs(m) - 1;
      int id = s_rank[i] + __popc(s_key[i] & ((1u << b) - 1u));
      prog.p_t[id] = (uint8_t)((i * 32 + b) & 255);
      m &= m - 1u;
    }
  }
  // groups = distinct (r, f): 8 key words per (r, f)
  for (int rf = tid; rf < kRF; rf += NT) {
    int c = 0;
    for (int k = 0; k < 8; k++) c += __popc(s_key[rf * 8 + k]);
    s_g[rf] = c > 0 ? 1 : 0;
  }
  if (tid == 0) s_g[kRF] = 0;
  __syncthreads();
  const int G = block_exclusive_scan<NT>(s_g, kRF + 1, s_warp);
  for (int rf = tid; rf < kRF; rf += NT) {
    int c = 0;
    for (int k = 0; k < 8; k++) c += __popc(s_key[rf * 8 + k]);
    if (c > 0) {
      prog.grp_poff[s_g[rf]] = (int16_t)s_rank[rf * 8];
      prog.grp_f[s_g[rf]] = (uint8_t)(rf % kNumFields);
    }
  }
  if (tid == 0) prog.grp_poff[G] = (int16_t)P;
  for (int r0 = tid; r0 <= R; r0 += NT) prog.rg_off[r0] = (int16_t)s_g[r0 * kNumFields];
  // used fields
  if (tid == 0) {
    int nfu = 0;
    for (int f = 0; f < kNumFields; f++) {
      bool used = false;
      for (int r0 = 0; r0 < R && !used; r0++) {
        int rf = r0 * kNumFields + f;
        used = s_g[rf + 1] > s_g[rf];
      }
      s_fslot[f] = used ? nfu++ : -1;
    }
    for (int f = 0; f < kNumFields; f++) prog.fslot[f] = (int8_t)s_fslot[f];
    int nl = 0;
    for (int k = 0; k < 8; k++) {
      s_labrank[k] = nl;
      nl += __popc(s_lab[k]);
    }
    prog.d_meta->P = P;
    prog.d_meta->G = G;
    prog.d_meta->NFU = nfu;
    prog.d_meta->NLAB = nl;
    prog.d_meta->err = 0;
    for (int l = 0; l < 256; l++)
      if (s_lab[l >> 5] & (1u << (l & 31)))
        prog.lab_val[s_labrank[l >> 5] + __popc(s_lab[l >> 5] & ((1u << (l & 31)) - 1u))] = (uint8_t)l;
  }
  __syncthreads();
  // row programs
  for (int v = tid; v < VQ; v += NT) {
    int c = 0;
    for (int r0 = 0; r0 < R; r0++)
      for (int f = 0; f < kNumFields; f++) {
        int t = qc[((size_t)v * R + r0) * kNumFields + f];
        int prev = r0 > 0 ? qc[((size_t)v * R + r0 - 1) * kNumFields + f] : 0;
        c += t > prev;
      }
    prog.row_off[v] = c;
    int l = qlabel[v];
    prog.row_lab[v] = (uint8_t)(s_labrank[l >> 5] + __popc(s_lab[l >> 5] & ((1u << (l & 31)) - 1u)));
  }
  __syncthreads();
  const int RE = block_exclusive_scan<NT>(prog.row_off, VQ, s_warp);
  if (tid == 0) {
    prog.row_off[VQ] = RE;
    prog.d_meta->row_entries = RE;
  }
  for (int v = tid; v < VQ; v += NT) {
    int pos = prog.row_off[v];
    for (int r0 = 0; r0 < R; r0++)
      for (int f = 0; f < kNumFields; f++) {
        int t = qc[((size_t)v * R + r0) * kNumFields + f];
        int prev = r0 > 0 ? qc[((size_t)v * R + r0 - 1) * kNumFields + f] : 0;
        if (t > prev) {
          int key = (r0 * kNumFields + f) * 256 + t;
          int id = s_rank[key >> 5] + __popc(s_key[key >> 5] & ((1u << (key & 31)) - 1u));
          prog.row_ids[pos++] = (uint16_t)id;
        }
      }
  }
}

cudaError_t launch_query_prep(const DevGraphs &q, int R, const uint8_t *qcounts, QueryProg &prog,
                              cudaStream_t st) {
  k_query_prep<<<1, kQueryPrepThreads, 0, st>>>(q.num_nodes, R, q.label, qcounts, prog);
  return cudaGetLastError();
}

// ===========================================================================
// k_filter: one CTA per tile of TW (<= 32) bitmap words = 32*TW data nodes.
// ===========================================================================
struct FilterSmem {
  size_t adj, ballA, ballB, fm, planes, win, molstart, molslot, fid, lab, mstart, sos, total;
};

__host__ __device__ inline size_t align16(size_t x) { return (x + 15) & ~(size_t)15; }

__host__ __device__ inline FilterSmem filter_layout(int NW, int EXTN, int EXTW, int MOLCAP, int NFU, int NLAB,
                                                    int P) {
  FilterSmem L;
  const size_t mb = 8 * (size_t)NW;
  size_t o = 0;
  L.adj = o;      o = align16(o + mb * EXTN);
  L.ballA = o;    o = align16(o + mb * EXTN);
  L.ballB = o;    o = align16(o + mb * EXTN);
  L.fm = o;       o = align16(o + mb * (size_t)MOLCAP * (NFU > 0 ? NFU : 1));
  L.planes = o;   o = align16(o + 4 * (size_t)(NLAB + P) * EXTW);
  L.win = o;      o = align16(o + mb * (size_t)(kFilterThreads / 32) * (NLAB + P));
  L.molstart = o; o = align16(o + 2 * (size_t)EXTN);
  L.molslot = o;  o = align16(o + 2 * (size_t)EXTN);
  L.fid = o;      o = align16(o + (size_t)EXTN);
  L.lab = o;      o = align16(o + (size_t)EXTN);
  L.mstart = o;   o = align16(o + 4 * (size_t)(MOLCAP + 1));
  L.sos = o;      o = align16(o + 2 * (size_t)EXTN);
  L.total = o;
  return L;
}

size_t filter_smem_bytes(int NW, int EXTN, int EXTW, int MOLCAP, int NFU, int NLAB, int P) {
  return filter_layout(NW, EXTN, EXTW, MOLCAP, NFU, NLAB, P).total;
}

template <int NW>
__global__ void __launch_bounds__(kFilterThreads) k_filter(FilterParams fp) {
  using M = Mask<NW>;
  constexpr int NT = kFilterThreads, NWARP = NT / 32;
  extern __shared__ __align__(16) unsigned char smem[];
  const FilterSmem L = filter_layout(NW, fp.EXTN, fp.EXTW, fp.MOLCAP, fp.NFU, fp.NLAB, fp.P);
  M *s_adj = (M *)(smem + L.adj);
  M *s_cur = (M *)(smem + L.ballA);
  M *s_nxt = (M *)(smem + L.ballB);
  M *s_fm = (M *)(smem + L.fm);
  uint32_t *s_planes = (uint32_t *)(smem + L.planes);
  M *s_win = (M *)(smem + L.win);
  int16_t *s_molstart = (int16_t *)(smem + L.molstart);
  int16_t *s_molslot = (int16_t *)(smem + L.molslot);
  uint8_t *s_fid = smem + L.fid;
  uint8_t *s_lab = smem + L.lab;
  int *s_mstart = (int *)(smem + L.mstart);
  int16_t *s_sos = (int16_t *)(smem + L.sos);
  __shared__ int s_g0, s_g1;

  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int ND = fp.D.num_graphs, VD = fp.D.num_nodes;
  const int w0 = blockIdx.x * fp.TW;
  if (w0 >= fp.W) return;
  const int n0 = w0 * 32;
  const int n1 = min(n0 + fp.TW * 32, VD);
  const int32_t *goff = fp.D.goff;
  if (tid == 0) {
    s_g0 = graph_of(goff, ND, n0);
    s_g1 = graph_of(goff, ND, n1 - 1) + 1;
  }
  __syncthreads();
  const int g0 = s_g0, g1 = s_g1, nmol = g1 - g0;
  const int gs = __ldg(&goff[g0]);
  const int ge = __ldg(&goff[g1]);
  const int next = ge - gs;
  const int xb = gs >> 5;                       // first ext word (global word index)
  const int nxw = ((ge - 1) >> 5) - xb + 1;     // ext words
  const int NLAB = fp.NLAB, P = fp.P, NFU = fp.NFU, EXTW = fp.EXTW;

  // ---- phase 1: nodes of all molecules overlapping the tile ----
  for (int i = tid; i <= nmol; i += NT) s_mstart[i] = __ldg(&goff[g0 + i]) - gs;
  for (int i = tid; i < next; i += NT) {
    const int v = gs + i;
    const int loc = fp.D.local[v];
    M a;
    a.clear();
    const int e1 = fp.D.roff[v + 1];
    for (int e = fp.D.roff[v]; e < e1; e++) a.set(fp.D.nbr[e] >> 8);
    s_adj[i] = a;
    s_cur[i] = M::bit(loc);
    s_molstart[i] = (int16_t)(i - loc);
    const int lab = fp.D.label[v];
    s_lab[i] = (uint8_t)lab;
    s_fid[i] = (uint8_t)field_of(lab);
  }
  for (int i = tid; i < nmol * NFU; i += NT) s_fm[i].clear();
  __syncthreads();
  for (int mi = tid; mi < nmol; mi += NT)
    if (s_mstart[mi] < s_mstart[mi + 1]) s_sos[s_mstart[mi]] = (int16_t)mi;
  __syncthreads();
  for (int i = tid; i < next; i += NT) {
    const int ms = s_molstart[i];
    const int slot = s_sos[ms];
    s_molslot[i] = (int16_t)slot;
    const int fs = NFU > 0 ? fp.fslot[s_fid[i]] : -1;
    if (fs >= 0) {
      const int loc = i - ms;
      atomicOr(&s_fm[slot * NFU + fs].w[loc >> 6], 1ull << (loc & 63));
    }
  }
  // ---- label planes (InitializeCandidates, Alg.1 l.29-37) ----
  for (int k = wid; k < nxw; k += NWARP) {
    const int i = (xb + k) * 32 + lane - gs;
    const bool valid = (i >= 0) && (i < next);
    const int lab = valid ? s_lab[i] : -1;
    for (int c = 0; c < NLAB; c++) {
      const unsigned b = __ballot_sync(FULL_MASK, lab == (int)fp.lab_val[c]);
      if (lane == 0) s_planes[c * EXTW + k] = b;
    }
  }
  __syncthreads();

  // ---- radii 1..R: bitset BFS + threshold planes ----
  for (int r = 1; r <= fp.R; r++) {
    for (int i = tid; i < next; i += NT) {
      M x = s_cur[i];
      M a = s_adj[i];
      const int ms = s_molstart[i];
      for (int u = a.lowest(); u >= 0; a.clear_lowest(), u = a.lowest()) x |= s_cur[ms + u];
      s_nxt[i] = x;
    }
    __syncthreads();
    M *t = s_cur;
    s_cur = s_nxt;
    s_nxt = t;
    const int gb = fp.rg_off[r - 1], gend = fp.rg_off[r];
    if (gb < gend) {
      for (int k = wid; k < nxw; k += NWARP) {
        const int i = (xb + k) * 32 + lane - gs;
        const bool valid = (i >= 0) && (i < next);
        M ball;
        ball.clear();
        int slot = 0, fid = -1;
        if (valid) {
          ball = s_cur[i];
          slot = s_molslot[i];
          fid = s_fid[i];
        }
        for (int grp = gb; grp < gend; grp++) {
          const int f = fp.grp_f[grp];
          int cnt = 0;
          if (valid) cnt = (ball & s_fm[slot * NFU + fp.fslot[f]]).popc() - (fid == f ? 1 : 0);
          const int pe = fp.grp_poff[grp + 1];
          for (int p = fp.grp_poff[grp]; p < pe; p++) {
            const unsigned b = __ballot_sync(FULL_MASK, cnt >= (int)fp.p_t[p]);
            if (lane == 0) s_planes[(NLAB + p) * EXTW + k] = b;
          }
        }
      }
    }
    __syncthreads();
  }

  // ---- rows: C_L word = label plane AND its constraint planes; written once ----
  {
    const int w = w0 + lane;
    const bool active = (lane < fp.TW) && (w < fp.W);
    const int k = w - xb;
    for (int row = wid; row < fp.VQ; row += NWARP) {
      const int rl = fp.row_lab[row];
      const int j0 = fp.row_off[row], j1 = fp.row_off[row + 1];
      if (active) {
        uint32_t x = s_planes[rl * EXTW + k];
        for (int j = j0; j < j1; j++) x &= s_planes[(NLAB + fp.row_ids[j]) * EXTW + k];
        fp.bitmap[(size_t)row * fp.Wpad + w] = x;
      }
    }
  }

  // ---- GMCR test for molecules starting in this tile ----
  M *win = s_win + (size_t)wid * (NLAB + P);
  for (int mi = wid; mi < nmol; mi += NWARP) {
    const int g = g0 + mi;
    const int gst = __ldg(&goff[g]);
    if (gst < n0) continue;  // owned by the previous tile
    const int ms = s_mstart[mi];
    const int n = s_mstart[mi + 1] - ms;
    const long long s = (long long)(gs + ms) - (long long)xb * 32;
    for (int c = lane; c < NLAB + P; c += 32) win[c] = extract_window<NW>(s_planes + (size_t)c * EXTW, nxw, s, n);
    __syncwarp();
    long long np = 0, ncm = 0;
    for (int qb = 0; qb < fp.NQW; qb++) {
      const int q = qb * 32 + lane;
      bool ok = q < fp.NQ;
      int nq = 0;
      if (ok) {
        const int r0 = fp.qgoff[q], r1 = fp.qgoff[q + 1];
        nq = r1 - r0;
        for (int row = r0; row < r1 && ok; row++) {
          M x = win[fp.row_lab[row]];
          const int j1 = fp.row_off[row + 1];
          for (int j = fp.row_off[row]; j < j1; j++) x &= win[NLAB + fp.row_ids[j]];
          ok = x.any();
        }
      }
      const unsigned bits = __ballot_sync(FULL_MASK, ok);
      if (lane == 0) fp.gm[(size_t)g * fp.NQW + qb] = bits;
      np += __popc(bits);
      int c = ok ? nq : 0;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(FULL_MASK, c, o);
      ncm += c;
    }
    if (lane == 0) {
      I64x2 v;
      v.a = np;
      v.b = ncm;
      fp.mol_cnt[g] = v;
    }
    __syncwarp();
  }
}

cudaError_t launch_filter(int NW, const FilterParams &p, int num_tiles, cudaStream_t st) {
  if (num_tiles <= 0) return cudaSuccess;
  cudaError_t e = cudaSuccess;
#define SIGMO_FILTER_CASE(K)                                                                         \
  case K:                                                                                            \
    e = cudaFuncSetAttribute(k_filter<K>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p.smem_bytes); \
    if (e != cudaSuccess) return e;                                                                  \
    k_filter<K><<<num_tiles, kFilterThreads, p.smem_bytes, st>>>(p);                                 \
    break;
  switch (NW) {
    SIGMO_FILTER_CASE(1)
    SIGMO_FILTER_CASE(2)
    SIGMO_FILTER_CASE(4)
    default: return cudaErrorInvalidValue;
  }
#undef SIGMO_FILTER_CASE
  return cudaGetLastError();
}

// ===========================================================================
// GMCR offsets: exclusive scan of (pairs, candidate-mask entries) per graph.
// ===========================================================================
struct AddI64x2 {
  __host__ __device__ __forceinline__ I64x2 operator()(const I64x2 &x, const I64x2 &y) const {
    I64x2 r;
    r.a = x.a + y.a;
    r.b = x.b + y.b;
    return r;
  }
};

cudaError_t launch_scan(const I64x2 *in, I64x2 *out, int n, void *temp, size_t *temp_bytes, cudaStream_t st) {
  I64x2 zero;
  zero.a = 0;
  zero.b = 0;
  return cub::DeviceScan::ExclusiveScan(temp, *temp_bytes, in, out, AddI64x2(), zero, n, st);
}

// ===========================================================================
// k_chunks: chunk key(g) = floor(pairs_before/PC) + floor(atoms_before/AC)
// + floor(cm_before/CMC) + floor(g/MC) is non-decreasing; chunk k is the run
// of graphs with key == k, so every chunk fits the join's smem capacities
// (PC + NQ pairs, AC + max_nodes atoms, CMC + VQ masks, MC graphs).
// ===========================================================================
__global__ void k_chunks(ChunkParams p) {
  const int g = blockIdx.x * blockDim.x + threadIdx.x;
  auto key = [&](int x) -> long long {
    const I64x2 o = p.off[x];
    return o.a / p.PC + (long long)p.goff[x] / p.AC + o.b / p.CMC + (long long)x / p.MC;
  };
  if (g == 0) {
    p.chunk_start[0] = 0;
    const long long K = (p.ND > 0) ? key(p.ND - 1) + 1 : 0;
    *p.nchunks = (int)K;
    p.chunk_start[K] = p.ND;
  } else if (g < p.ND) {
    const long long kp = key(g - 1), kg = key(g);
    for (long long k = kp + 1; k <= kg; k++) p.chunk_start[k] = g;
  }
}

cudaError_t launch_chunks(const ChunkParams &p, cudaStream_t st) {
  const int n = p.ND > 0 ? p.ND : 1;
  k_chunks<<<(n + 255) / 256, 256, 0, st>>>(p);
  return cudaGetLastError();
}

// ===========================================================================
// k_join: persistent CTAs pull molecule chunks; within a chunk, lanes pull
// (pair, root candidate) items and run an explicit-stack DFS
// over molecule-local bitsets.  Per depth e of the query's plan:
//   cand(e) = cm[e] & ~used & AND_{(j,b) in back(e)} adj_b[f(j)]
// and the last depth is counted with popc instead of being enumerated.
// ===========================================================================
struct JoinSmem {
  size_t adj, cm, cand, cnt, tot, pq, pcm, pitem, pmol, mstart, map, found, total;
};

__host__ __device__ inline JoinSmem join_layout(int NW, int NB, int ACAP, int CMCAP, int PCAP, int MCAP, int NQ,
                                                int maxq) {
  JoinSmem L;
  const size_t mb = 8 * (size_t)NW;
  const int NT = kJoinThreads;
  size_t o = 0;
  L.adj = o;    o = align16(o + mb * (size_t)NB * ACAP);
  L.cm = o;     o = align16(o + mb * (size_t)CMCAP);
  L.cand = o;   o = align16(o + mb * (size_t)maxq * NT);
  L.cnt = o;    o = align16(o + 8 * (size_t)PCAP);
  L.tot = o;    o = align16(o + 8 * (size_t)NQ);
  L.pq = o;     o = align16(o + 4 * (size_t)PCAP);
  L.pcm = o;    o = align16(o + 4 * (size_t)PCAP);
  L.pitem = o;  o = align16(o + 4 * (size_t)(PCAP + 1));
  L.pmol = o;   o = align16(o + 2 * (size_t)PCAP);
  L.mstart = o; o = align16(o + 4 * (size_t)(MCAP + 1));
  L.map = o;    o = align16(o + (size_t)maxq * NT);
  L.found = o;  o = align16(o + (size_t)PCAP);
  L.total = o;
  return L;
}

size_t join_smem_bytes(int NW, const JoinParams &p) {
  return join_layout(NW, p.NB, p.ACAP, p.CMCAP, p.PCAP, p.MCAP, p.NQ, p.maxq).total;
}

template <int NW, int MODE>
__global__ void __launch_bounds__(kJoinThreads) k_join(JoinParams jp) {
  using M = Mask<NW>;
  constexpr int NT = kJoinThreads, NWARP = NT / 32;
  extern __shared__ __align__(16) unsigned char smem[];
  const JoinSmem L = join_layout(NW, jp.NB, jp.ACAP, jp.CMCAP, jp.PCAP, jp.MCAP, jp.NQ, jp.maxq);
  M *s_adj = (M *)(smem + L.adj);
  M *s_cm = (M *)(smem + L.cm);
  M *s_cand = (M *)(smem + L.cand);
  unsigned long long *s_cnt = (unsigned long long *)(smem + L.cnt);
  unsigned long long *s_tot = (unsigned long long *)(smem + L.tot);
  int *s_pq = (int *)(smem + L.pq);
  int *s_pcm = (int *)(smem + L.pcm);
  int *s_pitem = (int *)(smem + L.pitem);
  int16_t *s_pmol = (int16_t *)(smem + L.pmol);
  int *s_mstart = (int *)(smem + L.mstart);
  uint8_t *s_map = smem + L.map;
  uint8_t *s_found = smem + L.found;
  __shared__ int s_chunk, s_next, s_warp[32];

  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int ACAP = jp.ACAP;
  for (int i = tid; i < jp.NQ; i += NT) s_tot[i] = 0ull;

  while (true) {
    __syncthreads();
    if (tid == 0) s_chunk = atomicAdd(jp.chunk_counter, 1);
    __syncthreads();
    const int c = s_chunk;
    if (c >= *jp.nchunks) break;
    const int g0 = jp.chunk_start[c], g1 = jp.chunk_start[c + 1];
    if (g0 >= g1) continue;
    const I64x2 o0 = jp.off[g0], o1 = jp.off[g1];
    const long long p0 = o0.a, c0 = o0.b;
    const int np = (int)(o1.a - p0);
    if (np == 0) continue;
    const int a0 = jp.goff[g0];
    const int na = jp.goff[g1] - a0;
    const int nm = g1 - g0;

    // ---- stage: molecule starts, bond-class adjacency masks ----
    for (int i = tid; i <= nm; i += NT) s_mstart[i] = jp.goff[g0 + i] - a0;
    for (int i = tid; i < na; i += NT) {
      const int v = a0 + i;
      const int e0 = jp.roff[v], e1 = jp.roff[v + 1];
      for (int b = 0; b < jp.NB; b++) {
        M m;
        m.clear();
        for (int e = e0; e < e1; e++) {
          const int x = jp.nbr[e];
          if (jp.bclass[x & 255] == b) m.set(x >> 8);
        }
        s_adj[b * ACAP + i] = m;
      }
    }
    // ---- stage: GMCR pairs of the chunk (warp per molecule) ----
    for (int mi = wid; mi < nm; mi += NWARP) {
      const int g = g0 + mi;
      const I64x2 og = jp.off[g];
      int run_p = (int)(og.a - p0), run_c = (int)(og.b - c0);
      for (int blk = 0; blk < jp.NQW; blk += 32) {
        const int qw = blk + lane;
        const uint32_t bits = (qw < jp.NQW) ? jp.gm[(size_t)g * jp.NQW + qw] : 0u;
        int myp = __popc(bits), myc = 0;
        for (uint32_t m = bits; m; m &= m - 1u) {
          const int q = qw * 32 + __ffs(m) - 1;
          myc += jp.qgoff[q + 1] - jp.qgoff[q];
        }
        int xp = myp, xc = myc;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int yp = __shfl_up_sync(FULL_MASK, xp, o), yc = __shfl_up_sync(FULL_MASK, xc, o);
          if (lane >= o) {
            xp += yp;
            xc += yc;
          }
        }
        int pos = run_p + xp - myp, cpos = run_c + xc - myc;
        for (uint32_t m = bits; m; m &= m - 1u) {
          const int q = qw * 32 + __ffs(m) - 1;
          s_pq[pos] = q;
          s_pmol[pos] = (int16_t)mi;
          s_pcm[pos] = cpos;
          pos++;
          cpos += jp.qgoff[q + 1] - jp.qgoff[q];
        }
        run_p += __shfl_sync(FULL_MASK, xp, 31);
        run_c += __shfl_sync(FULL_MASK, xc, 31);
      }
    }
    __syncthreads();
    // ---- stage: candidate masks of every pair (molecule window of each row) ----
    for (int i = tid; i < np; i += NT) {
      const int q = s_pq[i], mi = s_pmol[i];
      const int ms = s_mstart[mi], n = s_mstart[mi + 1] - ms;
      const long long gstart = (long long)a0 + ms;
      const int qb = jp.qgoff[q], nq = jp.qgoff[q + 1] - qb;
      const int cb = s_pcm[i];
      for (int e = 0; e < nq; e++) {
        const int row = jp.qp_row[qb + e];
        s_cm[cb + e] = extract_window<NW>(jp.bitmap + (size_t)row * jp.Wpad, jp.Wpad, gstart, n);
      }
      s_pitem[i] = s_cm[cb].popc();
      s_cnt[i] = 0ull;
      s_found[i] = 0;
    }
    __syncthreads();
    const int nitems = block_exclusive_scan<NT>(s_pitem, np, s_warp);
    if (tid == 0) s_next = 0;
    __syncthreads();

    // ---- DFS: lanes pull (pair, root) items ----
    int p = -1;
    bool exhausted = false;
    int d = 0, nq = 0, qb = 0, cmoff = 0, mbase = 0;
    M used, cset;
    used.clear();
    cset.clear();
    unsigned long long cnt = 0ull;

    auto compute = [&](int e, const M &u) -> M {
      M x = s_cm[cmoff + e].andnot(u);
      const int k1 = __ldg(&jp.qp_beoff[qb + e + 1]);
      for (int k = __ldg(&jp.qp_beoff[qb + e]); k < k1; k++) {
        const int be = __ldg(&jp.qp_be[k]);
        const int v = s_map[(be >> 8) * NT + tid];
        x &= s_adj[(be & 255) * ACAP + mbase + v];
      }
      return x;
    };
    auto finish = [&]() {
      if (cnt) {
        atomicAdd(&s_cnt[p], cnt);
        if (MODE == 1) s_found[p] = 1;
      }
      p = -1;
    };

    while (true) {
      const bool need = (p < 0) && !exhausted;
      const unsigned nmask = __ballot_sync(FULL_MASK, need);
      if (nmask) {
        const int leader = __ffs(nmask) - 1;
        int base = 0;
        if (lane == leader) base = atomicAdd(&s_next, __popc(nmask));
        base = __shfl_sync(FULL_MASK, base, leader);
        if (need) {
          const int it = base + __popc(nmask & ((1u << lane) - 1u));
          if (it >= nitems) {
            exhausted = true;
          } else {
            int lo = 0, hi = np - 1;
            while (lo < hi) {
              const int mid = (lo + hi + 1) >> 1;
              if (s_pitem[mid] <= it) lo = mid;
              else hi = mid - 1;
            }
            p = lo;
            const int k = it - s_pitem[p];
            const int q = s_pq[p];
            qb = jp.qgoff[q];
            nq = jp.qgoff[q + 1] - qb;
            cmoff = s_pcm[p];
            mbase = s_mstart[s_pmol[p]];
            M r = s_cm[cmoff];
            for (int j = 0; j < k; j++) r.clear_lowest();
            const int v0 = r.lowest();
            cnt = 0ull;
            if (MODE == 1 && s_found[p]) {
              p = -1;
            } else if (nq == 1) {
              cnt = 1ull;
              finish();
            } else {
              s_map[tid] = (uint8_t)v0;
              used = M::bit(v0);
              const M x = compute(1, used);
              if (nq == 2) {
                cnt = (unsigned long long)x.popc();
                finish();
              } else {
                d = 1;
                cset = x;
              }
            }
          }
        }
      }
      if (__ballot_sync(FULL_MASK, !exhausted) == 0u) break;
      if (p >= 0) {
        if (MODE == 1 && s_found[p]) {
          p = -1;  // another lane found this pair's first embedding
        } else if (!cset.any()) {
          if (d == 1) {
            finish();
          } else {
            d--;
            used.reset(s_map[d * NT + tid]);
            cset = s_cand[d * NT + tid];
          }
        } else {
          const int v = cset.lowest();
          cset.clear_lowest();
          s_map[d * NT + tid] = (uint8_t)v;
          M u2 = used;
          u2.set(v);
          const M x = compute(d + 1, u2);
          if (d + 1 == nq - 1) {
            cnt += (unsigned long long)x.popc();
            if (MODE == 1 && cnt) finish();
          } else if (x.any()) {
            s_cand[d * NT + tid] = cset;
            used = u2;
            d++;
            cset = x;
          }
        }
      }
    }
    __syncthreads();
    // ---- results: GMCR pair list + per-pair result + per-query totals ----
    for (int i = tid; i < np; i += NT) {
      unsigned long long r = s_cnt[i];
      if (MODE == 1) r = r ? 1ull : 0ull;
      const int q = s_pq[i];
      jp.pair_query[p0 + i] = q;
      jp.pair_result[p0 + i] = r;
      if (r) atomicAdd(&s_tot[q], r);
    }
  }
  __syncthreads();
  for (int i = tid; i < jp.NQ; i += NT)
    if (s_tot[i]) atomicAdd(&jp.totals[i], s_tot[i]);
}

template <int NW, int MODE>
static cudaError_t launch_join_t(const JoinParams &p, int grid, cudaStream_t st) {
  cudaError_t e = cudaFuncSetAttribute(k_join<NW, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)p.smem_bytes);
  if (e != cudaSuccess) return e;
  k_join<NW, MODE><<<grid, kJoinThreads, p.smem_bytes, st>>>(p);
  return cudaGetLastError();
}

cudaError_t launch_join(int NW, int mode, const JoinParams &p, int grid, cudaStream_t st) {
  if (grid <= 0) return cudaSuccess;
  switch (NW * 2 + mode) {
    case 2: return launch_join_t<1, 0>(p, grid, st);
    case 3: return launch_join_t<1, 1>(p, grid, st);
    case 4: return launch_join_t<2, 0>(p, grid, st);
    case 5: return launch_join_t<2, 1>(p, grid, st);
    case 8: return launch_join_t<4, 0>(p, grid, st);
    case 9: return launch_join_t<4, 1>(p, grid, st);
    default: return cudaErrorInvalidValue;
  }
}

int join_blocks_per_sm(int NW, int mode, size_t smem) {
  int n = 0;
  cudaError_t e = cudaSuccess;
  switch (NW * 2 + mode) {
    case 2:
      cudaFuncSetAttribute(k_join<1, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_join<1, 0>, kJoinThreads, smem);
      break;
    case 3:
      cudaFuncSetAttribute(k_join<1, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_join<1, 1>, kJoinThreads, smem);
      break;
    case 4:
      cudaFuncSetAttribute(k_join<2, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_join<2, 0>, kJoinThreads, smem);
      break;
    case 5:
      cudaFuncSetAttribute(k_join<2, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_join<2, 1>, kJoinThreads, smem);
      break;
    case 8:
      cudaFuncSetAttribute(k_join<4, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_join<4, 0>, kJoinThreads, smem);
      break;
    case 9:
      cudaFuncSetAttribute(k_join<4, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_join<4, 1>, kJoinThreads, smem);
      break;
    default: return 1;
  }
  if (e != cudaSuccess || n < 1) return 1;
  return n;
}

}  // namespace sigmo
