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

#include <type_traits>

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
    if (NW == 1) {
      // branch-free count of trailing zeros (w != 0 assumed by callers; 64 if 0 -> -1)
      const unsigned long long x = w[0];
      const int t = __popcll((x & (0ull - x)) - 1ull);
      return x ? t : -1;
    }
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
// skip0: wildcard query batches (R22) -- a label-0 atom ('*') adds
// to no field of the other atoms' counts
__global__ void __launch_bounds__(128) k_sig_counts(DevGraphs g, int R, uint8_t *counts,
                                                    unsigned long long *packed, int pack_radius, int skip0) {
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
    if (!(skip0 && g.label[base + i] == 0)) atomicOr(&s_fm[s_fid[i]].w[i >> 6], 1ull << (i & 63));
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
        // the node itself is not counted (u != v); a skipped wildcard is in no field mask
        int c = (cur[i] & s_fm[f]).popc() - ((s_fid[i] == f && !(skip0 && g.label[base + i] == 0)) ? 1 : 0);
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

cudaError_t launch_sig_counts(const DevGraphs &g, int R, uint8_t *counts, int skip0, cudaStream_t st) {
  if (g.num_graphs == 0 || R <= 0) return cudaSuccess;
  k_sig_counts<<<g.num_graphs, 128, 0, st>>>(g, R, counts, nullptr, 0, skip0);
  return cudaGetLastError();
}

cudaError_t launch_sig_pack(const DevGraphs &g, int radius, unsigned long long *out, int skip0, cudaStream_t st) {
  if (g.num_graphs == 0) return cudaSuccess;
  k_sig_counts<<<g.num_graphs, 128, 0, st>>>(g, radius, nullptr, out, radius, skip0);
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
                                                                   const uint8_t *qc, QueryProg prog, int wild) {
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
  // label planes of the query labels; a wildcard atom ('*', label 0; R22) has
  // none -- its row starts from the all-ones channel NLAB
  for (int v = tid; v < VQ; v += NT)
    if (!(wild && qlabel[v] == 0)) atomicOr(&s_lab[qlabel[v] >> 5], 1u << (qlabel[v] & 31));
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
    prog.row_lab[v] = (wild && l == 0) ? (uint8_t)prog.d_meta->NLAB
                                       : (uint8_t)(s_labrank[l >> 5] + __popc(s_lab[l >> 5] & ((1u << (l & 31)) - 1u)));
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

cudaError_t launch_query_prep(const DevGraphs &q, int R, const uint8_t *qcounts, QueryProg &prog, int wild,
                              cudaStream_t st) {
  k_query_prep<<<1, kQueryPrepThreads, 0, st>>>(q.num_nodes, R, q.label, qcounts, prog, wild);
  return cudaGetLastError();
}

// ===========================================================================
// k_filter: one CTA per tile of TW (<= 32) bitmap words = 32*TW data nodes.
// Plane words are stored word-major (s_pl[k * PS + channel], PS odd), so the
// rows phase (lane = word) reads them without bank conflicts and the plane
// phase (warp = word) writes them with immediate offsets.
// ===========================================================================
struct FilterSmem {
  size_t nb, ballA, ballB, fm, pl, fpl, memb, win, nz, gmb, slotat, endb, own, molstart, molslot, loc, fid, lab, mstart,
      sos, grec, tab, bdone, rowpoff, rowp, dnz, qdr, stg, total;
};

__host__ __device__ inline size_t align16(size_t x) { return (x + 15) & ~(size_t)15; }
__host__ __device__ inline int plane_stride(int NLAB, int P) { return (NLAB + 1 + P) | 1; }

__host__ __device__ inline FilterSmem filter_layout(int NW, int EXTN, int EXTW, int MOLCAP, int NFU, int NLAB,
                                                    int P, int NREC, int VQ, int NRP, int rows_smem, int NQW,
                                                    int TS, int mol = 0, int NDR = 0, int NQ = 0, int NQWL = 0) {
  FilterSmem L;
  const size_t mb = 8 * (size_t)NW;
  const int NWARP = kFilterThreads / 32;
  const int VQW = (VQ + 31) / 32;
  const int NCH = NLAB + 1 + P;
  size_t o = 0;
  L.nb = o;       o = align16(o + 4 * (size_t)EXTN);
  L.ballA = o;    o = align16(o + mb * EXTN);
  L.ballB = o;    o = align16(o + (NW == 1 ? 0 : mb * EXTN));  // NW == 1: in-place BFS via registers
  L.fm = o;       o = align16(o + mb * (size_t)MOLCAP * (NFU > 0 ? NFU : 1));
  L.pl = o;       o = align16(o + 4 * (size_t)plane_stride(NLAB, P) * EXTW);
  L.fpl = o;      o = align16(o + 4 * (size_t)(NFU > 0 ? NFU : 1) * EXTW);
  L.memb = o;     o = align16(o + 4 * 32 * (size_t)EXTW);
  // window path (dense tiles): per warp one molecule's channel windows
  L.win = o;      o = align16(o + mb * (size_t)(mol ? 0 : NWARP) * NCH);
  L.nz = o;       o = align16(o + (mol ? 0 : 4 * (size_t)NWARP * (VQW + 1)));
  L.gmb = o;      o = align16(o + 4 * (size_t)MOLCAP * (NQW > 0 ? NQW : 1));
  L.slotat = o;   o = align16(o + (mol ? 0 : 2 * 32 * 32));
  L.endb = o;     o = align16(o + 4 * 32);
  L.own = o;      o = align16(o + 4 * 32);
  L.molstart = o; o = align16(o + 2 * (size_t)EXTN);
  L.molslot = o;  o = align16(o + 2 * (size_t)EXTN);
  L.loc = o;      o = align16(o + (size_t)EXTN);
  L.fid = o;      o = align16(o + (size_t)EXTN);
  L.lab = o;      o = align16(o + (size_t)EXTN);
  L.mstart = o;   o = align16(o + 4 * (size_t)(MOLCAP + 1));
  // start-of-segment slots: used while loading the tile, before the plane
  // phase writes memb (molecule tiles: alias memb)
  if (mol && 2 * (size_t)EXTN <= 4 * 32 * (size_t)EXTW) {
    L.sos = L.memb;
  } else {
    L.sos = o; o = align16(o + 2 * (size_t)EXTN);
  }
  L.grec = o;     o = align16(o + sizeof(GroupRec) * (size_t)(NREC > 0 ? NREC : 1));
  L.tab = o;      o = align16(o + 4 * (size_t)TS * (NREC > 0 ? NREC : 1));
  L.bdone = o;    o = align16(o + (size_t)(P / 32 + 1));
  L.rowpoff = o;  o = align16(o + (rows_smem && !mol ? 4 * (size_t)(VQ + 1) : 0));
  L.rowp = o;     o = align16(o + (rows_smem ? 4 * (size_t)NRP : 0));
  // molecule tiles, rows phase only: non-empty bits of the distinct rows
  // [NDR/32][32 molecules], the per-query GMCR lists, the store staging (4
  // rows x 33 per warp).  They live after the plane phase, so they alias the
  // BFS arrays (nb, balls) and the plane-batch carry words (memb) when they fit
  if (mol) {
    const size_t dnz_b = align16(4 * (size_t)32 * ((NDR + 31) / 32));
    const size_t qdr_b = align16(align16(4 * (size_t)(NQ + 1)) + 8 * (size_t)NQWL);
    const size_t stg_b = align16(8 * (size_t)NWARP * 4 * 33);
    if (stg_b <= L.fm - L.nb) {  // nb + ballA (+ ballB) are contiguous
      L.stg = L.nb;
    } else {
      L.stg = o; o = align16(o + stg_b);
    }
    if (dnz_b + qdr_b <= 4 * 32 * (size_t)EXTW) {
      L.dnz = L.memb;
      L.qdr = L.memb + dnz_b;
    } else {
      L.dnz = o; o = align16(o + dnz_b);
      L.qdr = o; o = align16(o + qdr_b);
    }
  } else {
    L.dnz = L.qdr = L.stg = o;
  }
  L.total = o;
  return L;
}

size_t filter_smem_bytes(int NW, int EXTN, int EXTW, int MOLCAP, int NFU, int NLAB, int P, int NREC, int VQ, int NRP,
                         int rows_smem, int NQW, int TS, int mol, int NDR, int NQ, int NQWL) {
  return filter_layout(NW, EXTN, EXTW, MOLCAP, NFU, NLAB, P, NREC, VQ, NRP, rows_smem, NQW, TS, mol, NDR, NQ, NQWL).total;
}

// 32x32 bit-matrix transpose across the warp: lane L holds row L (bit p =
// element (L, p)); returns column `lane` (bit L = element (L, lane)).  Each of
// the five stages exchanges bit j of the row index with bit j of the column
// index.
__device__ __forceinline__ uint32_t transpose32(uint32_t x, int lane) {
#pragma unroll
  for (int j = 16; j >= 1; j >>= 1) {
    const uint32_t m = j == 16 ? 0x0000ffffu : j == 8 ? 0x00ff00ffu : j == 4 ? 0x0f0f0f0fu : j == 2 ? 0x33333333u
                                                                                                     : 0x55555555u;
    const uint32_t sw = ((x << j) & ~m) | ((x >> j) & m);
    const uint32_t y = __shfl_xor_sync(FULL_MASK, sw, j);
    const uint32_t K = (lane & j) ? ~m : m;
    x = (x & K) | (y & ~K);
  }
  return x;
}

// extract_window over one channel of the word-major plane array
template <int NW>
__device__ __forceinline__ Mask<NW> extract_window_strided(const uint32_t *words, int stride, long long nw,
                                                           long long s, int n) {
  Mask<NW> m;
#pragma unroll
  for (int k = 0; k < NW; k++) {
    long long b = s + 64ll * k;
    long long wi = b >> 5;
    int sh = (int)(b & 31);
    unsigned long long w0 = (wi < nw) ? words[wi * stride] : 0u;
    unsigned long long w1 = (wi + 1 < nw) ? words[(wi + 1) * stride] : 0u;
    unsigned long long w2 = (wi + 2 < nw) ? words[(wi + 2) * stride] : 0u;
    unsigned long long x = (w0 | (w1 << 32)) >> sh;
    if (sh) x |= w2 << (64 - sh);
    int rem = n - 64 * k;
    if (rem <= 0) x = 0ull;
    else if (rem < 64) x &= (1ull << rem) - 1ull;
    m.w[k] = x;
  }
  return m;
}

// MOL: molecule tiles (32 consecutive data graphs per CTA, <= 64 nodes each)
// writing the molecule-padded candidate layout cmol[g][row] (u64 window of
// graph g in the row of query node `row`; a pair's rows are contiguous), used
// by k_join_lane.  Otherwise
// dense tiles of TW words writing the row-major bitmap.
template <int NW, bool MOL>
__global__ void __launch_bounds__(kFilterThreads, MOL ? 5 : 4) k_filter(const __grid_constant__ FilterParams fp) {
  using M = Mask<NW>;
  constexpr int NT = kFilterThreads, NWARP = NT / 32;
  extern __shared__ __align__(16) unsigned char smem[];
  const FilterSmem L = filter_layout(NW, fp.EXTN, fp.EXTW, fp.MOLCAP, fp.NFU, fp.NLAB, fp.P, fp.NREC, fp.VQ, fp.NRP,
                                     fp.rows_smem, fp.NQW, fp.TS, MOL ? 1 : 0, fp.NDR, fp.NQ, fp.NQWL);
  uint32_t *s_nb = (uint32_t *)(smem + L.nb);
  M *s_cur = (M *)(smem + L.ballA);
  M *s_nxt = (M *)(smem + L.ballB);
  M *s_fm = (M *)(smem + L.fm);
  uint32_t *s_pl = (uint32_t *)(smem + L.pl);
  uint32_t *s_fpl = (uint32_t *)(smem + L.fpl);
  uint32_t *s_memb = (uint32_t *)(smem + L.memb);
  M *s_win = (M *)(smem + L.win);
  uint32_t *s_nz = (uint32_t *)(smem + L.nz);
  uint32_t *s_gm = (uint32_t *)(smem + L.gmb);
  int16_t *s_slotat = (int16_t *)(smem + L.slotat);
  uint32_t *s_endb = (uint32_t *)(smem + L.endb);
  uint32_t *s_own = (uint32_t *)(smem + L.own);
  int16_t *s_molstart = (int16_t *)(smem + L.molstart);
  int16_t *s_molslot = (int16_t *)(smem + L.molslot);
  uint8_t *s_loc = smem + L.loc;
  uint8_t *s_fid = smem + L.fid;
  uint8_t *s_lab = smem + L.lab;
  int *s_mstart = (int *)(smem + L.mstart);
  int16_t *s_sos = (int16_t *)(smem + L.sos);
  GroupRec *s_grec = (GroupRec *)(smem + L.grec);
  uint32_t *s_tab = (uint32_t *)(smem + L.tab);
  uint8_t *s_bdone = smem + L.bdone;
  __shared__ int s_g0, s_g1, s_strad;
  __shared__ unsigned s_cwb[33];  // molecule tiles: cmol word base of each molecule (bit 31: 64-bit windows)
  __shared__ int s_rrec[kMaxRadius + 1];
  __shared__ int s_rcarry[kMaxRadius];
  __shared__ uint8_t s_fused[kNumFields];
  __shared__ int8_t s_fslot[kNumFields];
  __shared__ uint8_t s_labval[256];
  __shared__ uint8_t s_labch[256];

  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int ND = fp.D.num_graphs, VD = fp.D.num_nodes;
  const int w0 = MOL ? 0 : blockIdx.x * fp.TW;
  if (!MOL && w0 >= fp.W) return;
  const int n0 = w0 * 32;
  const int n1 = MOL ? 0 : min(n0 + fp.TW * 32, VD);
  const int32_t *goff = fp.D.goff;
  const int NLAB = fp.NLAB, NFU = fp.NFU, EXTW = fp.EXTW;
  const int PS = plane_stride(NLAB, fp.P);
  if (tid == 0) {
    if (MOL) {
      s_g0 = __ldg(&fp.mtile[blockIdx.x]);
      s_g1 = __ldg(&fp.mtile[blockIdx.x + 1]);
    } else if (fp.tile_g0) {
      s_g0 = __ldg(&fp.tile_g0[blockIdx.x]);
      s_g1 = __ldg(&fp.tile_g1[blockIdx.x]);
    } else {
      s_g0 = graph_of(goff, ND, n0);
      s_g1 = graph_of(goff, ND, n1 - 1) + 1;
    }
    s_strad = -1;
  }
  {
    const int4 *src = (const int4 *)fp.grec;
    int4 *dst = (int4 *)s_grec;
    for (int i = tid; i < fp.NREC; i += NT) dst[i] = __ldg(&src[i]);
    const uint4 *ts = (const uint4 *)fp.tab;
    uint4 *td = (uint4 *)s_tab;
    for (int i = tid; i < fp.NREC * fp.TS / 4; i += NT) td[i] = __ldg(&ts[i]);
  }
  for (int i = tid; i < fp.NBATCH; i += NT) s_bdone[i] = (uint8_t)fp.bdone[i];
  for (int i = tid; i <= fp.R; i += NT) s_rrec[i] = fp.rrec_off[i];
  for (int i = tid; i < fp.R; i += NT) s_rcarry[i] = fp.rcarry[i];
  for (int i = tid; i < 256; i += NT) s_labch[i] = 0xff;
  for (int i = tid; i < NLAB; i += NT) s_labval[i] = fp.lab_val[i];
  for (int i = tid; i < kNumFields; i += NT) {
    s_fslot[i] = fp.fslot[i];
    if (fp.fslot[i] >= 0) s_fused[fp.fslot[i]] = (uint8_t)i;
  }
  if (fp.rows_smem) {
    int32_t *b = (int32_t *)(smem + L.rowpoff);
    uint32_t *c = (uint32_t *)(smem + L.rowp);
    if (!MOL)
      for (int i = tid; i <= fp.VQ; i += NT) b[i] = fp.rowp_off[i];
    for (int i = tid; i < fp.NRP; i += NT) c[i] = fp.rowp[i];
  }
  if (tid < 32) {
    s_endb[tid] = 0u;
    s_own[tid] = 0u;
  }
  __syncthreads();
  const int g0 = s_g0, g1 = s_g1, nmol = g1 - g0;
  const int gs = __ldg(&goff[g0]);
  const int ge = __ldg(&goff[g1]);
  const int next = ge - gs;
  // node i (relative to gs) sits at bit (xo - gs + i) of the ext words; dense
  // tiles use the global 32-bit word grid, molecule tiles start at gs
  const int xb = gs >> 5;                       // first ext word (global word index, dense)
  const int xo = MOL ? gs : xb * 32;
  const int nxw = MOL ? (next + 31) >> 5 : ((ge - 1) >> 5) - xb + 1;  // ext words
  const int tw_eff = min(fp.TW, fp.W - w0);     // words written by this tile
  const int tbits = 32 * tw_eff;

  // ---- phase 1: molecules and nodes overlapping the tile ----
  for (int i = tid; i < nmol * fp.NQW; i += NT) s_gm[i] = 0u;
  for (int i = tid; i <= nmol; i += NT) {
    const int st = __ldg(&goff[g0 + i]) - gs;
    s_mstart[i] = st;
    if (MOL && i < nmol) {
      const int n = __ldg(&goff[g0 + i + 1]) - gs - st;
      s_cwb[i] = ((unsigned)fp.NDR * __ldg(&fp.cand_units[g0 + i])) | (n > 32 ? 0x80000000u : 0u);
    }
    if (i < nmol) {
      const int n = __ldg(&goff[g0 + i + 1]) - gs - st;
      const int tb = gs + st - n0;  // tile bit of the molecule's first node
      const int te = tb + n - 1;    // ... and of its last node
      if (n > 0 && !MOL) {
        if (te >= 0 && te < tbits) atomicOr(&s_endb[te >> 5], 1u << (te & 31));  // segment end
        if (tb >= 0 && tb < tbits) {  // starts here: this tile owns its GMCR bits
          if (te < tbits && NW == 1) {
            atomicOr(&s_own[te >> 5], 1u << (te & 31));
            s_slotat[te] = (int16_t)i;
          } else {
            s_strad = i;  // ends beyond the tile (or needs the multi-word path)
          }
        }
      }
    }
  }
  for (int i = tid; i < next; i += NT) {
    const int v = gs + i;
    const int loc = __ldg(&fp.D.local[v]);
    const int e0 = __ldg(&fp.D.roff[v]), e1 = __ldg(&fp.D.roff[v + 1]);
    // up to 4 neighbours packed (unused slots = the node itself: OR-neutral)
    uint32_t nb = (uint32_t)loc * 0x01010101u;
    if (e1 - e0 <= 4)
      for (int e = e0; e < e1; e++) {
        const int sh = 8 * (e - e0);
        nb = (nb & ~(0xffu << sh)) | ((uint32_t)(__ldg(&fp.D.nbr[e]) >> 8) << sh);
      }
    s_nb[i] = nb;
    s_cur[i] = M::bit(loc);
    s_molstart[i] = (int16_t)(i - loc);
    s_loc[i] = (uint8_t)loc;
    const int lab = __ldg(&fp.D.label[v]);
    s_lab[i] = (uint8_t)lab;
    s_fid[i] = (uint8_t)(field_of(lab) | (e1 - e0 > 4 ? 0x80 : 0));
  }
  __syncthreads();
  for (int mi = tid; mi < nmol; mi += NT)
    if (s_mstart[mi] < s_mstart[mi + 1]) s_sos[s_mstart[mi]] = (int16_t)mi;
  for (int c = tid; c < NLAB; c += NT) s_labch[s_labval[c]] = (uint8_t)c;
  __syncthreads();
  // ---- label planes (InitializeCandidates, Alg.1 l.29-37) and field planes:
  // lane = node builds its one-hot membership word, a warp transpose turns
  // it into plane words (lane = channel) ----
  const bool onehot_fits = NLAB + 1 + NFU <= 32;
  for (int k = wid; k < nxw; k += NWARP) {
    const int i = xo + k * 32 + lane - gs;
    const bool valid = (i >= 0) && (i < next);
    const int lab = valid ? s_lab[i] : -1;
    const int fid = valid ? (s_fid[i] & 0x7f) : -1;
    uint32_t *plw = s_pl + (size_t)k * PS;
    if (onehot_fits) {
      uint32_t mb = 0u;
      if (valid) {
        const int lc = s_labch[lab];
        const int fs = s_fslot[fid];
        if (lc != 0xff) mb |= 1u << lc;
        if (fs >= 0) mb |= 1u << (NLAB + 1 + fs);
      }
      const uint32_t T = transpose32(mb, lane);
      const uint32_t vw = __ballot_sync(FULL_MASK, valid);  // channel NLAB: existing nodes (wildcard rows, R22)
      if (lane < NLAB) plw[lane] = T;
      else if (lane == NLAB) plw[NLAB] = vw;
      else if (lane < NLAB + 1 + NFU) s_fpl[(lane - NLAB - 1) * EXTW + k] = T;
    } else {
      for (int c = 0; c < NLAB; c++) {
        const unsigned b = __ballot_sync(FULL_MASK, lab == (int)s_labval[c]);
        if (lane == 0) plw[c] = b;
      }
      const uint32_t vw = __ballot_sync(FULL_MASK, valid);
      if (lane == 0) plw[NLAB] = vw;
      for (int fs = 0; fs < NFU; fs++) {
        const unsigned b = __ballot_sync(FULL_MASK, fid == (int)s_fused[fs]);
        if (lane == 0) s_fpl[fs * EXTW + k] = b;
      }
    }
  }
  __syncthreads();
  // per-molecule field masks = windows of the field planes
  for (int t = tid; t < nmol * NFU; t += NT) {
    const int mi = t / NFU, fs = t - mi * NFU;
    const int ms = s_mstart[mi], n = s_mstart[mi + 1] - ms;
    s_fm[t] = extract_window<NW>(s_fpl + (size_t)fs * EXTW, nxw, (long long)(gs + ms) - (long long)xo, n);
  }
  for (int i = tid; i < next; i += NT) s_molslot[i] = s_sos[s_molstart[i]];
  __syncthreads();

  // ---- radii 1..R: bitset BFS + threshold planes (RefineCandidates, l.19-28) ----
  auto bfs_node = [&](int i) -> M {  // ball_r(v) = ball_{r-1}(v) | OR_{u in N(v)} ball_{r-1}(u)
    M x = s_cur[i];
    const int ms = s_molstart[i];
    if (!(s_fid[i] & 0x80)) {
      const uint32_t nb = s_nb[i];
      x |= s_cur[ms + (nb & 0xff)];
      x |= s_cur[ms + ((nb >> 8) & 0xff)];
      x |= s_cur[ms + ((nb >> 16) & 0xff)];
      x |= s_cur[ms + (nb >> 24)];
    } else {
      const int v = gs + i;
      const int e1 = __ldg(&fp.D.roff[v + 1]);
      for (int e = __ldg(&fp.D.roff[v]); e < e1; e++) x |= s_cur[ms + (__ldg(&fp.D.nbr[e]) >> 8)];
    }
    return x;
  };
  for (int r = 1; r <= fp.R; r++) {
    if (NW == 1) {
      // in place: all new balls are computed into registers before any is written
      // EXTN <= 32 * TW + 2 * 63 (dense) or 1,024 (molecule tiles) for <= 64-node graphs
      constexpr int kIt = MOL ? (1024 + NT - 1) / NT : (1024 + 2 * 63 + NT - 1) / NT;
      M tmp[kIt];
#pragma unroll
      for (int it = 0; it < kIt; it++) {
        const int i = tid + it * NT;
        if (i < next) tmp[it] = bfs_node(i);
      }
      __syncthreads();
#pragma unroll
      for (int it = 0; it < kIt; it++) {
        const int i = tid + it * NT;
        if (i < next) s_cur[i] = tmp[it];
      }
    } else {
      for (int i = tid; i < next; i += NT) s_nxt[i] = bfs_node(i);
      __syncthreads();
      M *t = s_cur;
      s_cur = s_nxt;
      s_nxt = t;
    }
    __syncthreads();
    const int r0 = r - 1;
    const int rb = s_rrec[r0], re = s_rrec[r0 + 1];
    if (rb < re) {
      const int TSm = fp.TS - 1;
      const bool carry = s_rcarry[r0] != 0;
      for (int k = wid; k < nxw; k += NWARP) {
        const int i = xo + k * 32 + lane - gs;
        const bool valid = (i >= 0) && (i < next);
        M ball;
        ball.clear();
        const M *fmb = s_fm;
        if (valid) {
          ball = s_cur[i];
          ball.reset(s_loc[i]);  // the node itself is not counted (u != v)
          fmb = s_fm + (size_t)s_molslot[i] * NFU;
        }
        uint32_t *plw = s_pl + (size_t)k * PS + NLAB + 1;
        // membership word of the current 32-plane batch: bit (p % 32) = [count >= t_p]
        uint32_t mb = carry ? s_memb[k * 32 + lane] : 0u;
        int cur_b = s_grec[rb].batch;
        for (int rec = rb; rec < re; rec++) {  // (r, f) group parts sorted by batch
          const GroupRec g = s_grec[rec];
          if (g.batch != cur_b) {
            const uint32_t T = transpose32(mb, lane);
            if (32 * cur_b + lane < fp.P) plw[32 * cur_b + lane] = T;
            mb = 0u;
            cur_b = g.batch;
          }
          const int pc = (ball & fmb[g.fslot]).popc();
          const int c = NW == 1 ? pc : min(pc, TSm);  // <= 64-node graphs: pc <= 63 < TS
          mb |= s_tab[g.toff + c];
        }
        if (s_bdone[cur_b] == r0) {
          const uint32_t T = transpose32(mb, lane);
          if (32 * cur_b + lane < fp.P) plw[32 * cur_b + lane] = T;
        } else {
          s_memb[k * 32 + lane] = mb;  // the batch continues at the next radius
        }
      }
    }
    __syncthreads();
  }

  if (MOL) {
    // ---- molecule tiles: rows in the word domain (lane = 32-node word k of
    // the tile, C_L word = AND of the row's plane words, as in the dense
    // path), then lane = molecule gathers its <= 3 words by shuffles and
    // writes its window once to cmol[g][row]; GMCR: every row
    // of the query non-empty ----
    const int mi = lane;
    const bool valid = mi < nmol;
    const int ms = valid ? s_mstart[mi] : 0;
    const int n = valid ? s_mstart[mi + 1] - ms : 0;
    const unsigned long long nmask = n >= 64 ? ~0ull : ((1ull << n) - 1ull);
    const int ws = ms >> 5, sh = ms & 31;
    uint32_t *dnz = (uint32_t *)(smem + L.dnz);  // [NDR/32][32 molecules]
    {  // these regions alias the BFS / plane-carry arrays, dead from here on
      int32_t *qwo = (int32_t *)(smem + L.qdr);
      uint2 *qw = (uint2 *)(smem + L.qdr + align16(4 * (size_t)(fp.NQ + 1)));
      for (int i = tid; i < 32 * ((fp.NDR + 31) >> 5); i += NT) dnz[i] = 0u;
      for (int i = tid; i <= fp.NQ; i += NT) qwo[i] = __ldg(&fp.qw_off[i]);
      for (int i = tid; i < fp.NQWL; i += NT) qw[i] = make_uint2(__ldg(&fp.qw[2 * i]), __ldg(&fp.qw[2 * i + 1]));
    }
    __syncthreads();
    // per warp: 4 rows x 32 molecules of windows, staged so that the stores
    // to cmol[g][row] (molecule-major) go out as 32-B sectors per molecule
    unsigned long long *stg = (unsigned long long *)(smem + L.stg) + (size_t)wid * (4 * 33);
    // tiles hold <= 1,024 nodes: nxw <= 32 words, one per lane
    auto mol_rows = [&](auto RWc, const uint32_t *rowp, auto GLc) {
      constexpr int RWk = decltype(RWc)::value;
      constexpr bool GL = decltype(GLc)::value;  // row programs in global memory (read-only path)
      const int RW = RWk ? RWk : fp.RW;
      const unsigned char *pl0 = (const unsigned char *)(s_pl + (size_t)(lane < nxw ? lane : 0) * PS);
      for (int rb = 4 * wid; rb < fp.NDR; rb += 4 * NWARP) {  // blocks of 4 rows per warp
      const int nr = min(4, fp.NDR - rb);
      uint32_t nzb = 0u;
      for (int r = 0; r < nr; r++) {
        const int row = rb + r;
        const uint32_t *pr = rowp + (size_t)row * RW;
        uint32_t x0 = 0xffffffffu;
#pragma unroll
        for (int j = 0; j < (RWk ? RWk : 1); j++) {
          const uint32_t two = GL ? __ldg(&pr[j]) : pr[j];
          x0 &= *(const uint32_t *)(pl0 + (two & 0xffffu)) & *(const uint32_t *)(pl0 + (two >> 16));
        }
        for (int j = RWk; j < RW; j++) {
          const uint32_t two = GL ? __ldg(&pr[j]) : pr[j];
          x0 &= *(const uint32_t *)(pl0 + (two & 0xffffu)) & *(const uint32_t *)(pl0 + (two >> 16));
        }
        const uint32_t w0 = __shfl_sync(FULL_MASK, x0, ws);
        const uint32_t w1 = __shfl_sync(FULL_MASK, x0, (ws + 1) & 31);
        const uint32_t w2 = __shfl_sync(FULL_MASK, x0, (ws + 2) & 31);
        const unsigned long long x =
            (((unsigned long long)__funnelshift_r(w1, w2, sh) << 32) | __funnelshift_r(w0, w1, sh)) & nmask;
        stg[r * 33 + mi] = x;
        nzb |= (x != 0ull ? 1u : 0u) << r;
      }
      if (valid && nzb) atomicOr(&dnz[(rb >> 5) * 32 + mi], nzb << (rb & 31));  // rb % 4 == 0: one word
      __syncwarp();
#pragma unroll
      for (int k = 0; k < 4; k++) {  // lane = (molecule, row): 8 molecules x 4 rows per store
        const int e = k * 32 + lane, m = e >> 2, r = e & 3;
        if (m < nmol && r < nr) {
          const unsigned b = s_cwb[m];
          if (b & 0x80000000u)
            *(unsigned long long *)(fp.cmol + (b & 0x7fffffffu) + 2u * (unsigned)(rb + r)) = stg[r * 33 + m];
          else
            fp.cmol[b + (unsigned)(rb + r)] = (uint32_t)stg[r * 33 + m];
        }
      }
      __syncwarp();
      }
    };
    if (fp.rows_smem) {
      const uint32_t *rs = (const uint32_t *)(smem + L.rowp);
      switch (fp.RW) {
        case 1: mol_rows(std::integral_constant<int, 1>{}, rs, std::false_type{}); break;
        case 2: mol_rows(std::integral_constant<int, 2>{}, rs, std::false_type{}); break;
        case 3: mol_rows(std::integral_constant<int, 3>{}, rs, std::false_type{}); break;
        case 4: mol_rows(std::integral_constant<int, 4>{}, rs, std::false_type{}); break;
        default: mol_rows(std::integral_constant<int, 0>{}, rs, std::false_type{}); break;
      }
    } else {  // row programs read through the read-only cache (warp-uniform loads)
      const uint32_t *rg = fp.rowp;
      switch (fp.RW) {
        case 2: mol_rows(std::integral_constant<int, 2>{}, rg, std::true_type{}); break;
        case 3: mol_rows(std::integral_constant<int, 3>{}, rg, std::true_type{}); break;
        case 4: mol_rows(std::integral_constant<int, 4>{}, rg, std::true_type{}); break;
        default: mol_rows(std::integral_constant<int, 0>{}, rg, std::true_type{}); break;
      }
    }
    __syncthreads();
    // GMCR: lane = molecule, warp per query: every node's distinct row
    // non-empty = each (word, bits) entry of the query's list fully set
    const int32_t *qwo = (const int32_t *)(smem + L.qdr);
    const uint2 *qwl = (const uint2 *)(smem + L.qdr + align16(4 * (size_t)(fp.NQ + 1)));
    for (int q = wid; q < fp.NQ && valid; q += NWARP) {
      bool all = true;
      const int k1 = qwo[q + 1];
      for (int k = qwo[q]; k < k1; k++) {
        const uint2 wm = qwl[k];
        all = all && (dnz[wm.x * 32 + mi] & wm.y) == wm.y;
      }
      if (all) atomicOr(&s_gm[mi * fp.NQW + (q >> 5)], 1u << (q & 31));
    }
  }

  // ---- rows (query-major): C_L word = AND of the row's channels, written
  // once; GMCR of the molecules contained in the tile from the row words:
  // per-segment any by a carry chain (segments end at end bits E), the
  // segment that continues from the previous word(s) by a ballot ----
  // RWc: compile-time row width (0 = runtime fp.RW)
  auto rows_phase = [&](auto RWc, const uint32_t *rowp) {
    constexpr int RWk = decltype(RWc)::value;
    const int RW = RWk ? RWk : fp.RW;
    const int w = w0 + lane;
    const bool active = lane < tw_eff;
    const int k = active ? w - xb : 0;
    const unsigned char *plk = (const unsigned char *)(s_pl + (size_t)k * PS);
    const uint32_t E = s_endb[lane], OWN = s_own[lane];
    const uint32_t m = ~E;
    const uint32_t above = E ? ((0xffffffffu << (31 - __clz(E))) << 1) : 0xffffffffu;  // bits above the last end
    const uint32_t firstE = E & (0u - E);
    const uint32_t NoE = __ballot_sync(FULL_MASK, active && E == 0u);
    const int lsh = lane > 0 ? lane - 1 : 31;  // lane 0: no continuation into word 0 is needed
    const uint32_t firstE0 = lane > 0 ? firstE : 0u;
    const size_t Wpad = fp.Wpad;
    for (int q = wid; q < fp.NQ; q += NWARP) {
      const int r0 = __ldg(&fp.qgoff[q]), r1 = __ldg(&fp.qgoff[q + 1]);
      uint32_t Aq = 0xffffffffu;
      uint32_t *bp = fp.bitmap + (size_t)r0 * Wpad + w;
      const uint32_t *pr = rowp + (size_t)r0 * RW;
      for (int row = r0; row < r1; row++, bp += Wpad, pr += RW) {
        uint32_t x = 0xffffffffu;
        if (RWk) {
#pragma unroll
          for (int j = 0; j < (RWk ? RWk : 1); j++) {
            const uint32_t two = pr[j];
            x &= *(const uint32_t *)(plk + (two & 0xffffu)) & *(const uint32_t *)(plk + (two >> 16));
          }
        } else {
          for (int j = 0; j < RW; j++) {
            const uint32_t two = pr[j];
            x &= *(const uint32_t *)(plk + (two & 0xffffu)) & *(const uint32_t *)(plk + (two >> 16));
          }
        }
        if (active) *bp = x;
        if (NW == 1) {
          uint32_t A = (((x & m) + m) | x) & E;
          const uint32_t H = __ballot_sync(FULL_MASK, (x & above) != 0u);
          const uint32_t G = H | ((H << 1) & NoE);
          A |= ((G >> lsh) & 1u) ? firstE0 : 0u;
          Aq &= A;
        }
      }
      if (NW == 1) {
        uint32_t bits = Aq & OWN;
        while (bits) {
          const int b = __ffs(bits) - 1;
          bits &= bits - 1u;
          const int mi = s_slotat[lane * 32 + b];
          atomicOr(&s_gm[mi * fp.NQW + (q >> 5)], 1u << (q & 31));
        }
      }
    }
  };
  if (!MOL) {
    const uint32_t *rp = fp.rows_smem ? (const uint32_t *)(smem + L.rowp) : fp.rowp;
    if (fp.rows_smem) {
      switch (fp.RW) {
        case 1: rows_phase(std::integral_constant<int, 1>{}, (const uint32_t *)(smem + L.rowp)); break;
        case 2: rows_phase(std::integral_constant<int, 2>{}, (const uint32_t *)(smem + L.rowp)); break;
        case 3: rows_phase(std::integral_constant<int, 3>{}, (const uint32_t *)(smem + L.rowp)); break;
        case 4: rows_phase(std::integral_constant<int, 4>{}, (const uint32_t *)(smem + L.rowp)); break;
        default: rows_phase(std::integral_constant<int, 0>{}, (const uint32_t *)(smem + L.rowp)); break;
      }
    } else {
      rows_phase(std::integral_constant<int, 0>{}, rp);
    }
  }

  // ---- GMCR by plane windows: the molecule straddling the tile end (and,
  // for multi-word masks, every molecule starting in the tile) ----
  const int NCH = NLAB + 1 + fp.P;
  M *win = s_win + (size_t)wid * NCH;
  const int VQW = (fp.VQ + 31) >> 5;
  uint32_t *nz = s_nz + (size_t)wid * (VQW + 1);
  const int strad = s_strad;
  const int32_t *rowpoff = fp.rows_smem ? (const int32_t *)(smem + L.rowpoff) : fp.rowp_off;
  const uint32_t *rowp = fp.rows_smem ? (const uint32_t *)(smem + L.rowp) : fp.rowp;
  for (int mi = wid; mi < nmol && !MOL; mi += NWARP) {
    if (NW == 1 && mi != strad) continue;
    const int g = g0 + mi;
    const int gst = __ldg(&goff[g]);
    if (gst < n0) continue;  // owned by the previous tile
    const int ms = s_mstart[mi];
    const int n = s_mstart[mi + 1] - ms;
    const long long s = (long long)(gs + ms) - (long long)xo;
    for (int c = lane; c < NCH; c += 32) win[c] = extract_window_strided<NW>(s_pl + c, PS, nxw, s, n);
    __syncwarp();
    for (int rb = 0; rb < VQW; rb++) {
      const int row = rb * 32 + lane;
      bool ok = false;
      if (row < fp.VQ) {
        M x = win[NLAB];
        const int j1 = rowpoff[row + 1];
        for (int j = rowpoff[row]; j < j1; j++) {
          const uint32_t two = rowp[j];
          x &= win[(two & 0xffffu) >> 2];
          x &= win[two >> 18];
        }
        ok = x.any();
      }
      const unsigned bits = __ballot_sync(FULL_MASK, ok);
      if (lane == 0) nz[rb] = bits;
    }
    if (lane == 0) nz[VQW] = 0u;
    __syncwarp();
    for (int qb = 0; qb < fp.NQW; qb++) {
      const int q = qb * 32 + lane;
      bool ok = false;
      if (q < fp.NQ) {
        const int r0 = __ldg(&fp.qgoff[q]), r1 = __ldg(&fp.qgoff[q + 1]);
        const int nq = r1 - r0;
        const int wi = r0 >> 5, sh = r0 & 31;
        uint32_t v = nz[wi] >> sh;
        if (sh) v |= nz[wi + 1] << (32 - sh);
        const uint32_t want = nq >= 32 ? 0xffffffffu : ((1u << nq) - 1u);
        ok = (v & want) == want;
      }
      const unsigned bits = __ballot_sync(FULL_MASK, ok);
      if (lane == 0) s_gm[mi * fp.NQW + qb] = bits;
    }
    __syncwarp();
  }
  __syncthreads();
  // ---- write the GMCR bits and pair counts of the molecules starting here ----
  for (int mi = tid; mi < nmol; mi += NT) {
    const int g = g0 + mi;
    if (!MOL && gs + s_mstart[mi] < n0) continue;
    long long np = 0;
    for (int qb = 0; qb < fp.NQW; qb++) {
      const uint32_t bits = s_gm[mi * fp.NQW + qb];
      fp.gm[(size_t)g * fp.NQW + qb] = bits;
      np += __popc(bits);
    }
    I64x2 v;
    // molecule tiles: pairs of <= 32-node molecules counted in .a, of larger
    // ones in .b (the lane join runs the two classes as separate launches)
    const bool wide = MOL && s_mstart[mi + 1] - s_mstart[mi] > 32;
    v.a = wide ? 0 : np;
    v.b = wide ? np : 0;
    fp.mol_cnt[g] = v;
  }
}

cudaError_t launch_filter(int NW, const FilterParams &p, int num_tiles, cudaStream_t st) {
  if (num_tiles <= 0) return cudaSuccess;
  cudaError_t e = cudaSuccess;
#define SIGMO_FILTER_CASE(K, MOLF)                                                                              \
  case K * 2 + MOLF:                                                                                            \
    e = cudaFuncSetAttribute(k_filter<K, MOLF>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p.smem_bytes); \
    if (e != cudaSuccess) return e;                                                                             \
    k_filter<K, MOLF><<<num_tiles, kFilterThreads, p.smem_bytes, st>>>(p);                                      \
    break;
  switch (NW * 2 + (p.cmol ? 1 : 0)) {
    SIGMO_FILTER_CASE(1, 0)
    SIGMO_FILTER_CASE(2, 0)
    SIGMO_FILTER_CASE(4, 0)
    default: return cudaErrorInvalidValue;
  }
#undef SIGMO_FILTER_CASE
  return cudaGetLastError();
}

// ===========================================================================
// k_support: neighbour-support refinement to the greatest fixed point
// (BASELINE.json north_star; R9).  For every (query q, molecule g)
// the candidate masks cm[v_q] (molecule-local) are refined by
//   cm[v_q] &= OR_{u in cm[u_q]} adj_b[u]   for every query edge (v_q,u_q,b)
// (v has a b-neighbour in C(u_q)  <=>  v lies in the b-neighbourhood of some
// u in C(u_q)) until nothing changes.  The fixed point is unique, so any
// update order gives the same bitmap; cleared bits are removed from the global
// bitmap with atomicAnd (molecule windows share words), and the GMCR bits /
// pair counts of the molecule are recomputed.  One CTA per group of SUPPORT_MOLS
// molecules; one thread per (molecule, query) pair at a time.
// ===========================================================================
template <int NW> struct SupportCfg {
  static constexpr int kMols = 16 / NW;        // molecules per CTA
  static constexpr int kThreads = 256 / NW;    // threads per CTA
};

template <int NW>
__global__ void __launch_bounds__(SupportCfg<NW>::kThreads) k_support(SupportParams sp) {
  using M = Mask<NW>;
  constexpr int kSupportMols = SupportCfg<NW>::kMols, kSupportThreads = SupportCfg<NW>::kThreads;
  extern __shared__ __align__(16) unsigned char smem[];
  const int NB = sp.NB;
  const int ACAP = kSupportMols * 64 * NW;
  M *s_adj = (M *)smem;                                              // [NB][ACAP]
  M *s_cm = s_adj + (size_t)(NB + sp.any_bond) * ACAP;              // [threads][maxq]
  uint32_t *s_gm = (uint32_t *)(s_cm + (size_t)kSupportThreads * sp.maxq);  // [mols][NQW]
  __shared__ int s_mstart[kSupportMols + 1];
  const int tid = threadIdx.x;
  const int g0 = blockIdx.x * kSupportMols;
  const int g1 = min(g0 + kSupportMols, sp.ND);
  const int nm = g1 - g0;
  if (nm <= 0) return;
  const int a0 = sp.goff[g0];
  const int na = sp.goff[g1] - a0;
  for (int i = tid; i <= nm; i += kSupportThreads) s_mstart[i] = sp.goff[g0 + i] - a0;
  for (int i = tid; i < nm * sp.NQW; i += kSupportThreads) s_gm[i] = 0u;
  for (int i = tid; i < na; i += kSupportThreads) {
    const int v = a0 + i;
    const int e0 = __ldg(&sp.roff[v]), e1 = __ldg(&sp.roff[v + 1]);
    M m[8], mall;
#pragma unroll
    for (int b = 0; b < 8; b++) m[b].clear();
    mall.clear();
    for (int e = e0; e < e1; e++) {
      const int x = __ldg(&sp.nbr[e]);
      const int cls = sp.bclass[x & 255];
#pragma unroll
      for (int b = 0; b < 8; b++)
        if (cls == b) m[b].set(x >> 8);
      mall.set(x >> 8);
    }
#pragma unroll
    for (int b = 0; b < 8; b++)
      if (b < NB) s_adj[b * ACAP + i] = m[b];
    if (sp.any_bond) s_adj[NB * ACAP + i] = mall;  // '~' query bonds (R22): class NB = every bond
  }
  __syncthreads();
  M *cm = s_cm + (size_t)tid * sp.maxq;
  const long long npairs = (long long)nm * sp.NQ;
  for (long long t = tid; t < npairs; t += kSupportThreads) {
    const int mi = (int)(t / sp.NQ), q = (int)(t % sp.NQ);
    const int ms = s_mstart[mi], n = s_mstart[mi + 1] - ms;
    const int qb = __ldg(&sp.qgoff[q]), nq = __ldg(&sp.qgoff[q + 1]) - qb;
    const long long gstart = (long long)a0 + ms;
    bool all = n > 0;
    for (int i = 0; i < nq; i++) {
      cm[i] = extract_window<NW>(sp.bitmap + (size_t)(qb + i) * sp.Wpad, sp.Wpad, gstart, n);
      all = all && cm[i].any();
    }
    // fixed point
    bool changed = true;
    bool any_change = false;
    while (changed) {
      changed = false;
      for (int i = 0; i < nq; i++) {
        M c = cm[i];
        if (!c.any()) continue;
        const int e1 = __ldg(&sp.qroff[qb + i + 1]);
        for (int e = __ldg(&sp.qroff[qb + i]); e < e1; e++) {
          const int x = __ldg(&sp.qnbr[e]);
          const int j = x >> 8, b = sp.bclass[x & 255];
          M supp;
          supp.clear();
          M u = cm[j];
          while (u.any()) {
            const int w = u.lowest();
            u.clear_lowest();
            supp |= s_adj[b * ACAP + ms + w];
          }
          c &= supp;
        }
        bool diff = false;
#pragma unroll
        for (int k = 0; k < NW; k++) diff |= c.w[k] != cm[i].w[k];
        if (diff) {
          cm[i] = c;
          changed = true;
          any_change = true;
        }
      }
    }
    if (any_change) {
      all = n > 0;
      for (int i = 0; i < nq; i++) {
        all = all && cm[i].any();
        // clear removed bits of this molecule window in the global bitmap
        const M orig = extract_window<NW>(sp.bitmap + (size_t)(qb + i) * sp.Wpad, sp.Wpad, gstart, n);
#pragma unroll
        for (int k = 0; k < NW; k++) {
          const unsigned long long rem = orig.w[k] & ~cm[i].w[k];
          if (!rem) continue;
          const long long bit = gstart + 64ll * k;
          const long long wi = bit >> 5;
          const int sh = (int)(bit & 31);
          uint32_t *row = sp.bitmap + (size_t)(qb + i) * sp.Wpad;
          const unsigned long long lo = rem << sh;
          const uint32_t r0 = (uint32_t)lo, r1 = (uint32_t)(lo >> 32);
          const uint32_t r2 = sh ? (uint32_t)(rem >> (64 - sh)) : 0u;
          if (r0) atomicAnd(&row[wi], ~r0);
          if (r1) atomicAnd(&row[wi + 1], ~r1);
          if (r2) atomicAnd(&row[wi + 2], ~r2);
        }
      }
    }
    if (all) atomicOr(&s_gm[mi * sp.NQW + (q >> 5)], 1u << (q & 31));
  }
  __syncthreads();
  for (int mi = tid; mi < nm; mi += kSupportThreads) {
    long long np = 0;
    for (int qb = 0; qb < sp.NQW; qb++) {
      const uint32_t bits = s_gm[mi * sp.NQW + qb];
      sp.gm[(size_t)(g0 + mi) * sp.NQW + qb] = bits;
      np += __popc(bits);
    }
    I64x2 v;
    v.a = np;
    v.b = 0;
    sp.mol_cnt[g0 + mi] = v;
  }
}

template <int NW>
static size_t support_smem_t(int NB, int maxq, int NQW) {
  constexpr int mols = SupportCfg<NW>::kMols, thr = SupportCfg<NW>::kThreads;
  return (size_t)8 * NW * ((size_t)(NB + 1) * mols * 64 * NW + (size_t)thr * maxq) + 4 * (size_t)mols * NQW;
}

size_t support_smem_bytes(int NW, int NB, int maxq, int NQW) {
  return NW == 1 ? support_smem_t<1>(NB, maxq, NQW) : NW == 2 ? support_smem_t<2>(NB, maxq, NQW)
                                                              : support_smem_t<4>(NB, maxq, NQW);
}

template <int NW>
static cudaError_t launch_support_t(const SupportParams &p, cudaStream_t st) {
  constexpr int mols = SupportCfg<NW>::kMols, thr = SupportCfg<NW>::kThreads;
  const int grid = (p.ND + mols - 1) / mols;
  if (grid <= 0) return cudaSuccess;
  const size_t smem = support_smem_t<NW>(p.NB, p.maxq, p.NQW);
  cudaError_t e = cudaFuncSetAttribute(k_support<NW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k_support<NW><<<grid, thr, smem, st>>>(p);
  return cudaGetLastError();
}

cudaError_t launch_support(int NW, const SupportParams &p, cudaStream_t st) {
  switch (NW) {
    case 1: return launch_support_t<1>(p, st);
    case 2: return launch_support_t<2>(p, st);
    case 4: return launch_support_t<4>(p, st);
    default: return cudaErrorInvalidValue;
  }
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
// Enumerate mode helpers: inclusive sum of the per-pair
// embedding counts (u64), and the distinct node sets of every pair (NLSM's
// X = f(V_q)) from its embeddings' molecule-local node masks.
// ===========================================================================
cudaError_t launch_u64_inclusive_sum(const unsigned long long *in, unsigned long long *out, long long n, void *temp,
                                     size_t *temp_bytes, cudaStream_t st) {
  return cub::DeviceScan::InclusiveSum(temp, *temp_bytes, in, out, n, st);
}

// one thread per pair: sort its node masks (insertion sort, segments are
// short; the shared-lane join writes them in any order) and count the distinct
__global__ void k_nodeset_count(const unsigned long long *eoff, long long P, unsigned long long *sets,
                                unsigned long long *ucnt) {
  const long long p = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= P) return;
  const unsigned long long a = eoff[p], b = eoff[p + 1];
  for (unsigned long long i = a + 1; i < b; i++) {
    const unsigned long long x = sets[i];
    unsigned long long j = i;
    while (j > a && sets[j - 1] > x) {
      sets[j] = sets[j - 1];
      j--;
    }
    sets[j] = x;
  }
  unsigned long long u = 0;
  for (unsigned long long i = a; i < b; i++) u += (i == a || sets[i] != sets[i - 1]) ? 1ull : 0ull;
  ucnt[p] = u;
}

__global__ void k_nodeset_write(const unsigned long long *eoff, const unsigned long long *uoff, long long P,
                                const unsigned long long *sets, unsigned long long *uniq) {
  const long long p = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= P) return;
  const unsigned long long a = eoff[p], b = eoff[p + 1];
  unsigned long long o = uoff[p];
  for (unsigned long long i = a; i < b; i++)
    if (i == a || sets[i] != sets[i - 1]) uniq[o++] = sets[i];
}

cudaError_t launch_nodesets(const unsigned long long *eoff, long long P, unsigned long long *sets,
                            unsigned long long *ucnt, const unsigned long long *uoff, unsigned long long *uniq,
                            cudaStream_t st) {
  if (P <= 0) return cudaSuccess;
  const unsigned blocks = (unsigned)((P + 255) / 256);
  if (!uoff) k_nodeset_count<<<blocks, 256, 0, st>>>(eoff, P, sets, ucnt);
  else k_nodeset_write<<<blocks, 256, 0, st>>>(eoff, uoff, P, sets, uniq);
  return cudaGetLastError();
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
    (void)o;
    return (long long)p.goff[x] / p.AC + (long long)x / p.MC;
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
// ---------------------------------------------------------------------------
// k_join shared-memory layout.  CTA-wide: the query plans (optional copy) and
// the per-query totals; then one private region per warp (warps work on their
// own molecule chunks and never wait for each other).
// ---------------------------------------------------------------------------
struct JoinWarpSmem {
  size_t adj, cm, cinfo, pinfo, cnt, found, mstart, scratch, total;  // scratch = bitmap slice (staging) | DFS stack
};
struct JoinSmem {
  size_t plan, tot, warps;
  JoinWarpSmem w;
  size_t total;
};

// plan block: qgoff[NQ+1] | qp_beoff[VQ+1] i32 | qp_row[VQ] i32 | qp_be[NBE] u16
__host__ __device__ inline size_t join_plan_bytes(int NQ, int VQ, int NBE) {
  return align16(4 * (size_t)(NQ + 1)) + align16(4 * (size_t)(VQ + 1)) + align16(4 * (size_t)VQ) +
         align16(2 * (size_t)NBE);
}

// DFS iterator stack: safe capacity (global promotion) and shared-memory capacity
__host__ __device__ inline int join_stack_cap(int maxq) { return 32 * (maxq + 1) + 64; }
__host__ __device__ inline size_t join_entry_bytes(int NW, int MQ) { return align16(8 * (2 * (size_t)NW + MQ) + 4); }
__host__ __device__ inline size_t join_stack_bytes(int NW, int MQ, int cap) { return join_entry_bytes(NW, MQ) * cap; }

// one DFS iterator (array-of-structs, 16-byte aligned: vector loads/stores)
template <int NW, int MQ>
struct __align__(16) DfsEntry {
  unsigned long long R[NW];     // candidates of depth d not yet tried
  unsigned long long used[NW];  // data nodes of the partial mapping
  unsigned long long map[MQ];   // f(pi_0..pi_{d-1}), one byte each
  uint32_t hdr;                 // pair | d << 16
};

__host__ __device__ inline JoinSmem join_layout(const JoinParams &p, int NW, int MQ) {
  JoinSmem L;
  const size_t mb = 8 * (size_t)NW;
  const int NWARP = kJoinThreads / 32;
  size_t o = 0;
  L.plan = o;  o = align16(o + (p.plan_smem ? join_plan_bytes(p.NQ, p.VQ, p.NBE) : 0));
  L.tot = o;   o = align16(o + 8 * (size_t)p.NQ);
  L.warps = o;
  size_t w = 0;
  L.w.adj = w;     w = align16(w + mb * (size_t)(p.NB + ((p.induced || p.any_bond) ? 1 : 0)) * p.ACAP);
  L.w.cm = w;      w = align16(w + mb * (size_t)p.CMCAP);
  L.w.cinfo = w;   w = align16(w + 4 * (size_t)p.CMCAP);
  L.w.pinfo = w;   w = align16(w + 16 * (size_t)p.PCAP);
  L.w.cnt = w;     w = align16(w + 8 * (size_t)p.PCAP);
  L.w.found = w;   w = align16(w + (size_t)p.PCAP);
  L.w.mstart = w;  w = align16(w + 4 * (size_t)(p.MCAP + 1));
  L.w.scratch = w;
  w = align16(w + join_stack_bytes(NW, MQ, p.SCS));
  L.w.total = w;
  o += w * NWARP;
  L.total = o;
  return L;
}

static inline int join_mq(int maxq) { return maxq <= 8 ? 1 : (maxq <= 16 ? 2 : 4); }

size_t join_smem_bytes(int NW, const JoinParams &p) { return join_layout(p, NW, join_mq(p.maxq)).total; }
size_t join_gstack_bytes(int NW, const JoinParams &p, int grid) {
  return join_stack_bytes(NW, join_mq(p.maxq), join_stack_cap(p.maxq)) * (size_t)grid * (kJoinThreads / 32) + 256;
}

// byte j of a packed mapping (MQ u64 words)
template <int MQ>
__device__ __forceinline__ int map_get(const unsigned long long (&m)[MQ], int j) {
  unsigned long long w = m[0];
#pragma unroll
  for (int k = 1; k < MQ; k++)
    if ((j >> 3) == k) w = m[k];
  return (int)((w >> ((j & 7) * 8)) & 0xffull);
}
template <int MQ>
__device__ __forceinline__ void map_set(unsigned long long (&m)[MQ], int j, int v) {
#pragma unroll
  for (int k = 0; k < MQ; k++)
    if ((j >> 3) == k) m[k] = (m[k] & ~(0xffull << ((j & 7) * 8))) | ((unsigned long long)v << ((j & 7) * 8));
}

// ===========================================================================
// k_join: every warp independently pulls molecule chunks (persistent, atomic
// chunk counter).  Per chunk the warp stages, in its private smem region:
// the bond-class adjacency masks of the chunk's molecules, its GMCR pairs and,
// per pair, the candidate mask of every query node restricted to the molecule
// (cut from a coalesced copy of the chunk's bitmap slice).  The DFS
// runs on the warp's stack of iterators
//   E = (pair, d, f(pi_0..pi_{d-1}), used, R)
// where R holds the not-yet-tried candidates of plan depth d.  Each step every
// lane pops one iterator, takes v = lowest(R), pushes the remainder and, for
// the extended mapping, the child iterator with
//   R' = cm[d+1] & ~used' & AND_{(j,b) in back(d+1)} adj_b[f(j)]
// (children above remainders: depth-first).  At the last depth embeddings are
// counted with popc instead of being pushed.  The warp keeps >= 32 iterators
// by seeding new pairs, so all lanes run the same instruction stream.
// ===========================================================================
template <int NW, int MQ, int MODE>
__global__ void __launch_bounds__(kJoinThreads) k_join(JoinParams jp) {
  using M = Mask<NW>;
  constexpr int NT = kJoinThreads, NWARP = NT / 32;
  extern __shared__ __align__(16) unsigned char smem[];
  const JoinSmem L = join_layout(jp, NW, MQ);
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  unsigned long long *s_tot = (unsigned long long *)(smem + L.tot);
  unsigned char *wb = smem + L.warps + (size_t)wid * L.w.total;
  M *s_adj = (M *)(wb + L.w.adj);
  M *s_cm = (M *)(wb + L.w.cm);
  uint32_t *s_cinfo = (uint32_t *)(wb + L.w.cinfo);  // plan info of (pair, depth), parallel to s_cm
  int4 *s_pinfo = (int4 *)(wb + L.w.pinfo);  // {cm offset, plan base qb, mbase | n << 16, q << 8 | nq}
  unsigned long long *s_cnt = (unsigned long long *)(wb + L.w.cnt);
  uint8_t *s_found = wb + L.w.found;
  int *s_mstart = (int *)(wb + L.w.mstart);
  // DFS stack (shared memory; promoted to a global area if it ever fills)
  using E = DfsEntry<NW, MQ>;
  const int SCS = jp.SCS;
  E *const st = (E *)(wb + L.w.scratch);
  const int SCG = join_stack_cap(jp.maxq);
  const size_t gwarp = (size_t)blockIdx.x * NWARP + wid;
  E *const spill = (E *)(jp.gstack + gwarp * join_stack_bytes(NW, MQ, SCG));

  const int ACAP = jp.ACAP;
  const int32_t *qgoff = jp.qgoff, *qp_beoff = jp.qp_beoff, *qp_row = jp.qp_row;
  const uint16_t *qp_be = jp.qp_be;
  if (jp.plan_smem) {
    unsigned char *b = smem + L.plan;
    int32_t *a0 = (int32_t *)b;
    int32_t *a1 = (int32_t *)(b + align16(4 * (size_t)(jp.NQ + 1)));
    int32_t *a2 = (int32_t *)((unsigned char *)a1 + align16(4 * (size_t)(jp.VQ + 1)));
    uint16_t *a3 = (uint16_t *)((unsigned char *)a2 + align16(4 * (size_t)jp.VQ));
    for (int i = tid; i <= jp.NQ; i += NT) a0[i] = jp.qgoff[i];
    for (int i = tid; i <= jp.VQ; i += NT) a1[i] = jp.qp_beoff[i];
    for (int i = tid; i < jp.VQ; i += NT) a2[i] = jp.qp_row[i];
    for (int i = tid; i < jp.NBE; i += NT) a3[i] = jp.qp_be[i];
    qgoff = a0;
    qp_beoff = a1;
    qp_row = a2;
    qp_be = a3;
  }
  for (int i = tid; i < jp.NQ; i += NT) s_tot[i] = 0ull;
  __syncthreads();
  int nodes = 0, iters = 0;
  const unsigned lt = (1u << lane) - 1u;

  while (true) {
    int c = 0;
    if (lane == 0) c = atomicAdd(jp.chunk_counter, 1);
    c = __shfl_sync(FULL_MASK, c, 0);
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

    // ---- stage: molecule starts and bond-class adjacency masks ----
    for (int i = lane; i <= nm; i += 32) s_mstart[i] = __ldg(&jp.goff[g0 + i]) - a0;
    for (int i = lane; i < na; i += 32) {
      const int v = a0 + i;
      const int e0 = __ldg(&jp.roff[v]), e1 = __ldg(&jp.roff[v + 1]);
      M m[8], mall;
#pragma unroll
      for (int b = 0; b < 8; b++) m[b].clear();
      mall.clear();
      for (int e = e0; e < e1; e++) {
        const int x = __ldg(&jp.nbr[e]);
        const int cls = jp.bclass[x & 255];
#pragma unroll
        for (int b = 0; b < 8; b++)
          if (cls == b) m[b].set(x >> 8);
        mall.set(x >> 8);
      }
#pragma unroll
      for (int b = 0; b < 8; b++)
        if (b < jp.NB) s_adj[b * ACAP + i] = m[b];
      if (jp.induced || jp.any_bond) s_adj[jp.NB * ACAP + i] = mall;  // every bond, whatever its label
    }
    __syncwarp();
    // The chunk's pairs are processed in passes that fit the warp's pair /
    // candidate-mask capacity (PCAP, CMCAP >= the largest query); pairs are
    // taken in GMCR order, so a pass is the contiguous range [done, done+pnp).
    int done = 0, mi_start = 0;
    while (done < np) {
    // ---- stage: the pass's GMCR pairs (lane = query) ----
    int pnp = 0;
    {
      int pos = 0, cpos = 0;
      bool full = false;
      for (int mi = mi_start; mi < nm && !full; mi++) {
        const int g = g0 + mi;
        const int first = (int)(jp.off[g].a - p0);
        if ((int)(jp.off[g + 1].a - p0) <= done) {
          mi_start = mi + 1;
          continue;
        }
        const int mbase = s_mstart[mi], n = s_mstart[mi + 1] - mbase;
        int gi = first;
        for (int qb = 0; qb < jp.NQW; qb++) {
          const uint32_t bits = __ldg(&jp.gm[(size_t)g * jp.NQW + qb]);
          const int q = qb * 32 + lane;
          const bool take = ((bits >> lane) & 1u) && (gi + __popc(bits & lt) >= done);
          int nq = 0, qbase = 0;
          if (take) {
            qbase = qgoff[q];
            nq = qgoff[q + 1] - qbase;
          }
          const unsigned tm = __ballot_sync(FULL_MASK, take);
          int xc = nq;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(FULL_MASK, xc, o);
            if (lane >= o) xc += y;
          }
          const int tp = __popc(tm & lt);
          const bool fits = take && (pos + tp < jp.PCAP) && (cpos + xc <= jp.CMCAP);
          const unsigned fm = __ballot_sync(FULL_MASK, fits);
          if (fits) {
            s_pinfo[pos + tp] = make_int4(cpos + xc - nq, qbase, mbase | (n << 16), (q << 8) | nq);
            s_cnt[pos + tp] = 0ull;
            s_found[pos + tp] = 0;
          }
          pos += __popc(fm);
          cpos += __shfl_sync(FULL_MASK, fits ? xc : 0, fm ? 31 - __clz(fm) : 0);
          if (tm & ~fm) {
            full = true;
            break;
          }
          gi += __popc(bits);
        }
      }
      pnp = pos;
    }
    __syncwarp();
    // ---- stage: candidate masks cm[pair][e] (molecule window of each query-node row) ----
    for (int i = lane; i < pnp; i += 32) {
      const int4 pi = s_pinfo[i];
      const int nq = pi.w & 0xff, mbase = pi.z & 0xffff, n = pi.z >> 16;
#pragma unroll 2
      for (int e = 0; e < nq; e++) {
        const int row = __ldg(&qp_row[pi.y + e]);
        s_cm[pi.x + e] = extract_window<NW>(jp.bitmap + (size_t)row * jp.Wpad, jp.Wpad, (long long)a0 + mbase, n);
        s_cinfo[pi.x + e] = __ldg(&jp.qp_info[pi.y + e]);
      }
    }
    __syncwarp();

    // ---- DFS on the warp's iterator stack ----
    // hot part of the stack in shared memory (SCS entries); the oldest
    // entries spill to the warp's global area when it fills (never on the
    // common path) and come back when the shared part runs low.
    int top = 0, nspill = 0, next_pair = 0;
    while (true) {
      if (top < 32 && nspill > 0) {
        // restore: shift the shared entries up by r, bring back r spilled ones
        const int r = min(nspill, SCS / 2);
        E keep;
        if (lane < top) keep = st[lane];
        __syncwarp();
        if (lane < top) st[r + lane] = keep;
        for (int i = lane; i < r; i += 32) st[i] = spill[nspill - r + i];
        nspill -= r;
        top += r;
        __syncwarp();
      }
      if (top < 32 && next_pair < pnp) {
        // seed iterators of new pairs: E = (pair, d = 0, R = root candidates)
        const int pi = next_pair + lane;
        const bool ok = lane < 32 - top && pi < pnp;
        if (ok) {
          E en;
#pragma unroll
          for (int k = 0; k < NW; k++) {
            en.R[k] = s_cm[s_pinfo[pi].x].w[k];
            en.used[k] = 0ull;
          }
#pragma unroll
          for (int k = 0; k < MQ; k++) en.map[k] = 0ull;
          en.hdr = (uint32_t)pi;
          st[top + lane] = en;
        }
        const int added = __popc(__ballot_sync(FULL_MASK, ok));
        top += added;
        next_pair += added;
        __syncwarp();
      }
      if (top == 0) break;
      const int take = min(32, top);
      iters++;
      top -= take;
      const bool act = lane < take;
      E en;
      if (act) en = st[top + lane];
      __syncwarp();
      nodes += take;
      M R, used;
#pragma unroll
      for (int k = 0; k < NW; k++) {
        R.w[k] = act ? en.R[k] : 0ull;
        used.w[k] = act ? en.used[k] : 0ull;
      }
      const uint32_t hdr = act ? en.hdr : 0u;
      const int pair = hdr & 0xffff;
      const int d = hdr >> 16;
      bool alive = act;
      if (MODE == 1 && alive && s_found[pair]) alive = false;
      const int4 pinf = s_pinfo[pair];  // pair 0 is always staged; dead lanes are masked below
      const int nq = pinf.w & 0xff;
      const int mbase = pinf.z & 0xffff;
      // one candidate v of depth d; the remainder keeps the others
      const int v = R.lowest();
      R.clear_lowest();
      const bool push_rem = alive && R.any();
#pragma unroll
      for (int k = 0; k < NW; k++) en.R[k] = R.w[k];
      unsigned long long mp[MQ];
#pragma unroll
      for (int k = 0; k < MQ; k++) mp[k] = en.map[k];
      map_set<MQ>(mp, d, v & 0xff);
      M u2 = used;
      u2.set(v & (64 * NW - 1));
      const int e = d + 1;  // mapped nodes after this step (plan depth of the next node)
      // candidates of depth e: cm & ~used & adj of its (<= 2 inline) back-edges
      const int ec = min(e, nq - 1);
      const uint32_t info = s_cinfo[pinf.x + ec];
      M x = s_cm[pinf.x + ec].andnot(u2);
      {
        const int j0 = info & 0x3f, j1 = (info >> 9) & 0x3f;
        const M a0 = s_adj[((info >> 6) & 7) * ACAP + mbase + map_get<MQ>(mp, j0 & 31)];
        const M a1 = s_adj[((info >> 15) & 7) * ACAP + mbase + map_get<MQ>(mp, j1 & 31)];
        if (j0 != 0x3f) x &= a0;
        if (j1 != 0x3f) x &= a1;
      }
      const int nex = (info >> 18) & 0x3f;
      if (nex) {  // > 2 back-edges at this depth (fused ring systems): rare
        const int k0 = __ldg(&jp.qp_beoff[pinf.y + ec]) + 2;
#pragma unroll 1
        for (int k = 0; k < nex; k++) {
          const int be = __ldg(&jp.qp_be[k0 + k]);
          x &= s_adj[(be & 255) * ACAP + mbase + map_get<MQ>(mp, be >> 8)];
        }
      }
      if (jp.induced && e < nq) {
        // induced mode (condition (3), R21): v' must not be adjacent
        // (any bond) to f(j) for every mapped depth j that is not a back-edge
        unsigned long long bm = 0ull;
        {
          const int j0 = info & 0x3f, j1 = (info >> 9) & 0x3f;
          if (j0 != 0x3f) bm |= 1ull << j0;
          if (j1 != 0x3f) bm |= 1ull << j1;
          if (nex) {
            const int k0 = __ldg(&jp.qp_beoff[pinf.y + ec]) + 2;
#pragma unroll 1
            for (int k = 0; k < nex; k++) bm |= 1ull << (__ldg(&jp.qp_be[k0 + k]) >> 8);
          }
        }
#pragma unroll 1
        for (int j = 0; j < e; j++)
          if (!((bm >> j) & 1ull)) x = x.andnot(s_adj[jp.NB * ACAP + mbase + map_get<MQ>(mp, j)]);
      }
      // leaf sum (e == nq-2 and the last node is not adjacent to depth nq-2):
      // X = candidates of the last depth given f(0..e-1) and v; then
      // sum_{w in x} |X \ {w}| = |x||X| - |x & X|
      const int lastd = max(nq - 1, 0);
      const uint32_t li = s_cinfo[pinf.x + lastd];
      const bool lsum = !jp.induced && (e == nq - 2) && ((li >> 24) & 1u);
      unsigned long long cnt = 0ull;
      if (__any_sync(FULL_MASK, lsum && alive)) {
        M X = s_cm[pinf.x + lastd].andnot(u2);
        const int j0 = li & 0x3f, j1 = (li >> 9) & 0x3f;
        const M a0 = s_adj[((li >> 6) & 7) * ACAP + mbase + map_get<MQ>(mp, j0 & 31)];
        const M a1 = s_adj[((li >> 15) & 7) * ACAP + mbase + map_get<MQ>(mp, j1 & 31)];
        if (j0 != 0x3f) X &= a0;
        if (j1 != 0x3f) X &= a1;
        const int lnex = (li >> 18) & 0x3f;
        if (lsum && lnex) {
          const int k0 = __ldg(&jp.qp_beoff[pinf.y + lastd]) + 2;
#pragma unroll 1
          for (int k = 0; k < lnex; k++) {
            const int be = __ldg(&jp.qp_be[k0 + k]);
            X &= s_adj[(be & 255) * ACAP + mbase + map_get<MQ>(mp, be >> 8)];
          }
        }
        if (lsum) cnt = (unsigned long long)x.popc() * (unsigned long long)X.popc() - (unsigned long long)(x & X).popc();
      }
      if (e == nq - 1) cnt = (unsigned long long)x.popc();  // last depth: count
      if (e == nq) cnt = 1ull;                                // single-node query
      if (!alive) cnt = 0ull;
      const bool push_child = alive && (e < nq - 1) && !lsum && x.any();
      if (cnt) {
        // 64-bit per-pair count kept as two 32-bit words with carry
        uint32_t *w = (uint32_t *)&s_cnt[pair];
        const uint32_t add = (uint32_t)cnt;
        const uint32_t old = atomicAdd(w, add);
        const uint32_t hi = (uint32_t)(cnt >> 32) + ((old + add < old) ? 1u : 0u);
        if (hi) atomicAdd(w + 1, hi);
        if (MODE == 1) s_found[pair] = 1;
      }
      // push: remainders first, then children (children end on top)
      const unsigned mr = __ballot_sync(FULL_MASK, push_rem);
      const unsigned mc = __ballot_sync(FULL_MASK, push_child);
      const int nr = __popc(mr);
      const int npush = nr + __popc(mc);
      if (top + npush > SCS) {
        // spill the oldest m shared entries to global, shift the rest down
        const int m = min(top, max(SCS / 2, top + npush - SCS));
        if (nspill + m > SCG) {
          if (lane == 0) atomicOr(jp.error, 1);
          top = 0;
          nspill = 0;
          next_pair = pnp;
          continue;
        }
        for (int i = lane; i < m; i += 32) spill[nspill + i] = st[i];
        __syncwarp();
        for (int base = m; base < top; base += 32) {
          E t;
          const int i = base + lane;
          if (i < top) t = st[i];
          __syncwarp();
          if (i < top) st[i - m] = t;
          __syncwarp();
        }
        nspill += m;
        top -= m;
      }
      if (push_rem) st[top + __popc(mr & lt)] = en;
      if (push_child) {
        E ch;
#pragma unroll
        for (int k = 0; k < NW; k++) {
          ch.R[k] = x.w[k];
          ch.used[k] = u2.w[k];
        }
#pragma unroll
        for (int k = 0; k < MQ; k++) ch.map[k] = mp[k];
        ch.hdr = (uint32_t)pair | ((uint32_t)e << 16);
        st[top + nr + __popc(mc & lt)] = ch;
      }
      top += npush;
      __syncwarp();
    }
    // ---- results: GMCR pair list + per-pair result + per-query totals ----
    for (int i = lane; i < pnp; i += 32) {
      unsigned long long r = s_cnt[i];
      if (MODE == 1) r = r ? 1ull : 0ull;
      const int q = s_pinfo[i].w >> 8;
      jp.pair_query[p0 + done + i] = q;
      jp.pair_result[p0 + done + i] = r;
      if (r) atomicAdd(&s_tot[q], r);
    }
    done += pnp;
    __syncwarp();
    }  // passes
    (void)c0;
  }
  __syncthreads();
  for (int i = tid; i < jp.NQ; i += NT)
    if (s_tot[i]) atomicAdd(&jp.totals[i], s_tot[i]);
  if (jp.stats && lane == 0) {
    atomicAdd(jp.stats, (unsigned long long)nodes);
    atomicAdd(jp.stats + 1, (unsigned long long)iters);
  }
}

template <int NW, int MQ, int MODE>
static cudaError_t launch_join_t(const JoinParams &p, int grid, cudaStream_t st) {
  cudaError_t e = cudaFuncSetAttribute(k_join<NW, MQ, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)p.smem_bytes);
  if (e != cudaSuccess) return e;
  k_join<NW, MQ, MODE><<<grid, kJoinThreads, p.smem_bytes, st>>>(p);
  return cudaGetLastError();
}

template <int NW, int MQ, int MODE>
static int occ_join_t(size_t smem) {
  int n = 0;
  cudaFuncSetAttribute(k_join<NW, MQ, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_join<NW, MQ, MODE>, kJoinThreads, smem) != cudaSuccess) {
    cudaGetLastError();
    return 1;
  }
  return n < 1 ? 1 : n;
}

#define SIGMO_JOIN_DISPATCH(FN, ...)                                             \
  switch ((NW == 1 ? 0 : NW == 2 ? 1 : 2) * 6 + (MQ == 1 ? 0 : MQ == 2 ? 1 : 2) * 2 + mode) { \
    case 0: return FN<1, 1, 0>(__VA_ARGS__);                                     \
    case 1: return FN<1, 1, 1>(__VA_ARGS__);                                     \
    case 2: return FN<1, 2, 0>(__VA_ARGS__);                                     \
    case 3: return FN<1, 2, 1>(__VA_ARGS__);                                     \
    case 4: return FN<1, 4, 0>(__VA_ARGS__);                                     \
    case 5: return FN<1, 4, 1>(__VA_ARGS__);                                     \
    case 6: return FN<2, 1, 0>(__VA_ARGS__);                                     \
    case 7: return FN<2, 1, 1>(__VA_ARGS__);                                     \
    case 8: return FN<2, 2, 0>(__VA_ARGS__);                                     \
    case 9: return FN<2, 2, 1>(__VA_ARGS__);                                     \
    case 10: return FN<2, 4, 0>(__VA_ARGS__);                                    \
    case 11: return FN<2, 4, 1>(__VA_ARGS__);                                    \
    case 12: return FN<4, 1, 0>(__VA_ARGS__);                                    \
    case 13: return FN<4, 1, 1>(__VA_ARGS__);                                    \
    case 14: return FN<4, 2, 0>(__VA_ARGS__);                                    \
    case 15: return FN<4, 2, 1>(__VA_ARGS__);                                    \
    case 16: return FN<4, 4, 0>(__VA_ARGS__);                                    \
    default: return FN<4, 4, 1>(__VA_ARGS__);                                    \
  }

cudaError_t launch_join(int NW, int mode, const JoinParams &p, int grid, cudaStream_t st) {
  if (grid <= 0) return cudaSuccess;
  if (NW != 1 && NW != 2 && NW != 4) return cudaErrorInvalidValue;
  const int MQ = join_mq(p.maxq);
  SIGMO_JOIN_DISPATCH(launch_join_t, p, grid, st)
}

int join_blocks_per_sm(int NW, int mode, const JoinParams &p, size_t smem) {
  const int MQ = join_mq(p.maxq);
  SIGMO_JOIN_DISPATCH(occ_join_t, smem)
}

// ===========================================================================
// GMCR pair list (paper section 4.5, "mapping #2"): expand the
// per-graph surviving-query bits into pair records at the scanned offsets
// (k_join_lane: molecule start node, query, cmol index of the pair's first
// candidate row, query plan info).  One warp per data graph, lane = query of
// a 32-query block.
// ===========================================================================
__global__ void __launch_bounds__(256) k_pairs(PairsParams pp) {
  const int lane = threadIdx.x & 31;
  const unsigned lt = (1u << lane) - 1u;
  // grid-stride over graphs, one warp per graph (one block per 8 graphs was
  // bound by block scheduling)
  const int nwarps = (int)((gridDim.x * blockDim.x) >> 5);
  for (int g = (int)((blockIdx.x * blockDim.x + threadIdx.x) >> 5); g < pp.ND; g += nwarps) {
  // lane join: records of <= 32-node molecules first (off.a), then the others
  // at P_narrow + off.b; the general path only uses .a
  long long o = pp.off[g].a;
  if (pp.prec && pp.off[g + 1].b > pp.off[g].b) o = pp.off[pp.ND].a + pp.off[g].b;
  const int a = __ldg(&pp.goff[g]);
  const uint32_t ng8 = (uint32_t)(__ldg(&pp.goff[g + 1]) - a) << 8;  // molecule size, bits 8-15 of the query info
  const int aw = pp.prec ? (int)__ldg(&pp.adj_off[g]) : 0;  // adjacency word offset (pair record .x)
  const int cw = pp.prec ? (int)((unsigned)pp.rowstride * __ldg(&pp.cand_units[g])) : 0;  // cmol word base (.z)
  // neighbour-support mode: the pair's pre-support index (its refined windows)
  long long oo = 0;
  const bool ns = pp.gm_old != nullptr;
  const bool wide_g = (ng8 >> 8) > 32u;
  if (ns) oo = wide_g ? pp.off_old[g].b : pp.off_old[g].a;
  for (int qb = 0; qb < pp.NQW; qb++) {
    const uint32_t bits = __ldg(&pp.gm[(size_t)g * pp.NQW + qb]);
    const uint32_t obits = ns ? __ldg(&pp.gm_old[(size_t)g * pp.NQW + qb]) : 0u;
    if ((bits >> lane) & 1u) {
      const int q = qb * 32 + lane;
      const long long p = o + __popc(bits & lt);
      if (!pp.prec) {
        pp.pair_query[p] = q;
      } else {  // the lane join reads the records only (queries from .y)
        const uint32_t qi = (__ldg(&pp.qinfo[q]) & ~0xff00u) | ng8;
        const int z = ns ? (int)((unsigned long long)(oo + __popc(obits & lt)) * (unsigned)pp.ns_mq * (wide_g ? 2u : 1u))
                         : cw;
        pp.prec[p] = make_int4(aw, q, z, (int)qi);
      }
    }
    o += __popc(bits);
    oo += __popc(obits);
  }
  }
}

// ===========================================================================
// k_support_lane: neighbour support to the greatest fixed point (north_star;
// DESIGN.md R9) on the lane path.  One thread per pre-support GMCR pair: the
// windows of its query nodes (plan-depth order) are refined by
//   C(w) &= OR_{u in C(v)} adj_b[u]   for every query edge (v, w, b)
// until nothing changes (an AC-3 worklist; the fixed point is unique, so the
// order is free); the refined windows are written per
// pair for the join, and a pair with an emptied node leaves the GMCR
// (k_gmcr_update rebuilds the GMCR bits and pair counts from the alive flags,
// then the pair records are rebuilt from the remaining bits).
// ===========================================================================
constexpr int kSupportLaneThreads = 128;

template <bool W64>
__global__ void __launch_bounds__(kSupportLaneThreads) k_support_lane(const __grid_constant__ SupportLaneParams sp) {
  using MT = typename std::conditional<W64, unsigned long long, unsigned>::type;
  constexpr unsigned sw = W64 ? 1u : 0u;
  extern __shared__ __align__(16) unsigned char smem[];
  MT *const wv = (MT *)smem + threadIdx.x;  // window of depth e at wv[e * blockDim.x]
  const long long p = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long P = W64 ? sp.Pw : sp.Pn;
  if (p >= P) return;
  const int4 r = __ldg(&sp.prec[(W64 ? sp.Pn : 0) + p]);
  const unsigned ca = (unsigned)r.x, cmb = (unsigned)r.z, info = (unsigned)r.w;
  const unsigned nq = info & 0xffu, ng = (info >> 8) & 0xffu, qb = info >> 16;
  const unsigned T = blockDim.x;
  auto adj = [&](unsigned i) -> MT {
    if (W64) return (MT)__ldg((const unsigned long long *)(sp.adjw + i));
    return (MT)__ldg(sp.adjw + i);
  };
  auto low = [](MT x) -> unsigned {
    return W64 ? (unsigned)(__ffsll((long long)x) - 1) : (unsigned)(__ffs((unsigned)x) - 1);
  };
  bool empty = false;
  for (unsigned e = 0; e < nq; e++) {
    const unsigned row = __ldg(&sp.qp_ent2[qb + e]).y >> 12;
    const MT w = W64 ? (MT)__ldg((const unsigned long long *)(sp.cmol + (cmb + 2u * row))) : (MT)__ldg(sp.cmol + (cmb + row));
    wv[e * T] = w;
    empty |= w == (MT)0;
  }
  // support of S along the bond-class row base a: the nodes with a b-neighbour
  // in S (up to four independent adjacency loads per round)
  auto supp = [&](MT S, unsigned a) -> MT {
    MT x = 0;
    while (S) {
      const unsigned u0 = low(S);
      S &= S - (MT)1;
      const bool h1 = S != (MT)0;
      const unsigned u1 = h1 ? low(S) : 0u;
      S &= S - (MT)(h1 ? 1 : 0);
      const bool h2 = S != (MT)0;
      const unsigned u2 = h2 ? low(S) : 0u;
      S &= S - (MT)(h2 ? 1 : 0);
      const bool h3 = S != (MT)0;
      const unsigned u3 = h3 ? low(S) : 0u;
      S &= S - (MT)(h3 ? 1 : 0);
      const MT y0 = adj(a + (u0 << sw));
      const MT y1 = h1 ? adj(a + (u1 << sw)) : (MT)0;
      const MT y2 = h2 ? adj(a + (u2 << sw)) : (MT)0;
      const MT y3 = h3 ? adj(a + (u3 << sw)) : (MT)0;
      x |= (y0 | y1) | (y2 | y3);
    }
    return x;
  };
  // AC-3 worklist over query nodes: revising every neighbour w of a dirty
  // node u against C(u) (C(w) &= supp(C(u), b)) and marking w dirty when it
  // shrinks reaches the greatest fixed point with no confirmation pass
  unsigned dirty = empty ? 0u : (nq >= 32 ? 0xffffffffu : (1u << nq) - 1u);
  while (dirty) {
    const unsigned u = (unsigned)(__ffs(dirty) - 1);
    dirty &= dirty - 1u;
    const uint2 nb = __ldg(&sp.qp_nbr[qb + u]);  // up to 8 neighbours: depth | class << 4 | 0x80
    const MT cu = wv[u * T];
#pragma unroll
    for (int k = 0; k < 8; k++) {
      const unsigned byte = ((k < 4 ? nb.x : nb.y) >> (8 * (k & 3))) & 0xffu;
      if (!(byte & 0x80u)) break;
      const unsigned w = byte & 15u, cls = (byte >> 4) & 7u;
      const MT cw = wv[w * T];
      const MT nw = cw & supp(cu, ca + ((cls * ng) << sw));
      if (nw != cw) {
        wv[w * T] = nw;
        if (!nw) {
          empty = true;
          dirty = 0u;
          break;
        }
        dirty |= 1u << w;
      }
    }
  }
  sp.alive[(W64 ? sp.Pn : 0) + p] = empty ? 0 : 1;  // k_gmcr_update rebuilds the GMCR bits from these
  if (empty) return;
  for (unsigned e = 0; e < nq; e++) {
    if (W64) sp.win64[(size_t)p * sp.MQ + e] = (unsigned long long)wv[e * T];
    else sp.win32[(size_t)p * sp.MQ + e] = (uint32_t)wv[e * T];
  }
}

cudaError_t launch_support_lane(const SupportLaneParams &p, cudaStream_t st) {
  const size_t s32 = 4 * (size_t)p.MQ * kSupportLaneThreads, s64 = 8 * (size_t)p.MQ * kSupportLaneThreads;
  if (p.Pn > 0) {
    k_support_lane<false><<<(unsigned)((p.Pn + kSupportLaneThreads - 1) / kSupportLaneThreads), kSupportLaneThreads, s32,
                            st>>>(p);
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
  }
  if (p.Pw > 0) {
    k_support_lane<true><<<(unsigned)((p.Pw + kSupportLaneThreads - 1) / kSupportLaneThreads), kSupportLaneThreads, s64,
                           st>>>(p);
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

// GMCR bits and pair counts after neighbour support: warp per data graph,
// lane = query of a 32-query block; a pre-support pair survives iff its
// alive flag is set (pre-support index = the graph's offset + rank of the bit)
__global__ void __launch_bounds__(256) k_gmcr_update(int ND, int NQW, const uint32_t *gm_old, const I64x2 *off_old,
                                                      const int32_t *goff, const uint8_t *alive, uint32_t *gm,
                                                      I64x2 *mol_cnt) {
  const int lane = threadIdx.x & 31;
  const int g = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (g >= ND) return;
  const unsigned lt = (1u << lane) - 1u;
  const bool wide = __ldg(&goff[g + 1]) - __ldg(&goff[g]) > 32;
  long long oo = wide ? off_old[ND].a + off_old[g].b : off_old[g].a;  // alive[] index of the graph's first pair
  long long np = 0;
  for (int qb = 0; qb < NQW; qb++) {
    const uint32_t obits = __ldg(&gm_old[(size_t)g * NQW + qb]);
    const bool mine = (obits >> lane) & 1u;
    const bool keep = mine && alive[oo + __popc(obits & lt)];
    const uint32_t nb = __ballot_sync(0xffffffffu, keep);
    if (lane == 0) gm[(size_t)g * NQW + qb] = nb;
    np += __popc(nb);
    oo += __popc(obits);
  }
  if (lane == 0) {
    I64x2 v;
    v.a = wide ? 0 : np;
    v.b = wide ? np : 0;
    mol_cnt[g] = v;
  }
}

cudaError_t launch_gmcr_update(int ND, int NQW, const uint32_t *gm_old, const I64x2 *off_old, const int32_t *goff,
                               const uint8_t *alive, uint32_t *gm, I64x2 *mol_cnt, cudaStream_t st) {
  if (ND <= 0) return cudaSuccess;
  k_gmcr_update<<<(unsigned)((32ll * ND + 255) / 256), 256, 0, st>>>(ND, NQW, gm_old, off_old, goff, alive, gm, mol_cnt);
  return cudaGetLastError();
}

// S7 count reduction for the lane path: totals[q] += sum over the GMCR pairs (g, q)
// of pair_result (Find All counts or Find First flags).  One warp per molecule
// (grid-stride), lane = query within a 32-query word of the GMCR bits; per-warp
// accumulators in shared memory owned by one lane each (no atomics), summed
// over the CTA's warps and added to the global totals once per CTA.
constexpr int kTotThreads = 256;
__global__ void __launch_bounds__(kTotThreads) k_lane_totals(int ND, int NQ, int NQW, const uint32_t *gm, const I64x2 *off,
                                                            const unsigned long long *presult, unsigned long long *totals) {
  extern __shared__ unsigned long long s_acc[];  // [warps][NQW * 32]
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const unsigned lt = (1u << lane) - 1u;
  const int QS = NQW * 32;
  unsigned long long *acc = s_acc + (size_t)wid * QS;
  for (int i = lane; i < QS; i += 32) acc[i] = 0ull;
  const long long pn = off[ND].a;
  const int nwarps = (int)((gridDim.x * blockDim.x) >> 5);
  for (int g = (int)((blockIdx.x * blockDim.x + threadIdx.x) >> 5); g < ND; g += nwarps) {
    const I64x2 o0 = off[g], o1 = off[g + 1];
    long long o = o1.b > o0.b ? pn + o0.b : o0.a;  // the records' order (k_pairs)
    for (int qb = 0; qb < NQW; qb++) {
      const uint32_t bits = __ldg(&gm[(size_t)g * NQW + qb]);
      SIGMO_BOUND(!((bits >> lane) & 1u) || o + __popc(bits & lt) < pn + off[ND].b);
      if ((bits >> lane) & 1u) acc[qb * 32 + lane] += __ldg(&presult[o + __popc(bits & lt)]);
      o += __popc(bits);
    }
  }
  __syncthreads();
  for (int q = threadIdx.x; q < NQ; q += blockDim.x) {
    unsigned long long t = 0ull;
    for (int w = 0; w < nw; w++) t += s_acc[(size_t)w * QS + q];
    if (t) atomicAdd(&totals[q], t);
  }
}

cudaError_t launch_lane_totals(int ND, int NQ, int NQW, const uint32_t *gm, const I64x2 *off,
                               const unsigned long long *presult, unsigned long long *totals, int sm_count, cudaStream_t st) {
  if (ND <= 0 || NQ <= 0) return cudaSuccess;
  // warps per CTA so that the accumulators fit 96 KB
  int warps = kTotThreads / 32;
  while (warps > 1 && (size_t)warps * NQW * 32 * 8 > 96 * 1024) warps--;
  const size_t smem = (size_t)warps * NQW * 32 * 8;
  if (smem > 200 * 1024) return cudaErrorInvalidValue;
  if (smem > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(k_lane_totals, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
  }
  const long long blocks = std::min<long long>((ND + warps - 1) / warps, (long long)sm_count * 8);
  k_lane_totals<<<(unsigned)blocks, 32 * warps, smem, st>>>(ND, NQ, NQW, gm, off, presult, totals);
  return cudaGetLastError();
}

cudaError_t launch_pairs(const PairsParams &p, cudaStream_t st) {
  if (p.ND <= 0) return cudaSuccess;
  const long long blocks = std::min<long long>((32ll * p.ND + 255) / 256, 148ll * 16);
  k_pairs<<<(unsigned)blocks, 256, 0, st>>>(p);
  return cudaGetLastError();
}

// Dense (row-major, LSB-first) view of the molecule-padded candidates for
// sigmo_get_candidates: thread per (row, graph), OR the window into the rows.
__global__ void k_unpad(const uint32_t *cmol, const uint32_t *cand_units, const uint16_t *qdrow, int NDR,
                        const int32_t *goff, int ND, int VQ, int Wpad, uint32_t *dense) {
  const long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= (long long)ND * VQ) return;
  const int g = (int)(t / VQ), row = (int)(t - (long long)g * VQ);
  const int a = goff[g];
  const size_t base = (size_t)NDR * cand_units[g];  // window of the distinct row of query node `row`
  const unsigned long long w = goff[g + 1] - a > 32 ? *(const unsigned long long *)(cmol + base + 2 * (size_t)qdrow[row])
                                                    : (unsigned long long)cmol[base + qdrow[row]];
  if (!w) return;
  uint32_t *r = dense + (size_t)row * Wpad;
  const int wi = a >> 5, sh = a & 31;
  const unsigned long long lo = w << sh;
  atomicOr(&r[wi], (uint32_t)lo);
  if ((uint32_t)(lo >> 32)) atomicOr(&r[wi + 1], (uint32_t)(lo >> 32));
  if (sh && (uint32_t)(w >> (64 - sh))) atomicOr(&r[wi + 2], (uint32_t)(w >> (64 - sh)));
}

cudaError_t launch_unpad(const uint32_t *cmol, const uint32_t *cand_units, const uint16_t *qdrow, int NDR,
                         const int32_t *goff, int ND, int VQ, int Wpad, uint32_t *dense, cudaStream_t st) {
  const long long n = (long long)ND * VQ;
  if (n <= 0) return cudaSuccess;
  k_unpad<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(cmol, cand_units, qdrow, NDR, goff, ND, VQ, Wpad, dense);
  return cudaGetLastError();
}

// ===========================================================================
// Bond-class adjacency masks (molecule-local bits of the neighbours of v
// joined by a bond of class b), for <= 64-node graphs, class-major inside
// each molecule: adjb[a * NB + b * n + (v - a)] for the molecule [a, a + n)
// holding v, so that lanes reading the same class of one molecule touch few
// 32-B sectors.
// ===========================================================================
__global__ void k_adjb(DevGraphs d, const uint8_t *bclass, int NB, const uint32_t *adj_off, uint32_t *adjw,
                       uint32_t *nb4) {
  const int v = blockIdx.x * blockDim.x + threadIdx.x;
  if (v >= d.num_nodes) return;
  unsigned long long m[8], mall = 0ull;
#pragma unroll
  for (int b = 0; b < 8; b++) m[b] = 0ull;
  const int e0 = d.roff[v], e1 = d.roff[v + 1];
  for (int e = e0; e < e1; e++) {
    const int x = d.nbr[e];
    const int cls = bclass[x & 255];
#pragma unroll
    for (int b = 0; b < 8; b++)
      if (cls == b) m[b] |= 1ull << ((x >> 8) & 63);
    mall |= 1ull << ((x >> 8) & 63);
  }
  const int g = graph_of(d.goff, d.num_graphs, v);
  const int a = d.goff[g], n = d.goff[g + 1] - a;
  const uint32_t base = adj_off[g];
#pragma unroll
  for (int b = 0; b < 8; b++)
    if (b < NB) {
      if (n <= 32) adjw[base + (uint32_t)(b * n + (v - a))] = (uint32_t)m[b];
      else *(unsigned long long *)(adjw + base + 2u * (uint32_t)(b * n + (v - a))) = m[b];
    }
  // class NB: every bond, whatever its label (k_filter_lane's slow path for
  // degree > 4, the induced lane join, R21)
  if (n <= 32) adjw[base + (uint32_t)(NB * n + (v - a))] = (uint32_t)mall;
  else *(unsigned long long *)(adjw + base + 2u * (uint32_t)(NB * n + (v - a))) = mall;
  // nb4: the first <= 4 neighbours (molecule-local ids, byte k), unused bytes
  // = the node itself, bit 7 of byte 0 set when the degree exceeds 4
  const uint32_t self = (uint32_t)(v - a) & 63u;
  uint32_t w = self * 0x01010101u;
  unsigned long long rest = mall;
  for (int k = 0; k < 4 && rest; k++) {
    const uint32_t u = (uint32_t)(__ffsll((long long)rest) - 1);
    rest &= rest - 1ull;
    w = (w & ~(0xffu << (8 * k))) | (u << (8 * k));
  }
  if (rest) w |= 0x80u;
  nb4[v] = w;
}

cudaError_t launch_adjb(const DevGraphs &d, const uint8_t *bclass, int NB, const uint32_t *adj_off, uint32_t *adjw,
                        uint32_t *nb4, cudaStream_t st) {
  if (d.num_nodes <= 0) return cudaSuccess;
  k_adjb<<<(d.num_nodes + 255) / 256, 256, 0, st>>>(d, bclass, NB, adj_off, adjw, nb4);
  return cudaGetLastError();
}

// ===========================================================================
// k_join_lane: stack-based DFS (section 4.6) with ONE GMCR pair
// per lane, for queries of <= kJoinLaneMaxQ nodes in <= 64-node data graphs.
//   * Per lane, in shared memory: the DFS stack {R_d, U_d} (untried
//     candidates of depth d, used set of f(pi_0..pi_{d-1})) and the map
//     words (adjacency index of f(pi_d)); the candidate windows cm[u] are
//     read from the filter's cmol[g][row] layout.  A bitmask `ne` of open
//     depths makes every step productive: a step pops the highest candidate
//     v of the deepest open depth d (backtracking is free) and builds the
//     candidates of e = d + 1:
//        X = cm[pi_e] & ~(U_d | {v}) & AND_{(j,b) in back(e)} adjb[b][f(pi_j)]
//     pushed as {X, U_d | {v}} (a predicated store); at the last depth they
//     are counted with popc (Find All) or end the pair (Find First).  Absent
//     back-edges read the all-ones adjacency entry, so the step has no
//     selects; SIGMO_JL_UNROLL steps run between two checks of the free lanes.
//   * The warp claims blocks of kJoinClaim consecutive GMCR pairs (one atomic
//     per block, a block ahead).  Lanes whose pair finished refill together
//     (>= batchK at a time): write the result, activate the next pair they
//     hold (its record in registers, its root window loaded a pass earlier),
//     and the lanes left without one take the next records of the warp's
//     blocks.  Lanes of a warp thus run pairs of very different sizes without
//     waiting for each other (the paper runs one work-item per query of a
//     data graph and sits at ~48% occupancy, divergence-bound);
//     when the list is drained, idle lanes take the shallowest open depth of
//     a busy lane (heavy pairs).
//   * Per-query totals: k_lane_totals, from the pair results.
// ===========================================================================
#ifndef SIGMO_JL_CLAIM
#define SIGMO_JL_CLAIM 128  // configs[2] join: claims of 64/128/512 pairs -> 4.87/4.60/4.60 ms
#endif
constexpr int kJoinClaim = SIGMO_JL_CLAIM;  // GMCR pairs per warp claim (atomic on the launch's pair counter)

// stack entry {R, U}: 2 x 32-bit masks (<= 32-node molecules) or 2 x 64-bit
__host__ __device__ inline size_t join_lane_warp_bytes(int MQ, bool w64) {
  const int SD = MQ > 1 ? MQ - 1 : 1;  // pushed depths 0..n-2
  // {R, U} [SD][32] (8 or 16 B) | map words [SD + 1][32] (u32: adjacency index of f(pi_d); slot SD: all ones)
  return 32 * (size_t)(w64 ? 16 : 8) * SD + 128 * (size_t)(SD + 1);
}
// CTA: the window and adjacency base pointers (16 B), (optionally) the plan entries [VQ] uint2, then one
// region per warp
__host__ __device__ inline size_t join_lane_plan_bytes(int VQ, int pmax) { return VQ <= pmax ? align16(8 * (size_t)VQ) : 0; }
__host__ __device__ inline size_t join_lane_cta_bytes(int VQ, int pmax) { return 16 + join_lane_plan_bytes(VQ, pmax); }
__host__ __device__ inline size_t join_lane_smem(int VQ, int MQ, bool w64, int pmax, int threads) {
  return join_lane_cta_bytes(VQ, pmax) + join_lane_warp_bytes(MQ, w64) * (size_t)(threads / 32);
}
size_t join_lane_smem_bytes(const JoinParams &p, bool w64) { return join_lane_smem(p.VQ, p.maxq, w64, p.plan_smem_max, p.lane_threads); }

// n-th (0-based) set bit of m (m has > n set bits)
__device__ __forceinline__ int nth_set_bit(unsigned m, int n) {
  for (int i = 0; i < n; i++) m &= m - 1u;
  return __ffs(m) - 1;
}

// shared-space accesses at 32-bit shared addresses (volatile: kept in program
// order among themselves; stores are compiler memory barriers)
__device__ __forceinline__ unsigned lds32(unsigned a) {
  unsigned v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts32(unsigned a, unsigned v) { asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory"); }
__device__ __forceinline__ void lds_pair(unsigned a, unsigned &x, unsigned &y) {
  asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(x), "=r"(y) : "r"(a));
}
__device__ __forceinline__ void lds_pair(unsigned a, unsigned long long &x, unsigned long long &y) {
  asm volatile("ld.shared.v2.u64 {%0, %1}, [%2];" : "=l"(x), "=l"(y) : "r"(a));
}
__device__ __forceinline__ void sts_pair(unsigned a, unsigned x, unsigned y) {
  asm volatile("st.shared.v2.u32 [%0], {%1, %2};" ::"r"(a), "r"(x), "r"(y) : "memory");
}
__device__ __forceinline__ void sts_pair(unsigned a, unsigned long long x, unsigned long long y) {
  asm volatile("st.shared.v2.u64 [%0], {%1, %2};" ::"r"(a), "l"(x), "l"(y) : "memory");
}
__device__ __forceinline__ void sts_mask(unsigned a, unsigned x) { asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(x) : "memory"); }
__device__ __forceinline__ void sts_mask(unsigned a, unsigned long long x) {
  asm volatile("st.shared.u64 [%0], %1;" ::"r"(a), "l"(x) : "memory");
}

__device__ __forceinline__ uint2 lds_u2(unsigned a) {
  uint2 v;
  asm("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
  return v;
}

// W64: the launch's pairs are on > 32-node molecules (64-bit masks); else all
// masks, stack entries and loads are 32-bit
// PS: the plan entries are copied to shared memory (VQ <= kJoinLanePlanSmemMax)
#ifndef SIGMO_JL_UNROLL
#define SIGMO_JL_UNROLL 4  // DFS steps per check of the free lanes (configs[2] join: 1/2/3/4 -> 4.86/4.69/4.65/4.64 ms)
#endif
#ifndef SIGMO_JL_MAXNREG
#define SIGMO_JL_MAXNREG 56
#endif
template <int MODE, bool W64, bool PS>
__global__ void __launch_bounds__(jl_threads(W64)) __maxnreg__(W64 ? 64 : SIGMO_JL_MAXNREG) k_join_lane(const __grid_constant__ JoinParams jp) {
  using MT = typename std::conditional<W64, unsigned long long, unsigned>::type;
  constexpr unsigned ES = W64 ? 16u : 8u;  // stack entry bytes
  constexpr unsigned sw = W64 ? 1u : 0u;   // word shift of an adjacency / window entry
  extern __shared__ __align__(16) unsigned char smem[];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int MQ = jp.maxq, SD = MQ > 1 ? MQ - 1 : 1;
  // ---- CTA tables ----
  // plan entries (8 B, JoinParams::qp_ent2): a shared-memory copy when they fit, else through the read-only cache
  const unsigned o_plan = 16u;
  if (PS)
    for (int i = threadIdx.x; i < jp.VQ; i += blockDim.x) ((uint2 *)(smem + o_plan))[i] = __ldg(&jp.qp_ent2[i]);
  // plan entry at shared-space address / global index p (an explicit ld.shared:
  // a generic smem + offset re-derives the shared window every step)
  const unsigned sbase = (unsigned)__cvta_generic_to_shared(smem);
#define JL_PLAN(p) (PS ? lds_u2(p) : __ldg(&jp.qp_ent2[(p)]))
  const unsigned wbase = (unsigned)(join_lane_cta_bytes(jp.VQ, jp.plan_smem_max) + (size_t)wid * join_lane_warp_bytes(MQ, W64));
  constexpr unsigned LS = ES;  // stack entries {R, U} interleaved per lane
  const unsigned oRU = wbase + LS * lane;  // stack entry of depth d: oRU + 32 ES d
  const unsigned mA = oRU - LS * lane + 32u * ES * SD + 4u * lane;  // map word of depth d: mA + 128 d (slot SD: absent)
  // stack entry {R, U} and map word of depth d at 32-bit shared addresses
  // (explicit ld/st.shared: generic smem + offset accesses re-derive the
  // shared window every step)
  const unsigned sRU = sbase + oRU, sMA = sbase + mA;
#define JL_LDRU(a, r, u) lds_pair((a), r, u)
#define JL_STRU(a, r, u) sts_pair((a), (MT)(r), (MT)(u))
#define JL_MAPR(d) lds32(sMA + 128u * (unsigned)(d))
#define JL_MAPW(d, x) sts32(sMA + 128u * (unsigned)(d), (x))
  auto popc = [](MT x) -> int { return W64 ? __popcll((unsigned long long)x) : __popc((unsigned)x); };
  auto highest = [](MT x) -> unsigned {  // index of the highest set bit (x != 0)
    unsigned r;
    if (W64) {  // two 32-bit bfinds and a select (bfind.u64 compiles to a branch)
      const unsigned hi = (unsigned)((unsigned long long)x >> 32), lo = (unsigned)x;
      unsigned fh, fl;
      asm("bfind.u32 %0, %1;" : "=r"(fh) : "r"(hi));
      asm("bfind.u32 %0, %1;" : "=r"(fl) : "r"(lo));
      r = hi ? fh + 32u : fl;
    } else {
      asm("bfind.u32 %0, %1;" : "=r"(r) : "r"((unsigned)x));
    }
    return r;
  };
  auto bfind32 = [](unsigned x) -> unsigned {
    unsigned r;
    asm("bfind.u32 %0, %1;" : "=r"(r) : "r"(x));
    return r;
  };
  auto lowest = [](MT x) -> unsigned {  // index of the lowest set bit (x != 0)
    return W64 ? (unsigned)(__ffsll((long long)x) - 1) : (unsigned)(__ffs((unsigned)x) - 1);
  };
  JL_MAPW(SD, jp.adj_ones);  // absent back-edges read the all-ones entry (class field 0)
  // the two base pointers of the step's global loads pass through shared memory: read back from there
  // they stay in registers (a kernel-parameter value is re-loaded from the constant bank every step)
  if (threadIdx.x == 0) *(ulonglong2 *)smem = make_ulonglong2((unsigned long long)jp.cmol, (unsigned long long)jp.adjw);
  __syncthreads();
  const uint32_t *cmol, *adjw;
  {
    unsigned long long pc, pa;
    asm volatile("ld.shared.v2.u64 {%0, %1}, [%2];" : "=l"(pc), "=l"(pa) : "r"(sbase));
    cmol = (const uint32_t *)pc;
    adjw = (const uint32_t *)pa;
  }

  const unsigned lt = (1u << lane) - 1u;
  // this launch's pairs: records / results [pair_base, pair_base + pair_count)
  const I64x2 ptot = jp.off[jp.ND];  // (pairs of <= 32-node molecules, pairs of larger ones)
  const unsigned P = (unsigned)(W64 ? ptot.b : ptot.a);
  const long long pbase0 = W64 ? ptot.a : 0;
  const int4 *const recs = jp.prec + pbase0;
  unsigned long long *const presult = jp.pair_result + pbase0;
  unsigned *const counter = (unsigned *)jp.chunk_counter;
  // mask of adjacency word index i (entries of 1 or 2 words)
  auto adj = [&](unsigned i) -> MT {
    SIGMO_BOUND((unsigned long long)i + sw < jp.adj_limit);
    if (W64) return (MT)__ldg((const unsigned long long *)(adjw + i));
    return (MT)__ldg(adjw + i);
  };
  // candidate window at cmol word index i
  auto cand = [&](unsigned i) -> MT {
    SIGMO_BOUND((unsigned long long)i + sw < jp.cmol_limit);
    if (W64) return (MT)__ldg((const unsigned long long *)(cmol + i));
    return (MT)__ldg(cmol + i);
  };
  // plan address (smem byte offset, or global index) of plan position i
  auto paddr = [&](unsigned i) -> unsigned { return PS ? sbase + o_plan + 8u * i : i; };
  constexpr unsigned PSTEP = PS ? 8u : 1u;
  // plan position of depth 0 of the pair whose depth-1 plan address is a
  auto cqb_of = [&](unsigned a) -> unsigned { return PS ? (a - sbase - o_plan) / 8u - 1u : a - 1u; };

  // ---- the warp's pairs: blocks of kJoinClaim consecutive GMCR pairs claimed by one same-address
  // atomic per block (one atomic per chunk of 32 serialised the launch on the counter), a block ahead;
  // lane 0 holds the pre-claimed block's start until it is needed.  Warp-uniform: cursor = the next
  // pair to hand out, bend = the end of its block ----
  unsigned cursor, bend, bnext0 = 0u;
  {
    unsigned x = 0u;
    if (lane == 0) x = atomicAdd(counter, 2u * kJoinClaim);
    x = __shfl_sync(FULL_MASK, x, 0);
    cursor = x;
    bend = x + kJoinClaim;
    bnext0 = x + kJoinClaim;
  }
  unsigned drained = cursor >= P ? 1u : 0u;
  int keff = jp.batchK;  // free lanes that end a stepping phase (1 once the list is drained)
  if (drained) keff = 1;

  // ---- lane state ----
  unsigned ne = 0u;  // open depths of the current pair (0: no work)
  unsigned pend = 0u;  // holds a pair (part) whose result is not yet written
  unsigned shared = 0u;
  unsigned cmb = 0u;  // cmol index of the current pair's first candidate window
  unsigned ca = 0u, ngs = 0u, pe = 0u;  // ca: adjacency index of the molecule's node 0; pe: plan address of depth 1
  unsigned cp = 0u;
  unsigned long long cnt = 0ull;
  unsigned steps = 0u;
  unsigned nv = 0u;  // next pair assigned (its record in registers)
  unsigned nr = 0u;  // and the load of its root window issued (the refill pass after the record's)
  int4 nrec = make_int4(0, 0, 0, 0);
  unsigned nidx = 0u;
  MT nR0 = 0;

  // enumerate mode: the embeddings of a leaf step -- the
  // mapped depths 0..d (map words) plus each candidate w of the last depth --
  // written in query node order at the pair's cursor (count pass + scan set
  // it to the pair's first slot; several lanes may share a donated pair), and
  // the node set f(V_q) as a molecule-local bit mask
  auto emit = [&](MT X, int d, MT used) {
    const unsigned cqb = cqb_of(pe);
    unsigned long long r0 = 0ull, r1 = 0ull;
    for (int j = 0; j <= d; j++) {
      const unsigned qn = __ldg(&jp.qp_qn[cqb + (unsigned)j]);
      const unsigned long long b = (JL_MAPR(j) - ca) >> sw;
      if (qn < 8u) r0 |= b << (8u * qn);
      else r1 |= b << (8u * (qn - 8u));
    }
    const unsigned qe = __ldg(&jp.qp_qn[cqb + (unsigned)(d + 1)]);
    unsigned long long pos = atomicAdd(jp.ecur + pbase0 + cp, (unsigned long long)popc(X));
    while (X) {
      const unsigned w = lowest(X);
      X &= X - (MT)1;
      const unsigned long long a0 = r0 | (qe < 8u ? (unsigned long long)w << (8u * qe) : 0ull);
      const unsigned long long a1 = r1 | (qe >= 8u ? (unsigned long long)w << (8u * (qe - 8u)) : 0ull);
      if (jp.estride == 8) {
        ((unsigned long long *)jp.emaps)[pos] = a0;
      } else {
        ((ulonglong2 *)jp.emaps)[pos] = make_ulonglong2(a0, a1);
      }
      if (jp.esets) jp.esets[pos] = (unsigned long long)used | (1ull << w);
      pos++;
    }
  };

  while (true) {
    // ---- DFS steps: SIGMO_JL_UNROLL per check of the free lanes (the check is a ballot and a popcount) ----
#pragma unroll
    for (int u = 0; u < SIGMO_JL_UNROLL; u++) {
      if (ne) {
        const unsigned d = bfind32(ne);  // deepest open depth
        const unsigned bd = 1u << d;
        const unsigned od = sRU + 32u * ES * d;
        SIGMO_BOUND(d + 1u < (unsigned)MQ && od + ES <= sbase + (unsigned)jp.smem_bytes);
        // plan entry of depth e = d + 1 (x: back-edge map slots, leaf, #extra;
        // y: bond classes, distinct row)
        const uint2 en = JL_PLAN(pe + PSTEP * d);
        MT R, U;
        JL_LDRU(od, R, U);
        const unsigned v = highest(R);
        const MT bit = (MT)1 << v;
        const MT Rn = R ^ bit;
        sts_mask(od, Rn);
        ne ^= Rn ? 0u : bd;
        // map word of depth d = the adjacency index of f(pi_d); stored before the
        // back-edge slots are read, so a back-edge to d reads it
        JL_MAPW(d, ca + (v << sw));
        const unsigned a0 = lds32(sMA + (en.x & 0x7ffu));
        const unsigned a1 = lds32(sMA + (en.x >> 16));
        const unsigned i0 = (en.y & 7u) * ngs + a0, i1 = ((en.y >> 3) & 7u) * ngs + a1;
        const MT used = U | bit;
        MT X = cand(cmb + ((en.y >> 12) << sw)) & ~used & adj(i0) & adj(i1);
        if (!(MODE & 8) && (en.x & 0xf000u)) {  // > 2 back-edges at this depth (fused rings): rare
          const unsigned nex = (en.x >> 12) & 15u;
          const unsigned b0 = (unsigned)__ldg(&jp.qp_ent[cqb_of(pe) + d + 1u]).w;
  #pragma unroll 1
          for (unsigned k = 0; k < nex; k++) {
            const unsigned be = __ldg(&jp.qp_be[b0 + k]);
            X &= adj((be & 255u) * ngs + JL_MAPR(be >> 8));
          }
        }
        if (MODE & 2) {  // induced mode (R21): drop neighbours (any bond) of mapped non-adjacent depths
          const unsigned cn = (unsigned)jp.NB * ngs;
          // two depths per iteration (the second reads the all-zeros entry when absent)
  #pragma unroll 1
          for (unsigned nm = __ldg(&jp.qp_non[cqb_of(pe) + d + 1u]); nm;) {
            const unsigned ia = cn + JL_MAPR(__ffs(nm) - 1);
            nm &= nm - 1u;
            const unsigned ib = nm ? cn + JL_MAPR(__ffs(nm) - 1) : jp.adj_ones + 2u;
            nm &= nm - 1u;
            X &= ~(adj(ia) | adj(ib));
          }
        }
        // depth e is the last: count (or decide) its candidates; else push them
        // (no branches: the two outcomes are selects and a predicated store)
        const unsigned leaf = en.x & 0x800u;
        if ((MODE & 4) && leaf && X) emit(X, (int)d, used);  // enumerate mode: write the embeddings
        const MT Xl = leaf ? X : (MT)0;
        cnt += (unsigned long long)popc(Xl);
        if ((MODE & 1) && Xl) ne = 0u;  // Find First: the pair (part) is decided
        const bool push = X != Xl;
        if (push) JL_STRU(od + 32u * ES, X, used);
        ne += push ? bd + bd : 0u;  // bit d + 1 is clear: d is the deepest open depth
        if (!(MODE & 8)) steps++;  // the lean instantiation does not count steps
      }
    }
    if (__popc(__ballot_sync(FULL_MASK, ne == 0u)) < keff) continue;

    // ---- finished pairs (parts): result (the per-query totals are reduced from the results by
    // k_lane_totals) ----
    if (pend && ne == 0u) {
      SIGMO_BOUND(cp < P);
      if (MODE & 1) {
        if (!shared) presult[cp] = cnt ? 1ull : 0ull;
        else if (cnt) atomicOr(&presult[cp], 1ull);
      } else {
        if (!shared) presult[cp] = cnt;
        else if (cnt) atomicAdd(&presult[cp], cnt);
      }
      pend = false;
    }
    // ---- free lanes activate their prefetched next pair ----
    if (ne == 0u && nv) {
      if (!nr) nR0 = cand((unsigned)nrec.z + ((JL_PLAN(paddr((unsigned)nrec.w >> 16)).y >> 12) << sw));
      cp = nidx;
      cmb = (unsigned)nrec.z;
      ca = (unsigned)nrec.x;  // adjacency word offset of the molecule
      ngs = (((unsigned)nrec.w >> 8) & 0xffu) << sw;  // molecule size: class stride of the adjacency
      pe = paddr(((unsigned)nrec.w >> 16) + 1u);
      shared = false;
      pend = true;
      cnt = 0ull;
      const MT R0 = nR0;
      if ((nrec.w & 0xff) == 1) {
        cnt = (unsigned long long)popc(R0);
        if ((MODE & 4) && R0) emit(R0, -1, (MT)0);
      } else {
        JL_STRU(sRU, R0, (MT)0);
        ne = R0 ? 1u : 0u;
      }
      nv = false;
    }
    // ---- root window of the next pair, its record loaded a pass ago ----
    if (nv && !nr) {
      nR0 = cand((unsigned)nrec.z + ((JL_PLAN(paddr((unsigned)nrec.w >> 16)).y >> 12) << sw));
      nr = true;
    }
    // ---- lanes without a next pair take the next ones of the warp's blocks: record and root window
    // are loaded now and used when the current pair ends ----
    if (!drained) {
      const unsigned f = __ballot_sync(FULL_MASK, !nv);
      const unsigned n = (unsigned)__popc(f), rank = (unsigned)__popc(f & lt);
      const unsigned left = bend - cursor;  // >= 1
      unsigned bn = 0u;
      if (n >= left) {  // the pass reaches the pre-claimed block: claim the one after it
        bn = __shfl_sync(FULL_MASK, bnext0, 0);
        if (lane == 0) bnext0 = atomicAdd(counter, (unsigned)kJoinClaim);
      }
      const unsigned idx = rank < left ? cursor + rank : bn + (rank - left);
      if (((f >> lane) & 1u) && idx < P) {
        SIGMO_BOUND(idx < P);
        nrec = __ldg(recs + idx);
        nidx = idx;
        nv = true;
        nr = false;
      }
      if (n >= left) {
        cursor = bn + (n - left);
        bend = bn + kJoinClaim;
      } else {
        cursor += n;
      }
      if (cursor >= P) {
        drained = true;
        keff = 1;
      }
    }
    // ---- drained: idle lanes take the shallowest open depth of a busy lane ----
    const unsigned idle = __ballot_sync(FULL_MASK, ne == 0u && !nv && !pend);
    if (drained && idle) {
      const unsigned donors = __ballot_sync(FULL_MASK, (ne & (ne - 1u)) != 0u);
      const int npair = min(__popc(idle), __popc(donors));
      if (npair > 0) {
        const bool recv = ((idle >> lane) & 1u) && __popc(idle & lt) < npair;
        const bool give = ((donors >> lane) & 1u) && __popc(donors & lt) < npair;
        const int src = recv ? nth_set_bit(donors, __popc(idle & lt)) : lane;
        const int ds_own = __ffs(ne) - 1;  // shallowest open depth
        const int ds = __shfl_sync(FULL_MASK, ds_own, src);
        const unsigned s_cp = __shfl_sync(FULL_MASK, cp, src);
        const unsigned s_ngs = __shfl_sync(FULL_MASK, ngs, src);
        const unsigned s_pe = __shfl_sync(FULL_MASK, pe, src);
        const unsigned s_ca = __shfl_sync(FULL_MASK, ca, src);
        const unsigned s_cmb = __shfl_sync(FULL_MASK, cmb, src);
        if (give && !shared) {
          presult[cp] = 0ull;  // the pair's result is accumulated from several lanes from now on
          shared = true;
        }
        __syncwarp();
        if (recv) {
          const unsigned dl = (unsigned)(src - lane);  // donor offsets = mine + dl * (LS | 4)
          {
            MT r, u;
            JL_LDRU(sRU + 32u * ES * ds + LS * dl, r, u);
            JL_STRU(sRU + 32u * ES * ds, r, u);
          }
          for (int j = 0; j < ds; j++) JL_MAPW(j, lds32(sMA + 128u * j + 4u * dl));
          cmb = s_cmb;
          cp = s_cp;
          ngs = s_ngs;
          pe = s_pe;
          ca = s_ca;
          ne = 1u << ds;
          cnt = 0ull;
          shared = true;
          pend = true;
        }
        __syncwarp();
        if (give) ne &= ~(1u << ds_own);
      }
    }
    if (drained && __ballot_sync(FULL_MASK, ne != 0u || nv || pend) == 0u) break;
  }
  if (!(MODE & 8) && jp.stats) {
    unsigned long long s2 = steps;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s2 += __shfl_xor_sync(FULL_MASK, s2, o);
    if (lane == 0) atomicAdd(jp.stats, s2);
  }
#undef JL_LDRU
#undef JL_STRU
#undef JL_PLAN
#undef JL_MAPR
#undef JL_MAPW
}

// dynamic shared memory size and (optionally) the preferred shared-memory carveout of a k_join_lane instantiation
template <typename K>
static cudaError_t jl_attrs(K k, size_t smem, int carveout) {
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess && carveout >= 0)
    e = cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, carveout);
  return e;
}

template <int MODE, bool W64>
static cudaError_t launch_join_lane_t(const JoinParams &p, int grid, cudaStream_t st) {
  // plan entries in shared memory when they fit (join_lane_plan_bytes)
  if (join_lane_plan_bytes(p.VQ, p.plan_smem_max) > 0) {
    cudaError_t e = jl_attrs(k_join_lane<MODE, W64, true>, p.smem_bytes, p.carveout);
    if (e != cudaSuccess) return e;
    k_join_lane<MODE, W64, true><<<grid, p.lane_threads, p.smem_bytes, st>>>(p);
  } else {
    cudaError_t e = jl_attrs(k_join_lane<MODE, W64, false>, p.smem_bytes, p.carveout);
    if (e != cudaSuccess) return e;
    k_join_lane<MODE, W64, false><<<grid, p.lane_threads, p.smem_bytes, st>>>(p);
  }
  return cudaGetLastError();
}

// the k_join_lane instantiation of a launch: bit 0 Find First, bit 1 induced (p.induced), bit 2 enumerate
// (p.emaps, Find All semantics), bit 3 lean (p.lean: no plan position with > 2 back-edges and no DFS step
// counting; Find All / First only)
static int lane_mode(int mode, const JoinParams &p) {
  if (p.emaps) return p.induced ? 6 : 4;
  const int m = (mode & 1) | (p.induced ? 2 : 0);
  return (m < 2 && p.lean) ? (m | 8) : m;
}

#define SIGMO_JL_DISPATCH(F, ...)                                              \
  switch (lane_mode(mode, p)) {                                                \
    case 0: return w64 ? F<0, true>(__VA_ARGS__) : F<0, false>(__VA_ARGS__);   \
    case 1: return w64 ? F<1, true>(__VA_ARGS__) : F<1, false>(__VA_ARGS__);   \
    case 2: return w64 ? F<2, true>(__VA_ARGS__) : F<2, false>(__VA_ARGS__);   \
    case 3: return w64 ? F<3, true>(__VA_ARGS__) : F<3, false>(__VA_ARGS__);   \
    case 4: return w64 ? F<4, true>(__VA_ARGS__) : F<4, false>(__VA_ARGS__);   \
    case 6: return w64 ? F<6, true>(__VA_ARGS__) : F<6, false>(__VA_ARGS__);   \
    case 8: return w64 ? F<8, true>(__VA_ARGS__) : F<8, false>(__VA_ARGS__);   \
    default: return w64 ? F<9, true>(__VA_ARGS__) : F<9, false>(__VA_ARGS__);  \
  }

cudaError_t launch_join_lane(int mode, bool w64, const JoinParams &p, int grid, cudaStream_t st) {
  if (grid <= 0) return cudaSuccess;
  SIGMO_JL_DISPATCH(launch_join_lane_t, p, grid, st)
}

template <int MODE, bool W64>
static int join_lane_occ_t(size_t smem, bool ps, int carveout, int threads) {
  int n = 0;
  cudaError_t e;
  if (ps) {
    jl_attrs(k_join_lane<MODE, W64, true>, smem, carveout);
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_join_lane<MODE, W64, true>, threads, smem);
  } else {
    jl_attrs(k_join_lane<MODE, W64, false>, smem, carveout);
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k_join_lane<MODE, W64, false>, threads, smem);
  }
  if (e != cudaSuccess) {
    cudaGetLastError();
    return 1;
  }
  return n < 1 ? 1 : n;
}

int join_lane_blocks_per_sm(int mode, bool w64, const JoinParams &p, size_t smem) {
  // the instantiation launch_join_lane picks
  const bool ps = join_lane_plan_bytes(p.VQ, p.plan_smem_max) > 0;
  SIGMO_JL_DISPATCH(join_lane_occ_t, smem, ps, p.carveout, p.lane_threads)
}
#undef SIGMO_JL_DISPATCH

}  // namespace sigmo
