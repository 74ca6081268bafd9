// lane_filter_body.cuh -- device code of the lane-path filter (DESIGN.md
// section 6 "k_filter_lane"; Alg. 1, section 4.5
// P:1242-1246).  Compiled twice:
//   * by nvcc inside libsigmo.so (sigmo_filter_lane.cu): the generic kernel,
//     which reads the query program (plane records, row programs, GMCR lists)
//     from tables at run time;
//   * by NVRTC at run time (sigmo_jit.cu, SIGMO_LF_JIT defined): the same
//     body specialised for ONE query program, whose generated header
//     (lf_generated.h) supplies the constants and the straight-line record,
//     row-group and GMCR-group sequences (no table decode, no loop overhead).
// The filter of the lane-join path (every data graph
// <= 64 atoms, every query <= kJoinLaneMaxQ nodes): InitializeCandidates
// (Alg. 1 l.29-37), GenerateSignatures (l.11-18, read
// as cumulative counts R4, saturated R8), RefineCandidates (l.19-28,
// P:580-591, per field R5) for every level at once, and the GMCR mapping test
// (section 4.5), writing each candidate window once.
//
// B200 design ("k_filter_lane"):
//   * one warp per GROUP of 4 slots, persistent CTAs.  A slot is 32 data
//     nodes: a narrow group holds 4 molecules of <= 32 atoms (slot k =
//     molecule k), a wide group 2 molecules of 33-64 atoms (slots 2m, 2m+1 =
//     nodes 0-31 / 32-63 of molecule m).  Lane = node inside the slot.  The
//     4 slots run as SIMD lanes of one instruction stream: every decode of
//     the query program (plane records, row programs, GMCR lists) is paid
//     once per 4 slots.
//   * signatures: bitset BFS, ball_r(v) = ball_{r-1}(v) | OR_{u in N(v)}
//     ball_{r-1}(u), gathered with warp shuffles over the <= 4 packed
//     neighbour ids of the node (nb4, written at load); count of field f at
//     radius r = popc(ball_r(v) \ {v} & fieldmask_f).
//   * planes: plane p = (r, f, t) is the 32-bit word [count_{r,f}(v) >= t]
//     of a slot, one ballot per (plane, slot); label planes likewise; kept in
//     the warp's shared memory as [channel][4 slots].
//   * rows (lane = distinct row): window = AND of the row's channels, one
//     128-bit shared load per channel for the 4 slots; stored once to
//     cmol[g][row] (coalesced: lanes = consecutive rows of one molecule).
//   * GMCR (lane = query): a query survives in molecule g iff each of its
//     distinct rows has a non-empty window, tested from the per-slot
//     non-empty ballots through the query's (word, bits) list.
#include "lane_filter_types.h"

namespace sigmo {

#define LF_FULL 0xffffffffu

#ifdef SIGMO_LF_JIT
#define LF_C(x) J_##x
#else
#define LF_C(x) fp.x
#endif

// 128-bit shared store by lane 0 only (a store of the same value by all 32
// lanes still costs 4 shared wavefronts); a = shared-window address
__device__ __forceinline__ void lf_sts128_lane0(unsigned a, const uint4 v, int lane) {
  asm volatile(
      "{\n .reg .pred p;\n setp.eq.s32 p, %5, 0;\n @p st.shared.v4.u32 [%0], {%1, %2, %3, %4};\n}\n" ::"r"(a),
      "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "r"(lane)
      : "memory");
}

template <bool W> struct LfBall { typedef unsigned T; };
template <> struct LfBall<true> { typedef unsigned long long T; };

__host__ __device__ inline size_t lf_align16(size_t x) { return (x + 15) & ~(size_t)15; }

// shared-memory layout: CTA tables, then one region per warp
struct LaneFilterLayout {
  size_t rowp, rgn, grec, qwl, qwh, lut, rrec, warps;
  size_t w_planes, w_fm, w_dnz, w_ball, w_total;
  size_t total;
};

__host__ __device__ inline LaneFilterLayout lane_filter_layout(const FilterLaneParams &p) {
  LaneFilterLayout L;
  const int NDRW = (p.NDR + 31) / 32;
  size_t o = 0;
  L.rowp = o; o = lf_align16(o + (p.tables_global ? 0 : 16 * (size_t)p.NDR * p.RWV));
  L.rgn = o;  o = lf_align16(o + 4 * (size_t)NDRW);
  L.grec = o; o = lf_align16(o + 8 * (size_t)(p.NREC > 0 ? p.NREC : 1));
  L.qwl = o;  o = lf_align16(o + (p.tables_global ? 0 : 8 * (size_t)p.NQWE));
  L.qwh = o;  o = lf_align16(o + 8 * (size_t)(p.NQG > 0 ? p.NQG : 1));
  L.lut = o;  o = lf_align16(o + 2 * 256);
  L.rrec = o; o = lf_align16(o + 4 * (size_t)(4 * kMaxRadius + 1));
  L.warps = o;
  size_t w = 0;
  L.w_planes = w; w = lf_align16(w + 16 * (size_t)p.NCH);
  L.w_fm = w;     w = lf_align16(w + 16 * (size_t)(p.NFU > 0 ? p.NFU : 1));
  L.w_dnz = w;    w = lf_align16(w + 16 * (size_t)NDRW);
  L.w_ball = w;   w = lf_align16(w + 8 * 64 * 2);
  L.w_total = w;
  L.total = o + w * (kFilterLaneThreads / 32);
  return L;
}

__device__ __forceinline__ uint4 lds128(const unsigned char *p) { return *(const uint4 *)p; }
__device__ __forceinline__ void and4(uint4 &a, const uint4 b) {
  a.x &= b.x;
  a.y &= b.y;
  a.z &= b.z;
  a.w &= b.w;
}

// threshold planes of one record (NP planes of one (radius, field) group):
// c = |ball_r(v) \ {v}| in the record's field, plane word = ballot(c >= t)
// per slot, stored as [channel][4 slots] (every lane stores the same value:
// one unpredicated 128-bit shared store)
template <bool WIDE, int NP, typename BT>
__device__ __forceinline__ void lf_record(const BT (&bx)[4], const uint4 fm, unsigned pp, unsigned thr, int lane) {
  int c[4];
  if constexpr (WIDE) {
    const unsigned long long f0 = (unsigned long long)fm.x | ((unsigned long long)fm.y << 32);
    const unsigned long long f1 = (unsigned long long)fm.z | ((unsigned long long)fm.w << 32);
    c[0] = __popcll((unsigned long long)bx[0] & f0);
    c[1] = __popcll((unsigned long long)bx[1] & f0);
    c[2] = __popcll((unsigned long long)bx[2] & f1);
    c[3] = __popcll((unsigned long long)bx[3] & f1);
  } else {
    c[0] = __popc((unsigned)bx[0] & fm.x);
    c[1] = __popc((unsigned)bx[1] & fm.y);
    c[2] = __popc((unsigned)bx[2] & fm.z);
    c[3] = __popc((unsigned)bx[3] & fm.w);
  }
#pragma unroll
  for (int j = 0; j < NP; j++) {
    const int t = (int)((thr >> (8 * j)) & 0xffu);
    uint4 w;
    w.x = __ballot_sync(LF_FULL, c[0] >= t);
    w.y = __ballot_sync(LF_FULL, c[1] >= t);
    w.z = __ballot_sync(LF_FULL, c[2] >= t);
    w.w = __ballot_sync(LF_FULL, c[3] >= t);
    lf_sts128_lane0(pp + 16u * j, w, lane);
  }
}

// threshold planes of the records [e0, e1), each with exactly NP planes
template <bool WIDE, int NP, typename BT>
__device__ __forceinline__ void plane_records(int e0, int e1, const uint2 *grec, const unsigned char *wfm,
                                              unsigned wpl_s, const BT (&bx)[4], int lane) {
  for (int e = e0; e < e1; e++) {
    // record: x = field slot | #planes << 8 | first plane channel << 16, y = thresholds (bytes)
    const uint2 g = grec[e];
    lf_record<WIDE, NP>(bx, lds128(wfm + 16 * (g.x & 0xffu)), wpl_s + 16u * (g.x >> 16), g.y, lane);
  }
}

// 32x32 bit-matrix transpose across the warp: lane L holds row L (bit p =
// element (L, p)); returns column `lane` (bit L = element (L, lane))
__device__ __forceinline__ unsigned lf_transpose32(unsigned x, int lane) {
#pragma unroll
  for (int j = 16; j >= 1; j >>= 1) {
    const unsigned m = j == 16 ? 0x0000ffffu : j == 8 ? 0x00ff00ffu : j == 4 ? 0x0f0f0f0fu : j == 2 ? 0x33333333u
                                                                                               : 0x55555555u;
    const unsigned sw = ((x << j) & ~m) | ((x >> j) & m);
    const unsigned y = __shfl_xor_sync(LF_FULL, sw, j);
    const unsigned K = (lane & j) ? ~m : m;
    x = (x & K) | (y & ~K);
  }
  return x;
}

// one 32-row group: lane = distinct row 32 rg + lane; window = AND of the
// row's channels for the 4 slots, stored once; per-slot non-empty ballots
// into the warp's [row group][4 slots] array.  NWC = channel-pair words of
// the group (0: runtime nw, rows are sorted by length so it is uniform).
struct LFRowCtx {
  const uint4 *rowp;
  unsigned char *wpl, *wdz;
  uint32_t *cmol;
  unsigned obase[4];
  bool sval[4];
  int lane;
};

__device__ __forceinline__ void lf_and_pair(uint4 &acc, const unsigned char *wpl, unsigned pw) {
  and4(acc, lds128(wpl + (pw & 0xffffu)));
  and4(acc, lds128(wpl + (pw >> 16)));
}

template <bool WIDE, int NWC>
__device__ __forceinline__ void lf_row_group(int rg, int nw, int NDR, int RWV, const LFRowCtx &c) {
  constexpr unsigned OS = WIDE ? 2u : 1u;  // words per window
  const int row = 32 * rg + c.lane;
  uint4 acc = make_uint4(0u, 0u, 0u, 0u);
  if (row < NDR) {
    acc = make_uint4(LF_FULL, LF_FULL, LF_FULL, LF_FULL);
    const uint4 *pr = c.rowp + (size_t)row * RWV;
    if (NWC > 0) {
#pragma unroll
      for (int q = 0; q < NWC; q += 4) {
        const uint4 pw = pr[q >> 2];
        lf_and_pair(acc, c.wpl, pw.x);
        if (q + 1 < NWC) lf_and_pair(acc, c.wpl, pw.y);
        if (q + 2 < NWC) lf_and_pair(acc, c.wpl, pw.z);
        if (q + 3 < NWC) lf_and_pair(acc, c.wpl, pw.w);
      }
    } else {
      for (int q = 0; q < nw; q += 4) {
        const uint4 pw = pr[q >> 2];
        switch (nw - q) {  // uniform across the warp: rows are sorted by length
          default:
            lf_and_pair(acc, c.wpl, pw.w);
            [[fallthrough]];
          case 3:
            lf_and_pair(acc, c.wpl, pw.z);
            [[fallthrough]];
          case 2:
            lf_and_pair(acc, c.wpl, pw.y);
            [[fallthrough]];
          case 1:
            lf_and_pair(acc, c.wpl, pw.x);
        }
      }
    }
    const unsigned ro = OS * (unsigned)row;
    if (c.sval[0]) c.cmol[c.obase[0] + ro] = acc.x;
    if (c.sval[1]) c.cmol[c.obase[1] + ro] = acc.y;
    if (c.sval[2]) c.cmol[c.obase[2] + ro] = acc.z;
    if (c.sval[3]) c.cmol[c.obase[3] + ro] = acc.w;
  }
  uint4 ne;
  ne.x = __ballot_sync(LF_FULL, acc.x != 0u);
  ne.y = __ballot_sync(LF_FULL, acc.y != 0u);
  ne.z = __ballot_sync(LF_FULL, acc.z != 0u);
  ne.w = __ballot_sync(LF_FULL, acc.w != 0u);
  if (WIDE) {  // a molecule's row is non-empty if either half is
    ne.x |= ne.y;
    ne.y = ne.x;
    ne.z |= ne.w;
    ne.w = ne.z;
  }
  lf_sts128_lane0((unsigned)__cvta_generic_to_shared(c.wdz) + 16u * rg, ne, c.lane);
}

// one 32-query group of the GMCR test: lane = query; a query
// survives in a molecule iff every (word, bits) entry of its list is covered
// by the molecule's non-empty distinct rows.  EC = entries (0: runtime ne).
template <bool WIDE, int NM, int EC>
__device__ __forceinline__ void lf_gmcr_group(int qg, int e0, int ne, int NQ, int NQW, const uint2 *qwl,
                                              const unsigned char *wdz, int lane, int my_mol, uint32_t *gm,
                                              long long &cnt) {
  unsigned f0 = 0u, f1 = 0u, f2 = 0u, f3 = 0u;
  const int n = EC > 0 ? EC : ne;
#pragma unroll
  for (int j = 0; j < (EC > 0 ? EC : 1); j++) {
    if (EC == 0 && j >= n) break;
    const uint2 e = qwl[(size_t)(e0 + j) * 32 + lane];
    const uint4 d = lds128(wdz + 16 * e.x);
    f0 |= e.y & ~d.x;
    f1 |= e.y & ~d.y;
    f2 |= e.y & ~d.z;
    f3 |= e.y & ~d.w;
  }
  if (EC == 0)
    for (int j = 1; j < n; j++) {
      const uint2 e = qwl[(size_t)(e0 + j) * 32 + lane];
      const uint4 d = lds128(wdz + 16 * e.x);
      f0 |= e.y & ~d.x;
      f1 |= e.y & ~d.y;
      f2 |= e.y & ~d.z;
      f3 |= e.y & ~d.w;
    }
  const bool qv = 32 * qg + lane < NQ;
  unsigned w[4];
  w[0] = __ballot_sync(LF_FULL, qv && f0 == 0u);
  w[1] = __ballot_sync(LF_FULL, qv && f1 == 0u);
  w[2] = __ballot_sync(LF_FULL, qv && f2 == 0u);
  w[3] = __ballot_sync(LF_FULL, qv && f3 == 0u);
  // molecule m's word: slot m (narrow) or slot 2m (wide; both halves carry it)
  unsigned gmw = 0u;
#pragma unroll
  for (int m = 0; m < NM; m++)
    if (lane == m) gmw = w[WIDE ? 2 * m : m];
  if (my_mol >= 0) {
    gm[(size_t)my_mol * NQW + qg] = gmw;
    cnt += __popc(gmw);
  }
}

#ifdef SIGMO_LF_JIT
#include "lf_generated.h"
#endif

// one group of 4 slots.  WIDE: 2 molecules of 33-64 atoms (slots 2m + h =
// nodes 32h .. 32h+31 of molecule m), else 4 molecules of <= 32 atoms.
template <bool WIDE>
__device__ __forceinline__ void lane_filter_group(const FilterLaneParams &fp, int gi, int lane,
                                                  unsigned char *wsm, const LaneFilterLayout &L,
                                                  const unsigned char *smem, const uint4 *rowp,
                                                  const uint2 *qwl) {
  constexpr int NM = WIDE ? 2 : 4;  // molecules in the group
  unsigned char *wpl = wsm + L.w_planes;
  const unsigned wpl_s = (unsigned)__cvta_generic_to_shared(wpl);
  unsigned char *wfm = wsm + L.w_fm;
  unsigned char *wdz = wsm + L.w_dnz;
  unsigned long long *wball = (unsigned long long *)(wsm + L.w_ball);
  const uint16_t *lut = (const uint16_t *)(smem + L.lut);
  const uint2 *grec = (const uint2 *)(smem + L.grec);
  const int32_t *rrec = (const int32_t *)(smem + L.rrec);
  const int32_t *rgn = (const int32_t *)(smem + L.rgn);
  const int2 *qwh = (const int2 *)(smem + L.qwh);

  // ---- molecules of the group: {first node, n, adjacency word offset, candidate units} ----
  int mol[NM];
  if constexpr (WIDE) {
    const int2 m2 = __ldg((const int2 *)fp.grp_wide + gi);
    mol[0] = m2.x;
    mol[1] = m2.y;
  } else {
    const int4 m4 = __ldg((const int4 *)fp.grp_narrow + gi);
    mol[0] = m4.x;
    mol[1] = m4.y;
    mol[2] = m4.z;
    mol[3] = m4.w;
  }
  int my_mol = -1;  // lane m < NM: molecule m (GMCR words and pair counts)
#pragma unroll
  for (int m = 0; m < NM; m++)
    if (lane == m) my_mol = mol[m];
  uint4 mr[NM];
#pragma unroll
  for (int m = 0; m < NM; m++) mr[m] = mol[m] >= 0 ? __ldg(&fp.mrec[mol[m]]) : make_uint4(0u, 0u, 0u, 0u);

  // ---- nodes: slot k holds node v = 32 h + lane of molecule m ----
  unsigned lt[4], nb[4];
#pragma unroll
  for (int k = 0; k < 4; k++) {
    const int m = WIDE ? k >> 1 : k;
    const unsigned v = (WIDE ? 32u * (k & 1) : 0u) + (unsigned)lane;
    const bool ok = v < mr[m].y;
    lt[k] = 0xffffu;
    nb[k] = v * 0x01010101u;  // filler = the node itself (OR-neutral in the BFS)
    if (ok) {
      lt[k] = lut[__ldg(fp.label + mr[m].x + v)];
      nb[k] = __ldg(fp.nb4 + mr[m].x + v);
    }
  }
  // channel NLAB: the slot's existing atoms (row padding, and the start of a
  // wildcard '*' row, R22)
  {
    unsigned vm[4];
#pragma unroll
    for (int k = 0; k < 4; k++) {
      const int m = WIDE ? k >> 1 : k;
      const int lo = WIDE ? 32 * (k & 1) : 0;
      const int nk = (int)mr[m].y - lo;
      vm[k] = nk >= 32 ? LF_FULL : (nk <= 0 ? 0u : (1u << nk) - 1u);
    }
    lf_sts128_lane0(wpl_s + 16u * (unsigned)LF_C(NLAB), make_uint4(vm[0], vm[1], vm[2], vm[3]), lane);
  }
  // label planes (channels 0..NLAB-1) and field masks [NFU][4 slots]
  if (LF_C(NLAB) + LF_C(NFU) <= 32) {
    // per slot, lane = node builds its one-hot word (bit c: label channel c,
    // bit NLAB + f: field slot f); a warp transpose turns it into lane = channel
    unsigned tw[4];
#pragma unroll
    for (int k = 0; k < 4; k++) {
      const unsigned lc = lt[k] & 0xffu, fs = lt[k] >> 8;
      unsigned mb = lc < 32u ? 1u << lc : 0u;
      mb |= fs < 32u ? 1u << ((unsigned)LF_C(NLAB) + fs) : 0u;
      tw[k] = lf_transpose32(mb, lane);
    }
    const uint4 w = make_uint4(tw[0], tw[1], tw[2], tw[3]);
    if (lane < LF_C(NLAB)) *(uint4 *)(wpl + 16 * lane) = w;
    else if (lane < LF_C(NLAB) + LF_C(NFU)) *(uint4 *)(wfm + 16 * (lane - LF_C(NLAB))) = w;
  } else {
    for (int c = 0; c < LF_C(NLAB); c++) {
      uint4 w;
      w.x = __ballot_sync(LF_FULL, (lt[0] & 0xffu) == (unsigned)c);
      w.y = __ballot_sync(LF_FULL, (lt[1] & 0xffu) == (unsigned)c);
      w.z = __ballot_sync(LF_FULL, (lt[2] & 0xffu) == (unsigned)c);
      w.w = __ballot_sync(LF_FULL, (lt[3] & 0xffu) == (unsigned)c);
      *(uint4 *)(wpl + 16 * c) = w;
    }
    for (int f = 0; f < LF_C(NFU); f++) {
      uint4 w;
      w.x = __ballot_sync(LF_FULL, (lt[0] >> 8) == (unsigned)f);
      w.y = __ballot_sync(LF_FULL, (lt[1] >> 8) == (unsigned)f);
      w.z = __ballot_sync(LF_FULL, (lt[2] >> 8) == (unsigned)f);
      w.w = __ballot_sync(LF_FULL, (lt[3] >> 8) == (unsigned)f);
      *(uint4 *)(wfm + 16 * f) = w;
    }
  }
  __syncwarp();

  // ---- radii 1..R: BFS + threshold planes ----
  // balls: narrow u32 (bit = node of the molecule), wide u64
  using BT = typename LfBall<WIDE>::T;
  BT ball[4];
#pragma unroll
  for (int k = 0; k < 4; k++) {
    const int m = WIDE ? k >> 1 : k;
    const unsigned v = (WIDE ? 32u * (k & 1) : 0u) + (unsigned)lane;
    ball[k] = v < mr[m].y ? (BT)1 << v : (BT)0;
  }
  // nodes with > 4 neighbours (flag bit 7 of nb byte 0): slow path over the all-bonds adjacency mask
  bool slow[4];
#pragma unroll
  for (int k = 0; k < 4; k++) slow[k] = __any_sync(LF_FULL, (nb[k] & 0x80u) != 0u);

  for (int r = 1; r <= LF_C(R); r++) {
    if constexpr (!WIDE) {
      BT nx[4];
#pragma unroll
      for (int k = 0; k < 4; k++) {
        BT x = ball[k];
        x |= __shfl_sync(LF_FULL, ball[k], (int)(nb[k] & 31u));
        x |= __shfl_sync(LF_FULL, ball[k], (int)((nb[k] >> 8) & 31u));
        x |= __shfl_sync(LF_FULL, ball[k], (int)((nb[k] >> 16) & 31u));
        x |= __shfl_sync(LF_FULL, ball[k], (int)((nb[k] >> 24) & 31u));
        if (slow[k]) {  // rare: the 5th.. neighbours from the all-bonds adjacency mask
          const int m = k;
          const unsigned v = (unsigned)lane;
          unsigned rest = 0u;
          if ((nb[k] & 0x80u) && v < mr[m].y)
            rest = __ldg(fp.adjw + mr[m].z + (unsigned)fp.NB * mr[m].y + v);
          // drop the 4 neighbours already gathered
          rest &= ~((1u << (nb[k] & 31u)) | (1u << ((nb[k] >> 8) & 31u)) | (1u << ((nb[k] >> 16) & 31u)) |
                    (1u << ((nb[k] >> 24) & 31u)));
          unsigned any = __ballot_sync(LF_FULL, rest != 0u);
          while (any) {
            const int u = rest ? __ffs(rest) - 1 : lane;
            const unsigned y = __shfl_sync(LF_FULL, ball[k], u);
            if (rest) x |= y;
            rest &= rest - 1u;
            any = __ballot_sync(LF_FULL, rest != 0u);
          }
        }
        nx[k] = x;
      }
#pragma unroll
      for (int k = 0; k < 4; k++) ball[k] = nx[k];
    } else {
      // wide: balls of molecule m at wball[64 m + v]
#pragma unroll
      for (int k = 0; k < 4; k++) wball[64 * (k >> 1) + 32 * (k & 1) + lane] = ball[k];
      __syncwarp();
      BT nx[4];
#pragma unroll
      for (int k = 0; k < 4; k++) {
        const unsigned long long *bm = wball + 64 * (k >> 1);
        BT x = ball[k];
        x |= bm[nb[k] & 63u];
        x |= bm[(nb[k] >> 8) & 63u];
        x |= bm[(nb[k] >> 16) & 63u];
        x |= bm[(nb[k] >> 24) & 63u];
        const int m = k >> 1;
        const unsigned v = 32u * (k & 1) + (unsigned)lane;
        if (slow[k] && (nb[k] & 0x80u) && v < mr[m].y) {
          unsigned long long rest =
              __ldg((const unsigned long long *)(fp.adjw + mr[m].z + 2u * ((unsigned)fp.NB * mr[m].y + v)));
          rest &= ~((1ull << (nb[k] & 63u)) | (1ull << ((nb[k] >> 8) & 63u)) | (1ull << ((nb[k] >> 16) & 63u)) |
                    (1ull << ((nb[k] >> 24) & 63u)));
          while (rest) {
            x |= bm[__ffsll((long long)rest) - 1];
            rest &= rest - 1ull;
          }
        }
        nx[k] = x;
      }
      __syncwarp();
#pragma unroll
      for (int k = 0; k < 4; k++) ball[k] = nx[k];
    }
    // the node itself is not counted (u != v, R4)
    BT bx[4];
#pragma unroll
    for (int k = 0; k < 4; k++) {
      const unsigned v = (WIDE ? 32u * (k & 1) : 0u) + (unsigned)lane;
      bx[k] = ball[k] & ~((BT)1 << v);
    }
    __syncwarp();
#ifdef SIGMO_LF_JIT
    jit_records<WIDE>(r, bx, wfm, wpl_s, lane);  // generated: the query program's records of radius r, constants inlined
#else
    // records of radius r, in four runs of 1, 2, 3, 4 planes (no per-plane branches)
    const int *rr = rrec + 4 * (r - 1);
    plane_records<WIDE, 1>(rr[0], rr[1], grec, wfm, wpl_s, bx, lane);
    plane_records<WIDE, 2>(rr[1], rr[2], grec, wfm, wpl_s, bx, lane);
    plane_records<WIDE, 3>(rr[2], rr[3], grec, wfm, wpl_s, bx, lane);
    plane_records<WIDE, 4>(rr[3], rr[4], grec, wfm, wpl_s, bx, lane);
#endif
  }
  __syncwarp();

  // ---- rows: lane = distinct row; window = AND of the row's channels ----
  LFRowCtx rc;
  rc.rowp = rowp;
  rc.wpl = wpl;
  rc.wdz = wdz;
  rc.cmol = fp.cmol;
  rc.lane = lane;
#pragma unroll
  for (int k = 0; k < 4; k++) {
    const int m = WIDE ? k >> 1 : k;
    rc.sval[k] = mol[m] >= 0;
    rc.obase[k] = (unsigned)LF_C(NDR) * mr[m].w + (WIDE ? (unsigned)(k & 1) : 0u);
  }
#ifdef SIGMO_LF_JIT
  jit_rows<WIDE>(rc);  // generated: one call per 32-row group with its program length
#else
  for (int rg = 0; rg < (LF_C(NDR) + 31) / 32; rg++) lf_row_group<WIDE, 0>(rg, rgn[rg], LF_C(NDR), LF_C(RWV), rc);
#endif
  __syncwarp();

  // ---- GMCR: lane = query; its (word, bits) list over the
  // distinct-row non-empty bits, padded per 32-query group with (0, 0) ----
  long long cnt = 0;     // lane m < NM: surviving pairs of molecule m
#ifdef SIGMO_LF_JIT
  jit_gmcr<WIDE, NM>(qwl, wdz, lane, my_mol, fp.gm, cnt);  // generated: one call per 32-query group
#else
  for (int qg = 0; qg < LF_C(NQG); qg++) {
    const int2 h = qwh[qg];  // entry offset (x 32), entries
    lf_gmcr_group<WIDE, NM, 0>(qg, h.x, h.y, LF_C(NQ), LF_C(NQW), qwl, wdz, lane, my_mol, fp.gm, cnt);
  }
#endif
  if (my_mol >= 0) {
    I64x2 v;
    v.a = WIDE ? 0 : cnt;
    v.b = WIDE ? cnt : 0;
    fp.mol_cnt[my_mol] = v;
  }
  __syncwarp();
}

// kernel body (persistent CTAs, warp per group).  GL: row programs and GMCR
// lists read from global memory (tables too large for shared memory)
template <bool GL>
__device__ __forceinline__ void lf_kernel_body(const FilterLaneParams &fp) {
  extern __shared__ __align__(16) unsigned char smem[];
  constexpr int NWARP = kFilterLaneThreads / 32;
  const LaneFilterLayout L = lane_filter_layout(fp);
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  // ---- CTA tables ----
  if (!GL) {
    const uint4 *src = fp.rowp;
    uint4 *dst = (uint4 *)(smem + L.rowp);
    for (int i = tid; i < fp.NDR * fp.RWV; i += kFilterLaneThreads) dst[i] = __ldg(&src[i]);
    const uint2 *qs = fp.qwl;
    uint2 *qd = (uint2 *)(smem + L.qwl);
    for (int i = tid; i < fp.NQWE; i += kFilterLaneThreads) qd[i] = __ldg(&qs[i]);
  }
  {
    int32_t *rg = (int32_t *)(smem + L.rgn);
    for (int i = tid; i < (fp.NDR + 31) / 32; i += kFilterLaneThreads) rg[i] = __ldg(&fp.rgn[i]);
    uint2 *gr = (uint2 *)(smem + L.grec);
    for (int i = tid; i < fp.NREC; i += kFilterLaneThreads) gr[i] = __ldg(&fp.grec[i]);
    int2 *qh = (int2 *)(smem + L.qwh);
    for (int i = tid; i < fp.NQG; i += kFilterLaneThreads) qh[i] = __ldg(&fp.qwh[i]);
    uint16_t *lu = (uint16_t *)(smem + L.lut);
    for (int i = tid; i < 256; i += kFilterLaneThreads) lu[i] = __ldg(&fp.lut[i]);
    int32_t *rr = (int32_t *)(smem + L.rrec);
    for (int i = tid; i <= 4 * fp.R; i += kFilterLaneThreads) rr[i] = __ldg(&fp.rrec[i]);
  }
  unsigned char *wsm = smem + L.warps + (size_t)wid * L.w_total;
  __syncthreads();
  const uint4 *rowp = GL ? fp.rowp : (const uint4 *)(smem + L.rowp);
  const uint2 *qwl = GL ? fp.qwl : (const uint2 *)(smem + L.qwl);
  const int ng = fp.NGN + fp.NGW;
  for (int gi = blockIdx.x * NWARP + wid; gi < ng; gi += gridDim.x * NWARP) {
    if (gi < fp.NGN) lane_filter_group<false>(fp, gi, lane, wsm, L, smem, rowp, qwl);
    else lane_filter_group<true>(fp, gi - fp.NGN, lane, wsm, L, smem, rowp, qwl);
  }
}


#ifndef SIGMO_LF_JIT
template <bool GL>
__global__ void __launch_bounds__(kFilterLaneThreads) k_filter_lane(const __grid_constant__ FilterLaneParams fp) {
  lf_kernel_body<GL>(fp);
}
#endif

}  // namespace sigmo
