/*
 * synth.c -- seeded, counter-based generator of synthetic ZINC-like
 * heavy-atom molecule graphs (inputs only).
 *
 * This module holds NO arithmetic of the method (no signatures, no
 * filtering, no matching).  It is the one module shared by the oracle side
 * (tests, bench cpu_baseline) and the CUDA side (tests, bench): both consume
 * the CSR-GO arrays it produces.
 *
 * Molecule i of a stream is a pure function of (seed, i, mode) -- shards and
 * batches are therefore reproducible in any order (SURVEY.md 8(d) recipe):
 *   * n ~ round(N(25,6)) clipped to [6,64] heavy atoms (mode 0); mode 1 is a
 *     ring-rich variant (n in [30,45], 3-5 rings) used to cut ring-system
 *     queries; mode 2 is mode 0 plus a 0.5% tail of 65-128-atom molecules
 *     (tests only);
 *   * rings ~ round(N(2.3,1.2)) clipped to [0,5]; size 6 (72%), 5 (25%),
 *     3/4/7 (1% each); 6-rings aromatic with p=.65, 5-rings with p=.45;
 *     fused (shared bond) with p=.3, otherwise linked by a 0-2 atom chain;
 *   * ring heteroatoms N/O/S (pyridine-, pyrrole-, furan-, thiophene-like);
 *   * acyclic growth respects valence and max degree 4;
 *   * heavy-atom label mix (atomic numbers) C 72, N 12, O 12, S 2, F 1,
 *     Cl 1, Br .4, P .1, I .1 (percent);
 *   * bond labels: 1 single, 2 double, 3 triple, 4 aromatic; ~50% of
 *     terminal O on C/S/P become double (carbonyl, sulfonyl, phosphoryl);
 *     ~30% of terminal N on a low-degree C become triple (nitrile).
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define MAXA 160
#define MAXE 512

/* ---------------- counter-based RNG (splitmix64 stream) ---------------- */
typedef struct { uint64_t s; } rng;

static uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static void rng_init(rng *r, uint64_t seed, uint64_t index, uint64_t stream) {
  r->s = mix64(seed ^ mix64(index * 0x9E3779B97F4A7C15ull + 0x632BE59BD9B4E019ull) ^ mix64(stream + 0x12345));
}
static uint64_t rng_next(rng *r) {
  r->s += 0x9E3779B97F4A7C15ull;
  return mix64(r->s);
}
static double rng_u01(rng *r) { return (double)(rng_next(r) >> 11) * (1.0 / 9007199254740992.0); }
static int rng_int(rng *r, int n) { return (int)(rng_u01(r) * n); } /* [0,n) */
static double rng_normal(rng *r) {
  double u1 = rng_u01(r), u2 = rng_u01(r);
  if (u1 < 1e-300) u1 = 1e-300;
  return sqrt(-2.0 * log(u1)) * cos(6.283185307179586 * u2);
}

/* ---------------- molecule builder ---------------- */
enum { H_ = 1, B_ = 5, C_ = 6, N_ = 7, O_ = 8, F_ = 9, P_ = 15, S_ = 16, CL_ = 17, BR_ = 35, I_ = 53 };

typedef struct {
  int n, ne;
  uint8_t lab[MAXA];
  int deg[MAXA];
  int hval[MAXA];   /* used valence in half-bond units */
  uint8_t ring[MAXA];
  int eu[MAXE], ev[MAXE];
  uint8_t eb[MAXE];
  uint8_t ering[MAXE];
} mol;

static int max_hval(uint8_t lab, int in_ring) {
  switch (lab) {
    case C_: return 8;
    case N_: return 6;
    case O_: return 4;
    case S_: return in_ring ? 4 : 12;
    case P_: return 10;
    case B_: return 6;
    default: return 2; /* halogens */
  }
}
static int max_deg(uint8_t lab, int in_ring) {
  switch (lab) {
    case C_: return 4;
    case N_: return 3;
    case O_: return 2;
    case S_: return in_ring ? 2 : 4;
    case P_: return 4;
    case B_: return 3;
    default: return 1;
  }
}
static int bond_hval(int b) { return b == 4 ? 3 : 2 * b; }

static int add_atom(mol *m, uint8_t lab, int ring) {
  if (m->n >= MAXA) return -1;
  int i = m->n++;
  m->lab[i] = lab;
  m->deg[i] = 0;
  m->hval[i] = 0;
  m->ring[i] = (uint8_t)ring;
  return i;
}
static int has_edge(const mol *m, int u, int v) {
  for (int e = 0; e < m->ne; e++)
    if ((m->eu[e] == u && m->ev[e] == v) || (m->eu[e] == v && m->ev[e] == u)) return 1;
  return 0;
}
static int add_bond(mol *m, int u, int v, int b, int ring) {
  if (u == v || u < 0 || v < 0 || m->ne >= MAXE || has_edge(m, u, v)) return -1;
  int e = m->ne++;
  m->eu[e] = u;
  m->ev[e] = v;
  m->eb[e] = (uint8_t)b;
  m->ering[e] = (uint8_t)ring;
  m->deg[u]++;
  m->deg[v]++;
  m->hval[u] += bond_hval(b);
  m->hval[v] += bond_hval(b);
  return e;
}
static int can_bond(const mol *m, int u, int b) {
  return m->deg[u] < max_deg(m->lab[u], m->ring[u]) && m->deg[u] < 4 &&
         m->hval[u] + bond_hval(b) <= max_hval(m->lab[u], m->ring[u]);
}

static uint8_t sample_chain_label(rng *r) {
  double u = rng_u01(r) * 1.006;
  if ((u -= 0.72) < 0) return C_;
  if ((u -= 0.12) < 0) return N_;
  if ((u -= 0.12) < 0) return O_;
  if ((u -= 0.02) < 0) return S_;
  if ((u -= 0.01) < 0) return F_;
  if ((u -= 0.01) < 0) return CL_;
  if ((u -= 0.004) < 0) return BR_;
  if ((u -= 0.001) < 0) return P_;
  return I_;
}

static int sample_ring_size(rng *r) {
  double u = rng_u01(r);
  if (u < 0.72) return 6;
  if (u < 0.97) return 5;
  if (u < 0.98) return 3;
  if (u < 0.99) return 4;
  return 7;
}

/* labels for the atoms of a ring of size s (positions 0..s-1) */
static void ring_labels(rng *r, int s, int arom, uint8_t *lab) {
  for (int i = 0; i < s; i++) lab[i] = C_;
  if (arom && s == 6) {
    for (int i = 0; i < s; i++)
      if (rng_u01(r) < 0.10) lab[i] = N_;
  } else if (arom && s == 5) {
    if (rng_u01(r) < 0.85) {
      double u = rng_u01(r);
      lab[0] = u < 0.5 ? N_ : (u < 0.75 ? O_ : S_);
      if (rng_u01(r) < 0.25) lab[2] = N_; /* imidazole / oxazole / thiazole-like */
    }
  } else {
    for (int i = 0; i < s; i++) {
      double u = rng_u01(r);
      if (u < 0.07) lab[i] = N_;
      else if (u < 0.11) lab[i] = O_;
    }
  }
}

static void build_molecule(uint64_t seed, int64_t index, int mode, mol *m) {
  rng R;
  rng_init(&R, seed, (uint64_t)index, (uint64_t)mode);
  m->n = 0;
  m->ne = 0;
  int target, nrings;
  if (mode == 1) {
    target = 30 + rng_int(&R, 16);
    nrings = 3 + rng_int(&R, 3);
  } else {
    target = (int)lround(25.0 + 6.0 * rng_normal(&R));
    if (target < 6) target = 6;
    if (target > 64) target = 64;
    if (mode == 2 && rng_u01(&R) < 0.005) target = 65 + rng_int(&R, 64);
    nrings = (int)lround(2.3 + 1.2 * rng_normal(&R));
    if (nrings < 0) nrings = 0;
    if (nrings > 5) nrings = 5;
    if (target > 64) nrings = 5 + rng_int(&R, 4);
  }

  /* ---- ring systems ---- */
  for (int k = 0; k < nrings; k++) {
    int s = sample_ring_size(&R);
    int arom = (s == 6 && rng_u01(&R) < 0.65) || (s == 5 && rng_u01(&R) < 0.45);
    int bt = arom ? 4 : 1;
    uint8_t lab[8];
    ring_labels(&R, s, arom, lab);
    int fused = (k > 0 && rng_u01(&R) < 0.3);
    if (fused) {
      /* share a ring bond (u,v) whose atoms both have room for one more bond */
      int cand[MAXE], nc = 0;
      for (int e = 0; e < m->ne; e++) {
        int u = m->eu[e], v = m->ev[e];
        if (m->ering[e] && m->deg[u] <= 2 && m->deg[v] <= 2 && m->lab[u] == C_ && m->lab[v] == C_) cand[nc++] = e;
      }
      if (nc > 0 && m->n + s - 2 <= target) {
        int e = cand[rng_int(&R, nc)];
        int u = m->eu[e], v = m->ev[e];
        int prev = u;
        for (int i = 0; i < s - 2; i++) {
          int a = add_atom(m, lab[i + 1], 1);
          add_bond(m, prev, a, bt, 1);
          prev = a;
        }
        add_bond(m, prev, v, bt, 1);
        continue;
      }
    }
    int chain = (k > 0) ? rng_int(&R, 3) : 0;
    if (m->n + s + chain > target) break;
    int anchor = -1;
    if (k > 0 && m->n > 0) {
      int cand[MAXA], nc = 0;
      for (int i = 0; i < m->n; i++)
        if (can_bond(m, i, 1)) cand[nc++] = i;
      if (nc == 0) break;
      anchor = cand[rng_int(&R, nc)];
      for (int i = 0; i < chain; i++) {
        int a = add_atom(m, C_, 0);
        add_bond(m, anchor, a, 1, 0);
        anchor = a;
      }
    }
    int first = m->n;
    for (int i = 0; i < s; i++) add_atom(m, lab[i], 1);
    for (int i = 0; i < s; i++) add_bond(m, first + i, first + (i + 1) % s, bt, 1);
    if (anchor >= 0) {
      /* attach at a ring atom with room (prefer carbon) */
      int at = first;
      for (int i = 0; i < s; i++)
        if (m->lab[first + i] == C_) { at = first + i; break; }
      add_bond(m, anchor, at, 1, 0);
    }
  }
  if (m->n == 0) add_atom(m, C_, 0);

  /* ---- acyclic growth ---- */
  while (m->n < target) {
    int cand[MAXA], nc = 0;
    for (int i = 0; i < m->n; i++)
      if (can_bond(m, i, 1)) cand[nc++] = i;
    if (nc == 0) break;
    int a = cand[rng_int(&R, nc)];
    uint8_t lab = sample_chain_label(&R);
    int bo = 1;
    uint8_t la = m->lab[a];
    if (lab == O_ && (la == C_ || la == S_ || la == P_) && rng_u01(&R) < 0.45 && can_bond(m, a, 2))
      bo = 2; /* carbonyl / sulfonyl / phosphoryl */
    else if (lab == N_ && la == C_ && !m->ring[a] && m->deg[a] <= 1 && rng_u01(&R) < 0.10 && can_bond(m, a, 3))
      bo = 3; /* nitrile */
    else if (lab == C_ && la == C_ && !m->ring[a] && rng_u01(&R) < 0.04 && can_bond(m, a, 2))
      bo = 2; /* alkene */
    int b = add_atom(m, lab, 0);
    if (b < 0) break;
    add_bond(m, a, b, bo, 0);
  }

  /* ---- bond orders on acyclic bonds ---- */
  for (int e = 0; e < m->ne; e++) {
    if (m->ering[e]) continue;
    int u = m->eu[e], v = m->ev[e];
    for (int side = 0; side < 2; side++) {
      int t = side ? u : v, o = side ? v : u; /* t terminal, o its neighbour */
      if (m->deg[t] != 1 || m->eb[e] != 1) continue;
      if (m->lab[t] == O_ && (m->lab[o] == C_ || m->lab[o] == S_ || m->lab[o] == P_)) {
        if (rng_u01(&R) < 0.5 && m->hval[o] + 2 <= max_hval(m->lab[o], m->ring[o]) && m->hval[t] + 2 <= 4) {
          m->eb[e] = 2;
          m->hval[o] += 2;
          m->hval[t] += 2;
        }
      } else if (m->lab[t] == N_ && m->lab[o] == C_ && m->deg[o] <= 2 && !m->ring[o]) {
        if (rng_u01(&R) < 0.3 && m->hval[o] + 4 <= 8) {
          m->eb[e] = 3;
          m->hval[o] += 4;
          m->hval[t] += 4;
        }
      }
    }
  }
}

/* ---------------- CSR emission ---------------- */
static int mol_adj_entries(const mol *m) { return 2 * m->ne; }

static void emit(const mol *m, int64_t node_base, int64_t adj_base, int64_t *row_offsets, int32_t *col,
                 uint8_t *nlab, uint8_t *elab) {
  /* neighbours of each atom sorted by id */
  int64_t pos = adj_base;
  for (int u = 0; u < m->n; u++) {
    row_offsets[u] = pos;
    nlab[u] = m->lab[u];
    int nb[MAXA];
    uint8_t bl[MAXA];
    int k = 0;
    for (int e = 0; e < m->ne; e++) {
      if (m->eu[e] == u) { nb[k] = m->ev[e]; bl[k] = m->eb[e]; k++; }
      else if (m->ev[e] == u) { nb[k] = m->eu[e]; bl[k] = m->eb[e]; k++; }
    }
    for (int i = 1; i < k; i++) { /* insertion sort */
      int x = nb[i];
      uint8_t y = bl[i];
      int j = i - 1;
      while (j >= 0 && nb[j] > x) { nb[j + 1] = nb[j]; bl[j + 1] = bl[j]; j--; }
      nb[j + 1] = x;
      bl[j + 1] = y;
    }
    for (int i = 0; i < k; i++) {
      col[pos - adj_base] = (int32_t)(node_base + nb[i]);
      elab[pos - adj_base] = bl[i];
      pos++;
    }
  }
}

typedef struct {
  uint64_t seed;
  int64_t first;
  int mode;
  int64_t begin, end;
  int32_t *natoms, *nadj;
  /* fill */
  const int64_t *goff, *aoff; /* per-molecule node / adjacency offsets (relative) */
  int64_t *row_offsets;
  int32_t *col;
  uint8_t *nlab, *elab;
} sjob;

static void *sizes_worker(void *arg) {
  sjob *J = (sjob *)arg;
  mol m;
  for (int64_t i = J->begin; i < J->end; i++) {
    build_molecule(J->seed, J->first + i, J->mode, &m);
    J->natoms[i] = m.n;
    J->nadj[i] = mol_adj_entries(&m);
  }
  return NULL;
}

static void *fill_worker(void *arg) {
  sjob *J = (sjob *)arg;
  mol m;
  for (int64_t i = J->begin; i < J->end; i++) {
    build_molecule(J->seed, J->first + i, J->mode, &m);
    int64_t nb = J->goff[i], ab = J->aoff[i];
    emit(&m, nb, ab, J->row_offsets + nb, J->col + ab, J->nlab + nb, J->elab + ab);
  }
  return NULL;
}

static void run(sjob *tmpl, int64_t count, int nthreads, void *(*fn)(void *)) {
  if (nthreads < 1) nthreads = 1;
  if (nthreads > 256) nthreads = 256;
  if (count < nthreads) nthreads = count > 0 ? (int)count : 1;
  pthread_t th[256];
  sjob jobs[256];
  for (int t = 0; t < nthreads; t++) {
    jobs[t] = *tmpl;
    jobs[t].begin = count * t / nthreads;
    jobs[t].end = count * (t + 1) / nthreads;
    pthread_create(&th[t], NULL, fn, &jobs[t]);
  }
  for (int t = 0; t < nthreads; t++) pthread_join(th[t], NULL);
}

/* Pass 1: per-molecule atom and adjacency-entry counts for molecules
 * first..first+count-1 of stream (seed, mode). */
int synth_sizes(uint64_t seed, int64_t first, int64_t count, int mode, int nthreads, int32_t *natoms,
                int32_t *nadj) {
  sjob t;
  memset(&t, 0, sizeof(t));
  t.seed = seed; t.first = first; t.mode = mode; t.natoms = natoms; t.nadj = nadj;
  run(&t, count, nthreads, sizes_worker);
  return 0;
}

/* Pass 2: fill CSR arrays.  goff/aoff are the exclusive prefix sums of the
 * pass-1 sizes (length count+1); row_offsets has goff[count]+1 entries (the
 * last one is written here), col/elab have aoff[count] entries, node ids in
 * col are global (goff-based). */
int synth_fill(uint64_t seed, int64_t first, int64_t count, int mode, int nthreads, const int64_t *goff,
               const int64_t *aoff, int64_t *row_offsets, int32_t *col, uint8_t *nlab, uint8_t *elab) {
  sjob t;
  memset(&t, 0, sizeof(t));
  t.seed = seed; t.first = first; t.mode = mode;
  t.goff = goff; t.aoff = aoff; t.row_offsets = row_offsets; t.col = col; t.nlab = nlab; t.elab = elab;
  run(&t, count, nthreads, fill_worker);
  row_offsets[goff[count]] = aoff[count];
  return 0;
}
