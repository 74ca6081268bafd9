/*
 * sigmo_oracle.c -- TEST INFRASTRUCTURE ONLY (not the product path).
 *
 * Plain, slow, obviously-correct CPU oracle for the SIGMo join result.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  It shares no code, header,
 * table or helper with the CUDA path (paper_conf_sc_carocfc25_b200/csrc);
 * it does NOT use the signature filter.
 *
 * What it computes (Def. 2.1; NLSM; edge
 * labels "are evaluated to prevent invalid matches"; Find All /
 * Find First), under DESIGN.md readings R1-R3:
 *
 *   count(q,g) = #{ f : V_q -> V_g injective |
 *                   for all v: L_q(v) == L_g(f(v))                       (1)
 *                   for all (u,v,b) in E_q: (f(u),f(v)) in E_g and
 *                                           bond_g(f(u),f(v)) == b }    (2)
 *   flag(q,g)  = [count(q,g) > 0], computed by an early-exit search.
 *
 * Algorithm (SURVEY.md 8(c), VF2/Ullmann-style backtracking):
 *   1. if n_q > n_g return 0
 *   2. static order pi: pi_0 = query node 0; next = the smallest-id unordered
 *      node adjacent to an ordered node; if none (disconnected query), the
 *      smallest-id unordered node
 *   3. back[i] = {(j,b) : j < i, (pi_j, pi_i, b) in E_q}
 *   4. recurse on depth i over data nodes v = 0..n_g-1: skip used v and
 *      L_g(v) != L_q(pi_i); require every (j,b) in back[i] to be a data edge
 *      (f(pi_j), v) with bond label b; assign, recurse, unassign
 *   5. at depth n_q count one embedding; Find First returns at the first leaf.
 *
 * Induced mode (mode bit 1, the literal G_D[X] reading of
 * Def. 2.1): additionally
 *                   for all u != v in V_q with (u,v) not in E_q:
 *                         (f(u),f(v)) not in E_g (any bond label)       (3)
 *   step 3b: non[i] = {j < i : (pi_j, pi_i) not in E_q}
 *   step 4b: require no data edge between f(pi_j) and v for j in non[i].
 *
 * Wildcard mode (mode bit 2, value 4, the paper's stated
 * next step P:2639-2645; R22): a query atom label 0 is the SMARTS
 * '*' (any atom) and a query bond label 0 the SMARTS '~' (any bond):
 *                   (1') L_q(v) == 0  or  L_q(v) == L_g(f(v))
 *                   (2') (f(u),f(v)) in E_g and (b == 0 or bond_g(f(u),f(v)) == b)
 *
 * Enumerate mode (NLSM outputs the embeddings themselves,
 * P:446-453, and atom typing needs every isomorphism): the same
 * search, but step 5 appends the leaf's mapping f, written in query node
 * order (f[pi_i] = map[i]), to the caller's buffer instead of counting it.
 *
 * Threads (std pthreads) split the data graphs into static contiguous chunks
 * and write independent per-pair slots, so results are deterministic.
 * Counts are u64; an addition that would overflow sets *overflow (R19).
 */
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
  int64_t num_graphs;
  const int64_t *graph_offsets; /* [num_graphs+1] */
  const int64_t *row_offsets;   /* [num_nodes+1]  */
  const int32_t *col_indices;   /* global node ids */
  const uint8_t *node_labels;
  const uint8_t *edge_labels;
} oracle_batch;

/* ---- per-query search plan (step 2 and 3) ---- */
typedef struct {
  int n;
  int order[64];
  uint8_t label[64];     /* label of order[i] */
  int nback[64];
  int back_j[64][64];    /* depth index j < i */
  int back_b[64][64];    /* bond label */
  int nnon[64];
  int non_j[64][64];     /* depth index j < i with (pi_j, pi_i) NOT in E_q (induced mode) */
} qplan;

static int build_plan(const oracle_batch *Q, int64_t q, qplan *P) {
  int64_t base = Q->graph_offsets[q];
  int n = (int)(Q->graph_offsets[q + 1] - base);
  if (n > 64) return -1;
  P->n = n;
  int ordered[64];
  int pos[64];
  memset(ordered, 0, sizeof(ordered));
  for (int i = 0; i < n; i++) pos[i] = -1;
  for (int i = 0; i < n; i++) {
    int pick = -1;
    if (i == 0) {
      pick = 0;
    } else {
      /* smallest-id unordered node adjacent to an ordered node */
      for (int u = 0; u < n && pick < 0; u++) {
        if (ordered[u]) continue;
        for (int64_t e = Q->row_offsets[base + u]; e < Q->row_offsets[base + u + 1]; e++) {
          int w = (int)(Q->col_indices[e] - base);
          if (w >= 0 && w < n && ordered[w]) { pick = u; break; }
        }
      }
      if (pick < 0)
        for (int u = 0; u < n; u++)
          if (!ordered[u]) { pick = u; break; }
    }
    ordered[pick] = 1;
    pos[pick] = i;
    P->order[i] = pick;
    P->label[i] = Q->node_labels[base + pick];
    P->nback[i] = 0;
    for (int64_t e = Q->row_offsets[base + pick]; e < Q->row_offsets[base + pick + 1]; e++) {
      int w = (int)(Q->col_indices[e] - base);
      if (w >= 0 && w < n && pos[w] >= 0 && w != pick) {
        P->back_j[i][P->nback[i]] = pos[w];
        P->back_b[i][P->nback[i]] = Q->edge_labels[e];
        P->nback[i]++;
      }
    }
    /* step 3b (induced mode): earlier depths not adjacent to pi_i */
    P->nnon[i] = 0;
    for (int j = 0; j < i; j++) {
      int adj = 0;
      for (int k = 0; k < P->nback[i]; k++)
        if (P->back_j[i][k] == j) adj = 1;
      if (!adj) P->non_j[i][P->nnon[i]++] = j;
    }
  }
  return 0;
}

/* ---- recursive search (step 4 and 5) ---- */
typedef struct {
  const qplan *P;
  int ng;
  int32_t *emb;         /* enumerate mode: embeddings [cap][n] (query node order), else NULL */
  int64_t emb_cap, emb_n;
  const uint8_t *glab;  /* [ng] */
  const int16_t *adjm;  /* [ng*ng], -1 = no edge, else bond label */
  int map[64];
  uint8_t used[256];
  int find_first;
  int induced;
  int wildcard;         /* mode bit 2: query label 0 = any atom, bond 0 = any bond */
  int overflow;
  uint64_t work;        /* search-tree nodes visited (informational) */
} search;

static uint64_t rec(search *S, int depth) {
  S->work++;
  if (depth == S->P->n) {
    if (S->emb) { /* enumerate mode: record f in query node order */
      if (S->emb_n < S->emb_cap)
        for (int i = 0; i < S->P->n; i++) S->emb[S->emb_n * S->P->n + S->P->order[i]] = S->map[i];
      S->emb_n++;
    }
    return 1;
  }
  uint64_t total = 0;
  for (int v = 0; v < S->ng; v++) {
    if (S->used[v]) continue;
    if (S->glab[v] != S->P->label[depth] && !(S->wildcard && S->P->label[depth] == 0)) continue; /* (1), (1') */
    int ok = 1;
    for (int k = 0; k < S->P->nback[depth]; k++) {
      int u = S->map[S->P->back_j[depth][k]];
      const int16_t b = S->adjm[u * S->ng + v];
      if (b < 0 || (b != S->P->back_b[depth][k] && !(S->wildcard && S->P->back_b[depth][k] == 0))) { ok = 0; break; }
    }
    if (!ok) continue;
    if (S->induced)  /* step 4b: no data edge (any bond) between v and f(pi_j) for j in non[i] */
      for (int k = 0; k < S->P->nnon[depth]; k++)
        if (S->adjm[S->map[S->P->non_j[depth][k]] * S->ng + v] >= 0) { ok = 0; break; }
    if (!ok) continue;
    S->used[v] = 1;
    S->map[depth] = v;
    uint64_t sub = rec(S, depth + 1);
    S->used[v] = 0;
    if (total + sub < total) S->overflow = 1;
    total += sub;
    if (S->find_first && total) return total;
  }
  return total;
}

/* ---- one data graph: adjacency matrix, then all requested queries ---- */
typedef struct {
  const oracle_batch *Q, *D;
  const qplan *plans;
  int find_first;
  /* dense mode */
  int64_t g_begin, g_end;
  uint64_t *dense_out;     /* [NQ*ND] row = query */
  /* pair-list mode */
  int64_t p_begin, p_end;
  const int64_t *pq, *pg;
  uint64_t *pair_out;
  uint64_t work;
  int overflow;
  int err;
} job;

static int load_graph(const oracle_batch *D, int64_t g, uint8_t *glab, int16_t *adjm, int *ng_out) {
  int64_t base = D->graph_offsets[g];
  int ng = (int)(D->graph_offsets[g + 1] - base);
  if (ng > 256) return -1;
  for (int i = 0; i < ng * ng; i++) adjm[i] = -1;
  for (int u = 0; u < ng; u++) {
    glab[u] = D->node_labels[base + u];
    for (int64_t e = D->row_offsets[base + u]; e < D->row_offsets[base + u + 1]; e++) {
      int64_t w = D->col_indices[e] - base;
      if (w < 0 || w >= ng) return -1;
      adjm[u * ng + (int)w] = D->edge_labels[e];
    }
  }
  *ng_out = ng;
  return 0;
}

static uint64_t count_one(job *J, const qplan *P, int ng, const uint8_t *glab, const int16_t *adjm) {
  if (P->n > ng) return 0; /* step 1 */
  search S;
  S.P = P;
  S.ng = ng;
  S.glab = glab;
  S.adjm = adjm;
  S.find_first = J->find_first & 1;
  S.induced = (J->find_first >> 1) & 1;
  S.wildcard = (J->find_first >> 2) & 1;
  S.overflow = 0;
  S.work = 0;
  S.emb = NULL;
  S.emb_cap = S.emb_n = 0;
  memset(S.used, 0, sizeof(S.used));
  uint64_t c = rec(&S, 0);
  J->work += S.work;
  if (S.overflow) J->overflow = 1;
  return (J->find_first & 1) ? (c ? 1u : 0u) : c;
}

static void *dense_worker(void *arg) {
  job *J = (job *)arg;
  uint8_t glab[256];
  int16_t *adjm = (int16_t *)malloc(sizeof(int16_t) * 256 * 256);
  int64_t NQ = J->Q->num_graphs, ND = J->D->num_graphs;
  for (int64_t g = J->g_begin; g < J->g_end; g++) {
    int ng;
    if (load_graph(J->D, g, glab, adjm, &ng)) { J->err = 1; break; }
    for (int64_t q = 0; q < NQ; q++)
      J->dense_out[q * ND + g] = count_one(J, &J->plans[q], ng, glab, adjm);
  }
  free(adjm);
  return NULL;
}

static void *pair_worker(void *arg) {
  job *J = (job *)arg;
  uint8_t glab[256];
  int16_t *adjm = (int16_t *)malloc(sizeof(int16_t) * 256 * 256);
  int64_t cur = -1;
  int ng = 0;
  for (int64_t p = J->p_begin; p < J->p_end; p++) {
    int64_t g = J->pg[p], q = J->pq[p];
    if (g < 0 || g >= J->D->num_graphs || q < 0 || q >= J->Q->num_graphs) { J->err = 1; break; }
    if (g != cur) {
      if (load_graph(J->D, g, glab, adjm, &ng)) { J->err = 1; break; }
      cur = g;
    }
    J->pair_out[p] = count_one(J, &J->plans[q], ng, glab, adjm);
  }
  free(adjm);
  return NULL;
}

static qplan *make_plans(const oracle_batch *Q) {
  qplan *plans = (qplan *)malloc(sizeof(qplan) * (size_t)(Q->num_graphs > 0 ? Q->num_graphs : 1));
  for (int64_t q = 0; q < Q->num_graphs; q++)
    if (build_plan(Q, q, &plans[q])) { free(plans); return NULL; }
  return plans;
}

static int run_jobs(job *jobs, int nthreads, void *(*fn)(void *), uint64_t *work_out, int *overflow_out) {
  pthread_t th[1024];
  for (int t = 0; t < nthreads; t++) pthread_create(&th[t], NULL, fn, &jobs[t]);
  int err = 0;
  uint64_t work = 0;
  int ovf = 0;
  for (int t = 0; t < nthreads; t++) {
    pthread_join(th[t], NULL);
    err |= jobs[t].err;
    work += jobs[t].work;
    ovf |= jobs[t].overflow;
  }
  if (work_out) *work_out = work;
  if (overflow_out) *overflow_out = ovf;
  return err ? -2 : 0;
}

/* Dense results out[q*ND + g] for every (query, data graph) pair.
 * mode bit 0: 0 = Find All (counts), 1 = Find First (0/1); mode bit 1
 * (value 2): induced-subgraph mode (Def. 2.1 read literally as G_D[X],
 * P:427-440, R21).  Returns 0 on success. */
int oracle_count_dense(const oracle_batch *Q, const oracle_batch *D, int mode, int nthreads,
                       uint64_t *out, uint64_t *work_out, int *overflow_out) {
  if (nthreads < 1) nthreads = 1;
  if (nthreads > 1024) nthreads = 1024;
  qplan *plans = make_plans(Q);
  if (!plans) return -1;
  job *jobs = (job *)calloc((size_t)nthreads, sizeof(job));
  int64_t ND = D->num_graphs;
  for (int t = 0; t < nthreads; t++) {
    jobs[t].Q = Q; jobs[t].D = D; jobs[t].plans = plans; jobs[t].find_first = mode;
    jobs[t].g_begin = ND * t / nthreads;
    jobs[t].g_end = ND * (t + 1) / nthreads;
    jobs[t].dense_out = out;
  }
  int rc = run_jobs(jobs, nthreads, dense_worker, work_out, overflow_out);
  free(jobs);
  free(plans);
  return rc;
}

/* Results for an explicit pair list (query idx pq[p], data graph pg[p]).
 * Pairs sorted by data graph run fastest (adjacency matrix reused). */
int oracle_count_pairs(const oracle_batch *Q, const oracle_batch *D, int mode, int nthreads,
                       int64_t npairs, const int64_t *pq, const int64_t *pg,
                       uint64_t *out, uint64_t *work_out, int *overflow_out) {
  if (nthreads < 1) nthreads = 1;
  if (nthreads > 1024) nthreads = 1024;
  qplan *plans = make_plans(Q);
  if (!plans) return -1;
  job *jobs = (job *)calloc((size_t)nthreads, sizeof(job));
  for (int t = 0; t < nthreads; t++) {
    jobs[t].Q = Q; jobs[t].D = D; jobs[t].plans = plans; jobs[t].find_first = mode;
    jobs[t].p_begin = npairs * t / nthreads;
    jobs[t].p_end = npairs * (t + 1) / nthreads;
    jobs[t].pq = pq; jobs[t].pg = pg; jobs[t].pair_out = out;
  }
  int rc = run_jobs(jobs, nthreads, pair_worker, work_out, overflow_out);
  free(jobs);
  free(plans);
  return rc;
}

/* Enumerate mode: every embedding f of query q in data graph g (Find All;
 * mode bit 1 = induced).  out[k * n_q + i] = molecule-local data node of
 * query node i in the k-th embedding, for k < cap; *n = the number of
 * embeddings (may exceed cap: call again with a larger buffer).  Returns 0
 * on success. */
int oracle_enumerate_pair(const oracle_batch *Q, const oracle_batch *D, int64_t q, int64_t g, int mode,
                          int32_t *out, int64_t cap, int64_t *n) {
  if (q < 0 || q >= Q->num_graphs || g < 0 || g >= D->num_graphs) return -1;
  qplan *P = (qplan *)malloc(sizeof(qplan));
  if (build_plan(Q, q, P)) { free(P); return -1; }
  uint8_t glab[256];
  int16_t *adjm = (int16_t *)malloc(sizeof(int16_t) * 256 * 256);
  int ng = 0;
  int rc = load_graph(D, g, glab, adjm, &ng);
  *n = 0;
  if (rc == 0 && P->n <= ng) { /* step 1 */
    search S;
    S.P = P;
    S.ng = ng;
    S.glab = glab;
    S.adjm = adjm;
    S.find_first = 0;
    S.induced = (mode >> 1) & 1;
    S.wildcard = (mode >> 2) & 1;
    S.overflow = 0;
    S.work = 0;
    S.emb = out;
    S.emb_cap = cap;
    S.emb_n = 0;
    memset(S.used, 0, sizeof(S.used));
    rec(&S, 0);
    *n = S.emb_n;
  }
  free(adjm);
  free(P);
  return rc;
}
