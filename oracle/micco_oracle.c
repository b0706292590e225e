/*
 * oracle/micco_oracle.c — CPU ORACLE (test infrastructure only; see
 * micco_oracle.h).  Plain C99, complex double written out as (re, im) pairs,
 * compiled -O2 -ffp-contract=off (no fused multiply-add, no fast-math, no
 * BLAS).  Nothing here is blocked, fused or reordered beyond the definitions
 * it cites.
 *
 * Definitions followed (PAPER.md line numbers; SURVEY.md §8(c) readings):
 *  - A graph's vertices are quark legs of hadron nodes, its edges quark
 *    propagations joining two legs (L11, L17, L50; reading #1).
 *  - Graph contraction deletes one edge after another; each deletion is a
 *    tensor contraction between the two hadron (or intermediate) nodes the
 *    edge joins, until only two nodes are left whose contraction yields the
 *    value (L17-19, L56-60).  When an edge joins two distinct components
 *    every edge between them is contracted in the same step (reading #4);
 *    the result keeps the left component's open legs, then the right's
 *    (reading #9).  An edge whose endpoints already share a component and
 *    that was not yet contracted is a (partial) trace of that component
 *    (the meson self-edge of reading #4/§8(b)).
 *  - Disconnected graphs: val = product of component scalars (reading #6).
 *  - C(t) = Σ_g c_g val_g(t), in graph order (L11; readings #3, #5).
 */
#include "micco_oracle.h"

#include <pthread.h>
#include <stdlib.h>
#include <string.h>

#include "../micco_inputs/synth.h"

#define MAXLEG 64 /* legs of one component (the oracle has no rank cap of its own) */

typedef struct {
  int r;            /* rank = number of open legs */
  int leg[MAXLEG];  /* open legs: global leg id = instance * 8 + position */
  int dim[MAXLEG];
  int64_t size;     /* product of dims */
  double *x;        /* 2*size doubles, interleaved, row-major over leg[] */
  int owned;
} comp_t;

static int64_t prod_dims(const int *d, int n) {
  int64_t s = 1;
  for (int i = 0; i < n; ++i) s *= d[i];
  return s;
}

/* Row-major offsets of every multi-index over the sub-list `pos` of a tensor
 * with dims `dim` (the index runs over pos[0] slowest ... pos[n-1] fastest).
 * out has prod(dim[pos[i]]) entries. */
static void offsets(const int *dim, int r, const int *pos, int n, int64_t *out) {
  int64_t stride[MAXLEG];
  int64_t s = 1;
  for (int i = r - 1; i >= 0; --i) { stride[i] = s; s *= dim[i]; }
  int idx[MAXLEG];
  for (int i = 0; i < n; ++i) idx[i] = 0;
  int64_t count = 1;
  for (int i = 0; i < n; ++i) count *= dim[pos[i]];
  for (int64_t c = 0; c < count; ++c) {
    int64_t o = 0;
    for (int i = 0; i < n; ++i) o += (int64_t)idx[i] * stride[pos[i]];
    out[c] = o;
    for (int i = n - 1; i >= 0; --i) {  /* odometer */
      if (++idx[i] < dim[pos[i]]) break;
      idx[i] = 0;
    }
  }
}

/* Contract component L with component R over the leg pairs (lp[i], rp[i]):
 *   Res[fl, fr] = Σ_k L[fl, k] · R[fr, k]
 * with fl over L's other legs (in order), fr over R's other legs, k over the
 * contracted pairs (in pair order).  Sequential accumulation over k. */
static int contract(const comp_t *L, const comp_t *R, const int *lp, const int *rp, int c,
                    comp_t *Res) {
  int lfree[MAXLEG], rfree[MAXLEG], nlf = 0, nrf = 0;
  for (int i = 0; i < L->r; ++i) {
    int used = 0;
    for (int j = 0; j < c; ++j) used |= (lp[j] == i);
    if (!used) lfree[nlf++] = i;
  }
  for (int i = 0; i < R->r; ++i) {
    int used = 0;
    for (int j = 0; j < c; ++j) used |= (rp[j] == i);
    if (!used) rfree[nrf++] = i;
  }
  for (int j = 0; j < c; ++j)
    if (L->dim[lp[j]] != R->dim[rp[j]]) return ORC_ERR_GRAPH;
  if (nlf + nrf > MAXLEG) return ORC_ERR_GRAPH;
  Res->r = nlf + nrf;
  for (int i = 0; i < nlf; ++i) { Res->leg[i] = L->leg[lfree[i]]; Res->dim[i] = L->dim[lfree[i]]; }
  for (int i = 0; i < nrf; ++i) { Res->leg[nlf + i] = R->leg[rfree[i]]; Res->dim[nlf + i] = R->dim[rfree[i]]; }
  Res->size = prod_dims(Res->dim, Res->r);
  int64_t nfl = 1, nfr = 1, nk = 1;
  for (int i = 0; i < nlf; ++i) nfl *= L->dim[lfree[i]];
  for (int i = 0; i < nrf; ++i) nfr *= R->dim[rfree[i]];
  for (int j = 0; j < c; ++j) nk *= L->dim[lp[j]];
  int64_t *oLf = malloc(sizeof(int64_t) * nfl), *oRf = malloc(sizeof(int64_t) * nfr);
  int64_t *oLk = malloc(sizeof(int64_t) * nk), *oRk = malloc(sizeof(int64_t) * nk);
  Res->x = malloc(sizeof(double) * 2 * Res->size);
  Res->owned = 1;
  if (!oLf || !oRf || !oLk || !oRk || !Res->x) {
    free(oLf); free(oRf); free(oLk); free(oRk); free(Res->x); Res->x = NULL;
    return ORC_ERR_OOM;
  }
  offsets(L->dim, L->r, lfree, nlf, oLf);
  offsets(R->dim, R->r, rfree, nrf, oRf);
  offsets(L->dim, L->r, lp, c, oLk);
  offsets(R->dim, R->r, rp, c, oRk);
  for (int64_t a = 0; a < nfl; ++a) {
    for (int64_t b = 0; b < nfr; ++b) {
      double sr = 0.0, si = 0.0;
      for (int64_t k = 0; k < nk; ++k) {
        const double *x = L->x + 2 * (oLf[a] + oLk[k]);
        const double *y = R->x + 2 * (oRf[b] + oRk[k]);
        double pr = x[0] * y[0] - x[1] * y[1];
        double pi = x[0] * y[1] + x[1] * y[0];
        sr += pr;
        si += pi;
      }
      Res->x[2 * (a * nfr + b)] = sr;
      Res->x[2 * (a * nfr + b) + 1] = si;
    }
  }
  free(oLf); free(oRf); free(oLk); free(oRk);
  return ORC_OK;
}

/* Partial trace of component A over its legs i and j (i != j):
 *   Res[f] = Σ_k A[f with leg i = leg j = k]. */
static int ptrace(const comp_t *A, int i, int j, comp_t *Res) {
  if (A->dim[i] != A->dim[j]) return ORC_ERR_GRAPH;
  int fr[MAXLEG], nf = 0;
  for (int l = 0; l < A->r; ++l)
    if (l != i && l != j) fr[nf++] = l;
  Res->r = nf;
  for (int l = 0; l < nf; ++l) { Res->leg[l] = A->leg[fr[l]]; Res->dim[l] = A->dim[fr[l]]; }
  Res->size = prod_dims(Res->dim, nf);
  int64_t nk = A->dim[i];
  int64_t *of = malloc(sizeof(int64_t) * Res->size);
  Res->x = malloc(sizeof(double) * 2 * Res->size);
  Res->owned = 1;
  if (!of || !Res->x) { free(of); free(Res->x); Res->x = NULL; return ORC_ERR_OOM; }
  offsets(A->dim, A->r, fr, nf, of);
  int64_t si_ = 1, sj_ = 1;
  for (int l = A->r - 1; l > i; --l) si_ *= A->dim[l];
  for (int l = A->r - 1; l > j; --l) sj_ *= A->dim[l];
  for (int64_t f = 0; f < Res->size; ++f) {
    double sr = 0.0, sim = 0.0;
    for (int64_t k = 0; k < nk; ++k) {
      const double *x = A->x + 2 * (of[f] + k * si_ + k * sj_);
      sr += x[0];
      sim += x[1];
    }
    Res->x[2 * f] = sr;
    Res->x[2 * f + 1] = sim;
  }
  free(of);
  return ORC_OK;
}

static void comp_free(comp_t *c) {
  if (c->owned) free(c->x);
  c->x = NULL;
  c->owned = 0;
}

static int validate(const orc_node *nodes, int32_t n_inst, const int32_t *inst_node, int32_t n_edges,
                    const orc_edge *edges) {
  int total = 0;
  for (int u = 0; u < n_inst; ++u) {
    if (nodes[inst_node[u]].rank < 1 || nodes[inst_node[u]].rank > 8) return ORC_ERR_GRAPH;
    total += nodes[inst_node[u]].rank;
  }
  if (2 * n_edges != total) return ORC_ERR_GRAPH;
  int *seen = calloc((size_t)n_inst * 8, sizeof(int));
  if (!seen) return ORC_ERR_OOM;
  int rc = ORC_OK;
  for (int e = 0; e < n_edges && rc == ORC_OK; ++e) {
    const orc_edge *E = &edges[e];
    if (E->u < 0 || E->u >= n_inst || E->v < 0 || E->v >= n_inst) { rc = ORC_ERR_GRAPH; break; }
    if (E->p < 0 || E->p >= nodes[inst_node[E->u]].rank) { rc = ORC_ERR_GRAPH; break; }
    if (E->q < 0 || E->q >= nodes[inst_node[E->v]].rank) { rc = ORC_ERR_GRAPH; break; }
    if (E->u == E->v && E->p == E->q) { rc = ORC_ERR_GRAPH; break; }
    if (seen[E->u * 8 + E->p]++ || seen[E->v * 8 + E->q]++) rc = ORC_ERR_GRAPH;
    if (nodes[inst_node[E->u]].N != nodes[inst_node[E->v]].N) rc = ORC_ERR_GRAPH;
  }
  free(seen);
  return rc;
}

static int find_leg(const comp_t *c, int gleg) {
  for (int i = 0; i < c->r; ++i)
    if (c->leg[i] == gleg) return i;
  return -1;
}

/* Size of the result of processing edge e now (for the oracle's greedy order). */
static int64_t step_result_size(comp_t *comps, const int *comp_of, const int *done,
                                const orc_edge *edges, int n_edges, int e) {
  int a = comp_of[edges[e].u], b = comp_of[edges[e].v];
  if (a == b) return comps[a].size / ((int64_t)comps[a].dim[find_leg(&comps[a], edges[e].u * 8 + edges[e].p)] *
                                      comps[a].dim[find_leg(&comps[a], edges[e].v * 8 + edges[e].q)]);
  int64_t s = comps[a].size * comps[b].size;
  for (int f = 0; f < n_edges; ++f) {
    if (done[f]) continue;
    int cu = comp_of[edges[f].u], cv = comp_of[edges[f].v];
    if ((cu == a && cv == b) || (cu == b && cv == a)) {
      int li = find_leg(&comps[cu], edges[f].u * 8 + edges[f].p);
      int64_t d = comps[cu].dim[li];
      s /= d * d;
    }
  }
  return s;
}

int orc_graph_value(const orc_node *nodes, int32_t Lt, int32_t n_inst, const int32_t *inst_node,
                    int32_t n_edges, const orc_edge *edges, const int32_t *order, int32_t t,
                    double out[2]) {
  if (!nodes || !inst_node || (n_edges && !edges) || !out || t < 0 || t >= Lt || n_inst < 1)
    return ORC_ERR_ARG;
  int rc = validate(nodes, n_inst, inst_node, n_edges, edges);
  if (rc) return rc;
  if (order) {
    int *chk = calloc(n_edges + 1, sizeof(int));
    for (int i = 0; i < n_edges; ++i) {
      if (order[i] < 0 || order[i] >= n_edges || chk[order[i]]++) { free(chk); return ORC_ERR_GRAPH; }
    }
    free(chk);
  }
  comp_t *comps = calloc(n_inst, sizeof(comp_t));
  int *comp_of = malloc(sizeof(int) * n_inst);
  int *alive = malloc(sizeof(int) * n_inst);
  int *done = calloc(n_edges + 1, sizeof(int));
  /* one component per instance: its tensor on slice t and its legs in order */
  for (int u = 0; u < n_inst; ++u) {
    const orc_node *nd = &nodes[inst_node[u]];
    comp_t *c = &comps[u];
    c->r = nd->rank;
    for (int p = 0; p < nd->rank; ++p) { c->leg[p] = u * 8 + p; c->dim[p] = nd->N; }
    c->size = prod_dims(c->dim, c->r);
    c->x = (double *)(nd->data + 2 * (int64_t)t * c->size);
    c->owned = 0;
    comp_of[u] = u;
    alive[u] = 1;
  }
  for (int step = 0; step < n_edges && rc == ORC_OK; ++step) {
    int e;
    if (order) {
      e = order[step];
      if (done[e]) continue;
    } else { /* oracle greedy: smallest result, then lowest edge index */
      e = -1;
      int64_t best = 0;
      for (int f = 0; f < n_edges; ++f) {
        if (done[f]) continue;
        int64_t s = step_result_size(comps, comp_of, done, edges, n_edges, f);
        if (e < 0 || s < best) { e = f; best = s; }
      }
      if (e < 0) break;
    }
    const orc_edge *E = &edges[e];
    int a = comp_of[E->u], b = comp_of[E->v];
    comp_t res;
    memset(&res, 0, sizeof(res));
    if (a == b) { /* trace of two legs of one component */
      int i = find_leg(&comps[a], E->u * 8 + E->p), j = find_leg(&comps[a], E->v * 8 + E->q);
      rc = ptrace(&comps[a], i, j, &res);
      done[e] = 1;
    } else {
      int lp[MAXLEG], rp[MAXLEG], c = 0;
      for (int f = 0; f < n_edges; ++f) {
        if (done[f]) continue;
        const orc_edge *F = &edges[f];
        int cu = comp_of[F->u], cv = comp_of[F->v];
        if (cu == a && cv == b) {
          lp[c] = find_leg(&comps[a], F->u * 8 + F->p); rp[c] = find_leg(&comps[b], F->v * 8 + F->q);
        } else if (cu == b && cv == a) {
          lp[c] = find_leg(&comps[a], F->v * 8 + F->q); rp[c] = find_leg(&comps[b], F->u * 8 + F->p);
        } else {
          continue;
        }
        done[f] = 1;
        ++c;
      }
      rc = contract(&comps[a], &comps[b], lp, rp, c, &res);
      comp_free(&comps[b]);
      alive[b] = 0;
      for (int u = 0; u < n_inst; ++u)
        if (comp_of[u] == b) comp_of[u] = a;
    }
    comp_free(&comps[a]);
    comps[a] = res;
  }
  /* value = product of the rank-0 component scalars, components in slot
   * order (reading #6) */
  double vr = 1.0, vi = 0.0;
  for (int u = 0; u < n_inst && rc == ORC_OK; ++u) {
    if (!alive[u]) continue;
    if (comps[u].r != 0) { rc = ORC_ERR_GRAPH; break; }
    double xr = comps[u].x[0], xi = comps[u].x[1];
    double nr = vr * xr - vi * xi, ni = vr * xi + vi * xr;
    vr = nr; vi = ni;
  }
  for (int u = 0; u < n_inst; ++u) comp_free(&comps[u]);
  free(comps); free(comp_of); free(alive); free(done);
  if (rc == ORC_OK) { out[0] = vr; out[1] = vi; }
  return rc;
}

int orc_graph_value_brute(const orc_node *nodes, int32_t Lt, int32_t n_inst, const int32_t *inst_node,
                          int32_t n_edges, const orc_edge *edges, int32_t t, double out[2]) {
  if (!nodes || !inst_node || (n_edges && !edges) || !out || t < 0 || t >= Lt) return ORC_ERR_ARG;
  int rc = validate(nodes, n_inst, inst_node, n_edges, edges);
  if (rc) return rc;
  int *edge_at = malloc(sizeof(int) * n_inst * 8);
  int *sigma = calloc(n_edges + 1, sizeof(int));
  int *dim = malloc(sizeof(int) * (n_edges + 1));
  for (int e = 0; e < n_edges; ++e) {
    edge_at[edges[e].u * 8 + edges[e].p] = e;
    edge_at[edges[e].v * 8 + edges[e].q] = e;
    dim[e] = nodes[inst_node[edges[e].u]].N;
  }
  double sr = 0.0, si = 0.0;
  for (;;) {
    double pr = 1.0, pi = 0.0;
    for (int u = 0; u < n_inst; ++u) {
      const orc_node *nd = &nodes[inst_node[u]];
      int64_t size = 1, off = 0;
      for (int p = 0; p < nd->rank; ++p) size *= nd->N;
      for (int p = 0; p < nd->rank; ++p) off = off * nd->N + sigma[edge_at[u * 8 + p]];
      const double *x = nd->data + 2 * ((int64_t)t * size + off);
      double nr = pr * x[0] - pi * x[1], ni = pr * x[1] + pi * x[0];
      pr = nr; pi = ni;
    }
    sr += pr;
    si += pi;
    int e = n_edges - 1;
    for (; e >= 0; --e) {
      if (++sigma[e] < dim[e]) break;
      sigma[e] = 0;
    }
    if (e < 0) break;
  }
  free(edge_at); free(sigma); free(dim);
  out[0] = sr;
  out[1] = si;
  return ORC_OK;
}

typedef struct {
  const orc_node *nodes;
  int32_t Lt, n_graphs;
  const int32_t *inst_off, *inst_node, *edge_off, *orders, *has_order;
  const orc_edge *edges;
  double *vals;
  int64_t next;
  int rc;
  pthread_mutex_t mu;
} job_t;

static void *worker(void *arg) {
  job_t *J = (job_t *)arg;
  int64_t total = (int64_t)J->n_graphs * J->Lt;
  for (;;) {
    pthread_mutex_lock(&J->mu);
    int64_t it = J->next++;
    int stop = J->rc != ORC_OK;
    pthread_mutex_unlock(&J->mu);
    if (it >= total || stop) break;
    int g = (int)(it / J->Lt), t = (int)(it % J->Lt);
    int32_t e0 = J->edge_off[g], e1 = J->edge_off[g + 1];
    const int32_t *ord = (J->orders && (!J->has_order || J->has_order[g])) ? J->orders + e0 : NULL;
    double v[2];
    int rc = orc_graph_value(J->nodes, J->Lt, J->inst_off[g + 1] - J->inst_off[g],
                             J->inst_node + J->inst_off[g], e1 - e0, J->edges + e0, ord, t, v);
    if (rc) {
      pthread_mutex_lock(&J->mu);
      J->rc = rc;
      pthread_mutex_unlock(&J->mu);
      break;
    }
    J->vals[2 * it] = v[0];
    J->vals[2 * it + 1] = v[1];
  }
  return NULL;
}

int orc_correlator(const orc_node *nodes, int32_t Lt, int32_t n_graphs, const int32_t *inst_off,
                   const int32_t *inst_node, const int32_t *edge_off, const orc_edge *edges,
                   const int32_t *orders, const int32_t *has_order, const double *coefs,
                   int32_t nthreads, double *graph_vals, double *corr) {
  if (!nodes || Lt < 1 || n_graphs < 0 || !inst_off || !inst_node || !edge_off || !coefs || !corr)
    return ORC_ERR_ARG;
  if (nthreads < 1) nthreads = 1;
  job_t J;
  memset(&J, 0, sizeof(J));
  J.nodes = nodes; J.Lt = Lt; J.n_graphs = n_graphs; J.inst_off = inst_off; J.inst_node = inst_node;
  J.edge_off = edge_off; J.edges = edges; J.orders = orders; J.has_order = has_order;
  J.vals = graph_vals ? graph_vals : malloc(sizeof(double) * 2 * (size_t)n_graphs * Lt + 16);
  pthread_mutex_init(&J.mu, NULL);
  pthread_t *th = malloc(sizeof(pthread_t) * nthreads);
  for (int i = 0; i < nthreads; ++i) pthread_create(&th[i], NULL, worker, &J);
  for (int i = 0; i < nthreads; ++i) pthread_join(th[i], NULL);
  free(th);
  pthread_mutex_destroy(&J.mu);
  if (J.rc == ORC_OK) {
    for (int t = 0; t < Lt; ++t) {
      double sr = 0.0, si = 0.0;
      for (int g = 0; g < n_graphs; ++g) { /* C(t) = Σ_g c_g val_g(t), graph order */
        const double *v = J.vals + 2 * ((int64_t)g * Lt + t);
        double cr = coefs[2 * g], ci = coefs[2 * g + 1];
        sr += cr * v[0] - ci * v[1];
        si += cr * v[1] + ci * v[0];
      }
      corr[2 * t] = sr;
      corr[2 * t + 1] = si;
    }
  }
  if (!graph_vals) free(J.vals);
  return J.rc;
}

void orc_synth_node(double *dst, uint64_t seed, uint64_t key, int64_t n_complex, int32_t mode,
                    double scale) {
  micco_synth_fill(dst, seed, key, 0, n_complex, mode, scale);
}
