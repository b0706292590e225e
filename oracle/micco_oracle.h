/*
 * oracle/micco_oracle.h — CPU ORACLE (test infrastructure only).
 *
 * A plain, slow, obviously-correct implementation of what the MICCO hot path
 * computes: the correlation function C(t) = Σ_g c_g · val_g(t), where val_g(t)
 * is the full contraction of contraction graph g on time slice t
 * (§I, §II-A, §II-B).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  It shares no code with the
 * CUDA library; the only common source is the input generator
 * micco_inputs/synth.h.
 *
 * Element type: complex double, interleaved (re, im) — SURVEY.md §8(c)
 * reading #2.  Node tensor layout: [Lt][N]...[N] row-major, t slowest.
 */
#ifndef MICCO_ORACLE_H
#define MICCO_ORACLE_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  int32_t rank;        /* number of quark legs: 2 meson, 3 baryon */
  int32_t N;           /* dimension of every leg */
  const double *data;  /* 2 * Lt * N^rank doubles, interleaved re/im, t slowest */
} orc_node;

typedef struct { int32_t u, p, v, q; } orc_edge; /* leg p of instance u <-> leg q of instance v */

/* Status codes. */
#define ORC_OK 0
#define ORC_ERR_GRAPH -3
#define ORC_ERR_ARG -1
#define ORC_ERR_OOM -5

/* O2: naive pairwise contraction of one graph on slice t, along `order`
 * (a permutation of the edges; NULL = the oracle's own greedy order).
 * PAPER.md L17-19 / L56-60: reduce edges one after another; each reduction is
 * a tensor contraction between (intermediate) hadron nodes. */
int orc_graph_value(const orc_node *nodes, int32_t Lt, int32_t n_inst, const int32_t *inst_node,
                    int32_t n_edges, const orc_edge *edges, const int32_t *order, int32_t t,
                    double out[2]);

/* O1: brute-force full index summation (definition of val_g(t), SURVEY.md
 * §8(c)): Σ over all assignments σ of an index to every edge of
 * Π_u T_{h(u)}[t][σ(e(u,0)),...].  Only for tiny graphs (≤ ~10^7 terms). */
int orc_graph_value_brute(const orc_node *nodes, int32_t Lt, int32_t n_inst, const int32_t *inst_node,
                          int32_t n_edges, const orc_edge *edges, int32_t t, double out[2]);

/* The correlator C(t) = Σ_g c_g val_g(t), graphs in CSR form:
 * graph g has instances inst_node[inst_off[g] .. inst_off[g+1]) and edges
 * edges[edge_off[g] .. edge_off[g+1]); orders (same offsets as edges) may be
 * NULL, and has_order[g] == 0 selects the greedy order for graph g.
 * coefs: 2 doubles per graph.  val_g(t) are computed in parallel over
 * (g, t) with `nthreads` POSIX threads; the sum over g is sequential in graph
 * order.  graph_vals (optional, [G][Lt][2]) receives val_g(t); corr receives
 * [Lt][2]. */
int orc_correlator(const orc_node *nodes, int32_t Lt, int32_t n_graphs, const int32_t *inst_off,
                   const int32_t *inst_node, const int32_t *edge_off, const orc_edge *edges,
                   const int32_t *orders, const int32_t *has_order, const double *coefs,
                   int32_t nthreads, double *graph_vals, double *corr);

/* Input generation passthrough (micco_inputs/synth.h), so large parity cases
 * do not need Python-side buffers. */
void orc_synth_node(double *dst, uint64_t seed, uint64_t key, int64_t n_complex, int32_t mode,
                    double scale);

#ifdef __cplusplus
}
#endif
#endif
