/*
 * fastt_oracle.c -- plain, slow, single-threaded CPU ORACLE for the FastT
 * strategy-search hot path (Yi et al., "Fast Training of Deep Learning Models
 * over Multiple GPUs", Middleware '20; /root/reference/PAPER.md = "P:<line>").
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or helper with the CUDA product path in
 * paper_conf_middleware_0001lmwlwyl20_b200/csrc/ and never calls it.
 *
 * Every function follows the paper's algorithm step by step, in the paper's
 * order, under the readings R1-R22 listed in DESIGN.md ("Readings").  There is
 * no blocking, fusion or clever data structure: the ready set is an array
 * scanned linearly, the split is materialised as a new graph, ranks are
 * recomputed from scratch for every candidate.
 *
 * Pins (tests/test_oracle_*.py): hand-derived examples (tests/golden/),
 * brute force over placements x topological orders on <=8-op DAGs,
 * closed forms, schedule invariants, an independent greedy-step replay
 * checker, Theorem 1 and published splitmix64 outputs.
 *
 * All times are int64 nanoseconds, all sizes int64 bytes (R18).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define FO_OK 0
#define FO_EINVAL (-1)
#define FO_ECYCLE (-2)
#define FO_ENOMEM (-3)
#define FO_ERANGE (-5)
#define FO_EUNSUP (-6)

#define FO_CAND_OK 0
#define FO_CAND_INFEASIBLE 1
#define FO_CAND_BADSPEC 2

#define FO_KIND_BASE 0
#define FO_KIND_PIN 1
#define FO_KIND_SPLIT 2

#define FO_DIM_BATCH 0
#define FO_DIM_CHANNEL 1

#define FO_F_CP_PIN 1u
#define FO_F_POLICY_INSERT 2u
#define FO_F_MEM_LIVE 64u /* liveness-based memory (NEXT N3, R24) */

#define FO_INF INT64_MAX
#define FO_MAXG 32
#define FO_MAXK 16
#define FO_MAXPINS 4

/* ------------------------------------------------------------------ graph */

/* G(O,E) of P:321 plus the devices, memory limits and cost models of
 * P:322-328.  Adjacency is CSR in both directions; every list is sorted by
 * the neighbour's id (that is the "pred order" / "succ order" of R13). */
typedef struct fo_graph {
  int32_t V, G, K;
  int64_t E;
  int32_t *succ_off, *succ_dst;
  int64_t *succ_bytes;
  uint8_t *succ_param;
  int32_t *pred_off, *pred_src;
  int64_t *pred_bytes;
  uint8_t *pred_param;
  int64_t *cost;        /* V*G, [op][device], ns; 0 = unknown */
  int64_t *mem, *param; /* V bytes */
  uint8_t *split_mask;  /* V, bit per splittable dimension */
  uint8_t *alive;       /* V, 0 = op removed by SplitOperation (Alg. 2 line 28) */
  int64_t *cap;         /* G */
  uint8_t *link_class;  /* G*G */
  int64_t alpha[FO_MAXK], beta[FO_MAXK];
  int64_t copy_fs;
} fo_graph;

static void fo_graph_free(fo_graph *g) {
  if (!g) return;
  free(g->succ_off); free(g->succ_dst); free(g->succ_bytes); free(g->succ_param);
  free(g->pred_off); free(g->pred_src); free(g->pred_bytes); free(g->pred_param);
  free(g->cost); free(g->mem); free(g->param); free(g->split_mask); free(g->alive);
  free(g->cap); free(g->link_class);
  free(g);
}

typedef struct { int32_t s, d; int64_t b; uint8_t p; } fo_edge;

static int cmp_edge_sd(const void *a, const void *b) {
  const fo_edge *x = a, *y = b;
  if (x->s != y->s) return x->s < y->s ? -1 : 1;
  if (x->d != y->d) return x->d < y->d ? -1 : 1;
  return 0;
}
static int cmp_edge_ds(const void *a, const void *b) {
  const fo_edge *x = a, *y = b;
  if (x->d != y->d) return x->d < y->d ? -1 : 1;
  if (x->s != y->s) return x->s < y->s ? -1 : 1;
  return 0;
}

/* Build both CSRs from an edge list.  Parallel edges are merged: bytes summed,
 * parameter flag OR-ed (R11).  Returns FO_ECYCLE on a self loop. */
static int fo_build_adjacency(fo_graph *g, fo_edge *ed, int64_t ne) {
  int32_t V = g->V;
  qsort(ed, (size_t)ne, sizeof(fo_edge), cmp_edge_sd);
  int64_t m = 0;
  for (int64_t e = 0; e < ne; e++) {
    if (ed[e].s == ed[e].d) return FO_ECYCLE;
    if (m > 0 && ed[m - 1].s == ed[e].s && ed[m - 1].d == ed[e].d) {
      if (ed[m - 1].b > INT64_MAX / 4 - ed[e].b) return FO_ERANGE; /* merged bytes stay far inside int64 */
      ed[m - 1].b += ed[e].b;
      ed[m - 1].p |= ed[e].p;
    } else {
      ed[m++] = ed[e];
    }
  }
  g->E = m;
  g->succ_off = calloc((size_t)V + 1, sizeof(int32_t));
  g->pred_off = calloc((size_t)V + 1, sizeof(int32_t));
  g->succ_dst = malloc(sizeof(int32_t) * (size_t)(m + 1));
  g->succ_bytes = malloc(sizeof(int64_t) * (size_t)(m + 1));
  g->succ_param = malloc((size_t)(m + 1));
  g->pred_src = malloc(sizeof(int32_t) * (size_t)(m + 1));
  g->pred_bytes = malloc(sizeof(int64_t) * (size_t)(m + 1));
  g->pred_param = malloc((size_t)(m + 1));
  if (!g->succ_off || !g->pred_off || !g->succ_dst || !g->succ_bytes || !g->succ_param ||
      !g->pred_src || !g->pred_bytes || !g->pred_param)
    return FO_ENOMEM;
  for (int64_t e = 0; e < m; e++) {
    g->succ_off[ed[e].s + 1]++;
    g->succ_dst[e] = ed[e].d;
    g->succ_bytes[e] = ed[e].b;
    g->succ_param[e] = ed[e].p;
  }
  for (int32_t i = 0; i < V; i++) g->succ_off[i + 1] += g->succ_off[i];
  qsort(ed, (size_t)m, sizeof(fo_edge), cmp_edge_ds);
  for (int64_t e = 0; e < m; e++) {
    g->pred_off[ed[e].d + 1]++;
    g->pred_src[e] = ed[e].s;
    g->pred_bytes[e] = ed[e].b;
    g->pred_param[e] = ed[e].p;
  }
  for (int32_t i = 0; i < V; i++) g->pred_off[i + 1] += g->pred_off[i];
  return FO_OK;
}

/* Kahn's algorithm; fills topo[] with the live ops in a topological order.
 * Returns the number of ops emitted (== number of live ops iff acyclic). */
static int32_t fo_topo(const fo_graph *g, int32_t *topo) {
  int32_t V = g->V, n = 0, head = 0, live = 0;
  int32_t *deg = malloc(sizeof(int32_t) * ((size_t)V + 1));
  for (int32_t i = 0; i < V; i++) {
    deg[i] = g->pred_off[i + 1] - g->pred_off[i];
    if (g->alive[i]) live++;
    if (g->alive[i] && deg[i] == 0) topo[n++] = i;
  }
  while (head < n) {
    int32_t i = topo[head++];
    for (int32_t e = g->succ_off[i]; e < g->succ_off[i + 1]; e++)
      if (--deg[g->succ_dst[e]] == 0) topo[n++] = g->succ_dst[e];
  }
  free(deg);
  (void)live;
  return n;
}

static int32_t fo_live_count(const fo_graph *g) {
  int32_t n = 0;
  for (int32_t i = 0; i < g->V; i++) n += g->alive[i] ? 1 : 0;
  return n;
}

/* ----------------------------------------------------------- cost models */

/* Communication cost model (R10): a linear function of the tensor
 * size per device-pair class; zero between ops on the same device (R6). */
static int64_t fo_comm_class(const fo_graph *g, int64_t bytes, int k) {
  /* ceil(bytes * beta / 1e6) with beta in femtoseconds per byte */
  int64_t num = bytes * g->beta[k];
  return g->alpha[k] + (num + 999999) / 1000000;
}
static int64_t fo_comm(const fo_graph *g, int64_t bytes, int s, int t) {
  if (s == t) return 0;
  return fo_comm_class(g, bytes, g->link_class[s * g->G + t]);
}
static int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

/* ------------------------------------------------------------- load/free */

int32_t fastt_ref_load(int32_t n_ops, int64_t n_edges, int32_t n_devices, const int32_t *src,
                       const int32_t *dst, const int64_t *bytes, const uint8_t *eparam,
                       const int64_t *cost, const int64_t *mem, const int64_t *param,
                       const uint8_t *split_mask, const int64_t *cap, const uint8_t *link_class,
                       int32_t n_classes, const int64_t *alpha, const int64_t *beta,
                       int64_t split_copy_fs, fo_graph **out) {
  *out = NULL;
  if (n_ops < 0 || n_edges < 0 || n_devices < 1 || n_devices > FO_MAXG || n_classes < 1 ||
      n_classes > FO_MAXK || split_copy_fs < 0)
    return FO_EINVAL;
  int32_t V = n_ops, G = n_devices;
  for (int64_t e = 0; e < n_edges; e++)
    if (src[e] < 0 || src[e] >= V || dst[e] < 0 || dst[e] >= V || bytes[e] < 0) return FO_EINVAL;
  for (int64_t i = 0; i < (int64_t)V * G; i++)
    if (cost[i] < 0) return FO_EINVAL;
  for (int32_t i = 0; i < V; i++)
    if (mem[i] < 0 || param[i] < 0 || param[i] > mem[i]) return FO_EINVAL;
  for (int32_t d = 0; d < G; d++)
    if (cap[d] < 0) return FO_EINVAL;
  for (int32_t d = 0; d < G * G; d++)
    if (link_class[d] >= n_classes) return FO_EINVAL;
  for (int32_t k = 0; k < n_classes; k++)
    if (alpha[k] < 0 || beta[k] < 0) return FO_EINVAL;
  fo_graph *g = calloc(1, sizeof(fo_graph));
  if (!g) return FO_ENOMEM;
  g->V = V; g->G = G; g->K = n_classes; g->copy_fs = split_copy_fs;
  for (int32_t k = 0; k < n_classes; k++) { g->alpha[k] = alpha[k]; g->beta[k] = beta[k]; }
  g->cost = malloc(sizeof(int64_t) * ((size_t)V * G + 1));
  g->mem = malloc(sizeof(int64_t) * ((size_t)V + 1));
  g->param = malloc(sizeof(int64_t) * ((size_t)V + 1));
  g->split_mask = malloc((size_t)V + 1);
  g->alive = malloc((size_t)V + 1);
  g->cap = malloc(sizeof(int64_t) * (size_t)G);
  g->link_class = malloc((size_t)G * G);
  if (V) {
    memcpy(g->cost, cost, sizeof(int64_t) * (size_t)V * G);
    memcpy(g->mem, mem, sizeof(int64_t) * (size_t)V);
    memcpy(g->param, param, sizeof(int64_t) * (size_t)V);
    memcpy(g->split_mask, split_mask, (size_t)V);
  }
  memset(g->alive, 1, (size_t)V + 1);
  memcpy(g->cap, cap, sizeof(int64_t) * (size_t)G);
  memcpy(g->link_class, link_class, (size_t)G * G);
  fo_edge *ed = malloc(sizeof(fo_edge) * (size_t)(n_edges + 1));
  for (int64_t e = 0; e < n_edges; e++) {
    ed[e].s = src[e]; ed[e].d = dst[e]; ed[e].b = bytes[e]; ed[e].p = eparam[e] ? 1 : 0;
  }
  int rc = fo_build_adjacency(g, ed, n_edges);
  free(ed);
  if (rc != FO_OK) { fo_graph_free(g); return rc; }
  /* parallel-edge sums and the linear comm model must stay inside int64 */
  for (int64_t e = 0; e < g->E; e++)
    for (int k = 0; k < g->K; k++)
      if (g->beta[k] && g->succ_bytes[e] > (INT64_MAX / 4) / g->beta[k]) { fo_graph_free(g); return FO_ERANGE; }
  /* ... and so must the split/concat node cost bytes * copy_fs (R13) */
  for (int64_t e = 0; e < g->E; e++)
    if (g->copy_fs && g->succ_bytes[e] > (INT64_MAX / 4) / g->copy_fs) { fo_graph_free(g); return FO_ERANGE; }
  int32_t *topo = malloc(sizeof(int32_t) * ((size_t)V + 1));
  int32_t n = fo_topo(g, topo);
  free(topo);
  if (n != V) { fo_graph_free(g); return FO_ECYCLE; }
  /* overflow guard: everything the method adds stays far below 2^62 */
  __int128 tot = 0, totm = 0;
  for (int32_t i = 0; i < V; i++) {
    int64_t mx = 0;
    for (int d = 0; d < G; d++) if (cost[(int64_t)i * G + d] > mx) mx = cost[(int64_t)i * G + d];
    tot += mx + G;
    totm += (__int128)mem[i] * (G + 1);
  }
  for (int64_t e = 0; e < g->E; e++) {
    int64_t mx = 0;
    for (int k = 0; k < g->K; k++) { int64_t c = fo_comm_class(g, g->succ_bytes[e], k); if (c > mx) mx = c; }
    tot += (__int128)(mx + (g->copy_fs ? ceil_div(g->succ_bytes[e] * g->copy_fs, 1000000) : 0)) * (G + 2);
  }
  if (tot >= ((__int128)1 << 58) || totm >= ((__int128)1 << 60)) { fo_graph_free(g); return FO_ERANGE; }
  *out = g;
  return FO_OK;
}

void fastt_ref_free(fo_graph *g) { fo_graph_free(g); }

int32_t fastt_ref_num_ops(const fo_graph *g) { return g->V; }
int64_t fastt_ref_num_edges(const fo_graph *g) { return g->E; }

/* ------------------------------------------------- SplitOperation (Alg. 2) */

/* Partition k of n of a tensor of b bytes (R13). */
static int64_t fo_part(int64_t b, int n, int k) { return b / n + (k < b % n ? 1 : 0); }

/* Is an edge with parameter flag p cut along dimension dim?  Batch split
 * (fine-grained data parallelism) cuts activations and replicates
 * parameters; channel split (fine-grained model parallelism) cuts parameters
 * and replicates activations (R13). */
static int fo_edge_cut(int dim, int p) { return dim == FO_DIM_BATCH ? !p : p; }

/* SplitOperation(G, op, d, n), Alg. 2 lines 16-30, materialised
 * as a new graph under R13: new ids appended as [split node per predecessor
 * (pred order), s_1..s_n, concat node per successor (succ order)]; the split
 * op stays as a removed tombstone so every other id is stable. */
static int fo_split_view(const fo_graph *g, int32_t op, int dim, int n, fo_graph **out) {
  int32_t V = g->V, G = g->G;
  int32_t P = g->pred_off[op + 1] - g->pred_off[op];
  int32_t S = g->succ_off[op + 1] - g->succ_off[op];
  int32_t V2 = V + P + n + S;
  fo_graph *h = calloc(1, sizeof(fo_graph));
  *h = *g;
  h->V = V2;
  h->cost = calloc((size_t)V2 * G + 1, sizeof(int64_t));
  h->mem = calloc((size_t)V2 + 1, sizeof(int64_t));
  h->param = calloc((size_t)V2 + 1, sizeof(int64_t));
  h->split_mask = calloc((size_t)V2 + 1, 1);
  h->alive = calloc((size_t)V2 + 1, 1);
  h->cap = malloc(sizeof(int64_t) * (size_t)G);
  h->link_class = malloc((size_t)G * G);
  memcpy(h->cap, g->cap, sizeof(int64_t) * (size_t)G);
  memcpy(h->link_class, g->link_class, (size_t)G * G);
  memcpy(h->cost, g->cost, sizeof(int64_t) * (size_t)V * G);
  memcpy(h->mem, g->mem, sizeof(int64_t) * (size_t)V);
  memcpy(h->param, g->param, sizeof(int64_t) * (size_t)V);
  memcpy(h->split_mask, g->split_mask, (size_t)V);
  memcpy(h->alive, g->alive, (size_t)V);
  /* Alg. 2 line 28: remove op and the edges connecting to it */
  h->alive[op] = 0;
  for (int d = 0; d < G; d++) h->cost[(int64_t)op * G + d] = 0;
  h->mem[op] = 0; h->param[op] = 0; h->split_mask[op] = 0;
  int32_t sp0 = V, s0 = V + P, con0 = V + P + n;
  int64_t ne = 0, cap_e = g->E + (int64_t)P * (1 + n) + (int64_t)S * (1 + n) + 1;
  fo_edge *ed = malloc(sizeof(fo_edge) * (size_t)cap_e);
  for (int32_t i = 0; i < V; i++)
    for (int32_t e = g->succ_off[i]; e < g->succ_off[i + 1]; e++) {
      if (i == op || g->succ_dst[e] == op) continue;
      ed[ne].s = i; ed[ne].d = g->succ_dst[e]; ed[ne].b = g->succ_bytes[e]; ed[ne].p = g->succ_param[e]; ne++;
    }
  /* Alg. 2 lines 17-19: n sub-operations; cost ceil(cost/n) on every device;
   * memory = partition of the non-parameter part + (replicated or cut) params */
  for (int k = 0; k < n; k++) {
    int32_t s = s0 + k;
    h->alive[s] = 1;
    for (int d = 0; d < G; d++) h->cost[(int64_t)s * G + d] = ceil_div(g->cost[(int64_t)op * G + d], n);
    int64_t act = g->mem[op] - g->param[op];
    int64_t prm = dim == FO_DIM_BATCH ? g->param[op] : fo_part(g->param[op], n, k);
    h->mem[s] = fo_part(act, n, k) + prm;
    h->param[s] = prm;
  }
  /* Alg. 2 lines 20-23: a split node per predecessor, cutting edge (pre,op)
   * into p_1..p_n, p_k -> s_k */
  for (int32_t a = 0; a < P; a++) {
    int32_t e = g->pred_off[op] + a, pre = g->pred_src[e], sp = sp0 + a;
    int64_t b = g->pred_bytes[e];
    uint8_t p = g->pred_param[e];
    h->alive[sp] = 1;
    int64_t c = g->copy_fs ? ceil_div(b * g->copy_fs, 1000000) : 0;
    for (int d = 0; d < G; d++) h->cost[(int64_t)sp * G + d] = c;
    ed[ne].s = pre; ed[ne].d = sp; ed[ne].b = b; ed[ne].p = p; ne++;
    for (int k = 0; k < n; k++) {
      ed[ne].s = sp; ed[ne].d = s0 + k; ed[ne].b = fo_edge_cut(dim, p) ? fo_part(b, n, k) : b; ed[ne].p = p; ne++;
    }
  }
  /* Alg. 2 lines 24-27: a concat node per successor gathering s_1..s_n */
  for (int32_t a = 0; a < S; a++) {
    int32_t e = g->succ_off[op] + a, suc = g->succ_dst[e], con = con0 + a;
    int64_t b = g->succ_bytes[e];
    uint8_t p = g->succ_param[e];
    h->alive[con] = 1;
    int64_t c = g->copy_fs ? ceil_div(b * g->copy_fs, 1000000) : 0;
    for (int d = 0; d < G; d++) h->cost[(int64_t)con * G + d] = c;
    for (int k = 0; k < n; k++) {
      ed[ne].s = s0 + k; ed[ne].d = con; ed[ne].b = fo_part(b, n, k); ed[ne].p = p; ne++;
    }
    ed[ne].s = con; ed[ne].d = suc; ed[ne].b = b; ed[ne].p = p; ne++;
  }
  h->succ_off = h->succ_dst = h->pred_off = h->pred_src = NULL;
  h->succ_bytes = h->pred_bytes = NULL;
  h->succ_param = h->pred_param = NULL;
  int rc = fo_build_adjacency(h, ed, ne);
  free(ed);
  if (rc != FO_OK) { fo_graph_free(h); return rc; }
  *out = h;
  return FO_OK;
}

/* ------------------------------------------------------ DPOS (Algorithm 1) */

typedef struct {
  int64_t makespan;
  uint8_t status;
  int64_t *peak;    /* G */
  uint8_t *place;   /* V, 0xFF = not scheduled / removed */
  int64_t *start;   /* V, -1 = not scheduled */
  int64_t *finish;  /* V */
  int32_t *order;   /* V, execution order list A, -1 padded */
  int32_t *dq;      /* V, dequeue sequence number, -1 */
  int32_t *deq;     /* V, ops in dequeue order, -1 padded */
} fo_result;

static void fo_result_alloc(fo_result *r, int32_t V, int32_t G) {
  r->peak = malloc(sizeof(int64_t) * (size_t)G);
  r->place = malloc((size_t)V + 1);
  r->start = malloc(sizeof(int64_t) * ((size_t)V + 1));
  r->finish = malloc(sizeof(int64_t) * ((size_t)V + 1));
  r->order = malloc(sizeof(int32_t) * ((size_t)V + 1));
  r->dq = malloc(sizeof(int32_t) * ((size_t)V + 1));
  r->deq = malloc(sizeof(int32_t) * ((size_t)V + 1));
}
static void fo_result_free(fo_result *r) {
  free(r->peak); free(r->place); free(r->start); free(r->finish); free(r->order); free(r->dq); free(r->deq);
}
static void fo_result_infeasible(fo_result *r, int32_t V, int32_t G, uint8_t status) {
  r->makespan = FO_INF;
  r->status = status;
  for (int d = 0; d < G; d++) r->peak[d] = -1;
  for (int32_t i = 0; i < V; i++) {
    r->place[i] = 0xFF; r->start[i] = -1; r->finish[i] = -1; r->order[i] = -1; r->dq[i] = -1; r->deq[i] = -1;
  }
}

/* w_i: "the maximal execution time of operation o_i (over different devices
 * that it could be assigned to run)", allowed set per R5. */
static int64_t fo_w(const fo_graph *g, const int32_t *pin, uint32_t dset, int32_t i) {
  if (pin && pin[i] >= 0) return g->cost[(int64_t)i * g->G + pin[i]];
  int64_t mx = 0;
  for (int d = 0; d < g->G; d++) {
    if (!((dset >> d) & 1u)) continue; /* R25: only the candidate's devices */
    if (g->cost[(int64_t)i * g->G + d] > mx) mx = g->cost[(int64_t)i * g->G + d];
  }
  return mx;
}

/* c_ij: "the maximal transmission time of the tensor from o_i to o_j (over
 * different device pairs that they can be located on)", R5:
 * pairs with s != t only; 0 if there is no such pair. */
static int64_t fo_c(const fo_graph *g, const int32_t *pin, uint32_t dset, int32_t i, int32_t j, int64_t bytes) {
  int64_t mx = 0;
  for (int s = 0; s < g->G; s++) {
    if (pin && pin[i] >= 0 && s != pin[i]) continue;
    if (!(pin && pin[i] >= 0) && !((dset >> s) & 1u)) continue;
    for (int t = 0; t < g->G; t++) {
      if (pin && pin[j] >= 0 && t != pin[j]) continue;
      if (!(pin && pin[j] >= 0) && !((dset >> t) & 1u)) continue;
      if (s == t) continue;
      int64_t c = fo_comm(g, bytes, s, t);
      if (c > mx) mx = c;
    }
  }
  return mx;
}

/* rank_u(o_i) = w_i + max_{o_j in succ(o_i)} (c_ij + rank_u(o_j)),
 * rank_u(o_exit) = w_exit, evaluated in reverse topological order. */
static void fo_rank(const fo_graph *g, const int32_t *pin, uint32_t dset, int64_t *rank) {
  int32_t V = g->V;
  int32_t *topo = malloc(sizeof(int32_t) * ((size_t)V + 1));
  int32_t n = fo_topo(g, topo);
  for (int32_t i = 0; i < V; i++) rank[i] = -1;
  for (int32_t t = n - 1; t >= 0; t--) {
    int32_t i = topo[t];
    int64_t best = 0;
    for (int32_t e = g->succ_off[i]; e < g->succ_off[i + 1]; e++) {
      int32_t j = g->succ_dst[e];
      int64_t v = fo_c(g, pin, dset, i, j, g->succ_bytes[e]) + rank[j];
      if (v > best) best = v;
    }
    rank[i] = fo_w(g, pin, dset, i) + best;
  }
  free(topo);
}

/* priority: larger rank first, then smaller op id (R2, R3) */
static int fo_higher(const int64_t *rank, int32_t a, int32_t b) {
  if (rank[a] != rank[b]) return rank[a] > rank[b];
  return a < b;
}

/* Critical path (R4, R7): start at the highest-priority entry op,
 * then repeatedly step to the successor with the largest rank. */
static int32_t fo_critical_path(const fo_graph *g, const int64_t *rank, int32_t *cp) {
  int32_t cur = -1, n = 0;
  for (int32_t i = 0; i < g->V; i++) {
    if (!g->alive[i] || g->pred_off[i + 1] != g->pred_off[i]) continue;
    if (cur < 0 || fo_higher(rank, i, cur)) cur = i;
  }
  while (cur >= 0) {
    cp[n++] = cur;
    int32_t nxt = -1;
    for (int32_t e = g->succ_off[cur]; e < g->succ_off[cur + 1]; e++) {
      int32_t j = g->succ_dst[e];
      if (nxt < 0 || fo_higher(rank, j, nxt)) nxt = j;
    }
    cur = nxt;
  }
  return n;
}

/* INSERT policy (reading R1i): "avail[j] is the start time of"
 * the earliest idle time slot on d_j whose length suffices for the op and
 * which preserves precedence.  The ops already placed on d_j (zero-length
 * ones included) form a sequence sorted by (ST, FT); its idle time slots are
 * the gaps of positive length between consecutive ops -- [0, s_1),
 * [f_1, s_2), ... -- and the open-ended slot [f_last, inf) after the last
 * op.  The op, ready at r (its predecessors' data arrived), fits slot
 * [a, b) iff max(a, r) + w <= b; EST = max(a, r) of the first slot that
 * fits. */
static int64_t fo_idle_slot(const int64_t *s, const int64_t *f, int32_t n, int64_t r, int64_t w) {
  int64_t a = 0;
  for (int32_t k = 0; k < n; k++) {
    int64_t b = s[k];
    if (b > a) {
      int64_t t = a > r ? a : r;
      if (t + w <= b) return t;
    }
    a = f[k];
  }
  return a > r ? a : r;
}

/* The full device set D of P:322-323 as a bit mask. */
static uint32_t fo_all_devices(int G) { return G >= 32 ? 0xFFFFFFFFu : ((1u << G) - 1u); }

/* DPOS (Alg. 1) for one candidate: graph g (already split if the
 * candidate splits), perturbation pins pin[] (-1 = free), the candidate's
 * device subset dset (R25: "FastT may not use all the input
 * devices, and can choose a subset"; fo_all_devices = all), flags.
 * Ranks are written to rank[] (V entries). */
static void fo_dpos(const fo_graph *g, const int32_t *pin, uint32_t dset, uint32_t flags, int64_t *rank,
                    fo_result *r) {
  int32_t V = g->V, G = g->G;
  /* Alg. 1 line 3-4: w, c and rank_u */
  fo_rank(g, pin, dset, rank);
  /* Alg. 1 lines 4-5: SET_CP and the critical-path devices d_cp (P:600-609,
   * P:678-682, R9) */
  int32_t *cpdev = malloc(sizeof(int32_t) * ((size_t)V + 1));
  int64_t reserved[FO_MAXG], used[FO_MAXG], avail[FO_MAXG];
  for (int d = 0; d < G; d++) { reserved[d] = 0; used[d] = 0; avail[d] = 0; }
  for (int32_t i = 0; i < V; i++) cpdev[i] = -1;
  if (flags & FO_F_CP_PIN) {
    int32_t *cp = malloc(sizeof(int32_t) * ((size_t)V + 1));
    int32_t ncp = fo_critical_path(g, rank, cp);
    int32_t *fr = malloc(sizeof(int32_t) * ((size_t)ncp + 1));
    int32_t nf = 0;
    for (int32_t q = 0; q < ncp; q++)
      if (!(pin && pin[cp[q]] >= 0)) fr[nf++] = cp[q];
    int devs[FO_MAXG];
    for (int d = 0; d < G; d++) devs[d] = (dset >> d) & 1u;
    int32_t k = 0;
    while (k < nf) {
      int any_dev = 0;
      for (int d = 0; d < G; d++) any_dev |= devs[d];
      if (!any_dev) break;
      int32_t m[FO_MAXG];
      int64_t S[FO_MAXG];
      int best = -1;
      for (int d = 0; d < G; d++) {
        m[d] = 0; S[d] = 0;
        if (!devs[d]) continue;
        /* "place as many remaining operations on the critical path as possible
         * onto the device (within its memory capacity)": longest prefix */
        int64_t msum = 0;
        while (k + m[d] < nf && msum + g->mem[fr[k + m[d]]] <= g->cap[d]) {
          msum += g->mem[fr[k + m[d]]];
          S[d] += g->cost[(int64_t)fr[k + m[d]] * G + d];
          m[d]++;
        }
        if (m[d] == 0) continue;
        /* smallest average S_d / m_d, compared exactly; ties -> lowest id */
        if (best < 0 || (__int128)S[d] * m[best] < (__int128)S[best] * m[d]) best = d;
      }
      if (best < 0) break;
      for (int32_t q = 0; q < m[best]; q++) {
        cpdev[fr[k + q]] = best;
        reserved[best] += g->mem[fr[k + q]];
      }
      devs[best] = 0;
      k += m[best];
    }
    free(cp); free(fr);
  }
  /* Alg. 1 lines 6-22: list scheduling over the ready set (R2) */
  int32_t *indeg = malloc(sizeof(int32_t) * ((size_t)V + 1));
  int32_t *ready = malloc(sizeof(int32_t) * ((size_t)V + 1));
  int32_t nready = 0, seq = 0;
  /* INSERT (R1i): per device the [ST, FT] of the ops placed on it,
   * kept sorted by (ST, FT) */
  const int insert = (flags & FO_F_POLICY_INSERT) != 0;
  int64_t *bs = NULL, *bf = NULL;
  int32_t nb[FO_MAXG];
  for (int d = 0; d < G; d++) nb[d] = 0;
  if (insert) {
    bs = malloc(sizeof(int64_t) * ((size_t)V * G + 1));
    bf = malloc(sizeof(int64_t) * ((size_t)V * G + 1));
  }
  /* liveness memory (NEXT N3, R24): an op's parameters stay on its device;
   * its output activation (mem - param) is held from the step the op is
   * dequeued until the step its last consumer is dequeued.  rem[i] counts
   * the consumers of op i not dequeued yet. */
  const int live = (flags & FO_F_MEM_LIVE) != 0;
  int32_t *rem = malloc(sizeof(int32_t) * ((size_t)V + 1));
  for (int d = 0; d < G; d++) r->peak[d] = 0;
  for (int32_t i = 0; i < V; i++) {
    rem[i] = g->succ_off[i + 1] - g->succ_off[i];
    indeg[i] = g->pred_off[i + 1] - g->pred_off[i];
    r->place[i] = 0xFF; r->start[i] = -1; r->finish[i] = -1; r->order[i] = -1; r->dq[i] = -1; r->deq[i] = -1;
    if (g->alive[i] && indeg[i] == 0) ready[nready++] = i;
  }
  int64_t makespan = 0;
  while (nready > 0) {
    /* o_i <- L.dequeue(): the ready op with the largest rank (ties: lowest id) */
    int32_t bi = 0;
    for (int32_t q = 1; q < nready; q++)
      if (fo_higher(rank, ready[q], ready[bi])) bi = q;
    int32_t i = ready[bi];
    ready[bi] = ready[--nready];
    int64_t mi = g->mem[i];
    int dsel = -1;
    int64_t est_sel = 0;
    /* EST(o_i, d_j) = max{avail[j], max_{o_m in pred(o_i)} (FT(o_m) + c^j_{m,i})}
     * (R1 append, R6 actual transfer time, 0 when co-located) */
#define FO_EST(dev, outv)                                                          \
  do {                                                                             \
    int64_t est_ = insert ? 0 : avail[dev];                                        \
    for (int32_t e_ = g->pred_off[i]; e_ < g->pred_off[i + 1]; e_++) {             \
      int32_t m_ = g->pred_src[e_];                                                \
      int64_t t_ = r->finish[m_] + fo_comm(g, g->pred_bytes[e_], r->place[m_], dev); \
      if (t_ > est_) est_ = t_;                                                    \
    }                                                                              \
    if (insert) est_ = fo_idle_slot(bs + (int64_t)(dev) * V, bf + (int64_t)(dev) * V, nb[dev], est_, \
                                    g->cost[(int64_t)i * G + (dev)]);             \
    (outv) = est_;                                                                 \
  } while (0)
    if (pin && pin[i] >= 0) {
      /* perturbation pin: a hard constraint (R8) */
      int d = pin[i];
      if (used[d] + reserved[d] + mi > g->cap[d]) {
        fo_result_infeasible(r, V, G, FO_CAND_INFEASIBLE);
        goto done;
      }
      dsel = d;
      FO_EST(d, est_sel);
    } else if (cpdev[i] >= 0) {
      /* Alg. 1 lines 9-10: S_new[o_i] = d_cp(o_i); memory reserved up front */
      dsel = cpdev[i];
      reserved[dsel] -= mi;
      FO_EST(dsel, est_sel);
    } else {
      /* Alg. 1 lines 12-19: EFT = +inf if memory exceeds capacity; argmin EFT */
      int64_t best = FO_INF;
      for (int d = 0; d < G; d++) {
        if (!((dset >> d) & 1u)) continue; /* R25: a device outside the candidate's subset */
        if (used[d] + reserved[d] + mi > g->cap[d]) continue;
        int64_t est;
        FO_EST(d, est);
        int64_t eft = est + g->cost[(int64_t)i * G + d];
        if (eft < best) { best = eft; dsel = d; est_sel = est; }
      }
      if (dsel < 0) {
        fo_result_infeasible(r, V, G, FO_CAND_INFEASIBLE);
        goto done;
      }
    }
#undef FO_EST
    /* Alg. 1 line 20 (R12): ST/FT on the chosen device */
    r->start[i] = est_sel;
    r->finish[i] = est_sel + g->cost[(int64_t)i * G + dsel];
    r->place[i] = (uint8_t)dsel;
    avail[dsel] = r->finish[i];
    if (insert) {
      /* keep the device's op sequence sorted by (ST, FT) */
      int64_t *s_ = bs + (int64_t)dsel * V, *f_ = bf + (int64_t)dsel * V;
      int32_t pos = nb[dsel];
      while (pos > 0 && (s_[pos - 1] > r->start[i] || (s_[pos - 1] == r->start[i] && f_[pos - 1] > r->finish[i]))) {
        s_[pos] = s_[pos - 1];
        f_[pos] = f_[pos - 1];
        pos--;
      }
      s_[pos] = r->start[i];
      f_[pos] = r->finish[i];
      nb[dsel]++;
    }
    used[dsel] += mi;
    if (live) {
      /* peak = the largest live total seen at any step (R24) */
      if (used[dsel] > r->peak[dsel]) r->peak[dsel] = used[dsel];
      /* free each input whose last consumer this op is, then this op's own
       * output if nothing consumes it */
      for (int32_t e = g->pred_off[i]; e < g->pred_off[i + 1]; e++) {
        int32_t m = g->pred_src[e];
        if (--rem[m] == 0) used[r->place[m]] -= g->mem[m] - g->param[m];
      }
      if (rem[i] == 0) used[dsel] -= mi - g->param[i];
    }
    r->dq[i] = seq;
    r->deq[seq] = i;
    seq++;
    if (r->finish[i] > makespan) makespan = r->finish[i];
    for (int32_t e = g->succ_off[i]; e < g->succ_off[i + 1]; e++)
      if (--indeg[g->succ_dst[e]] == 0) ready[nready++] = g->succ_dst[e];
  }
  /* Alg. 1 line 23: A = ops sorted by ascending ST (ties: dequeue order, R17);
   * done as a plain insertion into the dequeue list */
  {
    int32_t n = 0;
    for (int32_t q = 0; q < seq; q++) {
      int32_t i = r->deq[q];
      int32_t pos = n;
      while (pos > 0 && r->start[r->order[pos - 1]] > r->start[i]) {
        r->order[pos] = r->order[pos - 1];
        pos--;
      }
      r->order[pos] = i;
      n++;
    }
  }
  /* Alg. 1 line 24 (R16): FT(o_exit) = max FT; peak memory per device (R8) */
  r->makespan = makespan;
  r->status = FO_CAND_OK;
  if (!live)
    for (int d = 0; d < G; d++) r->peak[d] = used[d];
done:
  free(cpdev); free(indeg); free(ready); free(rem);
  free(bs); free(bf);
}

/* ----------------------------------------------------- candidate handling */

/* Validate a candidate and produce (graph to schedule, pin array, device
 * set).  dev_mask = 0 means every device; otherwise it must be a subset of
 * the G devices and hold every pinned device (R25).
 * Returns FO_CAND_OK or FO_CAND_BADSPEC. *gs is g itself or a new split view. */
static int fo_prepare(const fo_graph *g, int kind, int npins, const int32_t *pin_op, const uint8_t *pin_dev,
                      int32_t split_op, int split_dim, int split_n, uint32_t dev_mask, fo_graph **gs,
                      int32_t **pin_out, uint32_t *dset) {
  *gs = (fo_graph *)g;
  *pin_out = NULL;
  *dset = dev_mask ? dev_mask : fo_all_devices(g->G);
  if (dev_mask & ~fo_all_devices(g->G)) return FO_CAND_BADSPEC;
  if (kind == FO_KIND_BASE) return FO_CAND_OK;
  if (kind == FO_KIND_PIN) {
    if (npins < 1 || npins > FO_MAXPINS) return FO_CAND_BADSPEC;
    int32_t *pin = malloc(sizeof(int32_t) * ((size_t)g->V + 1));
    for (int32_t i = 0; i < g->V; i++) pin[i] = -1;
    for (int q = 0; q < npins; q++) {
      int32_t o = pin_op[q];
      if (o < 0 || o >= g->V || !g->alive[o] || pin_dev[q] >= g->G || pin[o] >= 0 || !((*dset >> pin_dev[q]) & 1u)) {
        free(pin);
        return FO_CAND_BADSPEC;
      }
      pin[o] = pin_dev[q];
    }
    *pin_out = pin;
    return FO_CAND_OK;
  }
  if (kind == FO_KIND_SPLIT) {
    if (split_op < 0 || split_op >= g->V || !g->alive[split_op]) return FO_CAND_BADSPEC;
    if (split_dim < 0 || split_dim > 1 || !(g->split_mask[split_op] & (1u << split_dim))) return FO_CAND_BADSPEC;
    if (split_n < 2 || split_n > g->G) return FO_CAND_BADSPEC;
    if (fo_split_view(g, split_op, split_dim, split_n, gs) != FO_OK) return FO_CAND_BADSPEC;
    return FO_CAND_OK;
  }
  return FO_CAND_BADSPEC;
}

/* v_max: the largest graph any single-split candidate can produce (R13, n<=G) */
int32_t fastt_ref_v_max(const fo_graph *g) {
  int32_t mx = 0;
  for (int32_t i = 0; i < g->V; i++) {
    if (!g->alive[i] || !g->split_mask[i]) continue;
    int32_t extra = (g->pred_off[i + 1] - g->pred_off[i]) + g->G + (g->succ_off[i + 1] - g->succ_off[i]);
    if (extra > mx) mx = extra;
  }
  return g->V + mx;
}

/* One candidate through Alg. 1.  Outputs are sized v_max (entries beyond the
 * candidate's graph are 0xFF / -1).  Any output pointer may be NULL. */
int32_t fastt_ref_schedule(const fo_graph *g, int32_t kind, int32_t npins, const int32_t *pin_op,
                           const uint8_t *pin_dev, int32_t split_op, int32_t split_dim, int32_t split_n,
                           uint32_t dev_mask, uint32_t flags, int64_t *makespan, int64_t *peak, uint8_t *status,
                           uint8_t *placement, int32_t *order, int64_t *start, int64_t *rank_out,
                           int32_t *deq_out) {
  int32_t vmax = fastt_ref_v_max(g), G = g->G;
  fo_graph *gs;
  int32_t *pin;
  uint32_t dset;
  int st = fo_prepare(g, kind, npins, pin_op, pin_dev, split_op, split_dim, split_n, dev_mask, &gs, &pin, &dset);
  if (placement) memset(placement, 0xFF, (size_t)vmax);
  for (int32_t i = 0; i < vmax; i++) {
    if (order) order[i] = -1;
    if (start) start[i] = -1;
    if (rank_out) rank_out[i] = -1;
    if (deq_out) deq_out[i] = -1;
  }
  if (st != FO_CAND_OK) {
    *makespan = FO_INF;
    *status = FO_CAND_BADSPEC;
    if (peak) for (int d = 0; d < G; d++) peak[d] = -1;
    return FO_OK;
  }
  fo_result r;
  fo_result_alloc(&r, gs->V, G);
  int64_t *rank = malloc(sizeof(int64_t) * ((size_t)gs->V + 1));
  fo_dpos(gs, pin, dset, flags, rank, &r);
  *makespan = r.makespan;
  *status = r.status;
  if (peak) for (int d = 0; d < G; d++) peak[d] = r.peak[d];
  for (int32_t i = 0; i < gs->V; i++) {
    if (placement) placement[i] = r.place[i];
    if (order) order[i] = r.order[i];
    if (start) start[i] = r.start[i];
    if (rank_out) rank_out[i] = gs->alive[i] ? rank[i] : -1;
    if (deq_out) deq_out[i] = r.deq[i];
  }
  free(rank);
  fo_result_free(&r);
  free(pin);
  if (gs != g) fo_graph_free(gs);
  return FO_OK;
}

/* ----------------------------------------- OS-DPOS (Algorithm 2) */

/* Alg. 2 lines 4-5 (R15): the critical path of the *placed* graph, using the
 * actual cost of each op on its assigned device and the actual transfer time
 * between the assigned devices, then sorted by descending computation time
 * (ties: lower id); only ops with a splittable dimension are kept. */
static int32_t fo_split_list(const fo_graph *g, const uint8_t *place, int32_t *list) {
  int32_t V = g->V, G = g->G;
  int64_t *rk = malloc(sizeof(int64_t) * ((size_t)V + 1));
  int32_t *topo = malloc(sizeof(int32_t) * ((size_t)V + 1));
  int32_t *cp = malloc(sizeof(int32_t) * ((size_t)V + 1));
  int32_t n = fo_topo(g, topo);
  for (int32_t i = 0; i < V; i++) rk[i] = -1;
  for (int32_t t = n - 1; t >= 0; t--) {
    int32_t i = topo[t];
    int64_t best = 0;
    for (int32_t e = g->succ_off[i]; e < g->succ_off[i + 1]; e++) {
      int32_t j = g->succ_dst[e];
      int64_t v = fo_comm(g, g->succ_bytes[e], place[i], place[j]) + rk[j];
      if (v > best) best = v;
    }
    rk[i] = g->cost[(int64_t)i * G + place[i]] + best;
  }
  int32_t ncp = fo_critical_path(g, rk, cp);
  int32_t m = 0;
  for (int32_t q = 0; q < ncp; q++)
    if (g->split_mask[cp[q]]) list[m++] = cp[q];
  /* insertion sort: cost on assigned device desc, id asc */
  for (int32_t a = 1; a < m; a++) {
    int32_t x = list[a];
    int64_t cx = g->cost[(int64_t)x * G + place[x]];
    int32_t b = a;
    while (b > 0) {
      int32_t y = list[b - 1];
      int64_t cy = g->cost[(int64_t)y * G + place[y]];
      if (cy > cx || (cy == cx && y < x)) break;
      list[b] = y;
      b--;
    }
    list[b] = x;
  }
  free(rk); free(topo); free(cp);
  return m;
}

/* split counts n in "# of GPUs" (R14) */
static int fo_split_ns(int G, int pow2_only, int *ns) {
  int c = 0;
  for (int n = 2; n <= G; n++)
    if (!pow2_only || (n & (n - 1)) == 0) ns[c++] = n;
  return c;
}

/* OS-DPOS.  Outputs: SP list (op, dim, n) into caller arrays of capacity
 * sp_cap, final placement / order / start sized out_cap (must hold the final
 * graph's op count), final makespan, final op count. */
int32_t fastt_ref_split_search(const fo_graph *g0, uint32_t flags, int32_t pow2_only, int32_t sp_cap,
                               int32_t *sp_n, int32_t *sp_op, uint8_t *sp_dim, uint8_t *sp_cnt,
                               int32_t out_cap, int32_t *n_ops_final, uint8_t *placement, int32_t *order,
                               int64_t *start, int64_t *makespan, uint8_t *status) {
  int32_t G = g0->G;
  fo_graph *cur = (fo_graph *)g0;
  fo_result best_r;
  fo_result_alloc(&best_r, g0->V, G);
  int64_t *rank = malloc(sizeof(int64_t) * ((size_t)g0->V + 1));
  /* Alg. 2 line 3 */
  fo_dpos(cur, NULL, fo_all_devices(cur->G), flags, rank, &best_r);
  free(rank);
  *sp_n = 0;
  if (best_r.status != FO_CAND_OK) {
    *makespan = FO_INF; *status = best_r.status; *n_ops_final = g0->V;
    fo_result_free(&best_r);
    return FO_OK;
  }
  int64_t ft_old = best_r.makespan;
  /* Alg. 2 lines 4-5 */
  int32_t *list = malloc(sizeof(int32_t) * ((size_t)g0->V + 1));
  int32_t nl = fo_split_list(g0, best_r.place, list);
  int ns[FO_MAXG];
  int nns = fo_split_ns(G, pow2_only, ns);
  /* Alg. 2 lines 7-14 */
  for (int32_t li = 0; li < nl; li++) {
    int32_t op = list[li];
    int64_t bft = FO_INF;
    int bdim = -1, bn = -1;
    fo_graph *bg = NULL;
    fo_result br;
    memset(&br, 0, sizeof(br));
    for (int dim = 0; dim < 2; dim++) {
      if (!(cur->split_mask[op] & (1u << dim))) continue;
      for (int q = 0; q < nns; q++) {
        fo_graph *sv;
        if (fo_split_view(cur, op, dim, ns[q], &sv) != FO_OK) continue;
        fo_result r;
        fo_result_alloc(&r, sv->V, G);
        int64_t *rk = malloc(sizeof(int64_t) * ((size_t)sv->V + 1));
        fo_dpos(sv, NULL, fo_all_devices(sv->G), flags, rk, &r);
        free(rk);
        if (r.status == FO_CAND_OK && r.makespan < bft) {
          if (bg) { fo_graph_free(bg); fo_result_free(&br); }
          bg = sv; br = r; bft = r.makespan; bdim = dim; bn = ns[q];
        } else {
          fo_graph_free(sv);
          fo_result_free(&r);
        }
      }
    }
    if (bg && bft < ft_old) {
      if (*sp_n < sp_cap) { sp_op[*sp_n] = op; sp_dim[*sp_n] = (uint8_t)bdim; sp_cnt[*sp_n] = (uint8_t)bn; }
      (*sp_n)++;
      ft_old = bft;
      if (cur != g0) fo_graph_free(cur);
      cur = bg;
      fo_result_free(&best_r);
      best_r = br;
    } else {
      if (bg) { fo_graph_free(bg); fo_result_free(&br); }
      break;
    }
  }
  *makespan = ft_old;
  *status = FO_CAND_OK;
  *n_ops_final = cur->V;
  int32_t n = cur->V < out_cap ? cur->V : out_cap;
  for (int32_t i = 0; i < out_cap; i++) {
    if (placement) placement[i] = i < n ? best_r.place[i] : 0xFF;
    if (order) order[i] = i < n ? best_r.order[i] : -1;
    if (start) start[i] = i < n ? best_r.start[i] : -1;
  }
  fo_result_free(&best_r);
  free(list);
  if (cur != g0) fo_graph_free(cur);
  return FO_OK;
}

/* NEXT row N2: best-improvement OS-DPOS.  Same input and CP
 * list as Alg. 2 (lines 3-5), but every round evaluates every split (op, dim,
 * n) of every not-yet-split op of the list on the current graph and accepts
 * the one with the smallest FT (ties: list order, dim asc, n asc) if it is
 * strictly better; stops when no split improves.  (A variant of Alg. 2,
 * the paper stops at the first op that does not improve.)
 *
 * With FO_F_SPLIT_MULTI (reading R27, multi-split candidates): each op's
 * best variant (smallest FT, ties dim asc, n asc) among those that improve;
 * the improving ops ranked by (FT asc, list order); the candidates C_j =
 * the best variants of the first j ranked ops applied in rank order (each
 * SplitOperation on the graph the previous one produced; ops keep their ids,
 * R13), j = 1 .. min(4, #improving); the round accepts the C_j of smallest
 * FT (ties: smaller j) -- C_1 improves by construction -- and marks its ops
 * split. */
#define FO_F_SPLIT_MULTI (1u << 7)
int32_t fastt_ref_split_search_bi(const fo_graph *g0, uint32_t flags, int32_t pow2_only, int32_t sp_cap,
                                  int32_t *sp_n, int32_t *sp_op, uint8_t *sp_dim, uint8_t *sp_cnt,
                                  int32_t out_cap, int32_t *n_ops_final, uint8_t *placement, int32_t *order,
                                  int64_t *start, int64_t *makespan, uint8_t *status) {
  int32_t G = g0->G;
  fo_graph *cur = (fo_graph *)g0;
  fo_result best_r;
  fo_result_alloc(&best_r, g0->V, G);
  int64_t *rank = malloc(sizeof(int64_t) * ((size_t)g0->V + 1));
  fo_dpos(cur, NULL, fo_all_devices(cur->G), flags, rank, &best_r);
  free(rank);
  *sp_n = 0;
  if (best_r.status != FO_CAND_OK) {
    *makespan = FO_INF; *status = best_r.status; *n_ops_final = g0->V;
    fo_result_free(&best_r);
    return FO_OK;
  }
  int64_t ft_old = best_r.makespan;
  int32_t *list = malloc(sizeof(int32_t) * ((size_t)g0->V + 1));
  int32_t nl = fo_split_list(g0, best_r.place, list);
  uint8_t *done = calloc((size_t)nl + 1, 1);
  int ns[FO_MAXG];
  int nns = fo_split_ns(G, pow2_only, ns);
  const int multi = (flags & FO_F_SPLIT_MULTI) != 0;
  flags &= ~FO_F_SPLIT_MULTI;
  /* per list op: FT, dim and n of its best improving variant this round */
  int64_t *oft = malloc(sizeof(int64_t) * ((size_t)nl + 1));
  int *odim = malloc(sizeof(int) * ((size_t)nl + 1)), *on = malloc(sizeof(int) * ((size_t)nl + 1));
  for (;;) {
    for (int32_t li = 0; li < nl; li++) oft[li] = FO_INF;
    int64_t bft = FO_INF;
    int32_t bli = -1;
    int bdim = -1, bn = -1;
    fo_graph *bg = NULL;
    fo_result br;
    memset(&br, 0, sizeof(br));
    for (int32_t li = 0; li < nl; li++) {
      if (done[li]) continue;
      int32_t op = list[li];
      for (int dim = 0; dim < 2; dim++) {
        if (!(cur->split_mask[op] & (1u << dim))) continue;
        for (int q = 0; q < nns; q++) {
          fo_graph *sv;
          if (fo_split_view(cur, op, dim, ns[q], &sv) != FO_OK) continue;
          fo_result r;
          fo_result_alloc(&r, sv->V, G);
          int64_t *rk = malloc(sizeof(int64_t) * ((size_t)sv->V + 1));
          fo_dpos(sv, NULL, fo_all_devices(sv->G), flags, rk, &r);
          free(rk);
          if (r.status == FO_CAND_OK && r.makespan < oft[li]) {
            oft[li] = r.makespan;
            odim[li] = dim;
            on[li] = ns[q];
          }
          if (r.status == FO_CAND_OK && r.makespan < bft) {
            if (bg) { fo_graph_free(bg); fo_result_free(&br); }
            bg = sv; br = r; bft = r.makespan; bli = li; bdim = dim; bn = ns[q];
          } else {
            fo_graph_free(sv);
            fo_result_free(&r);
          }
        }
      }
    }
    if (!bg || bft >= ft_old) {
      if (bg) { fo_graph_free(bg); fo_result_free(&br); }
      break;
    }
    /* the accepted candidate: C_1 (the single best split), or a multi-split C_j */
    int32_t acc_li[4] = {bli, -1, -1, -1};
    int nacc = 1;
    if (multi) {
      /* the improving ops ranked by (FT asc, list order asc); the first is bli
         (the same order and tie rule as the single best) */
      int32_t rk_li[4];
      int nrk = 0;
      for (int32_t li = 0; li < nl; li++) {
        if (done[li] || oft[li] >= ft_old) continue;
        int pos = nrk;
        while (pos > 0 && oft[rk_li[pos - 1]] > oft[li]) pos--;
        if (pos >= 4) continue;
        for (int t = (nrk < 4 ? nrk : 3); t > pos; t--) rk_li[t] = rk_li[t - 1];
        rk_li[pos] = li;
        if (nrk < 4) nrk++;
      }
      /* C_j's graph: C_{j-1}'s graph with the j-th ranked op's best split */
      fo_graph *cg[5] = {NULL, bg, NULL, NULL, NULL};
      for (int j = 2; j <= nrk; j++) {
        const int32_t li = rk_li[j - 1];
        if (fo_split_view(cg[j - 1], list[li], odim[li], on[li], &cg[j]) != FO_OK) {
          cg[j] = NULL;
          break;
        }
        fo_result r;
        fo_result_alloc(&r, cg[j]->V, G);
        int64_t *rkj = malloc(sizeof(int64_t) * ((size_t)cg[j]->V + 1));
        fo_dpos(cg[j], NULL, fo_all_devices(cg[j]->G), flags, rkj, &r);
        free(rkj);
        if (r.status == FO_CAND_OK && r.makespan < bft) {  /* (ties: the smaller j stays) */
          fo_result_free(&br);
          br = r;
          bft = r.makespan;
          nacc = j;
        } else {
          fo_result_free(&r);
        }
      }
      for (int j = 1; j <= 4; j++)
        if (cg[j] && j != nacc) fo_graph_free(cg[j]);
      bg = cg[nacc];
      for (int t = 0; t < nacc; t++) acc_li[t] = rk_li[t];
    }
    for (int t = 0; t < nacc; t++) {
      const int32_t li = acc_li[t];
      const int dim = multi ? odim[li] : bdim, n = multi ? on[li] : bn;
      if (*sp_n < sp_cap) { sp_op[*sp_n] = list[li]; sp_dim[*sp_n] = (uint8_t)dim; sp_cnt[*sp_n] = (uint8_t)n; }
      (*sp_n)++;
      done[li] = 1;
    }
    ft_old = bft;
    if (cur != g0) fo_graph_free(cur);
    cur = bg;
    fo_result_free(&best_r);
    best_r = br;
  }
  free(oft);
  free(odim);
  free(on);
  *makespan = ft_old;
  *status = FO_CAND_OK;
  *n_ops_final = cur->V;
  int32_t n = cur->V < out_cap ? cur->V : out_cap;
  for (int32_t i = 0; i < out_cap; i++) {
    if (placement) placement[i] = i < n ? best_r.place[i] : 0xFF;
    if (order) order[i] = i < n ? best_r.order[i] : -1;
    if (start) start[i] = i < n ? best_r.start[i] : -1;
  }
  fo_result_free(&best_r);
  free(list);
  free(done);
  if (cur != g0) fo_graph_free(cur);
  return FO_OK;
}

/* ------------------------------------- the sweep's candidate stream (R21) */

typedef struct {
  uint8_t kind, n_pins, split_dim, split_n;
  int32_t split_op;
  int32_t pin_op[4];
  uint8_t pin_dev[4];
  uint32_t dev_mask; /* R25: device subset, 0 = all */
} fo_cand; /* 32 bytes */

static uint64_t fo_splitmix64(uint64_t *s) {
  *s += 0x9E3779B97F4A7C15ull;
  uint64_t z = *s;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

/* exported for the published-output pin */
uint64_t fastt_ref_splitmix64_next(uint64_t *state) { return fo_splitmix64(state); }

typedef struct {
  uint8_t *base_place; /* V */
  int32_t *split_op;   /* n_split */
  uint8_t *split_dim, *split_n;
  int64_t n_split;
  int32_t *live;
  int32_t n_live;
  int64_t n_subset; /* G-1 prefix-subset candidates when enabled (R25), else 0 */
} fo_stream;

static void fo_stream_free(fo_stream *s) { free(s->base_place); free(s->split_op); free(s->split_dim); free(s->split_n); free(s->live); }

/* gen_opts bits of the stream calls */
#define FO_GEN_POW2 1    /* split counts {2,4,8,..} only (R14) */
#define FO_GEN_SUBSETS 2 /* a block of device-subset candidates after the SPLITs (R25) */

/* One DPOS run on the base graph gives the base placement and, through
 * Alg. 2 lines 4-5, the ordered split-eligible CP ops (R21). */
static void fo_stream_init(const fo_graph *g, uint32_t flags, int gen_opts, fo_stream *s) {
  int pow2_only = gen_opts & FO_GEN_POW2;
  int32_t V = g->V, G = g->G;
  fo_result r;
  fo_result_alloc(&r, V, G);
  int64_t *rank = malloc(sizeof(int64_t) * ((size_t)V + 1));
  fo_dpos(g, NULL, fo_all_devices(g->G), flags, rank, &r);
  free(rank);
  s->base_place = malloc((size_t)V + 1);
  for (int32_t i = 0; i < V; i++) s->base_place[i] = r.status == FO_CAND_OK ? r.place[i] : 0;
  int32_t *list = malloc(sizeof(int32_t) * ((size_t)V + 1));
  int32_t nl = r.status == FO_CAND_OK ? fo_split_list(g, r.place, list) : 0;
  int ns[FO_MAXG];
  int nns = fo_split_ns(G, pow2_only, ns);
  s->split_op = malloc(sizeof(int32_t) * ((size_t)nl * 2 * (nns + 1) + 1));
  s->split_dim = malloc((size_t)nl * 2 * (nns + 1) + 1);
  s->split_n = malloc((size_t)nl * 2 * (nns + 1) + 1);
  s->n_split = 0;
  for (int32_t li = 0; li < nl; li++)
    for (int dim = 0; dim < 2; dim++) {
      if (!(g->split_mask[list[li]] & (1u << dim))) continue;
      for (int q = 0; q < nns; q++) {
        s->split_op[s->n_split] = list[li];
        s->split_dim[s->n_split] = (uint8_t)dim;
        s->split_n[s->n_split] = (uint8_t)ns[q];
        s->n_split++;
      }
    }
  s->live = malloc(sizeof(int32_t) * ((size_t)V + 1));
  s->n_live = 0;
  for (int32_t i = 0; i < V; i++) if (g->alive[i]) s->live[s->n_live++] = i;
  s->n_subset = (gen_opts & FO_GEN_SUBSETS) ? G - 1 : 0;
  free(list);
  fo_result_free(&r);
}

static void fo_stream_cand(const fo_graph *g, const fo_stream *s, uint64_t seed, int kmin, int kmax, int64_t c,
                           fo_cand *out) {
  memset(out, 0, sizeof(*out));
  out->split_op = -1;
  for (int q = 0; q < 4; q++) { out->pin_op[q] = -1; out->pin_dev[q] = 0; }
  if (c == 0) { out->kind = FO_KIND_BASE; return; }
  if (c <= s->n_split) {
    out->kind = FO_KIND_SPLIT;
    out->split_op = s->split_op[c - 1];
    out->split_dim = s->split_dim[c - 1];
    out->split_n = s->split_n[c - 1];
    return;
  }
  if (c <= s->n_split + s->n_subset) {
    /* R25: BASE on the first k devices, k = 1 .. G-1 */
    int k = (int)(c - s->n_split);
    out->kind = FO_KIND_BASE;
    out->dev_mask = (1u << k) - 1u;
    return;
  }
  out->kind = FO_KIND_PIN;
  uint64_t st = seed ^ ((uint64_t)c * 0x9E3779B97F4A7C15ull);
  uint64_t x0 = fo_splitmix64(&st);
  int K = kmin + (int)(x0 % (uint64_t)(kmax - kmin + 1));
  if (K > s->n_live) K = s->n_live;
  out->n_pins = (uint8_t)K;
  for (int k = 0; k < K; k++) {
    uint64_t xo = fo_splitmix64(&st);
    int32_t idx = (int32_t)(xo % (uint64_t)s->n_live);
    for (;;) {
      int taken = 0;
      for (int q = 0; q < k; q++) taken |= out->pin_op[q] == s->live[idx];
      if (!taken) break;
      idx = (idx + 1) % s->n_live;
    }
    int32_t op = s->live[idx];
    uint64_t xd = fo_splitmix64(&st);
    out->pin_op[k] = op;
    out->pin_dev[k] = (uint8_t)((s->base_place[op] + 1 + (int)(xd % (uint64_t)(g->G - 1))) % g->G);
  }
}

static int fo_stream_check(const fo_graph *g, const fo_stream *s, int kmin, int kmax, int64_t first, int64_t n,
                           int64_t stride) {
  if (kmin < 1 || kmax > 4 || kmin > kmax || first < 0 || n < 0 || stride < 1) return FO_EINVAL;
  if (n > 0 && (g->G == 1 || s->n_live == 0) && first + (n - 1) * stride > s->n_split + s->n_subset) return FO_EINVAL;
  return FO_OK;
}

int32_t fastt_ref_stream_info(const fo_graph *g, uint32_t flags, int32_t gen_opts, int64_t *n_split,
                              uint8_t *base_place) {
  fo_stream s;
  fo_stream_init(g, flags, gen_opts, &s);
  *n_split = s.n_split;
  if (base_place) memcpy(base_place, s.base_place, (size_t)g->V);
  fo_stream_free(&s);
  return FO_OK;
}

int32_t fastt_ref_generate(const fo_graph *g, uint32_t flags, uint64_t seed, int32_t kmin, int32_t kmax,
                           int32_t gen_opts, int64_t first, int64_t n, void *out) {
  fo_stream s;
  fo_stream_init(g, flags, gen_opts, &s);
  int rc = fo_stream_check(g, &s, kmin, kmax, first, n, 1);
  if (rc == FO_OK)
    for (int64_t q = 0; q < n; q++) fo_stream_cand(g, &s, seed, kmin, kmax, first + q, (fo_cand *)out + q);
  fo_stream_free(&s);
  return rc;
}

/* Sweep: evaluate candidates c = first + q*stride (q < n); best = smallest
 * makespan, then smallest index (R3).  Per-candidate makespans optional. */
int32_t fastt_ref_sweep(const fo_graph *g, uint32_t flags, uint64_t seed, int32_t kmin, int32_t kmax,
                        int32_t gen_opts, int64_t first, int64_t n, int64_t stride, int64_t *best_makespan,
                        int64_t *best_index, int64_t *makespans) {
  fo_stream s;
  fo_stream_init(g, flags, gen_opts, &s);
  int rc = fo_stream_check(g, &s, kmin, kmax, first, n, stride);
  *best_makespan = FO_INF;
  *best_index = -1;
  if (rc == FO_OK) {
    for (int64_t q = 0; q < n; q++) {
      int64_t c = first + q * stride;
      fo_cand cd;
      fo_stream_cand(g, &s, seed, kmin, kmax, c, &cd);
      int64_t ms;
      uint8_t stt;
      fastt_ref_schedule(g, cd.kind, cd.n_pins, cd.pin_op, cd.pin_dev, cd.split_op, cd.split_dim, cd.split_n,
                         cd.dev_mask, flags, &ms, NULL, &stt, NULL, NULL, NULL, NULL, NULL);
      if (makespans) makespans[q] = ms;
      if (ms < *best_makespan || (ms == *best_makespan && ms != FO_INF && c < *best_index)) {
        *best_makespan = ms;
        *best_index = c;
      }
    }
  }
  fo_stream_free(&s);
  return rc;
}

/* Upward ranks of a candidate's graph (base when kind == BASE). */
int32_t fastt_ref_rank(const fo_graph *g, int32_t kind, int32_t npins, const int32_t *pin_op, const uint8_t *pin_dev,
                       int32_t split_op, int32_t split_dim, int32_t split_n, uint32_t dev_mask, int64_t *rank_out) {
  int32_t vmax = fastt_ref_v_max(g);
  fo_graph *gs;
  int32_t *pin;
  uint32_t dset;
  for (int32_t i = 0; i < vmax; i++) rank_out[i] = -1;
  if (fo_prepare(g, kind, npins, pin_op, pin_dev, split_op, split_dim, split_n, dev_mask, &gs, &pin, &dset) !=
      FO_CAND_OK)
    return FO_EINVAL;
  int64_t *rank = malloc(sizeof(int64_t) * ((size_t)gs->V + 1));
  fo_rank(gs, pin, dset, rank);
  for (int32_t i = 0; i < gs->V; i++) rank_out[i] = gs->alive[i] ? rank[i] : -1;
  free(rank);
  free(pin);
  if (gs != g) fo_graph_free(gs);
  return FO_OK;
}

/* Base critical path (R7) on unpinned ranks, for the info call. */
int32_t fastt_ref_cp(const fo_graph *g, int32_t *cp_out) {
  int64_t *rank = malloc(sizeof(int64_t) * ((size_t)g->V + 1));
  int32_t *cp = malloc(sizeof(int32_t) * ((size_t)g->V + 1));
  fo_rank(g, NULL, fo_all_devices(g->G), rank);
  int32_t n = fo_critical_path(g, rank, cp);
  if (cp_out) memcpy(cp_out, cp, sizeof(int32_t) * (size_t)n);
  free(rank); free(cp);
  return n;
}

/* Export the graph a SPLIT candidate schedules (for the R13 property pins).
 * Arrays must hold v_max ops / (E + v_max * (G + 2) * 2) edges.  Returns the
 * edge count, or a negative status. */
int64_t fastt_ref_split_export(const fo_graph *g, int32_t op, int32_t dim, int32_t n, int32_t *V_out,
                               int32_t *src, int32_t *dst, int64_t *bytes, uint8_t *eparam, int64_t *cost,
                               int64_t *mem, int64_t *param, uint8_t *alive) {
  fo_graph *gs;
  int32_t *pin;
  uint8_t dummy = 0;
  uint32_t dset;
  if (fo_prepare(g, FO_KIND_SPLIT, 0, NULL, &dummy, op, dim, n, 0, &gs, &pin, &dset) != FO_CAND_OK) return FO_EINVAL;
  *V_out = gs->V;
  for (int32_t i = 0; i < gs->V; i++) {
    for (int d = 0; d < gs->G; d++) cost[(int64_t)i * gs->G + d] = gs->cost[(int64_t)i * gs->G + d];
    mem[i] = gs->mem[i];
    param[i] = gs->param[i];
    alive[i] = gs->alive[i];
    for (int32_t e = gs->succ_off[i]; e < gs->succ_off[i + 1]; e++) {
      src[e] = i; dst[e] = gs->succ_dst[e]; bytes[e] = gs->succ_bytes[e]; eparam[e] = gs->succ_param[e];
    }
  }
  int64_t E = gs->E;
  fo_graph_free(gs);
  return E;
}
