/*
 * fastt.h -- C-ABI of the B200-native FastT strategy-search hot path.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, "P:<line>"):
 *   Yi et al., "Fast Training of Deep Learning Models over Multiple GPUs"
 *   (FastT, Middleware '20).  Inputs are the problem of Sec. 3:
 *   (a) the DAG computing graph, (b) the device set with per-device memory
 *   limits, (c) the computation and communication cost models.  Outputs are
 *   those of P:330-336: (i) a partition (split) list, (ii) the placement of
 *   every (sub-)operation, (iii) the execution order.
 *   The library evaluates CANDIDATE DEPLOYMENTS of that graph with DPOS
 *   (Alg. 1): upward ranks, the critical path and its
 *   devices, and list scheduling with
 *       EST(o_i,d_j) = max{avail[j], max_{pred m} FT(o_m) + c^j_{m,i}},
 *       EFT = EST + w_{i,j}
 *   and runs OS-DPOS (Alg. 2) with SplitOperation.
 *   The exact semantics, including every reading of a garbled or silent
 *   passage (R1-R22), are in DESIGN.md "Readings".
 *
 * Conventions
 *   - All integers.  Time is int64 nanoseconds, sizes int64 bytes, the
 *     link model's slope is femtoseconds per byte.  No floats cross the ABI.
 *   - Op ids are the caller's ids 0..n_ops-1.  A split candidate appends new
 *     ids (R13): [one split node per predecessor of the split op, in
 *     ascending predecessor id] [the n sub-ops] [one concat node per
 *     successor, ascending successor id]; the split op is removed.
 *   - Per-op output arrays are sized v_max (fastt_graph_info) per candidate;
 *     entries of ops that do not exist or were not scheduled are 0xFF
 *     (placement) / -1 (order, start, rank).
 *   - Ownership: inputs are copied; the caller may free them after the call.
 *     Batch outputs are caller-allocated, host memory unless
 *     FASTT_F_OUT_DEVICE (then device memory on the graph's device).
 *     Candidate inputs are host memory unless FASTT_F_IN_DEVICE.
 *     fastt_split_result arrays are library-allocated (host) and released by
 *     fastt_free_split_result.
 *   - Errors: every call returns a status; nothing throws or aborts across
 *     the ABI.  On error fastt_last_error() (thread-local) explains why.
 *     Per-candidate infeasibility is a status value, not an error.
 *   - Synchronisation ("calls are asynchronous on
 *     cuda_stream; the caller synchronizes"): work is issued on
 *     opts->cuda_stream (NULL = the legacy default stream of the graph's
 *     device).  With FASTT_F_ASYNC, fastt_schedule_batch,
 *     fastt_sweep_best and fastt_generate_candidates return once the work
 *     is enqueued: nothing on their steady-state path waits for the device
 *     (how many preparation rounds a batch needs is decided on the device,
 *     by a CUDA-graph WHILE loop), and their outputs are valid once the
 *     stream -- or fastt_sync -- has completed.  Inputs are consumed before
 *     the call returns.  Host output buffers must then be page-locked for
 *     the copies to be asynchronous; device buffers (FASTT_F_OUT_DEVICE /
 *     FASTT_F_IN_DEVICE) always are.  The first call for a graph and flag
 *     set (the BASE run, snapshot, stream and arena setup) and a call that
 *     grows a workspace may block once.  Without FASTT_F_ASYNC a call
 *     returns after the stream has completed it.  fastt_rank and
 *     fastt_split_search are always blocking (their results come back
 *     through host decisions: Alg. 2's accept/stop rule).  Calls on one
 *     graph are ordered among themselves whatever stream they use (the
 *     graph's scratch is shared); calls on different graphs are
 *     independent and may overlap.
 *   - Determinism: every output is a pure function of (graph, candidates,
 *     flags, generator parameters); it is bit-identical to the CPU oracle.
 */
#ifndef FASTT_H
#define FASTT_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct fastt_graph fastt_graph; /* opaque; immutable after load except for the lazy stream cache */
typedef int32_t fastt_status;

enum {
  FASTT_OK = 0,
  FASTT_EINVAL = -1, /* malformed input */
  FASTT_ECYCLE = -2, /* the graph is not a DAG (R22) */
  FASTT_ENOMEM = -3, /* host or device allocation failed */
  FASTT_ECUDA = -4,  /* a CUDA runtime call failed (no device, launch failure) */
  FASTT_ERANGE = -5, /* an int64 bound would be exceeded */
  FASTT_EUNSUP = -6  /* outside the supported envelope (see fastt_load_graph) */
};

/* per-candidate status */
enum { FASTT_CAND_OK = 0, FASTT_CAND_INFEASIBLE = 1 /* memory, R8 */, FASTT_CAND_BADSPEC = 2 };
/* candidate kinds */
enum { FASTT_KIND_BASE = 0, FASTT_KIND_PIN = 1, FASTT_KIND_SPLIT = 2 };
/* split dimensions; split_mask bit (1 << dim) */
enum { FASTT_DIM_BATCH = 0, FASTT_DIM_CHANNEL = 1 };
/* option flags */
enum {
  FASTT_F_CP_PIN = 1u << 0,        /* pin critical-path ops to CP devices (Alg. 1 lines 4-5, 9-10) */
  FASTT_F_POLICY_INSERT = 1u << 1, /* insertion-based avail[j] (R1i; NEXT N1): earliest idle slot that fits */
  FASTT_F_OUT_DEVICE = 1u << 2,    /* output pointers are device pointers */
  FASTT_F_IN_DEVICE = 1u << 3,     /* candidate input pointer is a device pointer */
  FASTT_F_TIMING = 1u << 4,        /* record CUDA events around the kernels of this call (fastt_last_timing) */
  FASTT_F_SPLIT_BEST = 1u << 5,    /* fastt_split_search: best-improvement rounds */
  FASTT_F_SPLIT_MULTI = 1u << 7,   /* fastt_split_search: best-improvement rounds with multi-split candidates
                                      (reading R27): each round also evaluates C_j = the best
                                      split of each of the j best-improving ops, applied in rank order
                                      (j = 2..4), and accepts the best C_j (ties: fewer splits) */
  FASTT_F_ASYNC = 1u << 8,         /* return once enqueued on cuda_stream (see Synchronisation above) */
  FASTT_F_MEM_LIVE = 1u << 6       /* liveness memory (reading R24): an op's parameters stay on
                                      its device; its output (mem - param) is held from the step it is dequeued
                                      until the step its last consumer is dequeued.  The feasibility test of
                                      Alg. 1 line 13 uses that live total; peak_mem = its maximum */
};

/* The problem input of P:321-328.  Edges are a CSR by source: the edges of
 * op i are succ_dst[succ_off[i] .. succ_off[i+1]).  Parallel edges are
 * merged at load (bytes summed, param flag OR-ed, R11). */
typedef struct {
  int32_t n_ops;      /* V >= 0 */
  int32_t n_devices;  /* G, 1..32 */
  const int32_t *succ_off;    /* V+1, nondecreasing, succ_off[0] = 0 */
  const int32_t *succ_dst;    /* E = succ_off[V], each in [0, V) and != its source */
  const int64_t *edge_bytes;  /* E, >= 0: tensor size on the edge */
  const uint8_t *edge_param;  /* E, bit0 = parameter tensor (decides which edges a split cuts, R13) */
  const int64_t *cost_ns;     /* V*G row-major [op][device], >= 0; 0 = unknown */
  const int64_t *mem_bytes;   /* V, >= 0: memory the op occupies on its device (R8) */
  const int64_t *param_bytes; /* V, 0 <= param_bytes <= mem_bytes */
  const uint8_t *split_mask;  /* V, bit (1<<dim) = splittable along dim */
  const int64_t *dev_mem_cap; /* G, >= 0; INT64_MAX = unlimited */
  const uint8_t *link_class;  /* G*G [src][dst] in [0, K); the diagonal is ignored (same device = 0 ns) */
  int32_t n_link_classes;     /* K, 1..16 */
  const int64_t *link_alpha_ns;         /* K, >= 0 */
  const int64_t *link_beta_fs_per_byte; /* K, >= 0; comm(b,k) = alpha_k + ceil(b*beta_k/1e6) (R10) */
  int64_t split_copy_fs_per_byte;       /* >= 0; split/concat node cost = ceil(b*x/1e6) on every device (R13) */
} fastt_graph_desc;

/* A candidate deployment (32 bytes).
 *   BASE : the graph as loaded.
 *   PIN  : n_pins (1..4) distinct ops pin_op[k] forced onto device pin_dev[k]
 *          (a "placement perturbation"); pinned ops use w = cost on that
 *          device and c over the allowed device pairs (R5).
 *   SPLIT: SplitOperation(graph, split_op, split_dim, split_n), 2 <= n <= G,
 *          split_op must have split_mask bit split_dim (R13, R14).
 *   dev_mask (any kind, reading R25): "FastT may not use all
 *          the input devices, and can choose a subset".  0 = all
 *          G devices; otherwise bit d set = device d may be used.  The
 *          unpinned ops' allowed set (w, c of R5), the CP devices (R9) and
 *          the EFT argmin (Alg. 1 line 12) range over the subset; every
 *          pin_dev must be in it and no bit >= G may be set (else BADSPEC).
 *          Devices outside the subset report peak_mem 0. */
typedef struct {
  uint8_t kind, n_pins, split_dim, split_n;
  int32_t split_op;
  int32_t pin_op[4];
  uint8_t pin_dev[4];
  uint32_t dev_mask;
} fastt_candidate;

/* The seeded candidate stream of a sweep (R21):
 *   index 0 = BASE; indices 1..n_split = every SPLIT of the sorted
 *   split-eligible placement-aware critical path (Alg. 2 lines 4-5) x dims
 *   ascending x n ascending (2..G, or powers of two if n_pow2_only);
 *   every later index c is a PIN candidate drawn from splitmix64 with state
 *   seed ^ (c * 0x9E3779B97F4A7C15): K = pin_k_min + x0 mod (pin_k_max -
 *   pin_k_min + 1) pins; pin k takes op live[x_{1+2k} mod V_live] (linear
 *   probing past ops already chosen) and device (base_place + 1 +
 *   x_{2+2k} mod (G-1)) mod G.  base_place comes from one DPOS run of the
 *   BASE candidate under the same flags (0 for every op if that run is
 *   infeasible).  With subset_prefixes = 1 a block of G-1 device-subset
 *   candidates follows the SPLIT block (R25): index n_split + k, k = 1..G-1,
 *   is BASE with dev_mask = (1 << k) - 1 (the first k devices); the PIN
 *   block then starts at n_split + G.  With G == 1 the stream ends after
 *   the SPLIT (and subset) block. */
typedef struct {
  uint64_t seed;
  uint8_t pin_k_min, pin_k_max; /* 1 <= min <= max <= 4 */
  uint8_t n_pow2_only;          /* split counts {2,4,8,..} only (C4) */
  uint8_t subset_prefixes;      /* 0/1: include the device-subset block (R25) */
  uint8_t _pad[4];
} fastt_gen_params;

typedef struct {
  uint32_t flags;
  int32_t _pad;
  void *cuda_stream; /* cudaStream_t; NULL = legacy default stream */
} fastt_opts;

/* Load + encode: validates (acyclic, ranges), merges
 * parallel edges, builds both CSRs, computes the device-side base ranks and
 * priority order.  Supported envelope: G <= 32, K <= 16, in/out degree
 * < 65535, V + largest split overlay <= 2^23 ops; above 32,768 ops the base
 * priority order must be topological (EUNSUP otherwise: the ready-set
 * kernel's bitmap of one candidate lives in shared memory; a candidate whose
 * order is not topological on such a graph fails the call, see fastt_sync);
 * int64 guard
 * sum_i (max cost + G) + sum_e (max comm + copy cost) * (G+2) < 2^58 and
 * sum_i mem * (G+1) < 2^60 (ERANGE beyond; the oracle applies the same rule).
 * cuda_device: the CUDA device ordinal to use. */
fastt_status fastt_load_graph(const fastt_graph_desc *desc, int cuda_device, fastt_graph **out);
void fastt_free_graph(fastt_graph *g);

/* n_ops: V; v_max: V + the largest single-split overlay; cp_len: length of
 * the base critical path (R7, unpinned ranks); time_bits: 32 when every
 * schedule of this graph provably fits in uint32 ns (then the kernels run
 * 32-bit), else 64. Any pointer may be NULL. */
fastt_status fastt_graph_info(const fastt_graph *g, int32_t *n_ops, int32_t *v_max, int32_t *cp_len,
                              int32_t *time_bits);

/* Upward ranks rank_u of the candidate's graph (cand NULL =
 * BASE), indexed by op id, v_max entries (-1 for absent ops).  rank_out is
 * host memory unless FASTT_F_OUT_DEVICE; cand is host memory. */
fastt_status fastt_rank(const fastt_graph *g, const fastt_candidate *cand, const fastt_opts *opts, int64_t *rank_out);

/* DPOS of n candidates (S2-S7).  makespan[n] (INT64_MAX if not OK),
 * status[n]; optional (NULL to skip): peak_mem[n*G] (sum of mem per device,
 * -1 if not OK; with FASTT_F_MEM_LIVE the live peak of R24), placement[n*v_max] (device per op id), order[n*v_max]
 * (op ids sorted by (start, dequeue sequence), R17, -1 padded),
 * start_ns[n*v_max]. */
fastt_status fastt_schedule_batch(const fastt_graph *g, const fastt_candidate *cands, int64_t n,
                                  const fastt_opts *opts, int64_t *makespan, int64_t *peak_mem, uint8_t *status,
                                  uint8_t *placement, int32_t *order, int64_t *start_ns);

/* Stream size info: n_split = size of the SPLIT block of the stream. */
fastt_status fastt_stream_info(const fastt_graph *g, const fastt_gen_params *gen, const fastt_opts *opts,
                               int64_t *n_split);

/* Candidates first .. first+n-1 of the stream (S2) into out[n]. */
fastt_status fastt_generate_candidates(const fastt_graph *g, const fastt_gen_params *gen, const fastt_opts *opts,
                                       int64_t first, int64_t n, fastt_candidate *out);

/* Sweep (S2-S7 fused): evaluate stream candidates c = first + q*stride,
 * q < n, generated on the device, and return best[0] = smallest makespan,
 * best[1] = smallest index attaining it (R3); (INT64_MAX, -1) if none is
 * feasible.  best is host memory unless FASTT_F_OUT_DEVICE. */
fastt_status fastt_sweep_best(const fastt_graph *g, const fastt_gen_params *gen, const fastt_opts *opts,
                              int64_t first, int64_t n, int64_t stride, int64_t *best);

/* OS-DPOS (Alg. 2, S8): DPOS of the graph, the placement-aware critical path
 * (lines 4-5, R15), then for each split-eligible CP op in descending cost the
 * best of its splits (dims asc, n asc; n in 2..G or powers of two with
 * n_pow2_only) is accepted if strictly better, else the search stops.
 * With FASTT_F_SPLIT_BEST (NEXT row N2, a variant): every round evaluates all
 * splits of all not-yet-split list ops in one batch and accepts the best
 * (ties: list order, dim, n) while it strictly improves. */
typedef struct {
  int32_t n_splits; /* SP list */
  int32_t *op;
  uint8_t *dim, *n;
  int32_t n_ops_final;  /* ops of the final graph (ids of removed ops keep placement 0xFF) */
  uint8_t *placement;   /* n_ops_final */
  int32_t *order;       /* n_ops_final, -1 padded */
  int64_t *start_ns;    /* n_ops_final */
  int64_t makespan;     /* INT64_MAX if the initial DPOS is infeasible */
  uint8_t status;
} fastt_split_result;
fastt_status fastt_split_search(const fastt_graph *g, const fastt_opts *opts, int32_t n_pow2_only,
                                fastt_split_result *out);
void fastt_free_split_result(fastt_split_result *r);

/* Instrumentation of the last fastt_schedule_batch / fastt_sweep_best call on
 * this graph.  launches: kernels the library launched (always counted).
 * The *_ms fields are CUDA-event times on the call's stream, filled only when
 * that call had FASTT_F_TIMING: ms_sim = the main simulation kernel (S2-S7 for
 * the candidates whose ranks equal the base ranks), ms_prep = the
 * per-candidate preparation pipeline plus its simulation launches, ms_total =
 * the whole call on the device. */
typedef struct {
  int64_t launches;
  int64_t candidates;   /* candidates evaluated */
  int64_t deferred;     /* of which went through the preparation pipeline */
  float ms_sim, ms_prep, ms_total;
  int32_t topo;         /* 1 or 2: the main simulation ran a position-order kernel (the graph's priority
                           order is topological, so the dequeue order is the position order):
                           1 = one lane group per candidate (k_sim), 2 = one lane per candidate
                           (k_sim_lane: makespan, per-device peak memory, memory caps) */
  int32_t _pad;
  int64_t warp_steps;   /* k_sim_lane main launch: op-steps executed per warp, summed (every lane of a
                           warp executes the warp's steps; prefix-shared steps are not executed) */
  int64_t lane_steps;   /* of which the steps of running candidates (each from its warp's start step) */
} fastt_timing;
fastt_status fastt_last_timing(const fastt_graph *g, fastt_timing *out);

/* Completion of asynchronous calls (FASTT_F_ASYNC): waits until the work of
 * every call issued on g so far has completed (on opts->cuda_stream and the
 * graph's internal streams), then reports what a blocking call would have:
 * FASTT_EUNSUP if a candidate met the envelope check done on the device (a
 * non-topological priority order on a graph above 32,768 ops), FASTT_ECUDA
 * if the device work failed.  Afterwards fastt_last_timing's `deferred`
 * and `launches` describe the last asynchronous call. */
fastt_status fastt_sync(const fastt_graph *g, const fastt_opts *opts);

/* Communication cost-model fit ("we gather
 * tensors across the same source-destination device pairs into one group.
 * For each group, we use linear regression to obtain a linear model: tensor
 * size vs. transfer time"; reading R26).  Sample k is a transfer of
 * bytes[k] bytes from device src_dev[k] to dst_dev[k] (!= src) that took
 * time_ns[k].  For every ordered pair (s, t) the least-squares line
 * time = alpha + beta * bytes with alpha >= 0 and beta >= 0 is fitted in
 * exact integer arithmetic and reported as the nearest integers (halves up)
 * in the units of the model R10: alpha_ns[s*G+t] in ns,
 * beta_fs_per_byte[s*G+t] in fs/byte.  A pair with no sample gets 0, 0
 * (unknown costs are 0); a pair whose samples all have one size
 * gets beta = 0 and alpha = the mean time.  count[s*G+t] (NULL to skip) is
 * the number of samples of the pair; the diagonal is 0.
 * Envelope: 1 <= G <= 32, n_samples < 2^24, bytes and time in [0, 2^40)
 * (EINVAL otherwise).  Runs on cuda_device: one pass over the samples
 * (exact 64/128-bit moment sums per pair) and one thread per pair for the
 * constrained normal equations.  Inputs are host memory unless
 * FASTT_F_IN_DEVICE, outputs host memory unless FASTT_F_OUT_DEVICE. */
fastt_status fastt_fit_comm(int32_t n_devices, int64_t n_samples, const uint8_t *src_dev, const uint8_t *dst_dev,
                            const int64_t *bytes, const int64_t *time_ns, int cuda_device, const fastt_opts *opts,
                            int64_t *alpha_ns, int64_t *beta_fs_per_byte, int64_t *count);

/* Computation cost model ("The
 * computation cost model provides the execution time of a (sub-)operation on
 * a device, using the operation's name and device as the key"
 * unknown costs are 0).  Sample k says op[k] ran on dev[k] for time_ns[k];
 * cost_ns[o*G+d] = the mean of the (o, d) samples as the nearest integer ns
 * (halves up), 0 where there is none -- the cost_ns table of
 * fastt_graph_desc.  Envelope: 1 <= G <= 32, n_ops >= 1, n_samples < 2^24,
 * op in [0, n_ops), dev < G, time in [0, 2^40) (EINVAL otherwise).  Runs on
 * cuda_device (integer sums and counts per entry, order-independent, then
 * one thread per entry); host memory unless FASTT_F_IN_DEVICE /
 * FASTT_F_OUT_DEVICE. */
fastt_status fastt_cost_table(int32_t n_ops, int32_t n_devices, int64_t n_samples, const int32_t *op,
                              const uint8_t *dev, const int64_t *time_ns, int cuda_device, const fastt_opts *opts,
                              int64_t *cost_ns);

/* The link model of fastt_graph_desc from per-pair parameters (host only):
 * pairs with identical (alpha, beta) share a link class; classes are
 * numbered in row-major order of first appearance over the off-diagonal
 * pairs; the diagonal gets class 0.  Outputs: link_class[G*G],
 * *n_link_classes, link_alpha_ns[16], link_beta_fs_per_byte[16].
 * EUNSUP if more than 16 distinct pairs' parameters exist (K <= 16). */
fastt_status fastt_link_model(int32_t n_devices, const int64_t *alpha_ns, const int64_t *beta_fs_per_byte,
                              uint8_t *link_class, int32_t *n_link_classes, int64_t *link_alpha_ns,
                              int64_t *link_beta_fs_per_byte);

const char *fastt_last_error(void); /* thread-local; valid until the next call on this thread */
const char *fastt_version(void);

#ifdef __cplusplus
}
#endif
#endif /* FASTT_H */
