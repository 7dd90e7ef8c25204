// fastt_abi.cu -- host side of the C-ABI (include/fastt.h): validation,
// graph encoding (S1), device memory layout, and the orchestration of the
// device kernels for rank (S4), batched DPOS (S2-S7), the sweep and OS-DPOS
// (S8).  Every step of the method itself runs in the kernels of k_prep.cu /
// k_sim.cu; this file moves data, sizes buffers and sequences launches.
#include "../../include/fastt.h"
#include "fastt_internal.cuh"

#include <algorithm>
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <mutex>
#include <string>
#include <vector>

using namespace fastt;

static thread_local std::string g_err;

static fastt_status fail(fastt_status s, const char *fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return s;
}

#define CK(x)                                                                                \
  do {                                                                                       \
    cudaError_t e_ = (x);                                                                    \
    if (e_ != cudaSuccess) return fail(FASTT_ECUDA, "%s: %s", #x, cudaGetErrorString(e_));   \
  } while (0)
#define TRY(x)                            \
  do {                                    \
    fastt_status s_ = (x);                \
    if (s_ != FASTT_OK) return s_;        \
  } while (0)

static size_t al16(size_t x) { return (x + 15) & ~(size_t)15; }

// ------------------------------------------------------------------ layouts

struct RawLayout {
  int64_t vcap = 0, ecap = 0;
  size_t o[20] = {0};
  size_t total = 0;
};

static RawLayout raw_layout(int64_t vcap, int64_t ecap, int G) {
  RawLayout L;
  L.vcap = vcap;
  L.ecap = ecap;
  size_t sz[20] = {(size_t)vcap * 4, (size_t)vcap * 4, (size_t)vcap * 4, (size_t)vcap * 4,  // off/cnt
                   (size_t)ecap * 4, (size_t)ecap * 4,                                       // dst, src
                   (size_t)ecap * 8, (size_t)ecap * 8,                                       // bytes
                   (size_t)ecap, (size_t)ecap,                                               // param flags
                   (size_t)vcap * G * 8,                                                     // cost
                   (size_t)vcap * 8, (size_t)vcap * 8,                                       // mem, param
                   (size_t)vcap, (size_t)vcap,                                               // split_mask, alive
                   (size_t)vcap * 4,                                                         // topo
                   (size_t)vcap * 4, (size_t)(vcap + 2) * 4, (size_t)vcap * 4,               // height, levels
                   16};
  size_t off = 0;
  for (int k = 0; k < 20; k++) {
    L.o[k] = off;
    off += al16(sz[k]);
  }
  L.total = off;
  return L;
}

static RawGraph raw_struct(char *b, const RawLayout &L, int32_t V, int32_t nl, int64_t E) {
  RawGraph R;
  R.V = V;
  R.n_live = nl;
  R.E = E;
  R.succ_off = (uint32_t *)(b + L.o[0]);
  R.succ_cnt = (uint32_t *)(b + L.o[1]);
  R.pred_off = (uint32_t *)(b + L.o[2]);
  R.pred_cnt = (uint32_t *)(b + L.o[3]);
  R.succ_dst = (int32_t *)(b + L.o[4]);
  R.pred_src = (int32_t *)(b + L.o[5]);
  R.succ_bytes = (int64_t *)(b + L.o[6]);
  R.pred_bytes = (int64_t *)(b + L.o[7]);
  R.succ_param = (uint8_t *)(b + L.o[8]);
  R.pred_param = (uint8_t *)(b + L.o[9]);
  R.cost = (int64_t *)(b + L.o[10]);
  R.mem = (int64_t *)(b + L.o[11]);
  R.param = (int64_t *)(b + L.o[12]);
  R.split_mask = (uint8_t *)(b + L.o[13]);
  R.alive = (uint8_t *)(b + L.o[14]);
  R.topo = (int32_t *)(b + L.o[15]);
  R.height = (int32_t *)(b + L.o[16]);
  R.lvl_off = (int32_t *)(b + L.o[17]);
  R.lvl_ops = (int32_t *)(b + L.o[18]);
  R.H = 0;
  R.ov_o = R.ov_base = R.ov_n = R.ov_S = 0;
  R.ov_P = -1;
  return R;
}

struct PrepLayout {
  int64_t ncap = 0, ecap = 0;
  size_t o[20] = {0};
  size_t total = 0;
};

static PrepLayout prep_layout(int64_t ncap, int64_t ecap, int G, int K, int tbytes) {
  PrepLayout L;
  L.ncap = ncap;
  L.ecap = ecap;
  size_t sz[20] = {(size_t)ncap * CARD_WORDS * 4,        // card
                   (size_t)ncap * G * tbytes,           // costp
                   (size_t)ecap * 4,                    // pe_src
                   (size_t)(ecap + 64) * K * tbytes,    // pe_comm (+ padding for speculative reads)
                   (size_t)ecap * 4, (size_t)ecap * 4,  // se_dst, se_pe
                   (size_t)ncap * 4,                    // npred
                   (size_t)(ncap / 32 + 2) * 4,         // srcbits
                   (size_t)ncap * 4,                    // pos (V <= ncap)
                   (size_t)ncap * 4,                    // uid
                   (size_t)ncap * 8,                    // rank
                   (size_t)ncap * 4,                    // cp
                   (size_t)(ncap + 1) * 8,              // pmem
                   (size_t)(ncap + 1) * G * 8,          // pcost
                   (size_t)ncap * 8, (size_t)ncap * 8,  // keys
                   (size_t)ncap * 4, (size_t)ncap * 4,  // vals
                   33 * 4,                              // srcsumm
                   (size_t)ncap * 8};                   // act
  size_t off = 0;
  for (int k = 0; k < 20; k++) {
    L.o[k] = off;
    off += al16(sz[k]);
  }
  L.total = off;
  return L;
}

static PrepGraph prep_struct(char *b, const PrepLayout &L, int tbits) {
  PrepGraph P;
  memset(&P, 0, sizeof P);
  P.tbits = tbits;
  P.card = (uint32_t *)(b + L.o[0]);
  P.costp = (void *)(b + L.o[1]);
  P.pe_src = (uint32_t *)(b + L.o[2]);
  P.pe_comm = (void *)(b + L.o[3]);
  P.se_dst = (uint32_t *)(b + L.o[4]);
  P.se_pe = (uint32_t *)(b + L.o[5]);
  P.npred = (uint32_t *)(b + L.o[6]);
  P.srcbits = (uint32_t *)(b + L.o[7]);
  P.pos = (uint32_t *)(b + L.o[8]);
  P.uid = (uint32_t *)(b + L.o[9]);
  P.rank = (uint64_t *)(b + L.o[10]);
  P.cp = (uint32_t *)(b + L.o[11]);
  P.pmem = (int64_t *)(b + L.o[12]);
  P.pcost = (int64_t *)(b + L.o[13]);
  P.key0 = (uint64_t *)(b + L.o[14]);
  P.key1 = (uint64_t *)(b + L.o[15]);
  P.val0 = (uint32_t *)(b + L.o[16]);
  P.val1 = (uint32_t *)(b + L.o[17]);
  P.srcsumm = (uint32_t *)(b + L.o[18]);
  P.act = (int64_t *)(b + L.o[19]);
  return P;
}

// ----------------------------------------------------------------- graph

// A "base": a raw graph in HBM plus its prepared (priority-ordered) form.
// The loaded graph is one; OS-DPOS creates more as it accepts splits.
struct Base {
  int32_t V = 0, n_live = 0, n = 0, cp_len = 0;
  int64_t E = 0;  // edge slots used
  RawLayout rl;
  PrepLayout pl;
  char *raw_block = nullptr;
  RawGraph *raw_dev = nullptr;
  char *prep_block = nullptr;
  PrepGraph *pg_dev = nullptr;
  int tbits = 64, key_bits = 64;
  int topo = 0;  // the prepared priority order is topological (k_sim's TOPO path)
  unsigned long long bound = 0, maxextra = 0;
  // packed device keys of the lane kernel (32-bit time, one link class)
  uint32_t *costk = nullptr;  // [n][G] cost << gshift | d, then commk [n][4] (inline comm << gshift)
  uint32_t *commk = nullptr;
  uint32_t *pkc = nullptr;  // compact PK cards of k_lane_pk (same allocation)
  LvlRec *lvlrec = nullptr;  // k_rank's level records (LvlRec, n_live)
  uint32_t pk_lim = 0;
  // recorded BASE schedule for prefix sharing, per CP-pin flag value
  struct Snap {
    bool valid = false;
    int round_dev = -1;
    char *buf = nullptr;  // dq | avail | ms | rec | rounds | used | used + reserved | keys
    uint32_t *dq = nullptr, *key = nullptr;  // key: the records as packed keys FT << gshift | place (PK)
    uint32_t *key2 = nullptr;                // the keys doubled (k_lane_pk, two candidates per lane)
    uint32_t *key4 = nullptr;                // ... and four times (four candidates per lane)
    void *avail = nullptr, *ms = nullptr, *rec = nullptr, *used = nullptr, *ur = nullptr;
    int32_t *rounds = nullptr;
  } snap[2];
  void release() {
    cudaFree(raw_block);
    cudaFree(raw_dev);
    cudaFree(prep_block);
    cudaFree(pg_dev);
    cudaFree(costk);
    cudaFree(lvlrec);
    lvlrec = nullptr;
    costk = nullptr;
    commk = nullptr;
    pkc = nullptr;
    pk_lim = 0;
    for (auto &x : snap) {
      cudaFree(x.buf);
      x = Snap();
    }
    raw_block = prep_block = nullptr;
    raw_dev = nullptr;
    pg_dev = nullptr;
  }
};

struct StreamCache {
  bool valid = false;
  uint8_t *base_place = nullptr;
  int32_t *live = nullptr;
  int32_t n_live = 0;
  int64_t n_split = 0;
  int32_t *split_op = nullptr;
  uint8_t *split_dim = nullptr, *split_n = nullptr;
  void release() {
    cudaFree(base_place);
    cudaFree(live);
    cudaFree(split_op);
    cudaFree(split_dim);
    cudaFree(split_n);
    *this = StreamCache();
  }
};

struct fastt_graph {
  int dev = 0;
  int32_t V = 0, G = 1, K = 1;
  int64_t E = 0;
  int32_t maxP = 0, maxS = 0;
  int32_t v_max = 0;  // V + largest single-split overlay (user-facing per-op array size)
  GraphConst gch;
  GraphConst *gc_dev = nullptr;
  uint8_t *split_mask_dev = nullptr;
  Base base;
  std::vector<uint8_t> split_mask_h;
  StreamCache streams[16];
  // arena (per base layout)
  size_t arena_raw_total = 0, arena_prep_total = 0;
  int arena_slots = 0;
  bool arena_capped = false;  // the last allocation was limited by the memory cap
  char *arena = nullptr;
  RawGraph *tmpl_dev = nullptr, *slot_raws_dev = nullptr;
  PrepGraph *slot_pgs_dev = nullptr;
  Cand *slot_cands = nullptr;
  int64_t *slot_result = nullptr, *slot_index = nullptr;
  // simulation workspace
  int sms = 148, sim_block = SIM_BLOCK, sim_grid = 0, sim_tbits = 0, sim_cpw = 1, sim_bm_stride = 0;
  int sim_grid_topo = 0;  // resident blocks of the TOPO variant (no shared-memory ready set)
  bool use_topo = true;   // FASTT_NO_TOPO=1 forces the ready-set path (A/B parity)
  // resident blocks of the lane-per-candidate kernel per memory mode and packed keys
  int sim_grid_lane[3][2] = {{0, 0}, {0, 0}, {0, 0}};
  int lane_wpb[3][2] = {{4, 4}, {4, 4}, {4, 4}};  // warps per block of those launches (k_lane_pk: 1, 2 or 4)
  int pk_wpb_env = 0;  // FASTT_PK_WPB: force k_lane_pk's warps per block
  // device staging buffers of fastt_schedule_batch (host candidates in,
  // makespan/status out), kept across calls and grown on demand
  struct IoBuf {
    void *p = nullptr;
    size_t cap = 0;
  } io[4];  // candidates in, makespan, status, per-device peak memory out
  bool use_rank_reuse = true;  // FASTT_NO_RANK_REUSE=1: SPLIT slots recompute every rank (A/B parity)
  bool use_cost_hole = true;   // FASTT_NO_COST_HOLE=1: split slots copy the base cost table too (A/B parity)
  bool use_lvlrec = true;      // FASTT_NO_LVLREC=1: k_rank recomputes every op's terms on its chain (A/B parity)
  bool use_pk = true;      // FASTT_NO_PK=1: the lane kernel without packed device keys (A/B parity)
  bool use_pk_tma = true;  // FASTT_NO_PK_TMA=1: packed keys on k_sim_lane instead of k_lane_pk (A/B parity)
  int pk_cpl = 2;          // FASTT_PK_CPL=1: one candidate per lane in the makespan-only k_lane_pk (A/B)
  bool pk_cpl_peak = true;  // FASTT_PK_CPL_PEAK=0: one per lane with per-device peak memory
  uint32_t pk_lim_cap = 0xFFFFFFFFu;  // FASTT_PK_LIM=<ns>: lower the deferral bound (tests of the deferral path)
  bool use_lane = true;   // FASTT_NO_LANE=1 keeps position-order launches on the group kernel (A/B parity)
  int last_topo = 0;      // the last main launch: 0 ready-set kernel, 1 group position-order, 2 lane position-order
  int64_t sim_ncap = 0;
  size_t sim_smem = 0;
  void *slab = nullptr;
  void *gap = nullptr;  // INSERT idle-slot pools, one per candidate slot (lazy)
  void *gap_lane = nullptr;  // INSERT idle-slot arrays of the lane kernel (lazy)
  int32_t gap_cap = 0;       // idle slots per lane and device
  int ins_lane_grid = 0;
  // FASTT_LANE_INS=1 runs INSERT on the lane kernel; off by default: on C5 it
  // evaluates 53k candidates/s against the group kernel's 147k/s (one lane
  // searches its G devices' idle slots one after the other, the group kernel
  // searches them in parallel, a lane per device)
  bool use_lane_ins = false;
  int64_t ins_cap_env = 0;   // FASTT_INS_CAP=<slots>: lower the per-device capacity (tests of the deferral)
  int64_t gap_stride = 0;
  int ins_grid = 0;
  int64_t *wbest = nullptr, *best_dev = nullptr;
  unsigned long long *counters = nullptr;  // [0] work counter, [1] deferred count, [2..3] k_sim_lane step counts, [4] kernel error
  int64_t *defer_q = nullptr;
  int64_t defer_cap = 0;
  // misc scratch
  int64_t *scratch_rank = nullptr;
  int32_t *scratch_cp = nullptr, *scratch_list = nullptr, *scratch_n = nullptr;
  // instrumentation
  int64_t launches = 0;
  fastt_timing last;
  bool share = true;  // BASE-schedule prefix sharing (env FASTT_NO_SHARE=1 disables, for A/B checks)
  // start-step sorted candidate lists for prefix sharing
  char *sort_buf = nullptr;
  int64_t sort_cap = 0;
  Cand *srt_tmp_c = nullptr, *srt_c = nullptr;
  int64_t *srt_tmp_i = nullptr, *srt_i = nullptr, *srt_res = nullptr;
  uint32_t *srt_key = nullptr, *srt_hist = nullptr;
  cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
  cudaEvent_t ev_main = nullptr;  // the main launch's start when it waits for the preparation kernels
  bool ev_main_rec = false;
  // overlapped preparation: the deferred tail of a classified list is
  // prepared and simulated on a high-priority stream while the main launch
  // (non-persistent, on the call's stream) runs
  bool use_overlap = true;  // FASTT_NO_OVERLAP=1 (A/B parity)
  int lane_batches = 0;     // FASTT_LANE_BATCHES: batches per warp of a non-persistent main launch (0: persistent)
  int main_bps = 0;         // FASTT_MAIN_BPS: resident blocks per SM of a persistent overlapped main launch (0: all)
  // FASTT_OVL_MODE: 1 (default) the main launch starts once the preparation
  // kernels are done and overlaps the slot simulations; 0 it starts at once
  // (all three run together); 2 main_bps blocks per SM start at once, the
  // rest after the preparation kernels (measured on C5, 1e6 candidates, final
  // code: 93.6 / 103-104 / 97.7-107 ms per sweep: a latency-bound
  // preparation chain co-running with the issue-bound main launch slows by
  // more than the main launch gains)
  int ovl_mode = 1;
  cudaStream_t st_prep = nullptr;
  cudaEvent_t ov_ev[5] = {nullptr, nullptr, nullptr, nullptr, nullptr};  // classified, prep start, slots done, prepared, main 2 done
  cudaStream_t st_main2 = nullptr;  // the second main launch (ovl_mode 2)
  void *slab_mg = nullptr;  // slab columns of the concurrent slot launches
  int64_t slab_mg_cols = 0;
  unsigned long long *counters2 = nullptr;  // work counter of the concurrent slot launches
  uint32_t *ov_words = nullptr;             // [0] n_main (classified), [1] active preparation slots
  uint32_t *slot_bm = nullptr;              // slab-slot bitmap of the non-persistent main launch
  int32_t slot_bm_bits = 0;
  int64_t wbest_cap = 0;        // wbest entries allocated
  int64_t pin_defer_hint = 256; // rank-changing PINs seen by the last classified call
  int64_t seq_defer_hint = 256; // deferred candidates of the last sequential (non-overlapped) evaluation
  // device-driven deferral loop (run_defer_loop): a cached CUDA graph with a
  // WHILE node over the preparation rounds, rebuilt when its arguments change
  DeferBlock *dblk = nullptr;
  uint32_t *dwords = nullptr;      // zero words (n_main of a loop without a tail)
  cudaStream_t st_cap = nullptr;   // capture stream of the loop graph
  cudaGraphExec_t dl_exec = nullptr;
  std::vector<char> dl_key;
  cudaEvent_t dl_ev = nullptr;     // recorded after every launch of dl_exec
  std::vector<std::pair<cudaGraphExec_t, cudaEvent_t>> dl_retired;  // destroyed once their event completed
  int dl_round_launches = 0;       // kernels per loop round (fastt_last_timing)
  DeferBlock *dl_sum = nullptr;    // pinned host copy of the last loop's block (hints, deferred counts)
  cudaEvent_t dl_sum_ev = nullptr;
  bool dl_sum_pending = false;
  bool dl_ran = false;             // this call ran the loop
  // call ordering: every call on this graph waits for the previous one (its
  // internal scratch is shared), whatever stream either was issued on
  cudaEvent_t done_ev = nullptr;
  bool done_rec = false;
  std::mutex mu;
};

static void read_defer_summary(fastt_graph *g);
static void reap_defer(fastt_graph *g, bool wait);

// FASTT_HOST_TRACE=1: host wall-clock checkpoints of a call on stderr (where
// a call waits for the device)
static void host_trace(const char *what) {
  static int on = -1;
  if (on < 0) on = getenv("FASTT_HOST_TRACE") && atoi(getenv("FASTT_HOST_TRACE")) ? 1 : 0;
  if (!on) return;
  static auto t0 = std::chrono::steady_clock::now();
  const double us = std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t0).count();
  fprintf(stderr, "[fastt host] %12.1f us  %s\n", us, what);
}

// kernels each launcher issues (for the launch count of fastt_last_timing)
enum { NL_SIM = 1, NL_PREP = 9, NL_ARGMIN = 1, NL_GATHER = 1, NL_CANDGEN = 1, NL_ORDER = 1, NL_FILL = 1 };

static fastt_status timing_begin(fastt_graph *g, uint32_t flags, cudaStream_t st) {
  g->launches = 0;
  memset(&g->last, 0, sizeof g->last);
  if (!(flags & FASTT_F_TIMING)) return FASTT_OK;
  if (g->counters) CK(cudaMemsetAsync(g->counters + 2, 0, 2 * sizeof(unsigned long long), st));
  for (auto &e : g->ev)
    if (!e) CK(cudaEventCreate(&e));
  if (!g->ev_main) CK(cudaEventCreate(&g->ev_main));
  g->ev_main_rec = false;
  CK(cudaEventRecord(g->ev[0], st));
  return FASTT_OK;
}
static void timing_mark(fastt_graph *g, uint32_t flags, int k, cudaStream_t st) {
  if (flags & FASTT_F_TIMING) cudaEventRecord(g->ev[k], st);
}
// a ready-set launch met a graph above READY_SET_MAX positions (k_sim sets
// counters[4]): the call fails (reads and clears the flag; synchronises st)
static fastt_status check_kernel_err(fastt_graph *g, cudaStream_t st) {
  if (!g->counters) return FASTT_OK;
  unsigned long long e = 0;
  CK(cudaMemcpyAsync(&e, g->counters + 4, sizeof e, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (e) {
    CK(cudaMemsetAsync(g->counters + 4, 0, sizeof e, st));
    return fail(FASTT_EUNSUP, "a candidate's priority order is not topological and its graph has more than %d ops "
                              "(the ready-set kernel's bitmap)", (int)READY_SET_MAX);
  }
  return FASTT_OK;
}

// the last deferral loop of this call, once its summary has landed (host
// synchronised): deferred count and the loop's kernel launches
static void defer_stats(fastt_graph *g) {
  if (!g->dl_ran || g->dl_sum_pending) return;
  const DeferBlock &d = *g->dl_sum;
  const int64_t tail = d.do_tail && d.n_main >= 0 ? d.n - d.n_main : 0;
  const int64_t past = d.n - d.tail_lo;  // the tail past the arena: loop rounds
  const int64_t cap = d.cap > 0 ? d.cap : 1;
  g->last.deferred = tail + d.n_defer;
  g->last.launches += ((past + cap - 1) / cap + (d.n_defer + cap - 1) / cap) * g->dl_round_launches;
}

static fastt_status timing_end(fastt_graph *g, uint32_t flags, cudaStream_t st, int64_t cands) {
  g->last.launches = g->launches;
  g->last.candidates = cands;
  g->last.deferred = 0;
  g->last.topo = g->last_topo;
  if (!(flags & FASTT_F_TIMING)) return FASTT_OK;
  CK(cudaEventRecord(g->ev[3], st));
  CK(cudaEventSynchronize(g->ev[3]));
  if (g->counters) {
    unsigned long long ws[2] = {0, 0};
    CK(cudaMemcpy(ws, g->counters + 2, sizeof ws, cudaMemcpyDeviceToHost));
    g->last.warp_steps = (int64_t)ws[0];
    g->last.lane_steps = (int64_t)ws[1];
  }
  float a = 0, b = 0, c = 0;
  CK(cudaEventElapsedTime(&a, g->ev_main_rec ? g->ev_main : g->ev[0], g->ev[1]));
  CK(cudaEventElapsedTime(&b, g->ev[1], g->ev[2]));
  CK(cudaEventElapsedTime(&c, g->ev[0], g->ev[3]));
  g->last.ms_sim = a;
  g->last.ms_prep = b;
  g->last.ms_total = c;
  return FASTT_OK;
}

// Every ABI call that issues work: call_begin orders it after the previous
// call on this graph (any stream); call_end records the graph's completion
// event and -- unless FASTT_F_ASYNC -- waits for the stream, reports a
// kernel-side envelope error and fills the deferred statistics.
static fastt_status call_begin(fastt_graph *g, cudaStream_t st) {
  if (g->done_rec) CK(cudaStreamWaitEvent(st, g->done_ev, 0));
  read_defer_summary(g);
  g->dl_ran = false;
  return FASTT_OK;
}
static fastt_status call_end(fastt_graph *g, uint32_t flags, cudaStream_t st, fastt_status rc) {
  if (!g->done_ev && cudaEventCreateWithFlags(&g->done_ev, cudaEventDisableTiming) != cudaSuccess) g->done_ev = nullptr;
  if (g->done_ev && cudaEventRecord(g->done_ev, st) == cudaSuccess) g->done_rec = true;
  if (flags & FASTT_F_ASYNC) return rc;
  if (cudaStreamSynchronize(st) != cudaSuccess && rc == FASTT_OK) rc = fail(FASTT_ECUDA, "synchronize");
  if (rc == FASTT_OK) rc = check_kernel_err(g, st);
  read_defer_summary(g);
  defer_stats(g);
  // retired loop graphs are destroyed here, never on an asynchronous path
  // (cudaGraphExecDestroy waits for the device)
  reap_defer(g, false);
  return rc;
}

// the blocking calls (rank, split search, stream info): ordered after the
// previous call on the graph; their completion recorded at scope exit
struct CallGuard {
  fastt_graph *g;
  cudaStream_t st;
  CallGuard(fastt_graph *g_, cudaStream_t st_) : g(g_), st(st_) { call_begin(g, st); }
  ~CallGuard() {
    if (!g->done_ev && cudaEventCreateWithFlags(&g->done_ev, cudaEventDisableTiming) != cudaSuccess) g->done_ev = nullptr;
    if (g->done_ev && cudaEventRecord(g->done_ev, st) == cudaSuccess) g->done_rec = true;
  }
};

static int64_t overlay_v(const fastt_graph *g) { return (int64_t)g->maxP + g->G + g->maxS + 1; }
static int64_t overlay_e(const fastt_graph *g) {
  return (int64_t)g->maxP * (2 + g->G) + (int64_t)g->maxS * (2 + g->G) + (int64_t)g->G + 16;
}

struct Dev {  // RAII device guard
  int prev = -1;
  explicit Dev(int d) {
    cudaGetDevice(&prev);
    cudaSetDevice(d);
  }
  ~Dev() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

static cudaStream_t stream_of(const fastt_opts *o) { return o ? (cudaStream_t)o->cuda_stream : (cudaStream_t)0; }
static uint32_t flags_of(const fastt_opts *o) { return o ? o->flags : 0u; }

// ------------------------------------------------------ base preparation

static int bits_for(unsigned long long v) {
  int b = 1;
  while (b < 64 && (v >> b) != 0) b++;
  return b;
}

// bound -> time type; rank, sort, cards, CP for a base whose raw graph is in place
static fastt_status prepare_base(fastt_graph *g, Base &B, cudaStream_t st) {
  {
    int32_t *scratch = nullptr;
    CK(cudaMalloc(&scratch, sizeof(int32_t) * (3 * B.rl.vcap + 64)));
    launch_heights(B.raw_dev, scratch, B.rl.vcap, st);
    CK(cudaGetLastError());
    CK(cudaStreamSynchronize(st));
    cudaFree(scratch);
  }
  // k_rank's level records (fast path of the preparation slots)
  cudaFree(B.lvlrec);
  B.lvlrec = nullptr;
  if (B.n_live > 0) {
    CK(cudaMalloc(&B.lvlrec, sizeof(LvlRec) * (size_t)B.n_live));
    launch_lvlrec(B.raw_dev, g->gc_dev, B.n_live, B.lvlrec, st);
    CK(cudaGetLastError());
  }
  unsigned long long *d_b = nullptr;
  CK(cudaMalloc(&d_b, 16));
  CK(cudaMemsetAsync(d_b, 0, 16, st));
  launch_bound(B.raw_dev, g->gc_dev, g->G, d_b, st);
  unsigned long long hb[2];
  CK(cudaMemcpyAsync(hb, d_b, 16, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  cudaFree(d_b);
  B.bound = hb[0];
  B.maxextra = hb[1];
  unsigned long long tot = hb[0] + hb[1];
  B.tbits = tot < (1ull << 32) ? 32 : 64;
  B.key_bits = B.tbits == 32 ? 32 : bits_for(tot);
  // prepared block (capacity = raw capacity)
  B.pl = prep_layout(B.rl.vcap, B.rl.ecap, g->G, g->K, B.tbits / 8);
  CK(cudaMalloc(&B.prep_block, B.pl.total));
  CK(cudaMalloc(&B.pg_dev, sizeof(PrepGraph)));
  PrepGraph P = prep_struct(B.prep_block, B.pl, B.tbits);
  P.V = B.V;
  CK(cudaMemcpyAsync(B.pg_dev, &P, sizeof P, cudaMemcpyHostToDevice, st));
  launch_rank(B.raw_dev, B.pg_dev, g->gc_dev, nullptr, 1, g->G, st);
  launch_sort(B.pg_dev, B.raw_dev, 1, B.key_bits, B.n_live, st);
  launch_cards(B.raw_dev, B.pg_dev, g->gc_dev, 1, B.n_live, g->G, g->K, B.tbits, st, true);
  launch_cp(B.raw_dev, B.pg_dev, 1, g->G, B.tbits, st);
  CK(cudaGetLastError());
  CK(cudaMemcpyAsync(&P, B.pg_dev, sizeof P, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  B.n = P.n;
  B.cp_len = P.cp_len;
  B.topo = P.topo;
  if (B.rl.vcap > READY_SET_MAX && !B.topo)
    return fail(FASTT_EUNSUP,
                "a graph above %d ops needs a topological priority order (every edge with w_i + c_ij > 0, R2): "
                "the ready-set kernel's bitmap covers %d positions",
                READY_SET_MAX, READY_SET_MAX);
  // packed keys (k_sim_lane PK): the bound below which no key wraps
  if (g->use_pk && B.tbits == 32 && g->K == 1 && B.n > 0) {
    int gsh = 0;
    while ((1 << gsh) < g->G) gsh++;
    const size_t nck = ((size_t)B.n * g->G + 3) & ~(size_t)3;  // (commk, pkc 16-B aligned)
    const size_t pkw = (size_t)pk_card_words_host(gsh);
    CK(cudaMalloc(&B.costk, sizeof(uint32_t) * (nck + 4 * (size_t)B.n + pkw * (size_t)B.n)));
    B.commk = B.costk + nck;
    B.pkc = B.commk + 4 * (size_t)B.n;
    unsigned long long *d_m = nullptr, hm[2];
    CK(cudaMalloc(&d_m, 16));
    CK(cudaMemsetAsync(d_m, 0, 16, st));
    launch_pack_costs(B.pg_dev, B.n, g->G, gsh, P.E, B.costk, B.commk, B.pkc, d_m, st);
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(hm, d_m, 16, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    cudaFree(d_m);
    const long long lim = (1ll << (32 - gsh)) - (long long)hm[0] - (long long)hm[1];
    B.pk_lim = lim > 0 ? (uint32_t)std::min<long long>(lim, (long long)g->pk_lim_cap) : 0u;
  }
  return FASTT_OK;
}

// ------------------------------------------------------------- workspaces

// preparation slots for `need` deferred candidates: sized to the batch (a
// C5 sweep's ~4k split candidates prepare in one wave), capped at
// ARENA_MAX_SLOTS (small graphs' frequent deferrals -- C1 defers ~10 % of
// its candidates -- take fewer rounds) and by memory (below), and kept for
// later calls with the same layout
constexpr int64_t ARENA_MAX_SLOTS = 32768;  // (slot-indexed launches put the slot in gridDim.y)
static fastt_status ensure_arena(fastt_graph *g, const Base &B, cudaStream_t st, int64_t need) {
  size_t rt = B.rl.total, pt = B.pl.total;
  const int64_t want = std::min<int64_t>(std::max<int64_t>(need, 64), ARENA_MAX_SLOTS);
  const bool same = g->arena && g->arena_raw_total == rt && g->arena_prep_total == pt;
  if (same && g->arena_slots >= want) return FASTT_OK;
  // (an arena the memory cap already limited is not re-allocated for a
  // larger request of the same layout: the cap would bind again, and each
  // attempt frees and re-allocates tens of GB; more rounds run instead)
  if (same && g->arena_capped) return FASTT_OK;
  cudaFree(g->arena);
  cudaFree(g->tmpl_dev);
  cudaFree(g->slot_raws_dev);
  cudaFree(g->slot_pgs_dev);
  cudaFree(g->slot_cands);
  cudaFree(g->slot_result);
  cudaFree(g->slot_index);
  g->arena = nullptr;
  size_t freeb = 0, totb = 0;
  CK(cudaMemGetInfo(&freeb, &totb));
  size_t per = rt + pt;
  // at most 60 % of the free and 40 % of the total device memory per graph
  // (a wave that does not fit costs one more latency-bound preparation round;
  // C5R8's 4,038 split slots take ~53 GB)
  int64_t slots = std::min<int64_t>(want, (int64_t)(std::min(freeb * 3 / 5, totb * 2 / 5) / per));
  if (slots < 1) return fail(FASTT_ENOMEM, "device memory too small for one preparation slot (%zu bytes)", per);
  g->arena_slots = (int)slots;
  g->arena_capped = slots < want;
  CK(cudaMalloc(&g->arena, per * slots));
  std::vector<RawGraph> tm(slots);
  std::vector<PrepGraph> pg(slots);
  for (int64_t k = 0; k < slots; k++) {
    char *b = g->arena + per * k;
    tm[k] = raw_struct(b, B.rl, 0, 0, 0);
    pg[k] = prep_struct(b + rt, B.pl, B.tbits);
  }
  CK(cudaMalloc(&g->tmpl_dev, sizeof(RawGraph) * slots));
  CK(cudaMalloc(&g->slot_raws_dev, sizeof(RawGraph) * slots));
  CK(cudaMalloc(&g->slot_pgs_dev, sizeof(PrepGraph) * slots));
  CK(cudaMalloc(&g->slot_cands, sizeof(Cand) * slots));
  CK(cudaMalloc(&g->slot_result, sizeof(int64_t) * slots));
  CK(cudaMalloc(&g->slot_index, sizeof(int64_t) * slots));
  CK(cudaMemcpyAsync(g->tmpl_dev, tm.data(), sizeof(RawGraph) * slots, cudaMemcpyHostToDevice, st));
  CK(cudaMemcpyAsync(g->slot_pgs_dev, pg.data(), sizeof(PrepGraph) * slots, cudaMemcpyHostToDevice, st));
  CK(cudaStreamSynchronize(st));
  g->arena_raw_total = rt;
  g->arena_prep_total = pt;
  return FASTT_OK;
}

// candidates per lane of a k_lane_pk launch in memory mode mm: two for
// makespan-only sweeps and with per-device peak memory (mm 1; FASTT_PK_CPL_PEAK=0
// keeps one: its 4 KB more shared memory per warp need blocks of 1-2 warps to
// keep 10 warps per SM, measured 88.9 vs 90.8 ms for one candidate per lane
// on C5, 101.5 ms with 4-warp blocks)
static int pk_cpl(const fastt_graph *g, int mm) {
  if (!g->use_pk_tma || g->pk_cpl < 2) return 1;
  if (mm == 0) return g->pk_cpl;
  return mm == 1 && g->pk_cpl_peak ? 2 : 1;
}

static int gshift_of(int G) {
  int gsh = 0;
  while ((1 << gsh) < G) gsh++;
  return gsh;
}

// simulation workspace: one candidate per lane group (32 >> gshift per warp),
// each with a ready bitmap in shared memory and an 8/16 B-per-op slab in HBM
static fastt_status ensure_sim(fastt_graph *g, const Base &B, int64_t defer_need, uint32_t flags = 0) {
  int64_t ncap = B.pl.ncap;
  if (!g->slab || g->sim_tbits != B.tbits || g->sim_ncap < ncap) {
    cudaFree(g->slab);
    cudaFree(g->wbest);
    cudaFree(g->gap);
    cudaFree(g->gap_lane);
    g->slab = nullptr;
    g->wbest = nullptr;
    g->gap = nullptr;
    g->gap_lane = nullptr;
    g->ins_lane_grid = 0;
    const int gsh = gshift_of(g->G);
    const int cpw = 32 >> gsh;
    // (the ready-set bitmap: the ready-set kernel runs on at most
    // READY_SET_MAX positions, larger graphs are topological)
    int leaf = (int)((std::min<int64_t>(ncap, READY_SET_MAX) + 31) / 32);
    int stride = leaf + 32;
    while (stride % 32 != 8) stride++;  // candidates of one warp start on different banks
    size_t smem = (size_t)(g->sim_block / 32) * cpw * stride * 4;
    if (smem > 48 * 1024) CK(sim_set_smem(B.tbits, gsh, smem));
    int per_sm = sim_occupancy(B.tbits, gsh, g->sim_block, smem, false);
    if (per_sm < 1) return fail(FASTT_EUNSUP, "simulation kernel does not fit on an SM (smem %zu)", smem);
    g->sim_grid = g->sms * per_sm;
    g->sim_grid_topo = g->sms * std::max(1, sim_occupancy(B.tbits, gsh, g->sim_block, 0, true));
    for (int mm = 0; mm < 3; mm++)
      for (int pk = 0; pk < 2; pk++) {
        // k_lane_pk: the block size (1, 2 or 4 warps) with the most resident
        // warps (its shared memory per warp need not divide an SM's by 4)
        int best_w = 4, best_b = std::max(1, lane_occupancy(B.tbits, gsh, mm, pk != 0, pk ? pk_cpl(g, mm) : 1, 4));
        if (pk && B.tbits == 32)
          for (int w : {2, 1}) {
            if (g->pk_wpb_env > 0 && w != g->pk_wpb_env) continue;
            const int b = lane_occupancy(B.tbits, gsh, mm, true, pk_cpl(g, mm), w);
            // (ties: two candidates per lane run better in 1-warp blocks,
            // measured 70.5 vs 71.9 ms on C5 at equal resident warps)
            const bool tie_small = pk_cpl(g, mm) >= 2 && w == 1 && b * w == best_b * best_w;
            if (b * w > best_b * best_w || tie_small || (g->pk_wpb_env == w && b > 0)) {
              best_b = b;
              best_w = w;
            }
          }
        g->sim_grid_lane[mm][pk] = g->sms * best_b;
        g->lane_wpb[mm][pk] = best_w;
        if (getenv("FASTT_HOST_TRACE")) {
          char msg[96];
          snprintf(msg, sizeof msg, "lane launch mm %d pk %d: %d blocks/SM x %d warps", mm, pk, best_b, best_w);
          host_trace(msg);
          if (pk && B.tbits == 32) {
            char att[512] = "";
            lane_pk_attrs(gsh, mm, pk_cpl(g, mm), att, sizeof att);
            host_trace(att);
          }
        }
      }
    g->sim_smem = smem;
    g->sim_cpw = cpw;
    g->sim_bm_stride = stride;
    int64_t nslot = (int64_t)std::max(g->sim_grid, g->sim_grid_topo) * (g->sim_block / 32) * cpw;
    for (int mm = 0; mm < 3; mm++)
      for (int pk = 0; pk < 2; pk++)
        nslot = std::max<int64_t>(nslot, (int64_t)g->sim_grid_lane[mm][pk] * 32 * g->lane_wpb[mm][pk]);  // a column per lane
    size_t rec = B.tbits == 32 ? 8 : 16;
    CK(cudaMalloc(&g->slab, (size_t)nslot * ncap * rec));
    CK(cudaMalloc(&g->wbest, sizeof(int64_t) * 2 * nslot));
    g->wbest_cap = nslot;
    g->sim_tbits = B.tbits;
    g->sim_ncap = ncap;
  }
  if ((flags & FASTT_F_POLICY_INSERT) && !g->gap) {
    // INSERT: per candidate slot and device an array of at most (ops on
    // the device + 1) idle slots; the resident INSERT grid is capped so the
    // arrays take at most a third of the free device memory
    g->gap_stride = g->sim_ncap + 1;
    const size_t rec = B.tbits == 32 ? sizeof(GapSlot<uint32_t>) : sizeof(GapSlot<uint64_t>);
    const size_t per_block = (size_t)(g->sim_block / 32) * g->sim_cpw * g->G * g->gap_stride * rec;
    size_t fr = 0, tot = 0;
    CK(cudaMemGetInfo(&fr, &tot));
    int64_t ig = std::min<int64_t>(std::max(g->sim_grid, g->sim_grid_topo), (int64_t)(fr / 3 / per_block));
    if (ig > g->sms) ig -= ig % g->sms;
    if (ig < 1) return fail(FASTT_ENOMEM, "INSERT idle-slot arrays (%zu bytes per block)", per_block);
    if (cudaMalloc(&g->gap, (size_t)ig * per_block) != cudaSuccess) {
      cudaGetLastError();
      g->gap = nullptr;
      return fail(FASTT_ENOMEM, "INSERT idle-slot arrays (%lld blocks)", (long long)ig);
    }
    g->ins_grid = (int)ig;
  }
  if ((flags & FASTT_F_POLICY_INSERT) && !g->gap_lane && g->use_lane_ins) {
    // INSERT on the lane kernel: per lane and device gap_cap idle slots (a
    // device holding more is deferred to the group kernel), for as many
    // resident blocks as a third of the free memory allows
    const int G = g->G, GP = 1 << gshift_of(G);
    int64_t cap = std::min<int64_t>(g->sim_ncap + 1, 2 * ((g->sim_ncap + G - 1) / G) + 256);
    if (g->ins_cap_env > 0) cap = std::min<int64_t>(cap, g->ins_cap_env);
    const size_t rec = B.tbits == 32 ? sizeof(GapSlot<uint32_t>) : sizeof(GapSlot<uint64_t>);
    const size_t per_block = (size_t)LANE_BLOCK * GP * (size_t)cap * rec;
    size_t fr = 0, tot = 0;
    CK(cudaMemGetInfo(&fr, &tot));
    int64_t ig = std::min<int64_t>(g->sim_grid_lane[0][0], (int64_t)(fr / 3 / per_block));
    if (ig > g->sms) ig -= ig % g->sms;
    if (ig >= 1 && cudaMalloc(&g->gap_lane, (size_t)ig * per_block) == cudaSuccess) {
      g->gap_cap = (int32_t)cap;
      g->ins_lane_grid = (int)ig;
    } else {
      cudaGetLastError();
      g->gap_lane = nullptr;
      g->ins_lane_grid = 0;  // (INSERT stays on the group kernel)
    }
  }
  if (!g->counters) {
    CK(cudaMalloc(&g->counters, 5 * sizeof(unsigned long long)));
    CK(cudaMemset(g->counters, 0, 5 * sizeof(unsigned long long)));
    CK(cudaMalloc(&g->best_dev, 2 * sizeof(int64_t)));
  }
  if (g->defer_cap < defer_need) {
    cudaFree(g->defer_q);
    int64_t cap = std::max<int64_t>(defer_need, 1024);
    CK(cudaMalloc(&g->defer_q, sizeof(int64_t) * cap));
    g->defer_cap = cap;
  }
  return FASTT_OK;
}

// The launch shape of a base-graph simulation: the TOPO variant (no ready
// set, no shared memory, more resident blocks) when the base's priority order
// is topological, else the ready-set variant.  Slot launches (mode 2) use
// the ready-set variant (slots may differ).
static void main_shape(fastt_graph *g, const Base &B, SimArgs &a, int &grid, size_t &smem) {
  const bool topo = g->use_topo && B.topo && a.mode != 2;
  // the lane kernel covers makespan (+ per-device peak, + memory caps, or
  // INSERT without memory) without per-op outputs or liveness memory
  const int mm = a.cap_check ? 2 : (a.out.peak ? 1 : 0);
  const bool ins_ok = !a.ins || (mm == 0 && g->gap_lane != nullptr && g->ins_lane_grid > 0);
  const bool lane = topo && g->use_lane && !a.live_mem && ins_ok && !a.out.place && !a.out.start && !a.out.deq &&
                    a.snap_mode != 1;
  g->last_topo = lane ? 2 : topo ? 1 : 0;
  a.lane = lane;
  a.lane_mm = mm;
  if (lane && a.ins) {
    a.topo = 1;
    grid = g->ins_lane_grid;
    smem = 0;
  } else if (lane) {
    a.topo = 1;
    // (the packed-key variant: 32-bit time, one link class, keys prepared)
    const bool pk = B.tbits == 32 && g->K == 1 && a.costk != nullptr && a.pk_lim > 0;
    grid = g->sim_grid_lane[a.lane_mm][pk ? 1 : 0];
    a.pk_cpl = pk && a.pkc ? pk_cpl(g, a.lane_mm) : 1;
    a.pk_wpb = g->lane_wpb[a.lane_mm][pk ? 1 : 0];
    smem = 0;
  } else if (topo) {
    a.topo = 1;
    grid = g->sim_grid_topo;
    smem = 0;
  } else {
    a.topo = 0;
    grid = g->sim_grid;
    smem = g->sim_smem;
  }
}
static int max_slots(const fastt_graph *g) {
  int gl = 0;  // resident warps of the lane launches
  for (int mm = 0; mm < 3; mm++)
    for (int pk = 0; pk < 2; pk++) gl = std::max(gl, g->sim_grid_lane[mm][pk] * g->lane_wpb[mm][pk]);
  return std::max(std::max(g->sim_grid, g->sim_grid_topo) * (g->sim_block / 32) * g->sim_cpw, gl);
}

static SimArgs sim_args(fastt_graph *g, const Base &B, uint32_t flags) {
  SimArgs a;
  memset(&a, 0, sizeof a);
  a.flags = flags;
  a.base = B.pg_dev;
  a.slots = g->slot_pgs_dev;
  a.gc = g->gc_dev;
  a.split_mask = B.raw_block ? raw_struct(B.raw_block, B.rl, 0, 0, 0).split_mask : nullptr;
  a.counter = g->counters;
  a.ndefer = g->counters + 1;
  a.stat = g->counters + 2;
  a.err = (unsigned *)(g->counters + 4);
  a.defer_q = g->defer_q;
  a.wbest = g->wbest;
  a.slab = g->slab;
  a.slab_stride = g->sim_ncap;
  a.leaf_words = (int32_t)((g->sim_ncap + 31) / 32);
  a.bm_stride = g->sim_bm_stride;
  a.G = g->G;
  a.gc_K = g->K;
  while ((1 << a.gshift) < g->G) a.gshift++;
  for (int d = 0; d < g->G; d++)
    if (g->gch.cap[d] != I64MAX) a.cap_check = 1;
  a.need_mem = a.cap_check;
  a.fastcomm = B.tbits == 32 && g->K == 1;
  a.costk = B.costk;
  a.commk = B.commk;
  a.pkc = g->use_pk_tma ? B.pkc : nullptr;
  a.pk_lim = B.pk_lim;
  if (flags & FASTT_F_MEM_LIVE) {
    a.live_mem = 1;
    a.need_mem = 1;
  }
  if (flags & FASTT_F_POLICY_INSERT) {
    a.ins = 1;
    a.gap = g->gap;
    a.gap_stride = g->gap_stride;
    a.ins_grid = g->ins_grid;
    a.gap_lane = g->gap_lane;
    a.gap_cap = g->gap_cap;
  }
  return a;
}

// Preparation pipeline for nslots deferred candidates already in slot_cands
// (SURVEY 8(a) S3 + S4 + S5 per candidate): materialise splits, ranks with
// the candidate's allowed sets, priority sort, cards, critical path.
// (nact: the device count of active slots when the wave is sized on the
// device -- the grids cover nslots, slots past *nact exit at once)
static fastt_status run_prep(fastt_graph *g, const Base &B, int nslots, cudaStream_t st,
                             const uint32_t *nact = nullptr) {
  g->launches += NL_PREP;
  launch_slot_setup(g->slot_cands, g->tmpl_dev, B.raw_dev, g->slot_raws_dev, nslots, st);
  // the slot copy skips the base cost, mem and param tables (layout slots
  // 10-12, contiguous): k_rank, k_cards_pred and k_cards_hdr read a base op's
  // rows from the base graph; k_patch_split writes the overlay rows
  const RawGraph Rb = raw_struct(B.raw_block, B.rl, B.V, B.n_live, B.E);
  const int64_t c_lo = (int64_t)B.rl.o[10], c_hi = (int64_t)B.rl.o[13];
  const bool hole = g->use_cost_hole && (c_hi & 15) == 0 && (c_lo & 15) == 0;
  launch_copy_block(B.raw_block, g->arena, (int64_t)(g->arena_raw_total + g->arena_prep_total), (int64_t)B.rl.total,
                    g->slot_cands, nslots, st, nact, hole ? c_lo : 0, hole ? c_hi : 0);
  launch_patch_split(B.raw_dev, g->slot_raws_dev, g->gc_dev, g->slot_cands, nslots, st, nact);
  launch_rank(g->slot_raws_dev, g->slot_pgs_dev, g->gc_dev, g->slot_cands, nslots, g->G, st,
              g->use_rank_reuse ? prep_struct(B.prep_block, B.pl, B.tbits).rank : nullptr, nact,
              hole ? Rb.cost : nullptr, g->use_lvlrec ? B.lvlrec : nullptr);
  launch_sort(g->slot_pgs_dev, g->slot_raws_dev, nslots, B.key_bits, (int)B.rl.vcap, st, nact);
  // (successor lists only for slots the ready-set kernel will run: see launch_slots)
  launch_cards(g->slot_raws_dev, g->slot_pgs_dev, g->gc_dev, nslots, (int)B.rl.vcap, g->G, g->K, B.tbits, st,
               !g->use_topo, nact, hole ? Rb.cost : nullptr, hole ? Rb.mem : nullptr, hole ? Rb.param : nullptr);
  launch_cp(g->slot_raws_dev, g->slot_pgs_dev, nslots, g->G, B.tbits, st, nact);
  CK(cudaGetLastError());
  return FASTT_OK;
}

// Record the BASE schedule of base B under `flags` (one BASE run in
// snap_mode 1): per-position dequeue index, final records, avail and
// makespan before every step, the base CP rounds.
static fastt_status ensure_snapshot(fastt_graph *g, Base &B, uint32_t flags, cudaStream_t st) {
  Base::Snap &S = B.snap[flags & FASTT_F_CP_PIN ? 1 : 0];
  if (S.valid || (flags & FASTT_F_POLICY_INSERT)) return FASTT_OK;  // (no sharing under INSERT)
  const size_t tb = B.tbits / 8, n = (size_t)B.pl.ncap;
  const size_t o_dq = 0, o_av = al16(4 * n), o_ms = o_av + al16(tb * (n + 1) * g->G),
               o_rec = o_ms + al16(tb * (n + 1)), o_rd = o_rec + al16((B.tbits == 32 ? 8 : 16) * n),
               o_us = o_rd + 64, o_ur = o_us + al16(8 * (n + 1) * g->G), o_k = o_ur + al16(8 * (n + 1) * g->G),
               o_k2 = o_k + al16(4 * n), o_k4 = o_k2 + al16(8 * n), tot = o_k4 + al16(16 * n);
  CK(cudaMalloc(&S.buf, tot));
  S.dq = (uint32_t *)(S.buf + o_dq);
  S.avail = S.buf + o_av;
  S.ms = S.buf + o_ms;
  S.rec = S.buf + o_rec;
  S.rounds = (int32_t *)(S.buf + o_rd);
  S.used = S.buf + o_us;
  S.ur = S.buf + o_ur;
  S.key = (uint32_t *)(S.buf + o_k);
  S.key2 = (uint32_t *)(S.buf + o_k2);
  S.key4 = (uint32_t *)(S.buf + o_k4);
  CK(cudaMemsetAsync(S.rounds, 0, 16, st));
  Cand c;
  memset(&c, 0, sizeof c);
  c.split_op = -1;
  for (int k = 0; k < 4; k++) c.pin_op[k] = -1;
  Cand *d_c;
  int64_t *d_ms;
  uint8_t *d_st;
  CK(cudaMalloc(&d_c, sizeof c));
  CK(cudaMalloc(&d_ms, 8));
  CK(cudaMalloc(&d_st, 8));
  CK(cudaMemcpyAsync(d_c, &c, sizeof c, cudaMemcpyHostToDevice, st));
  TRY(ensure_sim(g, B, 1));
  CK(cudaMemsetAsync(g->counters, 0, 2 * sizeof(unsigned long long), st));
  SimArgs a = sim_args(g, B, flags);
  a.mode = 1;
  a.cands = d_c;
  a.n = 1;
  a.out.makespan = d_ms;
  a.out.status = d_st;
  a.snap_mode = 1;
  a.snap_dq = S.dq;
  a.snap_avail = S.avail;
  a.snap_ms = S.ms;
  a.snap_rec = S.rec;
  a.snap_rounds = S.rounds;
  a.snap_used = S.used;  // (memory tracked in the recording run: peak / caps of the lane kernel)
  a.snap_ur = S.ur;
  a.need_mem = 1;
  {
    int grid;
    size_t smem;
    main_shape(g, B, a, grid, smem);
    launch_sim(a, B.tbits, 1, g->sim_block, smem, st);
  }
  g->launches += NL_SIM;
  CK(cudaGetLastError());
  int32_t rd[4];
  uint8_t hst = 0;
  CK(cudaMemcpyAsync(rd, S.rounds, 16, cudaMemcpyDeviceToHost, st));
  CK(cudaMemcpyAsync(&hst, d_st, 1, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  cudaFree(d_c);
  cudaFree(d_ms);
  cudaFree(d_st);
  if (hst != FASTT_CAND_OK) return FASTT_OK;  // an infeasible BASE (caps): no sharing
  if (B.tbits == 32) {
    launch_snap_keys(S.rec, B.n, gshift_of(g->G), S.key, S.key2, S.key4, st);
    CK(cudaGetLastError());
  }
  S.round_dev = (rd[0] == 1 && rd[2] == 0 && rd[3] == B.cp_len) ? rd[1] : -1;
  S.valid = true;
  return FASTT_OK;
}

// enable prefix sharing on a launch when the snapshot exists
static void use_snapshot(const Base &B, uint32_t flags, SimArgs &a) {
  const Base::Snap &S = B.snap[flags & FASTT_F_CP_PIN ? 1 : 0];
  if (!S.valid || a.live_mem || a.out.place || a.ins) return;
  a.snap_mode = 2;
  a.snap_used = S.used;
  a.snap_ur = S.ur;
  a.snap_key = S.key;
  a.snap_key2 = S.key2;
  a.snap_key4 = S.key4;
  a.snap_round_dev = S.round_dev;
  a.snap_dq = S.dq;
  a.snap_avail = S.avail;
  a.snap_ms = S.ms;
  a.snap_rec = S.rec;
}

static fastt_status ensure_sort_buf(fastt_graph *g, int64_t n) {
  if (g->sort_cap >= n) return FASTT_OK;
  cudaFree(g->sort_buf);
  const int64_t c = std::max<int64_t>(n, 4096);
  const size_t oc = 0, oc2 = al16(32 * c), oi = oc2 + al16(32 * c), oi2 = oi + al16(8 * c), ores = oi2 + al16(8 * c),
               ok = ores + al16(8 * c), oh = ok + al16(4 * c), tot = oh + 4096;
  CK(cudaMalloc(&g->sort_buf, tot));
  g->srt_tmp_c = (Cand *)(g->sort_buf + oc);
  g->srt_c = (Cand *)(g->sort_buf + oc2);
  g->srt_tmp_i = (int64_t *)(g->sort_buf + oi);
  g->srt_i = (int64_t *)(g->sort_buf + oi2);
  g->srt_res = (int64_t *)(g->sort_buf + ores);
  g->srt_key = (uint32_t *)(g->sort_buf + ok);
  g->srt_hist = (uint32_t *)(g->sort_buf + oh);
  g->sort_cap = c;
  return FASTT_OK;
}

// Simulation of nc prepared slots (mode 2).  Slots whose priority order is
// topological (the flag the card kernels write into each slot's PrepGraph)
// run the position-order variant, the others the ready-set variant: two
// launches, each skipping the other kind of slot.
static void launch_slots(fastt_graph *g, SimArgs b, int tbits, int nc, cudaStream_t st) {
  b.mode = 2;
  b.stat = nullptr;  // (the step counts are the main launch's)
  const int per_block = (g->sim_block / 32) * g->sim_cpw;
  if (g->use_topo && b.lane && !b.ins) {
    // makespan-only evaluation without memory tracking: the multi-graph lane
    // kernel (one slot per lane, one warp per block) for topological slots
    b.lane = 2;
    b.topo = 1;
    b.slot_filter = 1;
    launch_sim(b, tbits, (nc + 31) / 32, 32, 0, st);
    cudaMemsetAsync(b.counter, 0, sizeof(unsigned long long), st);
    b.lane = 0;
    b.slot_filter = 2;
  } else if (g->use_topo) {
    b.lane = 0;
    b.topo = 1;
    b.slot_filter = 1;
    launch_sim(b, tbits, (int)std::min<int64_t>(g->sim_grid_topo, nc / per_block + 1), g->sim_block, 0, st);
    cudaMemsetAsync(b.counter, 0, sizeof(unsigned long long), st);
    b.slot_filter = 2;
  } else {
    b.lane = 0;
    b.slot_filter = 0;
  }
  b.topo = 0;
  launch_sim(b, tbits, (int)std::min<int64_t>(g->sim_grid, nc / per_block + 1), g->sim_block, g->sim_smem, st);
  g->launches += g->use_topo ? 1 : 0;
}

// ------------------------------------------- device-driven deferral loop
// The candidates a main launch hands to the preparation pipeline (the tail
// of a classified list past the arena, the deferral queue) are evaluated in
// rounds of at most `cap` slots: gather -> preparation -> slot simulations.
// How many rounds run is only known on the device, so the rounds are the
// body of a CUDA-graph WHILE node whose condition k_defer_begin /
// k_defer_plan set (cudaGraphSetConditional): the call enqueues the loop and
// never waits for a count (fastt.h: calls are asynchronous on cuda_stream).
// The instantiated graph depends only on the graph's buffers and the slot
// launches' arguments; per-call values (list length, sources) live in the
// device block dblk, written by k_defer_setup.

static fastt_status ensure_defer(fastt_graph *g) {
  if (g->dblk) return FASTT_OK;
  CK(cudaMalloc(&g->dblk, sizeof(DeferBlock)));
  CK(cudaMemset(g->dblk, 0, sizeof(DeferBlock)));
  CK(cudaMalloc(&g->dwords, 16));
  CK(cudaMemset(g->dwords, 0, 16));
  if (!g->counters2) CK(cudaMalloc(&g->counters2, 2 * sizeof(unsigned long long)));
  CK(cudaStreamCreateWithFlags(&g->st_cap, cudaStreamNonBlocking));
  CK(cudaEventCreateWithFlags(&g->dl_ev, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&g->dl_sum_ev, cudaEventDisableTiming));
  CK(cudaMallocHost(&g->dl_sum, sizeof(DeferBlock)));
  memset(g->dl_sum, 0, sizeof(DeferBlock));
  return FASTT_OK;
}

// destroy retired loop graphs whose last launch has completed (all of them
// when wait: the caller has synchronised the device); only from blocking
// calls: cudaGraphExecDestroy waits for the device
static void reap_defer(fastt_graph *g, bool wait) {
  for (size_t k = 0; k < g->dl_retired.size();) {
    auto &r = g->dl_retired[k];
    if (wait || cudaEventQuery(r.second) == cudaSuccess) {
      cudaGraphExecDestroy(r.first);
      cudaEventDestroy(r.second);
      g->dl_retired[k] = g->dl_retired.back();
      g->dl_retired.pop_back();
    } else {
      k++;
    }
  }
}

// the last loop's summary (pinned copy) once its event completed: the arena
// hint (rank-changing PINs of the last classified list)
static void read_defer_summary(fastt_graph *g) {
  if (!g->dl_sum_pending || cudaEventQuery(g->dl_sum_ev) != cudaSuccess) return;
  g->dl_sum_pending = false;
  if (g->dl_sum->do_tail && g->dl_sum->n_main >= 0) g->pin_defer_hint = g->dl_sum->n - g->dl_sum->n_main;
  else g->seq_defer_hint = g->dl_sum->n_defer;
}

// arena slots of a sequential (non-overlapped) evaluation: the last such
// call's deferral count (one round when the count repeats), at least `lo`
static int64_t seq_arena_want(const fastt_graph *g, int64_t lo) {
  return std::max<int64_t>(std::max<int64_t>(256, lo), std::min<int64_t>(g->seq_defer_hint, ARENA_MAX_SLOTS));
}

static fastt_status build_defer_graph(fastt_graph *g, Base &B, const SimArgs &b, int cap, bool results,
                                      const uint32_t *n_main, const unsigned long long *ndefer,
                                      cudaGraphExec_t *out) {
  cudaStream_t cs = g->st_cap;
  cudaGraph_t gr = nullptr, body = nullptr, tmp = nullptr;
  CK(cudaGraphCreate(&gr, 0));
  cudaGraphConditionalHandle h;
  fastt_status rc = FASTT_OK;
  auto ck = [&](cudaError_t e, const char *what) {
    if (e != cudaSuccess && rc == FASTT_OK) rc = fail(FASTT_ECUDA, "%s: %s", what, cudaGetErrorString(e));
  };
  ck(cudaGraphConditionalHandleCreate(&h, gr, 0, 0), "conditional handle");
  ck(cudaStreamBeginCaptureToGraph(cs, gr, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed), "capture");
  launch_defer_begin(g->dblk, n_main, ndefer, h, cs);
  cudaStreamCaptureStatus cst;
  cudaGraph_t cg = nullptr;
  const cudaGraphNode_t *deps = nullptr;
  size_t nd = 0;
  ck(cudaStreamGetCaptureInfo(cs, &cst, nullptr, &cg, &deps, &nd), "capture info");
  cudaGraphNodeParams cp = {};
  cp.type = cudaGraphNodeTypeConditional;
  cp.conditional.handle = h;
  cp.conditional.type = cudaGraphCondTypeWhile;
  cp.conditional.size = 1;
  cudaGraphNode_t cn = nullptr;
  if (rc == FASTT_OK) ck(cudaGraphAddNode(&cn, cg, deps, nd, &cp), "WHILE node");
  if (rc == FASTT_OK) ck(cudaStreamUpdateCaptureDependencies(cs, &cn, 1, cudaStreamSetCaptureDependencies), "deps");
  ck(cudaStreamEndCapture(cs, &tmp), "end capture");
  host_trace("loop build: WHILE node");
  if (rc == FASTT_OK) {
    body = cp.conditional.phGraph_out[0];
    const int64_t l0 = g->launches;
    ck(cudaStreamBeginCaptureToGraph(cs, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed), "body capture");
    launch_defer_plan(g->dblk, h, cs);
    launch_defer_gather(g->dblk, cap, g->srt_c, g->srt_i, results ? g->srt_res : nullptr, g->defer_q,
                        g->slot_cands, g->slot_index, results ? g->slot_result : nullptr, cs);
    fastt_status pr = run_prep(g, B, cap, cs, &g->dblk->nact);
    if (pr != FASTT_OK && rc == FASTT_OK) rc = pr;
    ck(cudaMemsetAsync(b.counter, 0, sizeof(unsigned long long), cs), "counter reset");
    launch_slots(g, b, B.tbits, cap, cs);
    g->launches += NL_SIM;
    g->dl_round_launches = 2 + (int)(g->launches - l0);
    g->launches = l0;
    ck(cudaGetLastError(), "body launches");
    ck(cudaStreamEndCapture(cs, &tmp), "end body capture");
  }
  host_trace("loop build: captured");
  if (rc == FASTT_OK) ck(cudaGraphInstantiate(out, gr, 0), "instantiate the deferral loop");
  host_trace("loop build: instantiated");
  cudaGraphDestroy(gr);
  return rc;
}

// Evaluate the deferred candidates of a finished main launch (b: the slot
// launches' arguments; src: defer_q entries index the sorted list (0), the
// candidate list cands (1) or the stream (2); do_tail: also the classified
// tail past the arena, positions [*n_main + cap, n) of the sorted list).
static fastt_status run_defer_loop(fastt_graph *g, Base &B, SimArgs b, int cap, int src, bool do_tail, int64_t n,
                                   const Cand *cands, const StreamState *ss, int64_t first, int64_t stride,
                                   bool results, const unsigned long long *ndefer, cudaStream_t st) {
  TRY(ensure_defer(g));
  const uint32_t *n_main = do_tail ? g->ov_words : g->dwords;
  b.slots = g->slot_pgs_dev;
  b.cands = g->slot_cands;
  b.slot_index = results ? nullptr : g->slot_index;
  b.slot_result = results ? g->slot_result : nullptr;
  b.n = cap;
  b.n_dev = &g->dblk->nact;
  b.counter = g->counters2;
  b.lane_batches = 0;
  b.preclassified = 0;
  b.stat = nullptr;
  b.flags &= ~(uint32_t)(FASTT_F_ASYNC | FASTT_F_TIMING | FASTT_F_OUT_DEVICE | FASTT_F_IN_DEVICE);  // (host-side)
  StreamState s0;
  memset(&s0, 0, sizeof s0);
  launch_defer_setup(g->dblk, n, cap, src, do_tail ? 1 : 0, results ? 1 : 0, cands, ss ? *ss : s0, first, stride, st);
  // the loop graph's identity: the slot launches' arguments and every buffer
  // the body touches
  const void *ptrs[] = {g->arena,     g->slot_raws_dev, g->slot_pgs_dev, g->slot_cands, g->slot_index,
                        g->slot_result, g->tmpl_dev,    B.raw_block,     B.raw_dev,     B.prep_block,
                        B.pg_dev,     g->srt_c,         g->srt_i,        g->srt_res,    g->defer_q,
                        n_main,       ndefer,           g->gc_dev};
  const int ints[] = {cap, B.tbits, B.key_bits, (int)B.rl.vcap, g->G, g->K, g->use_topo, g->use_rank_reuse,
                      results, (int)g->sim_block, (int)g->sim_grid, (int)g->sim_grid_topo, (int)g->sim_cpw};
  std::vector<char> key(sizeof b + sizeof ptrs + sizeof ints);
  memcpy(key.data(), &b, sizeof b);
  memcpy(key.data() + sizeof b, ptrs, sizeof ptrs);
  memcpy(key.data() + sizeof b + sizeof ptrs, ints, sizeof ints);
  if (!g->dl_exec || g->dl_key != key) {
    if (getenv("FASTT_HOST_TRACE") && g->dl_key.size() == key.size()) {
      char msg[96];
      for (size_t k = 0; k < key.size(); k++)
        if (key[k] != g->dl_key[k]) {
          snprintf(msg, sizeof msg, "loop: key differs at byte %zu (SimArgs %zu bytes)", k, sizeof b);
          host_trace(msg);
          break;
        }
    }
    if (g->dl_exec) {  // retire: destroyed once its last launch completed
      g->dl_retired.push_back({g->dl_exec, g->dl_ev});
      g->dl_exec = nullptr;
      g->dl_ev = nullptr;
      CK(cudaEventCreateWithFlags(&g->dl_ev, cudaEventDisableTiming));
    }
    TRY(build_defer_graph(g, B, b, cap, results, n_main, ndefer, &g->dl_exec));
    g->dl_key.swap(key);
  }
  host_trace("loop: setup + graph");
  CK(cudaGraphLaunch(g->dl_exec, st));
  host_trace("loop: graph launch");
  CK(cudaEventRecord(g->dl_ev, st));
  g->launches += 2;  // setup + begin (the rounds: fastt_last_timing)
  CK(cudaMemcpyAsync(g->dl_sum, g->dblk, sizeof(DeferBlock), cudaMemcpyDeviceToHost, st));
  CK(cudaEventRecord(g->dl_sum_ev, st));
  g->dl_sum_pending = true;
  g->dl_ran = true;
  return FASTT_OK;
}

// ------------------------------------------------- overlapped evaluation
// A start-step-sorted candidate list classified on the device (launch_t0_sort
// with T0Classify: the candidates that need their own prepared graph sorted
// to the tail, n_main = ov_words[0] the others) is evaluated by two
// concurrent pipelines: the main lane launch over [0, n_main) on the call's
// stream -- non-persistent (each warp takes lane_batches batches and a slab
// slot), so its blocks retire while it runs -- and, on a high-priority
// stream, the gather of the tail into the preparation arena, the
// preparation kernels and the slot simulations (their own slab columns,
// work counter and wbest entries after the main launch's).  The wave is
// sized on the device (nact); a tail longer than the arena, and candidates
// the main launch defers (packed-key bound), run after the join.

static fastt_status ensure_overlap(fastt_graph *g, const Base &B, int cap, int wmain) {
  if (!g->st_prep) {
    int lo = 0, hi = 0;
    CK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
    CK(cudaStreamCreateWithPriority(&g->st_prep, cudaStreamNonBlocking, hi));
    CK(cudaStreamCreateWithFlags(&g->st_main2, cudaStreamNonBlocking));
    for (auto &e : g->ov_ev) CK(cudaEventCreate(&e));
    CK(cudaMalloc(&g->counters2, 2 * sizeof(unsigned long long)));
    CK(cudaMalloc(&g->ov_words, 16));
    CK(cudaMemset(g->ov_words, 0, 16));
  }
  const int64_t cols = (int64_t)cap + 64;
  const size_t rec = B.tbits == 32 ? 8 : 16;
  if (!g->slab_mg || g->slab_mg_cols < cols) {
    cudaFree(g->slab_mg);
    g->slab_mg = nullptr;
    CK(cudaMalloc(&g->slab_mg, (size_t)cols * (size_t)g->sim_ncap * rec));
    g->slab_mg_cols = cols;
  }
  if (g->slot_bm_bits < wmain) {
    cudaFree(g->slot_bm);
    g->slot_bm = nullptr;
    CK(cudaMalloc(&g->slot_bm, sizeof(uint32_t) * (size_t)((wmain + 31) / 32)));
    g->slot_bm_bits = wmain;
  }
  if (g->wbest_cap < wmain + cols) {
    cudaFree(g->wbest);
    g->wbest = nullptr;
    CK(cudaMalloc(&g->wbest, sizeof(int64_t) * 2 * (size_t)(wmain + cols)));
    g->wbest_cap = wmain + cols;
  }
  return FASTT_OK;
}

// resident warps of the main lane launch (its slab slots and wbest entries)
static int lane_warps(const fastt_graph *g, const SimArgs &a) {
  return g->sim_grid_lane[a.lane_mm][1] * g->lane_wpb[a.lane_mm][1];
}

// the overlapped launches after the classified sort (a: the main launch's
// arguments, mode 3 over g->srt_*); results: per-candidate outputs through
// slot_result (schedule_batch) instead of per-warp bests (sweeps)
static fastt_status run_overlapped(fastt_graph *g, Base &B, SimArgs a, int64_t n, uint32_t flags, cudaStream_t st,
                                   bool results, int cap, int wmain) {
  cudaStream_t sp = g->st_prep;
  if (a.track_best) launch_init_best(g->wbest, (int64_t)wmain + cap + 64, st);
  CK(cudaMemsetAsync(g->slot_bm, 0, sizeof(uint32_t) * (size_t)((wmain + 31) / 32), st));
  CK(cudaMemsetAsync(g->counters2, 0, 2 * sizeof(unsigned long long), st));
  CK(cudaEventRecord(g->ov_ev[0], st));
  // preparation pipeline + slot simulations (high priority)
  CK(cudaStreamWaitEvent(sp, g->ov_ev[0], 0));
  if (flags & FASTT_F_TIMING) CK(cudaEventRecord(g->ov_ev[1], sp));
  launch_gather_tail(g->srt_c, g->srt_i, results ? g->srt_res : nullptr, g->ov_words, n, 0, cap, g->slot_cands,
                     g->slot_index, results ? g->slot_result : nullptr, g->ov_words + 1, sp);
  g->launches += NL_GATHER;
  TRY(run_prep(g, B, cap, sp, g->ov_words + 1));
  if (g->ovl_mode >= 1) CK(cudaEventRecord(g->ov_ev[3], sp));  // (prepared: the main launch may start)
  SimArgs b = a;
  b.slots = g->slot_pgs_dev;
  b.cands = g->slot_cands;
  b.slot_index = results ? nullptr : g->slot_index;
  b.slot_result = results ? g->slot_result : nullptr;
  b.n = cap;
  b.n_dev = g->ov_words + 1;
  b.counter = g->counters2;
  b.ndefer = g->counters2 + 1;
  b.wbest = g->wbest + 2 * (int64_t)wmain;
  b.slab = g->slab_mg;
  b.lane_batches = 0;
  b.preclassified = 0;
  b.stat = nullptr;
  launch_slots(g, b, B.tbits, cap, sp);
  g->launches += NL_SIM;
  CK(cudaGetLastError());
  host_trace("overlap: prep stream launches");
  CK(cudaEventRecord(g->ov_ev[2], sp));
  // the main launch (the call's stream)
  a.preclassified = 1;
  a.n_dev = g->ov_words;
  a.lane_batches = g->lane_batches;
  a.slot_bm = g->slot_bm;
  a.n_slab_slots = wmain;
  int64_t blocks;
  if (g->lane_batches > 0) {
    const int64_t rw = 32 * (int64_t)std::max(1, a.pk_cpl);  // candidates per warp batch
    const int64_t warps = (n + rw - 1) / rw;
    const int64_t wpb = std::max(1, a.pk_wpb);
    blocks = (warps + (int64_t)g->lane_batches * wpb - 1) / ((int64_t)g->lane_batches * wpb);
  } else {  // persistent, optionally leaving block slots to the preparation stream
    blocks = wmain / std::max(1, a.pk_wpb);
    if (g->main_bps > 0 && g->ovl_mode != 2) blocks = std::min<int64_t>(blocks, (int64_t)g->sms * g->main_bps);
  }
  if (g->ovl_mode == 2 && g->lane_batches == 0) {
    // two persistent launches on one work queue: main_bps blocks per SM at
    // once (beside the preparation kernels), the rest of the resident
    // blocks once the preparation kernels are done (their own slab columns
    // and wbest entries: gwarp_off)
    const int64_t ba = std::min<int64_t>(blocks, (int64_t)g->sms * std::max(1, g->main_bps));
    a.gwarp_off = 0;
    launch_sim(a, B.tbits, (int)std::max<int64_t>(1, ba), LANE_BLOCK, 0, st);
    if (blocks > ba) {
      CK(cudaStreamWaitEvent(g->st_main2, g->ov_ev[3], 0));
      SimArgs a2 = a;
      a2.gwarp_off = (int32_t)(ba * std::max(1, a.pk_wpb));
      launch_sim(a2, B.tbits, (int)(blocks - ba), LANE_BLOCK, 0, g->st_main2);
      CK(cudaEventRecord(g->ov_ev[4], g->st_main2));
      CK(cudaStreamWaitEvent(st, g->ov_ev[4], 0));
      g->launches += NL_SIM;
    }
  } else {
    if (g->ovl_mode == 1) {
      CK(cudaStreamWaitEvent(st, g->ov_ev[3], 0));
      if (flags & FASTT_F_TIMING) {  // ms_sim: the main launch's own duration
        CK(cudaEventRecord(g->ev_main, st));
        g->ev_main_rec = true;
      }
    }
    launch_sim(a, B.tbits, (int)std::max<int64_t>(1, std::min<int64_t>(blocks, 1 << 30)), LANE_BLOCK, 0, st);
  }
  g->launches += NL_SIM;
  CK(cudaGetLastError());
  timing_mark(g, flags, 1, st);
  CK(cudaStreamWaitEvent(st, g->ov_ev[2], 0));
  return FASTT_OK;
}

// after the join: a tail longer than the arena and the main launch's
// packed-key deferrals, sequentially on st (the device-driven loop)
static fastt_status finish_overlapped(fastt_graph *g, Base &B, SimArgs a, int64_t n, cudaStream_t st, bool results,
                                      int cap, int wmain) {
  SimArgs b = a;
  b.wbest = g->wbest + 2 * (int64_t)wmain;
  b.slab = g->slab_mg;
  b.n_dev = nullptr;
  return run_defer_loop(g, B, b, cap, 0, true, n, nullptr, nullptr, 0, 1, results, g->counters + 1, st);
}

struct DevOut {
  int64_t *makespan = nullptr;
  uint8_t *status = nullptr;
  int64_t *peak = nullptr;
  uint8_t *place = nullptr;
  int64_t *start = nullptr;
  int32_t *deq = nullptr;
  int32_t *order = nullptr;
  int64_t vmax = 0;
};

// DPOS of n candidates (device array) on base B.  Outputs: device pointers.
static fastt_status eval_batch(fastt_graph *g, Base &B, const Cand *d_cands, int64_t n, uint32_t flags,
                               cudaStream_t st, DevOut o) {
  if (n <= 0) return FASTT_OK;
  TRY(ensure_sim(g, B, n, flags));
  const bool sharing =
      g->share && !o.place && n >= 64 && !(flags & (FASTT_F_POLICY_INSERT | FASTT_F_MEM_LIVE));
  if (sharing) TRY(ensure_snapshot(g, B, flags, st));  // before the work counters are reset
  if (o.place) CK(cudaMemsetAsync(o.place, 0xFF, (size_t)n * o.vmax, st));
  if (o.start) {
    launch_fill_i64(o.start, n * o.vmax, -1, st);
    g->launches += NL_FILL;
  }
  if (o.deq) CK(cudaMemsetAsync(o.deq, 0xFF, (size_t)n * o.vmax * 4, st));
  CK(cudaMemsetAsync(g->counters, 0, 2 * sizeof(unsigned long long), st));
  SimArgs a = sim_args(g, B, flags);
  a.mode = 1;
  a.cands = d_cands;
  a.n = n;
  a.out.makespan = o.makespan;
  a.out.status = o.status;
  a.out.peak = o.peak;
  if (o.peak) a.need_mem = 1;
  a.out.place = o.place;
  a.out.start = o.start;
  a.out.deq = o.deq;
  a.out.vmax = (int32_t)o.vmax;
  if (sharing) use_snapshot(B, flags, a);
  const bool sorted = a.snap_mode == 2;
  // the overlapped path (see run_overlapped): packed-key lane kernel, no per-op outputs
  bool ovl = false;
  if (sorted && g->use_overlap && a.pkc && a.costk && a.pk_lim > 0 && !o.place && !o.start && !o.deq) {
    SimArgs t = a;
    int gr;
    size_t sm;
    main_shape(g, B, t, gr, sm);
    ovl = t.lane == 1;
  }
  if (ovl) {
    TRY(ensure_arena(g, B, st, std::max<int64_t>(256, std::min<int64_t>(g->pin_defer_hint, ARENA_MAX_SLOTS))));
    const int cap = g->arena_slots;
    int wmain;
    {
      SimArgs t = a;
      int gr;
      size_t sm;
      main_shape(g, B, t, gr, sm);
      wmain = lane_warps(g, t);
    }
    TRY(ensure_overlap(g, B, cap, wmain));
    TRY(ensure_sort_buf(g, n));
    const PrepGraph P = prep_struct(B.prep_block, B.pl, B.tbits);
    StreamState dummy;
    memset(&dummy, 0, sizeof dummy);
    T0Classify cl{1, B.tbits, B.pg_dev, g->gc_dev, a.split_mask, g->ov_words};
    launch_t0_sort(0, dummy, 0, 1, d_cands, n, P.pos, a.snap_dq, B.n, B.V, g->G, g->srt_tmp_c, g->srt_tmp_i,
                   g->srt_key, g->srt_hist, g->srt_c, g->srt_i, g->srt_res, st, cl);
    g->launches += 4;
    a.mode = 3;
    a.cands = g->srt_c;
    a.slot_index = g->srt_i;
    a.slot_result = g->srt_res;
    {
      int gr;
      size_t sm;
      main_shape(g, B, a, gr, sm);
    }
    TRY(run_overlapped(g, B, a, n, flags, st, true, cap, wmain));
    timing_mark(g, flags, 2, st);
    TRY(finish_overlapped(g, B, a, n, st, true, cap, wmain));
    if (!(flags & FASTT_F_ASYNC)) CK(cudaStreamSynchronize(st));
    return FASTT_OK;
  }
  // the arena of the deferral rounds (sized before the launch: the count is
  // only known on the device)
  TRY(ensure_arena(g, B, st, seq_arena_want(g, 0)));
  if (sorted) {
    // order the list by BASE-prefix start step (results keep their index)
    TRY(ensure_sort_buf(g, n));
    const PrepGraph P = prep_struct(B.prep_block, B.pl, B.tbits);
    StreamState dummy;
    memset(&dummy, 0, sizeof dummy);
    launch_t0_sort(0, dummy, 0, 1, d_cands, n, P.pos, a.snap_dq, B.n, B.V, g->G, g->srt_tmp_c, g->srt_tmp_i,
                   g->srt_key, g->srt_hist, g->srt_c, g->srt_i, g->srt_res, st);
    g->launches += 4;
    a.mode = 3;
    a.cands = g->srt_c;
    a.slot_index = g->srt_i;
    a.slot_result = g->srt_res;
  }
  {
    int grid;
    size_t smem;
    main_shape(g, B, a, grid, smem);
    launch_sim(a, B.tbits, grid, g->sim_block, smem, st);
  }
  g->launches += NL_SIM;
  CK(cudaGetLastError());
  timing_mark(g, flags, 1, st);
  TRY(run_defer_loop(g, B, a, g->arena_slots, sorted ? 0 : 1, false, n, d_cands, nullptr, 0, 1, true,
                     g->counters + 1, st));
  timing_mark(g, flags, 2, st);
  if (o.order) {
    // execution order list A (R17): per-result stable sort of the dequeue
    // list by start, 256 results per launch (stream-ordered scratch)
    const int64_t chunk = 256;
    uint64_t *k0 = nullptr, *k1 = nullptr;
    uint32_t *v0 = nullptr, *v1 = nullptr;
    int64_t *d_idx = nullptr;
    CK(cudaMallocAsync(&k0, (size_t)chunk * o.vmax * 8, st));
    CK(cudaMallocAsync(&k1, (size_t)chunk * o.vmax * 8, st));
    CK(cudaMallocAsync(&v0, (size_t)chunk * o.vmax * 4, st));
    CK(cudaMallocAsync(&v1, (size_t)chunk * o.vmax * 4, st));
    CK(cudaMallocAsync(&d_idx, sizeof(int64_t) * n, st));
    launch_iota_i64(d_idx, n, st);
    for (int64_t c0 = 0; c0 < n; c0 += chunk) {
      const int64_t nc = std::min(chunk, n - c0);
      launch_order_chunk(o.deq, o.start, o.order, d_idx + c0, nc, o.vmax, B.key_bits, k0, k1, v0, v1, st);
      g->launches += NL_ORDER;
    }
    CK(cudaFreeAsync(k0, st));
    CK(cudaFreeAsync(k1, st));
    CK(cudaFreeAsync(v0, st));
    CK(cudaFreeAsync(v1, st));
    CK(cudaFreeAsync(d_idx, st));
  }
  if (!(flags & FASTT_F_ASYNC)) CK(cudaStreamSynchronize(st));
  return FASTT_OK;
}

// ----------------------------------------------------------------- stream

static int split_counts(int G, int pow2, int *ns) {
  int c = 0;
  for (int n = 2; n <= G; n++)
    if (!pow2 || (n & (n - 1)) == 0) ns[c++] = n;
  return c;
}

// split-eligible placement-aware CP of a placement (Alg. 2 lines 4-5) -> host list
static fastt_status split_list(fastt_graph *g, Base &B, const uint8_t *d_place, std::vector<int32_t> &out,
                               cudaStream_t st) {
  if (!g->scratch_rank) {
    CK(cudaMalloc(&g->scratch_n, 16));
  }
  cudaFree(g->scratch_rank);
  cudaFree(g->scratch_cp);
  cudaFree(g->scratch_list);
  CK(cudaMalloc(&g->scratch_rank, sizeof(int64_t) * (B.V + 1)));
  CK(cudaMalloc(&g->scratch_cp, sizeof(int32_t) * (B.V + 1)));
  CK(cudaMalloc(&g->scratch_list, sizeof(int32_t) * (B.V + 1)));
  launch_splitlist(B.raw_dev, g->gc_dev, d_place, g->scratch_list, g->scratch_n, g->scratch_rank, g->scratch_cp,
                   g->G, st);
  CK(cudaGetLastError());
  int32_t m = 0;
  CK(cudaMemcpyAsync(&m, g->scratch_n, 4, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  out.resize(m);
  if (m) CK(cudaMemcpy(out.data(), g->scratch_list, sizeof(int32_t) * m, cudaMemcpyDeviceToHost));
  return FASTT_OK;
}

static fastt_status ensure_stream(fastt_graph *g, uint32_t flags, int pow2, cudaStream_t st, StreamCache **out) {
  int key = (int)(flags & FASTT_F_CP_PIN) | (pow2 ? 2 : 0) | (flags & FASTT_F_POLICY_INSERT ? 4 : 0) |
            (flags & FASTT_F_MEM_LIVE ? 8 : 0);
  StreamCache &S = g->streams[key];
  *out = &S;
  if (S.valid) return FASTT_OK;
  Base &B = g->base;
  const int64_t vm = B.rl.vcap;
  // one DPOS run of BASE (R21)
  Cand c;
  memset(&c, 0, sizeof c);
  c.split_op = -1;
  for (int k = 0; k < 4; k++) c.pin_op[k] = -1;
  Cand *d_c;
  int64_t *d_ms;
  uint8_t *d_st;
  CK(cudaMalloc(&d_c, sizeof c));
  CK(cudaMalloc(&d_ms, 8));
  CK(cudaMalloc(&d_st, 1));
  CK(cudaMalloc(&S.base_place, vm));
  CK(cudaMemcpyAsync(d_c, &c, sizeof c, cudaMemcpyHostToDevice, st));
  DevOut o;
  o.makespan = d_ms;
  o.status = d_st;
  o.place = S.base_place;
  o.vmax = vm;
  TRY(eval_batch(g, B, d_c, 1, flags & ~FASTT_F_ASYNC, st, o));  // (one-time setup: blocking)
  uint8_t hst = 0;
  CK(cudaMemcpy(&hst, d_st, 1, cudaMemcpyDeviceToHost));
  std::vector<int32_t> list;
  if (hst != FASTT_CAND_OK) {
    CK(cudaMemsetAsync(S.base_place, 0, vm, st));
  } else {
    TRY(split_list(g, B, S.base_place, list, st));
  }
  cudaFree(d_c);
  cudaFree(d_ms);
  cudaFree(d_st);
  int ns[MAXG];
  int nns = split_counts(g->G, pow2, ns);
  std::vector<int32_t> so;
  std::vector<uint8_t> sd, sn;
  for (int32_t op : list)
    for (int dim = 0; dim < 2; dim++) {
      if (!(g->split_mask_h[op] & (1u << dim))) continue;
      for (int q = 0; q < nns; q++) {
        so.push_back(op);
        sd.push_back((uint8_t)dim);
        sn.push_back((uint8_t)ns[q]);
      }
    }
  S.n_split = (int64_t)so.size();
  CK(cudaMalloc(&S.split_op, sizeof(int32_t) * (so.size() + 1)));
  CK(cudaMalloc(&S.split_dim, so.size() + 1));
  CK(cudaMalloc(&S.split_n, so.size() + 1));
  if (!so.empty()) {
    CK(cudaMemcpy(S.split_op, so.data(), sizeof(int32_t) * so.size(), cudaMemcpyHostToDevice));
    CK(cudaMemcpy(S.split_dim, sd.data(), sd.size(), cudaMemcpyHostToDevice));
    CK(cudaMemcpy(S.split_n, sn.data(), sn.size(), cudaMemcpyHostToDevice));
  }
  std::vector<int32_t> live(g->V);
  for (int32_t i = 0; i < g->V; i++) live[i] = i;
  S.n_live = g->V;
  CK(cudaMalloc(&S.live, sizeof(int32_t) * (g->V + 1)));
  if (g->V) CK(cudaMemcpy(S.live, live.data(), sizeof(int32_t) * g->V, cudaMemcpyHostToDevice));
  S.valid = true;
  return FASTT_OK;
}

static StreamState stream_state(const fastt_graph *g, const StreamCache &S, const fastt_gen_params *gp) {
  StreamState s;
  s.base_place = S.base_place;
  s.live = S.live;
  s.n_live = S.n_live;
  s.n_split = S.n_split;
  s.split_op = S.split_op;
  s.split_dim = S.split_dim;
  s.split_n = S.split_n;
  s.seed = gp->seed;
  s.kmin = gp->pin_k_min;
  s.kmax = gp->pin_k_max;
  s.G = g->G;
  s.n_subset = gp->subset_prefixes ? g->G - 1 : 0;
  return s;
}

static fastt_status check_gen(const fastt_graph *g, const StreamCache &S, const fastt_gen_params *gp, int64_t first,
                              int64_t n, int64_t stride) {
  if (!gp) return fail(FASTT_EINVAL, "gen params are NULL");
  if (gp->pin_k_min < 1 || gp->pin_k_max > 4 || gp->pin_k_min > gp->pin_k_max)
    return fail(FASTT_EINVAL, "need 1 <= pin_k_min <= pin_k_max <= 4");
  if (first < 0 || n < 0 || stride < 1) return fail(FASTT_EINVAL, "need first >= 0, n >= 0, stride >= 1");
  if (gp->subset_prefixes > 1) return fail(FASTT_EINVAL, "subset_prefixes must be 0 or 1");
  if (n > 0 && (g->G == 1 || S.n_live == 0) &&
      first + (n - 1) * stride > S.n_split + (gp->subset_prefixes ? g->G - 1 : 0))
    return fail(FASTT_EINVAL, "the stream has no PIN candidates (G == 1 or no ops)");
  return FASTT_OK;
}

// =================================================================== ABI

extern "C" {

const char *fastt_last_error(void) { return g_err.c_str(); }
const char *fastt_version(void) { return "fastt-b200 0.1 (sm_100a)"; }

fastt_status fastt_load_graph(const fastt_graph_desc *d, int cuda_device, fastt_graph **out) {
  g_err.clear();
  if (!d || !out) return fail(FASTT_EINVAL, "NULL argument");
  *out = nullptr;
  const int32_t V = d->n_ops, G = d->n_devices, K = d->n_link_classes;
  if (V < 0) return fail(FASTT_EINVAL, "n_ops < 0");
  if (G < 1 || G > MAXG) return fail(FASTT_EINVAL, "n_devices must be 1..32");
  if (K < 1 || K > MAXK) return fail(FASTT_EINVAL, "n_link_classes must be 1..16");
  if (!d->succ_off || !d->dev_mem_cap || !d->link_class || !d->link_alpha_ns || !d->link_beta_fs_per_byte)
    return fail(FASTT_EINVAL, "NULL array");
  if (V > 0 && (!d->cost_ns || !d->mem_bytes || !d->param_bytes || !d->split_mask))
    return fail(FASTT_EINVAL, "NULL per-op array");
  if (d->succ_off[0] != 0) return fail(FASTT_EINVAL, "succ_off[0] != 0");
  for (int32_t i = 0; i < V; i++)
    if (d->succ_off[i + 1] < d->succ_off[i]) return fail(FASTT_EINVAL, "succ_off not monotone at %d", i);
  const int64_t E = d->succ_off[V];
  if (E > 0 && (!d->succ_dst || !d->edge_bytes || !d->edge_param)) return fail(FASTT_EINVAL, "NULL edge array");
  if (d->split_copy_fs_per_byte < 0) return fail(FASTT_EINVAL, "split_copy_fs_per_byte < 0");
  for (int32_t k = 0; k < K; k++)
    if (d->link_alpha_ns[k] < 0 || d->link_beta_fs_per_byte[k] < 0) return fail(FASTT_EINVAL, "negative link model");
  for (int32_t q = 0; q < G * G; q++)
    if (d->link_class[q] >= K) return fail(FASTT_EINVAL, "link_class out of range");
  for (int32_t q = 0; q < G; q++)
    if (d->dev_mem_cap[q] < 0) return fail(FASTT_EINVAL, "negative memory cap");
  for (int64_t q = 0; q < (int64_t)V * G; q++)
    if (d->cost_ns[q] < 0) return fail(FASTT_EINVAL, "negative cost");
  for (int32_t i = 0; i < V; i++)
    if (d->mem_bytes[i] < 0 || d->param_bytes[i] < 0 || d->param_bytes[i] > d->mem_bytes[i])
      return fail(FASTT_EINVAL, "need 0 <= param_bytes <= mem_bytes (op %d)", i);
  // edges: validate, merge parallel edges (R11), sort both adjacency lists
  struct Ed { int32_t s, t; int64_t b; uint8_t p; };
  std::vector<Ed> ed;
  ed.reserve(E);
  for (int32_t i = 0; i < V; i++)
    for (int64_t e = d->succ_off[i]; e < d->succ_off[i + 1]; e++) {
      int32_t t = d->succ_dst[e];
      if (t < 0 || t >= V) return fail(FASTT_EINVAL, "edge destination out of range");
      if (t == i) return fail(FASTT_ECYCLE, "self loop at op %d", i);
      if (d->edge_bytes[e] < 0) return fail(FASTT_EINVAL, "negative edge bytes");
      ed.push_back({i, t, d->edge_bytes[e], (uint8_t)(d->edge_param[e] ? 1 : 0)});
    }
  std::sort(ed.begin(), ed.end(), [](const Ed &a, const Ed &b) { return a.s != b.s ? a.s < b.s : a.t < b.t; });
  size_t m = 0;
  for (size_t e = 0; e < ed.size(); e++) {
    if (m > 0 && ed[m - 1].s == ed[e].s && ed[m - 1].t == ed[e].t) {
      if (ed[m - 1].b > INT64_MAX / 4 - ed[e].b) return fail(FASTT_ERANGE, "merged edge bytes overflow");
      ed[m - 1].b += ed[e].b;
      ed[m - 1].p |= ed[e].p;
    } else {
      ed[m++] = ed[e];
    }
  }
  ed.resize(m);
  const int64_t Em = (int64_t)m;
  for (auto &x : ed)
    for (int k = 0; k < K; k++)
      if (d->link_beta_fs_per_byte[k] && x.b > (INT64_MAX / 4) / d->link_beta_fs_per_byte[k])
        return fail(FASTT_ERANGE, "bytes * beta overflows int64");
  for (auto &x : ed)
    if (d->split_copy_fs_per_byte && x.b > (INT64_MAX / 4) / d->split_copy_fs_per_byte)
      return fail(FASTT_ERANGE, "bytes * split_copy_fs_per_byte overflows int64");
  std::vector<uint32_t> so(V), sc(V, 0), po(V), pc(V, 0);
  std::vector<int32_t> sdst(Em), psrc(Em);
  std::vector<int64_t> sb(Em), pb(Em);
  std::vector<uint8_t> sp(Em), pp(Em);
  for (auto &x : ed) sc[x.s]++, pc[x.t]++;
  {
    uint32_t a = 0, b = 0;
    for (int32_t i = 0; i < V; i++) {
      so[i] = a;
      a += sc[i];
      po[i] = b;
      b += pc[i];
    }
  }
  {
    std::vector<uint32_t> fs(so), fp(po);
    for (auto &x : ed) {  // ed sorted by (s, t): succ lists ascending
      uint32_t q = fs[x.s]++;
      sdst[q] = x.t;
      sb[q] = x.b;
      sp[q] = x.p;
    }
    std::vector<Ed> byt(ed);
    std::sort(byt.begin(), byt.end(), [](const Ed &a, const Ed &b) { return a.t != b.t ? a.t < b.t : a.s < b.s; });
    for (auto &x : byt) {
      uint32_t q = fp[x.t]++;
      psrc[q] = x.s;
      pb[q] = x.b;
      pp[q] = x.p;
    }
  }
  int32_t maxdeg = 0, maxP = 0, maxS = 0, maxov = 0;
  for (int32_t i = 0; i < V; i++) {
    maxdeg = std::max<int32_t>(maxdeg, (int32_t)std::max(sc[i], pc[i]));
    if (d->split_mask[i]) {
      maxov = std::max<int32_t>(maxov, (int32_t)(pc[i] + G + sc[i]));
      maxP = std::max<int32_t>(maxP, (int32_t)pc[i]);
      maxS = std::max<int32_t>(maxS, (int32_t)sc[i]);
    }
  }
  if (maxdeg >= 65535) return fail(FASTT_EUNSUP, "an op has >= 65535 neighbours");
  // Kahn: acyclicity and a topological order
  std::vector<int32_t> topo;
  topo.reserve(V);
  {
    std::vector<uint32_t> deg(pc);
    for (int32_t i = 0; i < V; i++)
      if (deg[i] == 0) topo.push_back(i);
    for (size_t h = 0; h < topo.size(); h++) {
      int32_t i = topo[h];
      for (uint32_t q = so[i]; q < so[i] + sc[i]; q++)
        if (--deg[sdst[q]] == 0) topo.push_back(sdst[q]);
    }
    if ((int32_t)topo.size() != V) return fail(FASTT_ECYCLE, "the graph has a cycle (R22)");
  }
  // link-class masks and the int64 guard (same rule as the oracle's loader)
  GraphConst gc;
  memset(&gc, 0, sizeof gc);
  gc.G = G;
  gc.K = K;
  gc.copy_fs = d->split_copy_fs_per_byte;
  for (int q = 0; q < G; q++) gc.cap[q] = d->dev_mem_cap[q];
  for (int k = 0; k < K; k++) {
    gc.alpha[k] = d->link_alpha_ns[k];
    gc.beta[k] = d->link_beta_fs_per_byte[k];
  }
  for (int s = 0; s < G; s++)
    for (int t = 0; t < G; t++) {
      gc.link_class[s * G + t] = d->link_class[s * G + t];
      if (s != t) {
        uint32_t bit = 1u << d->link_class[s * G + t];
        gc.offdiag_mask |= bit;
        gc.row_mask[s] |= bit;
        gc.col_mask[t] |= bit;
      }
    }
  {
    __int128 tot = 0, totm = 0;
    for (int32_t i = 0; i < V; i++) {
      int64_t mx = 0;
      for (int q = 0; q < G; q++) mx = std::max(mx, d->cost_ns[(int64_t)i * G + q]);
      tot += mx + G;
      totm += (__int128)d->mem_bytes[i] * (G + 1);
    }
    for (auto &x : ed) {
      int64_t mx = 0;
      for (int k = 0; k < K; k++) mx = std::max(mx, comm_class(gc, x.b, k));
      int64_t cc = gc.copy_fs ? ceil_div64(x.b * gc.copy_fs, 1000000) : 0;
      tot += (__int128)(mx + cc) * (G + 2);
    }
    if (tot >= ((__int128)1 << 58) || totm >= ((__int128)1 << 60))
      return fail(FASTT_ERANGE, "costs/bytes exceed the int64 envelope");
  }
  fastt_graph *g = new (std::nothrow) fastt_graph();
  if (!g) return fail(FASTT_ENOMEM, "host allocation");
  g->dev = cuda_device;
  g->V = V;
  g->G = G;
  g->K = K;
  g->E = Em;
  g->maxP = maxP;
  g->maxS = maxS;
  g->v_max = V + maxov;
  g->gch = gc;
  g->split_mask_h.assign(d->split_mask, d->split_mask + V);
  {
    const char *e = getenv("FASTT_NO_SHARE");
    g->share = !(e && e[0] == '1');
    e = getenv("FASTT_NO_TOPO");
    g->use_topo = !(e && e[0] == '1');
    e = getenv("FASTT_NO_LANE");
    g->use_lane = !(e && e[0] == '1');
    e = getenv("FASTT_NO_RANK_REUSE");
    g->use_rank_reuse = !(e && e[0] == '1');
    e = getenv("FASTT_NO_COST_HOLE");
    g->use_cost_hole = !(e && e[0] == '1');
    e = getenv("FASTT_NO_LVLREC");
    g->use_lvlrec = !(e && e[0] == '1');
    e = getenv("FASTT_NO_PK");
    g->use_pk = !(e && e[0] == '1');
    e = getenv("FASTT_NO_PK_TMA");
    g->use_pk_tma = !(e && e[0] == '1');
    e = getenv("FASTT_LANE_INS");
    g->use_lane_ins = e && e[0] == '1';
    e = getenv("FASTT_INS_CAP");
    if (e && e[0]) g->ins_cap_env = std::max(1ll, atoll(e));
    e = getenv("FASTT_NO_OVERLAP");
    g->use_overlap = !(e && e[0] == '1');
    e = getenv("FASTT_LANE_BATCHES");
    if (e && e[0]) g->lane_batches = std::max(0, atoi(e));
    e = getenv("FASTT_MAIN_BPS");
    if (e && e[0]) g->main_bps = std::max(0, atoi(e));
    e = getenv("FASTT_PK_WPB");
    if (e && e[0]) g->pk_wpb_env = (atoi(e) == 1 || atoi(e) == 2) ? atoi(e) : 4;
    e = getenv("FASTT_PK_CPL_PEAK");
    if (e && e[0]) g->pk_cpl_peak = e[0] == '1';
    e = getenv("FASTT_OVL_MODE");
    if (e && e[0]) g->ovl_mode = atoi(e);
    e = getenv("FASTT_PK_CPL");
    if (e && e[0]) g->pk_cpl = atoi(e) == 1 ? 1 : atoi(e) == 4 ? 4 : 2;
    e = getenv("FASTT_PK_LIM");
    if (e && e[0]) g->pk_lim_cap = (uint32_t)std::max(1ll, std::min(0xFFFFFFFFll, atoll(e)));
  }
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || cuda_device < 0 || cuda_device >= ndev) {
    delete g;
    return fail(FASTT_ECUDA, "no CUDA device %d", cuda_device);
  }
  Dev guard(cuda_device);
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, cuda_device);
  g->sms = sms > 0 ? sms : 148;
  const int64_t vcap = (int64_t)V + overlay_v(g);
  const int64_t ecap = Em + overlay_e(g);
  // positions are 24-bit in the lane kernels' CP rounds and the group
  // kernel's records; the ready-set kernel's 3-level bitmap covers 32768
  // positions, so larger graphs need a topological priority order (checked
  // after the base is prepared)
  if (vcap > MAX_VCAP) {
    delete g;
    return fail(FASTT_EUNSUP, "graphs above %d ops (+ split overlay) are not supported (V=%d)", MAX_VCAP, V);
  }
  Base &B = g->base;
  B.V = V;
  B.n_live = V;
  B.E = Em;
  B.rl = raw_layout(vcap, ecap, G);
  // host image of the raw block, one H2D copy
  std::vector<char> img(B.rl.total, 0);
  auto put = [&](int k, const void *src, size_t bytes) {
    if (bytes) memcpy(img.data() + B.rl.o[k], src, bytes);
  };
  put(0, so.data(), 4 * (size_t)V);
  put(1, sc.data(), 4 * (size_t)V);
  put(2, po.data(), 4 * (size_t)V);
  put(3, pc.data(), 4 * (size_t)V);
  put(4, sdst.data(), 4 * (size_t)Em);
  put(5, psrc.data(), 4 * (size_t)Em);
  put(6, sb.data(), 8 * (size_t)Em);
  put(7, pb.data(), 8 * (size_t)Em);
  put(8, sp.data(), (size_t)Em);
  put(9, pp.data(), (size_t)Em);
  put(10, d->cost_ns, 8 * (size_t)V * G);
  put(11, d->mem_bytes, 8 * (size_t)V);
  put(12, d->param_bytes, 8 * (size_t)V);
  put(13, d->split_mask, (size_t)V);
  {
    std::vector<uint8_t> alive(V, 1);
    put(14, alive.data(), (size_t)V);
  }
  put(15, topo.data(), 4 * (size_t)V);
  cudaStream_t st = 0;
  fastt_status rc = FASTT_OK;
  do {
    if (cudaMalloc(&g->gc_dev, sizeof gc) != cudaSuccess || cudaMalloc(&B.raw_block, B.rl.total) != cudaSuccess ||
        cudaMalloc(&B.raw_dev, sizeof(RawGraph)) != cudaSuccess) {
      rc = fail(FASTT_ENOMEM, "device allocation for the graph");
      break;
    }
    RawGraph R = raw_struct(B.raw_block, B.rl, V, V, Em);
    if (cudaMemcpy(g->gc_dev, &gc, sizeof gc, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemcpy(B.raw_block, img.data(), B.rl.total, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemcpy(B.raw_dev, &R, sizeof R, cudaMemcpyHostToDevice) != cudaSuccess) {
      rc = fail(FASTT_ECUDA, "upload: %s", cudaGetErrorString(cudaGetLastError()));
      break;
    }
    rc = prepare_base(g, B, st);
  } while (0);
  if (rc != FASTT_OK) {
    fastt_free_graph(g);
    return rc;
  }
  *out = g;
  return FASTT_OK;
}

void fastt_free_graph(fastt_graph *g) {
  if (!g) return;
  {
    Dev guard(g->dev);
    cudaDeviceSynchronize();  // (in-flight asynchronous calls)
    g->base.release();
    for (auto &s : g->streams) s.release();
    cudaFree(g->gc_dev);
    cudaFree(g->arena);
    cudaFree(g->tmpl_dev);
    cudaFree(g->slot_raws_dev);
    cudaFree(g->slot_pgs_dev);
    cudaFree(g->slot_cands);
    cudaFree(g->slot_result);
    cudaFree(g->slot_index);
    cudaFree(g->slab);
    cudaFree(g->gap);
    cudaFree(g->gap_lane);
    cudaFree(g->wbest);
    cudaFree(g->best_dev);
    cudaFree(g->counters);
    cudaFree(g->defer_q);
    cudaFree(g->scratch_rank);
    cudaFree(g->scratch_cp);
    cudaFree(g->scratch_list);
    cudaFree(g->scratch_n);
    cudaFree(g->sort_buf);
    for (auto &b : g->io) cudaFree(b.p);
    for (auto &e : g->ev)
      if (e) cudaEventDestroy(e);
    for (auto &e : g->ov_ev)
      if (e) cudaEventDestroy(e);
    if (g->ev_main) cudaEventDestroy(g->ev_main);
    if (g->st_prep) cudaStreamDestroy(g->st_prep);
    if (g->st_main2) cudaStreamDestroy(g->st_main2);
    cudaFree(g->slab_mg);
    cudaFree(g->counters2);
    cudaFree(g->ov_words);
    cudaFree(g->slot_bm);
    reap_defer(g, true);
    if (g->dl_exec) cudaGraphExecDestroy(g->dl_exec);
    if (g->dl_ev) cudaEventDestroy(g->dl_ev);
    if (g->dl_sum_ev) cudaEventDestroy(g->dl_sum_ev);
    if (g->done_ev) cudaEventDestroy(g->done_ev);
    if (g->st_cap) cudaStreamDestroy(g->st_cap);
    cudaFreeHost(g->dl_sum);
    cudaFree(g->dblk);
    cudaFree(g->dwords);
  }
  delete g;
}

fastt_status fastt_graph_info(const fastt_graph *g, int32_t *n_ops, int32_t *v_max, int32_t *cp_len,
                              int32_t *time_bits) {
  if (!g) return fail(FASTT_EINVAL, "NULL graph");
  if (n_ops) *n_ops = g->V;
  if (v_max) *v_max = g->v_max;
  if (cp_len) *cp_len = g->base.cp_len;
  if (time_bits) *time_bits = g->base.tbits;
  return FASTT_OK;
}

// host or device candidates -> device array
static void *io_buf(fastt_graph *g, int k, size_t bytes) {
  auto &b = g->io[k];
  if (b.cap < bytes) {
    cudaFree(b.p);
    b.p = nullptr;
    b.cap = 0;
    if (cudaMalloc(&b.p, bytes) != cudaSuccess) return nullptr;
    b.cap = bytes;
  }
  return b.p;
}

static fastt_status upload_cands(const fastt_candidate *cands, int64_t n, uint32_t flags, Cand **d, bool *owned,
                                 cudaStream_t st) {
  *owned = false;
  if (flags & FASTT_F_IN_DEVICE) {
    *d = (Cand *)cands;
    return FASTT_OK;
  }
  CK(cudaMalloc(d, sizeof(Cand) * (n + 1)));
  *owned = true;
  if (n) CK(cudaMemcpyAsync(*d, cands, sizeof(Cand) * n, cudaMemcpyHostToDevice, st));
  return FASTT_OK;
}

fastt_status fastt_rank(const fastt_graph *gc_, const fastt_candidate *cand, const fastt_opts *opts,
                        int64_t *rank_out) {
  fastt_graph *g = (fastt_graph *)gc_;
  if (!g || !rank_out) return fail(FASTT_EINVAL, "NULL argument");
  std::lock_guard<std::mutex> lk(g->mu);
  Dev guard(g->dev);
  cudaStream_t st = stream_of(opts);
  CallGuard cg(g, st);  // (blocking: the ranks come back through the host)
  Base &B = g->base;
  const int64_t vm = g->v_max;
  std::vector<uint64_t> r(B.rl.vcap, ~0ull);
  const uint32_t all = all_devices(g->G);
  if (cand && (cand->dev_mask & ~all)) return fail(FASTT_EINVAL, "dev_mask names a device >= G");
  const uint32_t dset = cand && cand->dev_mask ? cand->dev_mask : all;
  if (!cand || (cand->kind == FASTT_KIND_BASE && dset == all)) {
    if (B.V) CK(cudaMemcpy(r.data(), prep_struct(B.prep_block, B.pl, B.tbits).rank, 8 * (size_t)B.V,
                           cudaMemcpyDeviceToHost));
  } else {
    // validate like the simulator does
    const Cand &c = *(const Cand *)cand;
    bool bad = false;
    if (c.kind == FASTT_KIND_PIN) {
      if (c.n_pins < 1 || c.n_pins > 4) bad = true;
      for (int k = 0; k < c.n_pins && !bad; k++) {
        if (c.pin_op[k] < 0 || c.pin_op[k] >= B.V || c.pin_dev[k] >= g->G || !((dset >> c.pin_dev[k]) & 1u))
          bad = true;
        for (int k2 = 0; k2 < k; k2++) bad |= c.pin_op[k2] == c.pin_op[k];
      }
    } else if (c.kind == FASTT_KIND_SPLIT) {
      if (c.split_op < 0 || c.split_op >= B.V || c.split_dim > 1 ||
          !(g->split_mask_h[c.split_op] & (1u << c.split_dim)) || c.split_n < 2 || c.split_n > g->G)
        bad = true;
    } else if (c.kind != FASTT_KIND_BASE) {
      bad = true;
    }
    if (bad) return fail(FASTT_EINVAL, "invalid candidate");
    TRY(ensure_arena(g, B, st, 1));
    CK(cudaMemcpyAsync(g->slot_cands, &c, sizeof c, cudaMemcpyHostToDevice, st));
    launch_slot_setup(g->slot_cands, g->tmpl_dev, B.raw_dev, g->slot_raws_dev, 1, st);
    launch_copy_block(B.raw_block, g->arena, (int64_t)(g->arena_raw_total + g->arena_prep_total),
                      (int64_t)B.rl.total, g->slot_cands, 1, st);
    launch_patch_split(B.raw_dev, g->slot_raws_dev, g->gc_dev, g->slot_cands, 1, st);
    launch_rank(g->slot_raws_dev, g->slot_pgs_dev, g->gc_dev, g->slot_cands, 1, g->G, st);
    CK(cudaGetLastError());
    RawGraph R;
    PrepGraph P;
    CK(cudaMemcpyAsync(&R, g->slot_raws_dev, sizeof R, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&P, g->slot_pgs_dev, sizeof P, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    CK(cudaMemcpy(r.data(), P.rank, 8 * (size_t)R.V, cudaMemcpyDeviceToHost));
  }
  std::vector<int64_t> ro(vm);
  for (int64_t i = 0; i < vm; i++) ro[i] = r[i] == ~0ull ? -1 : (int64_t)r[i];
  if (flags_of(opts) & FASTT_F_OUT_DEVICE) CK(cudaMemcpy(rank_out, ro.data(), 8 * vm, cudaMemcpyHostToDevice));
  else memcpy(rank_out, ro.data(), 8 * vm);
  return FASTT_OK;
}

fastt_status fastt_schedule_batch(const fastt_graph *gc_, const fastt_candidate *cands, int64_t n,
                                  const fastt_opts *opts, int64_t *makespan, int64_t *peak_mem, uint8_t *status,
                                  uint8_t *placement, int32_t *order, int64_t *start_ns) {
  fastt_graph *g = (fastt_graph *)gc_;
  if (!g || n < 0 || (n > 0 && (!cands || !makespan || !status))) return fail(FASTT_EINVAL, "bad argument");
  const uint32_t flags = flags_of(opts);
  if (n == 0) return FASTT_OK;
  std::lock_guard<std::mutex> lk(g->mu);
  Dev guard(g->dev);
  cudaStream_t st = stream_of(opts);
  TRY(call_begin(g, st));
  Base &B = g->base;
  const int64_t vm = g->v_max;
  const bool outdev = (flags & FASTT_F_OUT_DEVICE) != 0;
  Cand *d_c;
  if (flags & FASTT_F_IN_DEVICE) {
    d_c = (Cand *)cands;
  } else {
    d_c = (Cand *)io_buf(g, 0, sizeof(Cand) * (size_t)(n + 1));
    if (!d_c) return fail(FASTT_ENOMEM, "candidate staging buffer");
    CK(cudaMemcpyAsync(d_c, cands, sizeof(Cand) * n, cudaMemcpyHostToDevice, st));
  }
  DevOut o;
  o.vmax = vm;
  std::vector<void *> tmp;
  auto dalloc = [&](void *user, size_t bytes, bool need) -> void * {  // stream-ordered scratch
    if (!need) return nullptr;
    if (outdev && user) return user;
    void *p = nullptr;
    if (cudaMallocAsync(&p, bytes, st) != cudaSuccess) return nullptr;
    tmp.push_back(p);
    return p;
  };
  o.makespan = (int64_t *)(outdev ? dalloc(makespan, 8 * (size_t)n, true) : io_buf(g, 1, 8 * (size_t)n));
  o.status = (uint8_t *)(outdev ? dalloc(status, (size_t)n, true) : io_buf(g, 2, (size_t)n));
  // (host outputs: the graph's staging buffers, kept across calls -- a
  // stream-ordered allocation per call would return its pages to the OS at
  // every synchronisation)
  o.peak = (int64_t *)(outdev || !peak_mem ? dalloc(peak_mem, 8 * (size_t)n * g->G, peak_mem != nullptr)
                                           : io_buf(g, 3, 8 * (size_t)n * g->G));
  const bool want_sched = placement || order || start_ns;
  o.place = (uint8_t *)dalloc(placement, (size_t)n * vm, want_sched);
  o.start = (int64_t *)dalloc(start_ns, 8 * (size_t)n * vm, want_sched);
  o.deq = (int32_t *)dalloc(nullptr, 4 * (size_t)n * vm, order != nullptr);
  o.order = (int32_t *)dalloc(order, 4 * (size_t)n * vm, order != nullptr);
  fastt_status rc = FASTT_OK;
  if (!o.makespan || !o.status || (peak_mem && !o.peak) || (want_sched && (!o.place || !o.start)) ||
      (order && (!o.deq || !o.order)))
    rc = fail(FASTT_ENOMEM, "device output buffers");
  if (rc == FASTT_OK) rc = timing_begin(g, flags, st);
  if (rc == FASTT_OK) rc = eval_batch(g, B, d_c, n, flags | FASTT_F_ASYNC, st, o);
  if (rc == FASTT_OK && !outdev) {
    auto back = [&](void *h, void *dd, size_t bytes) {
      if (h && dd && cudaMemcpyAsync(h, dd, bytes, cudaMemcpyDeviceToHost, st) != cudaSuccess)
        rc = fail(FASTT_ECUDA, "download");
    };
    back(makespan, o.makespan, 8 * (size_t)n);
    back(status, o.status, (size_t)n);
    back(peak_mem, o.peak, 8 * (size_t)n * g->G);
    back(placement, o.place, (size_t)n * vm);
    back(start_ns, o.start, 8 * (size_t)n * vm);
    back(order, o.order, 4 * (size_t)n * vm);
  }
  for (void *p : tmp) cudaFreeAsync(p, st);
  if (rc == FASTT_OK) rc = timing_end(g, flags, st, n);
  return call_end(g, flags, st, rc);
}

fastt_status fastt_stream_info(const fastt_graph *gc_, const fastt_gen_params *gen, const fastt_opts *opts,
                               int64_t *n_split) {
  fastt_graph *g = (fastt_graph *)gc_;
  if (!g || !gen || !n_split) return fail(FASTT_EINVAL, "NULL argument");
  std::lock_guard<std::mutex> lk(g->mu);
  Dev guard(g->dev);
  CallGuard cg(g, stream_of(opts));
  StreamCache *S;
  TRY(ensure_stream(g, flags_of(opts), gen->n_pow2_only, stream_of(opts), &S));
  *n_split = S->n_split;
  return FASTT_OK;
}

fastt_status fastt_generate_candidates(const fastt_graph *gc_, const fastt_gen_params *gen, const fastt_opts *opts,
                                       int64_t first, int64_t n, fastt_candidate *out) {
  fastt_graph *g = (fastt_graph *)gc_;
  if (!g || !gen || (n > 0 && !out)) return fail(FASTT_EINVAL, "NULL argument");
  std::lock_guard<std::mutex> lk(g->mu);
  Dev guard(g->dev);
  cudaStream_t st = stream_of(opts);
  TRY(call_begin(g, st));
  StreamCache *S;
  TRY(ensure_stream(g, flags_of(opts), gen->n_pow2_only, st, &S));
  TRY(check_gen(g, *S, gen, first, n, 1));
  if (n == 0) return FASTT_OK;
  StreamState ss = stream_state(g, *S, gen);
  const bool outdev = (flags_of(opts) & FASTT_F_OUT_DEVICE) != 0;
  Cand *d = (Cand *)out;
  if (!outdev) {  // (the graph's candidate staging buffer, kept across calls)
    d = (Cand *)io_buf(g, 0, sizeof(Cand) * (size_t)(n + 1));
    if (!d) return fail(FASTT_ENOMEM, "candidate staging buffer");
  }
  launch_candgen(ss, first, n, d, st);
  CK(cudaGetLastError());
  if (!outdev) CK(cudaMemcpyAsync(out, d, sizeof(Cand) * n, cudaMemcpyDeviceToHost, st));
  return call_end(g, flags_of(opts), st, FASTT_OK);
}

fastt_status fastt_sweep_best(const fastt_graph *gc_, const fastt_gen_params *gen, const fastt_opts *opts,
                              int64_t first, int64_t n, int64_t stride, int64_t *best) {
  fastt_graph *g = (fastt_graph *)gc_;
  if (!g || !gen || !best) return fail(FASTT_EINVAL, "NULL argument");
  const uint32_t flags = flags_of(opts);
  std::lock_guard<std::mutex> lk(g->mu);
  Dev guard(g->dev);
  cudaStream_t st = stream_of(opts);
  host_trace("sweep: enter");
  TRY(call_begin(g, st));
  host_trace("sweep: call_begin");
  StreamCache *S;
  TRY(ensure_stream(g, flags, gen->n_pow2_only, st, &S));
  TRY(check_gen(g, *S, gen, first, n, stride));
  Base &B = g->base;
  host_trace("sweep: stream");
  TRY(ensure_sim(g, B, n, flags));
  host_trace("sweep: sim");
  if (g->share) TRY(ensure_snapshot(g, B, flags, st));
  host_trace("sweep: snapshot");
  int64_t nwarps = max_slots(g);  // candidate slots (per-warp bests)
  SimArgs a = sim_args(g, B, flags);
  a.mode = 0;
  a.stream = stream_state(g, *S, gen);
  a.first = first;
  a.n = n;
  a.stride = stride;
  a.track_best = 1;
  if (g->share) use_snapshot(B, flags, a);
  // the overlapped path: a sorted, classified list on the packed-key lane kernel
  bool ovl = false;
  if (n > 0 && g->use_overlap && a.snap_mode == 2 && a.pkc && a.costk && a.pk_lim > 0) {
    SimArgs t = a;
    int gr;
    size_t sm;
    main_shape(g, B, t, gr, sm);
    ovl = t.lane == 1;
  }
  int cap = 0, wmain = 0;
  if (ovl) {
    // arena: the window's SPLIT and device-subset candidates plus the
    // rank-changing PINs of the last call (a longer tail runs after the join)
    const int64_t hi = a.stream.n_split + a.stream.n_subset;
    int64_t nsp = 0;
    if (hi >= 1 && first <= hi) {
      const int64_t q_lo = first >= 1 ? 0 : (1 - first + stride - 1) / stride;
      const int64_t q_hi = std::min<int64_t>(n - 1, (hi - first) / stride);
      nsp = q_hi >= q_lo ? q_hi - q_lo + 1 : 0;
    }
    TRY(ensure_arena(g, B, st, std::max<int64_t>(nsp + 256, std::min<int64_t>(g->pin_defer_hint, ARENA_MAX_SLOTS))));
    cap = g->arena_slots;
    {
      SimArgs t = a;
      int gr;
      size_t sm;
      main_shape(g, B, t, gr, sm);
      wmain = lane_warps(g, t);
    }
    host_trace("sweep: arena");
    TRY(ensure_overlap(g, B, cap, wmain));
    host_trace("sweep: overlap bufs");
    nwarps = (int64_t)wmain + cap + 64;
  } else {
    launch_init_best(g->wbest, nwarps, st);
  }
  // (the non-overlapped path's deferral rounds: arena sized before the launch)
  if (!ovl && n > 0) {
    // the window's SPLIT and device-subset candidates are deferred for sure
    const int64_t hi = a.stream.n_split + a.stream.n_subset;
    int64_t nsp = 0;
    if (hi >= 1 && first <= hi) {
      const int64_t q_lo = first >= 1 ? 0 : (1 - first + stride - 1) / stride;
      const int64_t q_hi = std::min<int64_t>(n - 1, (hi - first) / stride);
      nsp = q_hi >= q_lo ? q_hi - q_lo + 1 : 0;
    }
    TRY(ensure_arena(g, B, st, seq_arena_want(g, nsp)));
    host_trace("sweep: arena (sequential path)");
  }
  TRY(timing_begin(g, flags, st));
  if (n > 0 && ovl) {
    CK(cudaMemsetAsync(g->counters, 0, 2 * sizeof(unsigned long long), st));
    TRY(ensure_sort_buf(g, n));
    const PrepGraph P = prep_struct(B.prep_block, B.pl, B.tbits);
    T0Classify cl{1, B.tbits, B.pg_dev, g->gc_dev, a.split_mask, g->ov_words};
    launch_t0_sort(1, a.stream, first, stride, nullptr, n, P.pos, a.snap_dq, B.n, B.V, g->G, g->srt_tmp_c,
                   g->srt_tmp_i, g->srt_key, g->srt_hist, g->srt_c, g->srt_i, nullptr, st, cl);
    g->launches += 4;
    a.mode = 3;
    a.cands = g->srt_c;
    a.slot_index = g->srt_i;
    a.slot_result = nullptr;
    {
      int gr;
      size_t sm;
      main_shape(g, B, a, gr, sm);
    }
    host_trace("sweep: sort");
    TRY(run_overlapped(g, B, a, n, flags, st, false, cap, wmain));
    host_trace("sweep: overlapped launches");
    timing_mark(g, flags, 2, st);
    TRY(finish_overlapped(g, B, a, n, st, false, cap, wmain));
    host_trace("sweep: deferral loop");
  } else if (n > 0) {
    CK(cudaMemsetAsync(g->counters, 0, 2 * sizeof(unsigned long long), st));
    if (a.snap_mode == 2) {
      TRY(ensure_sort_buf(g, n));
      const PrepGraph P = prep_struct(B.prep_block, B.pl, B.tbits);
      launch_t0_sort(1, a.stream, first, stride, nullptr, n, P.pos, a.snap_dq, B.n, B.V, g->G, g->srt_tmp_c,
                     g->srt_tmp_i, g->srt_key, g->srt_hist, g->srt_c, g->srt_i, nullptr, st);
      g->launches += 4;
      a.mode = 3;
      a.cands = g->srt_c;
      a.slot_index = g->srt_i;
      a.slot_result = nullptr;
    }
    host_trace("sweep: sorted (sequential path)");
    {
      int grid;
      size_t smem;
      main_shape(g, B, a, grid, smem);
      launch_sim(a, B.tbits, grid, g->sim_block, smem, st);
    }
    g->launches += NL_SIM;
    CK(cudaGetLastError());
    host_trace("sweep: main launch (sequential path)");
    timing_mark(g, flags, 1, st);
    TRY(run_defer_loop(g, B, a, g->arena_slots, a.mode == 3 ? 0 : 2, false, n, nullptr, &a.stream, first, stride,
                       false, g->counters + 1, st));
    timing_mark(g, flags, 2, st);
  } else {
    timing_mark(g, flags, 1, st);
    timing_mark(g, flags, 2, st);
  }
  launch_argmin(g->wbest, nwarps, g->best_dev, st);
  g->launches += NL_ARGMIN;
  CK(cudaGetLastError());
  if (flags & FASTT_F_OUT_DEVICE) {
    CK(cudaMemcpyAsync(best, g->best_dev, 16, cudaMemcpyDeviceToDevice, st));
  } else {
    CK(cudaMemcpyAsync(best, g->best_dev, 16, cudaMemcpyDeviceToHost, st));
  }
  TRY(timing_end(g, flags, st, n));
  if (ovl && (flags & FASTT_F_TIMING)) {  // the concurrent preparation stream's own duration
    float mp = 0;
    CK(cudaEventElapsedTime(&mp, g->ov_ev[1], g->ov_ev[2]));
    g->last.ms_prep = mp;
  }
  host_trace("sweep: argmin");
  const fastt_status rc = call_end(g, flags, st, FASTT_OK);
  host_trace("sweep: exit");
  return rc;
}

// materialise an accepted split into a new base with room for one more split
static fastt_status materialize_base(fastt_graph *g, Base &from, const Cand &c, Base &to, cudaStream_t st) {
  RawGraph Rf = raw_struct(from.raw_block, from.rl, from.V, from.n_live, from.E);
  (void)Rf;
  // sizes of the new graph
  std::vector<uint32_t> cnt(2);
  uint32_t P = 0, S = 0;
  {
    RawGraph R = raw_struct(from.raw_block, from.rl, 0, 0, 0);
    CK(cudaMemcpy(&P, R.pred_cnt + c.split_op, 4, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(&S, R.succ_cnt + c.split_op, 4, cudaMemcpyDeviceToHost));
  }
  to.V = from.V + (int32_t)(P + c.split_n + S);
  to.n_live = from.n_live - 1 + (int32_t)(P + c.split_n + S);
  const int64_t newE = from.E + (int64_t)P + (int64_t)P * c.split_n * 2 + (int64_t)S * c.split_n * 2 + S + 16;
  to.rl = raw_layout((int64_t)to.V + overlay_v(g), newE + overlay_e(g), g->G);
  if (to.rl.vcap > MAX_VCAP || (to.rl.vcap > READY_SET_MAX && !from.topo))
    return fail(FASTT_EUNSUP, "split search grew the graph above %d ops", to.rl.vcap > MAX_VCAP ? MAX_VCAP : READY_SET_MAX);
  CK(cudaMalloc(&to.raw_block, to.rl.total));
  CK(cudaMalloc(&to.raw_dev, sizeof(RawGraph)));
  CK(cudaMemsetAsync(to.raw_block, 0, to.rl.total, st));
  // array-wise copy (capacities differ)
  const int64_t vf = from.rl.vcap, ef = from.rl.ecap;
  size_t sz[16] = {(size_t)vf * 4, (size_t)vf * 4, (size_t)vf * 4, (size_t)vf * 4, (size_t)ef * 4, (size_t)ef * 4,
                   (size_t)ef * 8, (size_t)ef * 8, (size_t)ef, (size_t)ef, (size_t)vf * g->G * 8, (size_t)vf * 8,
                   (size_t)vf * 8, (size_t)vf, (size_t)vf, (size_t)vf * 4};
  for (int k = 0; k < 16; k++)
    CK(cudaMemcpyAsync(to.raw_block + to.rl.o[k], from.raw_block + from.rl.o[k], sz[k], cudaMemcpyDeviceToDevice, st));
  RawGraph Rt = raw_struct(to.raw_block, to.rl, from.V, from.n_live, from.E);
  CK(cudaMemcpyAsync(to.raw_dev, &Rt, sizeof Rt, cudaMemcpyHostToDevice, st));
  Cand *d_c;
  CK(cudaMalloc(&d_c, sizeof c));
  CK(cudaMemcpyAsync(d_c, &c, sizeof c, cudaMemcpyHostToDevice, st));
  launch_patch_split(from.raw_dev, to.raw_dev, g->gc_dev, d_c, 1, st);
  CK(cudaGetLastError());
  CK(cudaMemcpyAsync(&Rt, to.raw_dev, sizeof Rt, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  cudaFree(d_c);
  to.E = Rt.E;
  Rt.ov_P = -1;  // a materialised base, not a slot: its levels are recomputed by prepare_base
  CK(cudaMemcpy(to.raw_dev, &Rt, sizeof Rt, cudaMemcpyHostToDevice));
  return prepare_base(g, to, st);
}

fastt_status fastt_split_search(const fastt_graph *gc_, const fastt_opts *opts, int32_t n_pow2_only,
                                fastt_split_result *out) {
  fastt_graph *g = (fastt_graph *)gc_;
  if (!g || !out) return fail(FASTT_EINVAL, "NULL argument");
  const uint32_t flags = flags_of(opts) & (FASTT_F_CP_PIN | FASTT_F_POLICY_INSERT | FASTT_F_MEM_LIVE);
  const bool multi_mode = (flags_of(opts) & FASTT_F_SPLIT_MULTI) != 0;
  const bool best_mode = (flags_of(opts) & FASTT_F_SPLIT_BEST) != 0 || multi_mode;
  memset(out, 0, sizeof *out);
  std::lock_guard<std::mutex> lk(g->mu);
  Dev guard(g->dev);
  cudaStream_t st = stream_of(opts);
  CallGuard cg(g, st);  // (blocking: Alg. 2's accept/stop decisions are taken on the host)
  std::deque<Base> owned;  // bases created by accepted splits (stable addresses)
  Base *cur = &g->base;
  // Alg. 2 line 3: DPOS of the input graph
  int64_t vm = cur->rl.vcap;
  const int maxc = 2 * MAXG;
  Cand *d_c;
  int64_t *d_ms, *d_start;
  uint8_t *d_st, *d_place;
  int32_t *d_deq, *d_order;
  // per-op output buffers of a round: the graph grows by at most one split
  // overlay per accepted split (checked before every round below)
  int64_t cap_v = std::max<int64_t>(READY_SET_MAX + 64, 2 * cur->rl.vcap);
  CK(cudaMalloc(&d_c, sizeof(Cand) * maxc));
  CK(cudaMalloc(&d_ms, 8 * maxc));
  CK(cudaMalloc(&d_st, maxc));
  CK(cudaMalloc(&d_place, (size_t)maxc * cap_v));
  CK(cudaMalloc(&d_start, 8 * (size_t)maxc * cap_v));
  CK(cudaMalloc(&d_deq, 4 * (size_t)maxc * cap_v));
  CK(cudaMalloc(&d_order, 4 * (size_t)maxc * cap_v));
  auto cleanup = [&]() {
    cudaFree(d_c);
    cudaFree(d_ms);
    cudaFree(d_st);
    cudaFree(d_place);
    cudaFree(d_start);
    cudaFree(d_deq);
    cudaFree(d_order);
    for (auto &b : owned) b.release();
    if (g->arena_raw_total != g->base.rl.total) {  // arena was sized for a split-search base
      cudaFree(g->arena);
      g->arena = nullptr;
      g->arena_raw_total = g->arena_prep_total = 0;
    }
  };
  Cand base;
  memset(&base, 0, sizeof base);
  base.split_op = -1;
  for (int k = 0; k < 4; k++) base.pin_op[k] = -1;
  CK(cudaMemcpy(d_c, &base, sizeof base, cudaMemcpyHostToDevice));
  DevOut o;
  o.makespan = d_ms;
  o.status = d_st;
  o.place = d_place;
  o.start = d_start;
  o.deq = d_deq;
  o.order = d_order;
  o.vmax = vm;
  fastt_status rc = eval_batch(g, *cur, d_c, 1, flags, st, o);
  if (rc != FASTT_OK) {
    cleanup();
    return rc;
  }
  int64_t ft_old = 0;
  uint8_t s0 = 0;
  CK(cudaMemcpy(&ft_old, d_ms, 8, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(&s0, d_st, 1, cudaMemcpyDeviceToHost));
  std::vector<uint8_t> bplace(vm);
  std::vector<int64_t> bstart(vm);
  std::vector<int32_t> border(vm);
  CK(cudaMemcpy(bplace.data(), d_place, vm, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(bstart.data(), d_start, 8 * vm, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(border.data(), d_order, 4 * vm, cudaMemcpyDeviceToHost));
  std::vector<int32_t> sp_op;
  std::vector<uint8_t> sp_dim, sp_n;
  int32_t vfinal = g->V;
  if (s0 == FASTT_CAND_OK) {
    // Alg. 2 lines 4-5
    std::vector<int32_t> list;
    rc = split_list(g, *cur, d_place, list, st);
    if (rc != FASTT_OK) {
      cleanup();
      return rc;
    }
    int ns[MAXG];
    int nns = split_counts(g->G, n_pow2_only, ns);
    if (best_mode) {
      // NEXT N2: best-improvement rounds -- every remaining split of every
      // not-yet-split list op in one batch, accept the best if it improves
      std::vector<char> done(list.size(), 0);
      const size_t cap_round = list.size() * 2 * (size_t)nns + 1;
      Cand *d_round = nullptr;
      int64_t *d_rms = nullptr;
      uint8_t *d_rst = nullptr;
      if (cudaMalloc(&d_round, sizeof(Cand) * cap_round) != cudaSuccess ||
          cudaMalloc(&d_rms, 8 * cap_round) != cudaSuccess || cudaMalloc(&d_rst, cap_round) != cudaSuccess) {
        cudaFree(d_round);
        cudaFree(d_rms);
        cleanup();
        return fail(FASTT_ENOMEM, "split-search round buffers");
      }
      for (;;) {
        std::vector<Cand> cs;
        std::vector<size_t> li_of;
        for (size_t li = 0; li < list.size(); li++) {
          if (done[li]) continue;
          const int32_t op = list[li];
          for (int dim = 0; dim < 2; dim++) {
            if (!(g->split_mask_h[op] & (1u << dim))) continue;
            for (int q = 0; q < nns; q++) {
              Cand c;
              memset(&c, 0, sizeof c);
              c.kind = FASTT_KIND_SPLIT;
              c.split_op = op;
              c.split_dim = (uint8_t)dim;
              c.split_n = (uint8_t)ns[q];
              for (int k = 0; k < 4; k++) c.pin_op[k] = -1;
              cs.push_back(c);
              li_of.push_back(li);
            }
          }
        }
        if (cs.empty()) break;
        CK(cudaMemcpy(d_round, cs.data(), sizeof(Cand) * cs.size(), cudaMemcpyHostToDevice));
        DevOut mo;
        mo.makespan = d_rms;
        mo.status = d_rst;
        mo.vmax = cur->rl.vcap;
        rc = eval_batch(g, *cur, d_round, (int64_t)cs.size(), flags, st, mo);
        std::vector<int64_t> ms(cs.size());
        std::vector<uint8_t> sts(cs.size());
        if (rc == FASTT_OK && (cudaMemcpy(ms.data(), d_rms, 8 * cs.size(), cudaMemcpyDeviceToHost) != cudaSuccess ||
                               cudaMemcpy(sts.data(), d_rst, cs.size(), cudaMemcpyDeviceToHost) != cudaSuccess))
          rc = fail(FASTT_ECUDA, "download round results");
        int bi = -1;
        for (size_t q = 0; rc == FASTT_OK && q < cs.size(); q++)
          if (sts[q] == FASTT_CAND_OK && (bi < 0 || ms[q] < ms[bi])) bi = (int)q;
        // R27 multi-split candidates: each op's best improving variant (the
        // first minimum in (dim, n) order), the ops ranked by (makespan, list
        // order), C_j = the first j ranked splits applied in rank order
        // (materialised one after the other), the C_j of smallest makespan
        // (ties: smaller j) is accepted -- C_1 is the single best (bi)
        if (multi_mode && rc == FASTT_OK && bi >= 0 && ms[bi] < ft_old) {
          std::vector<int> bestq(list.size(), -1), rk;
          for (size_t q = 0; q < cs.size(); q++) {
            const size_t li = li_of[q];
            if (sts[q] == FASTT_CAND_OK && ms[q] < ft_old && (bestq[li] < 0 || ms[q] < ms[bestq[li]])) bestq[li] = (int)q;
          }
          for (size_t li = 0; li < list.size(); li++)
            if (bestq[li] >= 0) rk.push_back(bestq[li]);
          std::stable_sort(rk.begin(), rk.end(), [&](int x, int y) { return ms[x] < ms[y]; });  // (list order kept)
          if (rk.size() > 4) rk.resize(4);
          if (rk.size() >= 2) {
            std::vector<Base *> chain(rk.size() + 1, nullptr);
            std::vector<int64_t> ftj(rk.size() + 1, I64MAX);
            chain[0] = cur;
            ftj[1] = ms[rk[0]];
            int bj = 1;
            for (size_t j = 1; j <= rk.size() && rc == FASTT_OK; j++) {
              owned.emplace_back();
              chain[j] = &owned.back();
              rc = materialize_base(g, *chain[j - 1], cs[rk[j - 1]], *chain[j], st);
              if (rc != FASTT_OK || j == 1) continue;
              DevOut jo;
              jo.makespan = d_rms;
              jo.status = d_rst;
              jo.vmax = chain[j]->rl.vcap;
              CK(cudaMemcpy(d_round, &base, sizeof base, cudaMemcpyHostToDevice));
              rc = eval_batch(g, *chain[j], d_round, 1, flags, st, jo);
              int64_t m = I64MAX;
              uint8_t s1 = 1;
              if (rc == FASTT_OK && (cudaMemcpy(&m, d_rms, 8, cudaMemcpyDeviceToHost) != cudaSuccess ||
                                     cudaMemcpy(&s1, d_rst, 1, cudaMemcpyDeviceToHost) != cudaSuccess))
                rc = fail(FASTT_ECUDA, "download a multi-split result");
              if (rc == FASTT_OK && s1 == FASTT_CAND_OK) {
                ftj[j] = m;
                if (m < ftj[bj]) bj = (int)j;
              }
            }
            if (rc == FASTT_OK && bj >= 2) {  // accept C_bj: outputs of its graph
              for (size_t j = 1; j <= rk.size(); j++)  // (each base is a copy: the others can go)
                if (j != (size_t)bj) chain[j]->release();
              vm = chain[bj]->rl.vcap;
              if (vm > cap_v) rc = fail(FASTT_EUNSUP, "split search grew the graph past its output buffers");
              o.vmax = vm;
              CK(cudaMemcpy(d_c, &base, sizeof base, cudaMemcpyHostToDevice));
              if (rc == FASTT_OK) rc = eval_batch(g, *chain[bj], d_c, 1, flags, st, o);
              if (rc == FASTT_OK) {
                ft_old = ftj[bj];
                for (int j = 1; j <= bj; j++) {
                  const Cand &cj = cs[rk[j - 1]];
                  done[li_of[rk[j - 1]]] = 1;
                  sp_op.push_back(cj.split_op);
                  sp_dim.push_back(cj.split_dim);
                  sp_n.push_back(cj.split_n);
                }
                vfinal = chain[bj]->V;
                bplace.resize(vm);
                bstart.resize(vm);
                border.resize(vm);
                CK(cudaMemcpy(bplace.data(), d_place, vm, cudaMemcpyDeviceToHost));
                CK(cudaMemcpy(bstart.data(), d_start, 8 * vm, cudaMemcpyDeviceToHost));
                CK(cudaMemcpy(border.data(), d_order, 4 * vm, cudaMemcpyDeviceToHost));
                cur = chain[bj];
                continue;
              }
            } else if (rc == FASTT_OK) {  // C_1 wins: drop the chain beyond it (C_1 is re-made below)
              for (size_t j = 1; j <= rk.size(); j++) chain[j]->release();
            }
          }
        }
        if (rc == FASTT_OK && bi >= 0 && ms[bi] < ft_old) {
          // the winner's placement / order / start (one more evaluation with outputs)
          vm = cur->rl.vcap;
          if (vm > cap_v) rc = fail(FASTT_EUNSUP, "split search grew the graph past its output buffers");
          o.vmax = vm;
          CK(cudaMemcpy(d_c, &cs[bi], sizeof(Cand), cudaMemcpyHostToDevice));
          if (rc == FASTT_OK) rc = eval_batch(g, *cur, d_c, 1, flags, st, o);
          if (rc == FASTT_OK) {
            owned.emplace_back();
            Base &nb = owned.back();
            rc = materialize_base(g, *cur, cs[bi], nb, st);
            if (rc == FASTT_OK) {
              ft_old = ms[bi];
              done[li_of[bi]] = 1;
              sp_op.push_back(cs[bi].split_op);
              sp_dim.push_back(cs[bi].split_dim);
              sp_n.push_back(cs[bi].split_n);
              vfinal = nb.V;
              bplace.resize(vm);
              bstart.resize(vm);
              border.resize(vm);
              CK(cudaMemcpy(bplace.data(), d_place, vm, cudaMemcpyDeviceToHost));
              CK(cudaMemcpy(bstart.data(), d_start, 8 * vm, cudaMemcpyDeviceToHost));
              CK(cudaMemcpy(border.data(), d_order, 4 * vm, cudaMemcpyDeviceToHost));
              cur = &nb;
              continue;
            }
          }
        }
        cudaFree(d_round);
        cudaFree(d_rms);
        cudaFree(d_rst);
        if (rc != FASTT_OK) {
          cleanup();
          return rc;
        }
        break;
      }
    } else
    // Alg. 2 lines 7-14
    for (int32_t op : list) {
      std::vector<Cand> cs;
      for (int dim = 0; dim < 2; dim++) {
        if (!(g->split_mask_h[op] & (1u << dim))) continue;
        for (int q = 0; q < nns; q++) {
          Cand c;
          memset(&c, 0, sizeof c);
          c.kind = FASTT_KIND_SPLIT;
          c.split_op = op;
          c.split_dim = (uint8_t)dim;
          c.split_n = (uint8_t)ns[q];
          for (int k = 0; k < 4; k++) c.pin_op[k] = -1;
          cs.push_back(c);
        }
      }
      if (cs.empty()) continue;
      CK(cudaMemcpy(d_c, cs.data(), sizeof(Cand) * cs.size(), cudaMemcpyHostToDevice));
      vm = cur->rl.vcap;
      if (vm > cap_v) rc = fail(FASTT_EUNSUP, "split search grew the graph past its output buffers");
      o.vmax = vm;
      if (rc == FASTT_OK) rc = eval_batch(g, *cur, d_c, (int64_t)cs.size(), flags, st, o);
      if (rc != FASTT_OK) {
        cleanup();
        return rc;
      }
      std::vector<int64_t> ms(cs.size());
      std::vector<uint8_t> sts(cs.size());
      CK(cudaMemcpy(ms.data(), d_ms, 8 * cs.size(), cudaMemcpyDeviceToHost));
      CK(cudaMemcpy(sts.data(), d_st, cs.size(), cudaMemcpyDeviceToHost));
      int bi = -1;
      for (size_t q = 0; q < cs.size(); q++)
        if (sts[q] == FASTT_CAND_OK && (bi < 0 || ms[q] < ms[bi])) bi = (int)q;
      if (bi < 0 || ms[bi] >= ft_old) break;
      // accept: Alg. 2 line 10
      owned.emplace_back();
      Base &nb = owned.back();
      rc = materialize_base(g, *cur, cs[bi], nb, st);
      if (rc != FASTT_OK) {
        cleanup();
        return rc;
      }
      ft_old = ms[bi];
      sp_op.push_back(op);
      sp_dim.push_back(cs[bi].split_dim);
      sp_n.push_back(cs[bi].split_n);
      vfinal = nb.V;
      bplace.resize(vm);
      bstart.resize(vm);
      border.resize(vm);
      CK(cudaMemcpy(bplace.data(), d_place + (size_t)bi * vm, vm, cudaMemcpyDeviceToHost));
      CK(cudaMemcpy(bstart.data(), d_start + (size_t)bi * vm, 8 * vm, cudaMemcpyDeviceToHost));
      CK(cudaMemcpy(border.data(), d_order + (size_t)bi * vm, 4 * vm, cudaMemcpyDeviceToHost));
      cur = &nb;
    }
  }
  rc = check_kernel_err(g, st);
  if (rc != FASTT_OK) {
    cleanup();
    return rc;
  }
  out->status = s0;
  out->makespan = s0 == FASTT_CAND_OK ? ft_old : I64MAX;
  out->n_splits = (int32_t)sp_op.size();
  out->op = (int32_t *)malloc(sizeof(int32_t) * (sp_op.size() + 1));
  out->dim = (uint8_t *)malloc(sp_op.size() + 1);
  out->n = (uint8_t *)malloc(sp_op.size() + 1);
  for (size_t q = 0; q < sp_op.size(); q++) {
    out->op[q] = sp_op[q];
    out->dim[q] = sp_dim[q];
    out->n[q] = sp_n[q];
  }
  out->n_ops_final = vfinal;
  out->placement = (uint8_t *)malloc(vfinal + 1);
  out->order = (int32_t *)malloc(sizeof(int32_t) * (vfinal + 1));
  out->start_ns = (int64_t *)malloc(sizeof(int64_t) * (vfinal + 1));
  for (int32_t i = 0; i < vfinal; i++) {
    out->placement[i] = i < (int32_t)bplace.size() ? bplace[i] : 0xFF;
    out->start_ns[i] = i < (int32_t)bstart.size() ? bstart[i] : -1;
    out->order[i] = i < (int32_t)border.size() ? border[i] : -1;
  }
  cleanup();
  return FASTT_OK;
}

// ------------------------------------------------- comm-model fit (N4)

fastt_status fastt_cost_table(int32_t V, int32_t G, int64_t n, const int32_t *op, const uint8_t *dev,
                              const int64_t *tns, int cuda_device, const fastt_opts *opts, int64_t *cost) {
  if (G < 1 || G > MAXG) return fail(FASTT_EINVAL, "n_devices must be in 1..%d", MAXG);
  if (V < 1) return fail(FASTT_EINVAL, "n_ops must be >= 1");
  if (n < 0 || n >= (1ll << 24)) return fail(FASTT_EINVAL, "n_samples must be in [0, 2^24)");
  if (!cost || (n > 0 && (!op || !dev || !tns))) return fail(FASTT_EINVAL, "NULL argument");
  const uint32_t flags = flags_of(opts);
  cudaStream_t st = stream_of(opts);
  Dev guard(cuda_device);
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, cuda_device);
  const bool in_dev = (flags & FASTT_F_IN_DEVICE) != 0, out_dev = (flags & FASTT_F_OUT_DEVICE) != 0;
  const size_t ne = (size_t)V * G;
  // one scratch block: [sum | count][err][cost][op][dev][time]
  const size_t o_err = al16(16 * ne), o_c = o_err + 16, o_op = o_c + al16(8 * ne),
               o_dv = o_op + (in_dev ? 0 : al16(4 * n)), o_t = o_dv + (in_dev ? 0 : al16(n)),
               tot = o_t + (in_dev ? 0 : al16(8 * n)) + 16;
  char *buf = nullptr;
  CK(cudaMalloc(&buf, tot));
  struct Free {
    char *p;
    ~Free() { cudaFree(p); }
  } fr{buf};
  const int32_t *d_op = op;
  const uint8_t *d_dv = dev;
  const int64_t *d_t = tns;
  if (!in_dev && n > 0) {
    CK(cudaMemcpyAsync(buf + o_op, op, 4 * n, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(buf + o_dv, dev, n, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(buf + o_t, tns, 8 * n, cudaMemcpyHostToDevice, st));
    d_op = (const int32_t *)(buf + o_op);
    d_dv = (const uint8_t *)(buf + o_dv);
    d_t = (const int64_t *)(buf + o_t);
  }
  unsigned *d_err = (unsigned *)(buf + o_err);
  CK(cudaMemsetAsync(d_err, 0, 4, st));
  int64_t *d_cost = out_dev ? cost : (int64_t *)(buf + o_c);
  launch_cost_table(V, G, n, d_op, d_dv, d_t, buf, d_err, d_cost, sms, st);
  CK(cudaGetLastError());
  unsigned herr = 0;
  CK(cudaMemcpyAsync(&herr, d_err, 4, cudaMemcpyDeviceToHost, st));
  if (!out_dev) CK(cudaMemcpyAsync(cost, d_cost, 8 * ne, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (herr) return fail(FASTT_EINVAL, "a sample is outside the envelope (op, device or time range)");
  return FASTT_OK;
}

fastt_status fastt_fit_comm(int32_t G, int64_t n, const uint8_t *src, const uint8_t *dst, const int64_t *bytes,
                            const int64_t *tns, int cuda_device, const fastt_opts *opts, int64_t *alpha,
                            int64_t *beta, int64_t *count) {
  if (G < 1 || G > MAXG) return fail(FASTT_EINVAL, "n_devices must be in 1..%d", MAXG);
  if (n < 0 || n >= (1ll << 24)) return fail(FASTT_EINVAL, "n_samples must be in [0, 2^24)");
  if (!alpha || !beta || (n > 0 && (!src || !dst || !bytes || !tns))) return fail(FASTT_EINVAL, "NULL argument");
  const uint32_t flags = flags_of(opts);
  cudaStream_t st = stream_of(opts);
  Dev guard(cuda_device);
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, cuda_device);
  const int P = G * G;
  const bool in_dev = (flags & FASTT_F_IN_DEVICE) != 0, out_dev = (flags & FASTT_F_OUT_DEVICE) != 0;
  // one scratch block: [sums][err][alpha][beta][count][src][dst][bytes][time]
  const size_t o_err = al16(fit_sums_bytes(G)), o_a = o_err + 16, o_b = o_a + al16(8 * P), o_c = o_b + al16(8 * P),
               o_s = o_c + al16(8 * P), o_d = o_s + (in_dev ? 0 : al16(n)), o_by = o_d + (in_dev ? 0 : al16(n)),
               o_t = o_by + (in_dev ? 0 : al16(8 * n)), tot = o_t + (in_dev ? 0 : al16(8 * n)) + 16;
  char *buf = nullptr;
  CK(cudaMalloc(&buf, tot));
  struct Free {
    char *p;
    ~Free() { cudaFree(p); }
  } fr{buf};
  const uint8_t *d_src = src, *d_dst = dst;
  const int64_t *d_by = bytes, *d_t = tns;
  if (!in_dev && n > 0) {
    CK(cudaMemcpyAsync(buf + o_s, src, n, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(buf + o_d, dst, n, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(buf + o_by, bytes, 8 * n, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(buf + o_t, tns, 8 * n, cudaMemcpyHostToDevice, st));
    d_src = (const uint8_t *)(buf + o_s);
    d_dst = (const uint8_t *)(buf + o_d);
    d_by = (const int64_t *)(buf + o_by);
    d_t = (const int64_t *)(buf + o_t);
  }
  int64_t *ra = out_dev ? alpha : (int64_t *)(buf + o_a), *rb = out_dev ? beta : (int64_t *)(buf + o_b);
  int64_t *rc = count ? (out_dev ? count : (int64_t *)(buf + o_c)) : nullptr;
  launch_fit(G, n, d_src, d_dst, d_by, d_t, buf, (unsigned *)(buf + o_err), ra, rb, rc, sms, st);
  CK(cudaGetLastError());
  unsigned err = 0;
  CK(cudaMemcpyAsync(&err, buf + o_err, 4, cudaMemcpyDeviceToHost, st));
  if (!out_dev) {
    CK(cudaMemcpyAsync(alpha, ra, 8 * P, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(beta, rb, 8 * P, cudaMemcpyDeviceToHost, st));
    if (count) CK(cudaMemcpyAsync(count, rc, 8 * P, cudaMemcpyDeviceToHost, st));
  }
  CK(cudaStreamSynchronize(st));
  if (err) return fail(FASTT_EINVAL, "a sample has a bad device pair or bytes/time outside [0, 2^40)");
  return FASTT_OK;
}

fastt_status fastt_link_model(int32_t G, const int64_t *alpha, const int64_t *beta, uint8_t *link_class,
                              int32_t *n_classes, int64_t *link_alpha, int64_t *link_beta) {
  if (G < 1 || G > MAXG) return fail(FASTT_EINVAL, "n_devices must be in 1..%d", MAXG);
  if (!alpha || !beta || !link_class || !n_classes || !link_alpha || !link_beta) return fail(FASTT_EINVAL, "NULL argument");
  int K = 0;
  int64_t ka[MAXK], kb[MAXK];
  for (int s = 0; s < G; s++)
    for (int t = 0; t < G; t++) {
      const int64_t a = alpha[s * G + t], b = beta[s * G + t];
      if (s == t) {
        link_class[s * G + t] = 0;
        continue;
      }
      if (a < 0 || b < 0) return fail(FASTT_EINVAL, "negative link parameters");
      int k = 0;
      while (k < K && !(ka[k] == a && kb[k] == b)) k++;
      if (k == K) {
        if (K == MAXK) return fail(FASTT_EUNSUP, "more than %d distinct link parameter pairs", MAXK);
        ka[K] = a;
        kb[K] = b;
        K++;
      }
      link_class[s * G + t] = (uint8_t)k;
    }
  if (K == 0) {  // G == 1: one (unused) class
    ka[0] = kb[0] = 0;
    K = 1;
  }
  *n_classes = K;
  for (int k = 0; k < K; k++) {
    link_alpha[k] = ka[k];
    link_beta[k] = kb[k];
  }
  return FASTT_OK;
}

fastt_status fastt_sync(const fastt_graph *gc_, const fastt_opts *opts) {
  fastt_graph *g = (fastt_graph *)gc_;
  if (!g) return fail(FASTT_EINVAL, "NULL argument");
  std::lock_guard<std::mutex> lk(g->mu);
  Dev guard(g->dev);
  cudaStream_t st = stream_of(opts);
  if (g->done_rec) CK(cudaStreamWaitEvent(st, g->done_ev, 0));
  return call_end(g, 0, st, FASTT_OK);
}

fastt_status fastt_last_timing(const fastt_graph *g, fastt_timing *out) {
  if (!g || !out) return fail(FASTT_EINVAL, "NULL argument");
  *out = g->last;
  return FASTT_OK;
}

void fastt_free_split_result(fastt_split_result *r) {
  if (!r) return;
  free(r->op);
  free(r->dim);
  free(r->n);
  free(r->placement);
  free(r->order);
  free(r->start_ns);
  memset(r, 0, sizeof *r);
}

}  // extern "C"
