// fastt_internal.cuh -- device-side data layout of the B200 FastT library.
//
// Two graph forms live in HBM:
//  * RawGraph  -- the problem graph in the caller's id space:
//    both CSRs with per-op (offset, count) so a split can be patched in place
//    and appended to (R13), per-edge bytes/param flags, cost/mem tables and a
//    topological order.  One for the loaded graph; one per SPLIT candidate
//    slot (materialised SplitOperation, Alg. 2 lines 16-30).
//  * PrepGraph -- what the schedule simulator reads.  Ops are renumbered by
//    their priority (rank_u desc, id asc; R2/R3), so a ready set is a bitmap
//    over positions and "pop max priority" is find-first-set.  Each op has a
//    128-byte CARD (header + up to 12 predecessor and 12 successor positions)
//    that one coalesced warp load brings in; costs are a [pos][G] table in
//    the time type T (uint32 when the schedule bound fits, else uint64).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

// simulation kernel launch shape (threads per block, min blocks per SM)
#ifndef SIM_BLOCK
#define SIM_BLOCK 128
#endif
#ifndef SIM_MINB
#define SIM_MINB 5
#endif
#ifndef SIM_MINB_TOPO
#define SIM_MINB_TOPO 7
#endif
// lane-per-candidate position-order kernel (k_sim_lane.cu)
#ifndef LANE_BLOCK
#define LANE_BLOCK 128
#endif
#ifndef LANE_MINB
#define LANE_MINB 4
#endif

namespace fastt {

constexpr int MAXG = 32;
constexpr int MAXK = 16;
constexpr int MAXPINS = 4;
constexpr int CARD_WORDS = 32;
constexpr int CARD_HDR = 8;
// card words 8..11: up to 4 predecessor positions; 12..15: their comm
// values (uint32 time, one link class); 16..31: up to 16 successor positions
constexpr int P_IN = 4;   // inline predecessor positions in a card
constexpr int S_IN = 16;  // inline successor positions in a card
constexpr int CW_PCOMM = CARD_HDR + P_IN;  // inline comm values
constexpr int CW_SUCC = CW_PCOMM + P_IN;   // inline successor positions
constexpr uint32_t NONE = 0xFFFFFFFFu;
constexpr int64_t I64MAX = INT64_MAX;
// graph size envelope: positions fit 24 bits (lane-kernel CP rounds, group
// kernel records); the ready-set kernel's 3-level bitmap covers 32768
constexpr int64_t MAX_VCAP = 1 << 23;
constexpr int64_t READY_SET_MAX = 32768;

// card header words
enum { CW_DEG = 0, CW_PBASE = 1, CW_SBASE = 2, CW_CPIDX = 3, CW_MEMLO = 4, CW_MEMHI = 5, CW_UID = 6, CW_FLAGS = 7 };

struct GraphConst {
  int32_t G, K;
  int64_t copy_fs;
  int64_t cap[MAXG];
  int64_t alpha[MAXK], beta[MAXK];
  uint8_t link_class[MAXG * MAXG];
  uint32_t offdiag_mask;          // classes k with some s != t, class[s][t] == k
  uint32_t row_mask[MAXG];        // classes in row s (t != s)
  uint32_t col_mask[MAXG];        // classes in column t (s != t)
};

struct RawGraph {
  int32_t V;       // op slots (dead ops included)
  int32_t n_live;  // live ops
  int64_t E;       // edge slots per side
  uint32_t *succ_off, *succ_cnt, *pred_off, *pred_cnt;
  int32_t *succ_dst, *pred_src;
  int64_t *succ_bytes, *pred_bytes;
  uint8_t *succ_param, *pred_param;
  int64_t *cost;   // V*G
  int64_t *mem, *param;
  uint8_t *split_mask, *alive;
  int32_t *topo;   // n_live, a topological order of the live ops
  // levels for the level-synchronous rank sweep (heights of the base graph;
  // a split slot keeps its base's levels and places its overlay nodes at
  // labels 4h(o)-2 (concat), 4h(o) (sub-ops), 4h(o)+2 (split nodes))
  int32_t *height;  // V: longest path (in edges) to a sink; -1 for dead ops
  int32_t *lvl_off; // H+2
  int32_t *lvl_ops; // n_live ops ordered by height
  int32_t H;        // max height
  // split overlay of a slot (ov_P < 0: none)
  int32_t ov_o, ov_base, ov_P, ov_n, ov_S;
};

struct PrepGraph {
  int32_t n;        // positions (= live ops)
  int32_t V;        // raw op slots
  int64_t E;        // live edges
  int32_t cp_len;   // written by the CP kernel
  int32_t tbits;    // 32 or 64
  int32_t topo;     // 1 iff every edge goes from a lower to a higher position (set by the card kernels)
  uint32_t *card;   // n * CARD_WORDS
  void *costp;      // n * G of T
  uint32_t *pe_src; // E: predecessor position, grouped by consumer position
  void *pe_comm;    // E * K of T: comm(bytes, k) of that edge per link class
  uint32_t *se_dst; // E: successor position, grouped by producer position
  uint32_t *se_pe;  // E: index of the same edge in pe_*
  uint32_t *npred;  // n
  uint32_t *srcbits;// ceil(n/32): positions with no predecessor
  uint32_t *srcsumm;// 33 words: summary of srcbits (bit b of word s = leaf word 32s+b nonzero), [32] = top
  uint32_t *pos;    // V: uid -> position (NONE for dead)
  uint32_t *uid;    // n: position -> uid
  uint64_t *rank;   // V: rank_u by uid (~0 for dead)
  uint32_t *cp;     // critical path (positions)
  int64_t *pmem;    // cp prefix sums of mem, cp_len+1
  int64_t *pcost;   // cp prefix sums of cost, (cp_len+1)*G
  int64_t *act;     // n: output bytes mem - param per position (liveness memory, R24)
  // scratch for the sort / scans
  uint64_t *key0, *key1;
  uint32_t *val0, *val1;
};

// the candidate record of the ABI (32 bytes)
struct Cand {
  uint8_t kind, n_pins, split_dim, split_n;
  int32_t split_op;
  int32_t pin_op[4];
  uint8_t pin_dev[4];
  uint32_t dev_mask;  // device subset (R25), 0 = all
};
static_assert(sizeof(Cand) == 32, "candidate record is 32 bytes");

// the sweep's candidate stream (R21)
struct StreamState {
  uint8_t *base_place;  // V
  int32_t *live;        // n_live uids
  int32_t n_live;
  int64_t n_split;
  int32_t n_subset;     // device-subset block after the SPLITs (R25): G-1 or 0
  int32_t *split_op;    // n_split
  uint8_t *split_dim, *split_n;
  uint64_t seed;
  int32_t kmin, kmax;
  int32_t G;
};

__host__ __device__ inline int64_t comm_class(const GraphConst &c, int64_t bytes, int k) {
  int64_t num = bytes * c.beta[k];
  return c.alpha[k] + (num + 999999) / 1000000;
}
__host__ __device__ inline uint32_t all_devices(int G) { return G >= 32 ? 0xFFFFFFFFu : ((1u << G) - 1u); }
__host__ __device__ inline int64_t ceil_div64(int64_t a, int64_t b) { return (a + b - 1) / b; }
__host__ __device__ inline int64_t part_bytes(int64_t b, int n, int k) { return b / n + (k < b % n ? 1 : 0); }

// ------------------------------------------------------------ launchers
// (defined in k_prep.cu / k_sim.cu; all asynchronous on `st`)

// base_rank (optional): rank_u of the base graph by uid; a SPLIT slot on all
// devices then copies the ranks below the split op's height instead of
// recomputing them (they have no path to the split op)
// nact (all prep launchers, nullable): device count of the active slots; the
// grid covers nslots, slots at or past *nact exit at once (a preparation
// wave sized on the device, without a host round trip)
// Level records of a base graph (k_rank's fast path): per op in level order
// (lvl_ops), its unpinned, full-device-set rank terms -- w = max cost, the
// first 4 successors and their c (R5) -- so a slot's level walk
// reads one 64-B record per op instead of recomputing them on its chain.
struct LvlRec {
  int32_t u, ns;    // op id (-1: dead), successor count
  int64_t w;
  int32_t s[4];     // successors (-1 past ns)
  int64_t c[4];
};
static_assert(sizeof(LvlRec) == 64, "level record");
void launch_lvlrec(const RawGraph *raw, const GraphConst *gc, int32_t n_live, LvlRec *out, cudaStream_t st);
// base_cost (nullable): a split slot's base-op cost rows are read from the
// base graph (the slot copy skips the cost table; the overlay rows are the
// slot's own)
void launch_rank(const RawGraph *raws, PrepGraph *pgs, const GraphConst *gc, const Cand *cands, int nslots,
                 int G, cudaStream_t st, const uint64_t *base_rank = nullptr, const uint32_t *nact = nullptr,
                 const int64_t *base_cost = nullptr, const LvlRec *lvlrec = nullptr);
void launch_heights(RawGraph *raw_dev, int32_t *scratch, int64_t vcap, cudaStream_t st);
void launch_sort(PrepGraph *pgs, const RawGraph *raws, int nslots, int key_bits, int max_n, cudaStream_t st,
                 const uint32_t *nact = nullptr);
void launch_cards(const RawGraph *raws, PrepGraph *pgs, const GraphConst *gc, int nslots, int max_n, int G, int K,
                  int tbits, cudaStream_t st, bool succ_all, const uint32_t *nact = nullptr,
                  const int64_t *base_cost = nullptr, const int64_t *base_mem = nullptr,
                  const int64_t *base_param = nullptr);
void launch_cp(const RawGraph *raws, PrepGraph *pgs, int nslots, int G, int tbits, cudaStream_t st,
               const uint32_t *nact = nullptr);
// (hole_lo, hole_hi: a byte range of the block not copied, 16-B aligned)
void launch_copy_block(const void *src, void *dst, int64_t slot_stride_bytes, int64_t bytes, const Cand *cands,
                       int nslots, cudaStream_t st, const uint32_t *nact = nullptr, int64_t hole_lo = 0,
                       int64_t hole_hi = 0);
void launch_patch_split(const RawGraph *base, RawGraph *raws, const GraphConst *gc, const Cand *cands, int nslots,
                        cudaStream_t st, const uint32_t *nact = nullptr);
void launch_bound(const RawGraph *raw, const GraphConst *gc, int G, unsigned long long *out /* [2] */,
                  cudaStream_t st);
void launch_splitlist(const RawGraph *raw, const GraphConst *gc, const uint8_t *place, int32_t *list,
                      int32_t *nlist, int64_t *scratch_rank, int32_t *scratch_cp, int G, cudaStream_t st);

struct SimOut {
  int64_t *makespan;   // per result index
  uint8_t *status;
  int64_t *peak;       // per result * G (nullable)
  uint8_t *place;      // per result * vmax (nullable)
  int64_t *start;      // per result * vmax (nullable)
  int32_t *deq;        // per result * vmax (nullable): uids in dequeue order
  int32_t vmax;
};

struct SimArgs {
  int mode;              // 0 sweep, 1 list, 2 prepared slots, 3 permuted list (slot_index/slot_result)
  uint32_t flags;
  const PrepGraph *base; // base prepared graph (modes 0, 1)
  const PrepGraph *slots;// prepared slot graphs (mode 2)
  const Cand *cands;     // mode 1: candidate list; mode 2: candidate per slot
  const int64_t *slot_result; // mode 2: result index per slot
  const int64_t *slot_index;  // mode 2: stream index per slot (sweep bests)
  const GraphConst *gc;
  const uint8_t *split_mask; // raw split masks of the base graph (validation)
  StreamState stream;    // mode 0
  int64_t first, n, stride;
  unsigned long long *counter;  // work counter
  int64_t *defer_q;      // deferred work items (q)
  unsigned long long *ndefer;
  int64_t *wbest;        // per candidate slot (makespan, index) pairs
  SimOut out;
  void *slab;            // per-warp state slabs
  int64_t slab_stride;   // elements (records) per warp
  int32_t leaf_words;    // ready-bitmap leaf words per candidate (smem)
  int32_t bm_stride;     // smem words per candidate: leaf_words + 32 summary words, padded
  int32_t G;
  int32_t gshift;        // ceil(log2(G)): lanes per predecessor group = 1 << gshift
  int32_t track_best;
  int32_t need_mem;      // track per-device memory (caps present or peak output)
  int32_t live_mem;      // liveness memory (R24, FASTT_F_MEM_LIVE); implies need_mem
  int32_t fastcomm;      // uint32 time and one link class: comm values inline in the cards
  int32_t topo;          // the graph's priority order is topological: dequeue order = position order
  int32_t lane;          // run the lane-per-candidate position-order kernel (k_sim_lane)
  int32_t gc_K;          // link classes (host copy of GraphConst::K)
  int32_t slot_filter;   // mode 2: 0 all slots, 1 only slots with a topological order, 2 only the others
  int32_t cap_check;     // some device has a finite memory cap (R8)
  // BASE-schedule prefix sharing: 1 = record the snapshot (one BASE run),
  // 2 = start eligible PIN candidates from it at their first pinned op
  int32_t snap_mode;
  int32_t snap_round_dev;  // device of the base's single CP round covering the whole CP, else -1
  uint32_t *snap_dq;       // [n] dequeue index of each position in the BASE schedule
  void *snap_avail;        // [(n+1)*G] T: avail[d] before step t
  void *snap_ms;           // [n+1] T: makespan before step t
  void *snap_rec;          // [n] final slab records of the BASE schedule
  int32_t *snap_rounds;    // [4] base CP rounds: count, dev0, lo0, hi0 (written when recording)
  // INSERT policy (R1i, NEXT N1): idle-slot arrays (GapSlot<T>) per
  // candidate slot and device, sorted by start,
  // gap_stride entries each; INSERT launches use at most ins_grid blocks
  int32_t ins;
  void *gap;
  int64_t gap_stride;
  int32_t ins_grid;
  // packed device keys of the lane kernel (k_sim_lane PK): cost rows
  // (cost << gshift) | d of the base graph, and the makespan at or above
  // which a candidate is deferred (0 = packed keys off)
  const uint32_t *costk;
  const uint32_t *commk;  // [n][4] inline predecessors' comm << gshift (PK, one class)
  const uint32_t *pkc;    // [n][pk_card_words] compact PK cards (k_lane_pk.cuh)
  uint32_t pk_lim;
  // memory mode of the lane kernel: 0 none, 1 per-device peak, 2 finite caps
  int32_t lane_mm;
  // BASE snapshot memory before step t ([(n+1)*G] int64, recorded with the
  // snapshot): used[d], and used[d] + reserved[d]
  void *snap_used;
  void *snap_ur;
  const uint32_t *snap_key;  // [n] BASE records as packed keys (PK records)
  // the list was classified by launch_t0_sort (deferred candidates sorted to
  // its tail): the kernel skips its own rank-change test and processes the
  // first *n_dev entries (n_dev nullable: a.n)
  int32_t preclassified;
  const uint32_t *n_dev;
  // k_sim_lane instrumentation (nullable): [0] += steps per warp batch,
  // [1] += steps of the batch's running lanes
  unsigned long long *stat;
  // k_lane_pk non-persistent mode (lane_batches > 0): a warp takes at most
  // lane_batches batches of 32 candidates, holding one of n_slab_slots slab
  // columns (and wbest entries) acquired from the bitmap slot_bm for its
  // lifetime, so the launch's blocks retire while it runs and a concurrent
  // higher-priority stream (the preparation pipeline) gets SM resources
  int32_t lane_batches;
  int32_t n_slab_slots;
  uint32_t *slot_bm;
  // set when a ready-set launch meets a graph above READY_SET_MAX positions
  // (the call then fails with FASTT_EUNSUP)
  unsigned *err;
  // INSERT on the lane kernel: per lane and device gap_cap idle slots
  void *gap_lane;
  int32_t gap_cap;
  // k_lane_pk with two candidates per lane: the BASE keys doubled ([2n],
  // key s at words 2s and 2s + 1, so an aligned 8-B load gives it to both)
  const uint32_t *snap_key2;
  const uint32_t *snap_key4;  // ... and four times ([4n], CPL 4)
  int32_t pk_cpl;  // candidates per lane of the k_lane_pk launch (1 or 2)
  int32_t gwarp_off;  // persistent k_lane_pk: first slab column block / wbest entry of this launch
  int32_t pk_wpb;     // k_lane_pk: warps per block (1, 2 or 4; 0 = 4)
};

// one idle slot [a, b) of a device under INSERT
template <typename T> struct GapSlot {
  T a, b;
};

void launch_sim(const SimArgs &a, int tbits, int grid, int block, size_t smem, cudaStream_t st);
// per-GSH kernel getters (k_sim_inst.cu / k_sim_lane_inst.cu, compiled once
// per lane-group width so the template instances build in parallel)
#define FASTT_CAT2(a, b) a##b
#define FASTT_CAT(a, b) FASTT_CAT2(a, b)
#define FASTT_DECL_SIM_FN(N) const void *sim_fn_g##N(int tbits, bool mem, bool ins, bool fc, bool topo);
FASTT_DECL_SIM_FN(0) FASTT_DECL_SIM_FN(1) FASTT_DECL_SIM_FN(2) FASTT_DECL_SIM_FN(3) FASTT_DECL_SIM_FN(4)
FASTT_DECL_SIM_FN(5)
#undef FASTT_DECL_SIM_FN
#define FASTT_DECL_LANE_FN(N, M) const void *lane_fn_g##N##_m##M(int tbits, int cm, bool exact, bool mg, bool pk);
#define FASTT_DECL_PK_FN(N) const void *lane_pk_fn_g##N(int mm, bool exact, int cpl); \
  const void *lane_ins_fn_g##N(int tbits, int cm, bool exact);
FASTT_DECL_PK_FN(0) FASTT_DECL_PK_FN(1) FASTT_DECL_PK_FN(2) FASTT_DECL_PK_FN(3) FASTT_DECL_PK_FN(4) FASTT_DECL_PK_FN(5)
#undef FASTT_DECL_PK_FN
#define FASTT_DECL_LANE_FN3(N) FASTT_DECL_LANE_FN(N, 0) FASTT_DECL_LANE_FN(N, 1) FASTT_DECL_LANE_FN(N, 2)
FASTT_DECL_LANE_FN3(0) FASTT_DECL_LANE_FN3(1) FASTT_DECL_LANE_FN3(2) FASTT_DECL_LANE_FN3(3) FASTT_DECL_LANE_FN3(4)
FASTT_DECL_LANE_FN3(5)
#undef FASTT_DECL_LANE_FN3
#undef FASTT_DECL_LANE_FN
void launch_argmin(const int64_t *wbest, int64_t nwarps, int64_t *best_dev, cudaStream_t st);
void launch_order_chunk(const int32_t *deq, const int64_t *start, int32_t *order, const int64_t *results, int64_t n,
                        int64_t vmax, int key_bits, uint64_t *k0, uint64_t *k1, uint32_t *v0, uint32_t *v1,
                        cudaStream_t st);
void launch_candgen(const StreamState &s, int64_t first, int64_t n, Cand *out, cudaStream_t st);
void launch_candgen_idx(const StreamState &s, int64_t first, int64_t stride, const int64_t *qlist, int64_t n,
                        Cand *out, int64_t *out_index, cudaStream_t st);
void launch_slot_setup(const Cand *cands, const RawGraph *tmpl, const RawGraph *base, RawGraph *raws, int nslots,
                       cudaStream_t st);
void launch_gather_cands(const Cand *src, const int64_t *idx, int64_t n, Cand *dst, int64_t *res, cudaStream_t st);
// Bucket-sort the candidates by BASE-prefix start step.  With `classify`
// (base PrepGraph pg, time bits tbits), candidates that need their own
// prepared graph (cand_classify) go to one extra bucket at the tail and
// *n_main receives the count of the others.
struct T0Classify {
  int on;
  int tbits;
  const PrepGraph *pg;
  const GraphConst *gc;
  const uint8_t *split_mask;
  uint32_t *n_main;
};
void launch_t0_sort(int from_stream, const StreamState &S, int64_t first, int64_t stride, const Cand *list, int64_t n,
                    const uint32_t *pos, const uint32_t *snap_dq, int32_t nops, int32_t vraw, int G, Cand *tmp_c,
                    int64_t *tmp_i, uint32_t *key, uint32_t *hist, Cand *out_c, int64_t *out_i, int64_t *out_res,
                    cudaStream_t st, T0Classify cl = T0Classify{0, 0, nullptr, nullptr, nullptr, nullptr});
void launch_gather_tail(const Cand *src, const int64_t *sidx, const int64_t *sres, const uint32_t *n_main, int64_t n,
                        int64_t off, int cap, Cand *dst, int64_t *didx, int64_t *dres, uint32_t *nslot,
                        cudaStream_t st);
void launch_init_best(int64_t *wb, int64_t nw, cudaStream_t st);
void launch_gather_sorted(const Cand *src, const int64_t *sidx, const int64_t *sres, const int64_t *qs, int64_t n,
                          Cand *dst, int64_t *didx, int64_t *dres, cudaStream_t st);
// Device-driven deferral loop (the ABI's asynchronous contract, fastt.h):
// the candidates a main launch hands to the preparation pipeline -- the
// tail of a classified sorted list past the arena (phase 0) and the
// deferral queue defer_q[0 .. *ndefer) (phase 1) -- are gathered into the
// arena in rounds of at most cap slots by a CUDA-graph WHILE node whose
// condition the kernels below set on the device, so no host round trip
// decides how many rounds run.
struct DeferBlock {
  // per call (k_defer_setup)
  int64_t n;            // sorted list length (phase 0 source)
  int32_t cap;          // arena slots per round
  int32_t src;          // phase-1 source: 0 sorted list, 1 candidate list (cands), 2 the stream
  int32_t do_tail;      // phase 0 runs (overlapped path)
  int32_t results;      // slot_result gets the result index (schedule_batch), else slot_index the stream index
  const Cand *cands;    // src 1
  StreamState ss;       // src 2
  int64_t first, stride;
  // k_defer_begin
  int64_t n_main;       // classified main-list length (do_tail), else -1
  int64_t tail_lo;      // first tail position (n_main + cap)
  int64_t n_defer;      // *ndefer when the loop starts
  int64_t total;        // candidates the loop evaluates (tail + deferrals)
  // cursor (k_defer_plan)
  int32_t phase;
  uint32_t nact;        // slots of this round (the preparation kernels' device count)
  int64_t off;          // consumed entries of the current phase
  int64_t q_lo, q_cnt;  // this round: positions (phase 0) or defer_q entries (phase 1)
  int32_t q_phase;      // this round's phase
};
void launch_defer_setup(DeferBlock *blk, int64_t n, int cap, int src, int do_tail, int results, const Cand *cands,
                        const StreamState &ss, int64_t first, int64_t stride, cudaStream_t st);
void launch_defer_begin(DeferBlock *blk, const uint32_t *n_main, const unsigned long long *ndefer,
                        cudaGraphConditionalHandle h, cudaStream_t st);
void launch_defer_plan(DeferBlock *blk, cudaGraphConditionalHandle h, cudaStream_t st);
void launch_defer_gather(const DeferBlock *blk, int cap, const Cand *srt_c, const int64_t *srt_i,
                         const int64_t *srt_res, const int64_t *defer_q, Cand *dst, int64_t *didx, int64_t *dres,
                         cudaStream_t st);
int sim_occupancy(int tbits, int gshift, int block, size_t smem, bool topo);
void launch_sim_lane(const SimArgs &a, int tbits, int grid, cudaStream_t st);
int lane_occupancy(int tbits, int gshift, int mm, bool pk, int cpl = 1, int wpb = 4);
void lane_pk_attrs(int gshift, int mm, int cpl, char *buf, size_t len);
// costk[p][d] = (cost[p][d] << gshift) | d over n positions; mx[0] = max
// cost, mx[1] = max edge comm (one link class) of the prepared graph
void launch_pack_costs(const PrepGraph *pg_dev, int32_t n, int G, int gshift, int64_t E, uint32_t *costk,
                       uint32_t *commk, uint32_t *pkc, unsigned long long *mx, cudaStream_t st);
// words of one compact PK card (k_lane_pk.cuh)
int pk_card_words_host(int gshift);
// BASE records (uint32 time: FT | place << 32) -> packed keys FT << gshift | place
void launch_snap_keys(const void *rec, int32_t n, int gshift, uint32_t *key, uint32_t *key2, uint32_t *key4,
                      cudaStream_t st);
void launch_fit(int G, int64_t n, const uint8_t *src, const uint8_t *dst, const int64_t *bytes, const int64_t *tns,
                void *sums, unsigned *err, int64_t *alpha, int64_t *beta, int64_t *count, int sms, cudaStream_t st);
size_t fit_sums_bytes(int G);
// computation cost table (N4): scratch = 16 * n_ops * G bytes
void launch_cost_table(int32_t V, int G, int64_t n, const int32_t *op, const uint8_t *dev, const int64_t *tns,
                       void *scratch, unsigned *err, int64_t *cost, int sms, cudaStream_t st);
cudaError_t sim_set_smem(int tbits, int gshift, size_t smem);
void launch_fill_i64(int64_t *p, int64_t n, int64_t v, cudaStream_t st);
void launch_iota_i64(int64_t *p, int64_t n, cudaStream_t st);

}  // namespace fastt
