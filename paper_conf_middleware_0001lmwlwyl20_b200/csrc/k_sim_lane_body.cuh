// k_sim_lane_body.cuh -- the lane-per-candidate position-order kernel
// (k_sim_lane) and its staging helpers; overview in k_sim_lane.cu.  Included
// by k_sim_lane_inst.cu, compiled once per device-count width GSH
// (build.py: -DFASTT_GSH=0..5), and by k_sim_lane.cu for the layout
// constants (no instances there).
#pragma once
#include "fastt_internal.cuh"
#include "sim_common.cuh"

namespace fastt {

// pipeline depth: records of positions at distance <= D-1 are read from the
// shared-memory ring of the last D records; older ones are staged by
// cp.async D-1 steps ahead (SLAB records are 8 B for 32-bit time, 16 B else)
#ifndef LANE_D
#define LANE_D 8
#endif
template <typename T> struct LaneDepth { static constexpr int D = sizeof(T) == 4 ? LANE_D : LANE_D / 2; };
// staged card of one position: header (words 0-3), predecessor positions
// (words 8-11), the inline predecessors' comm values (4 x T), with memory
// tracking (MM > 0) header words 4-7 (mem lo/hi), then the cost row padded
// to 16 B
template <typename T> __host__ __device__ constexpr int card_hdr1_off() { return 32 + 4 * (int)sizeof(T); }
template <typename T, int MM> __host__ __device__ constexpr int card_cost_off() {
  return card_hdr1_off<T>() + (MM ? 16 : 0);
}
template <typename T, int GP, int MM> __host__ __device__ constexpr int card_slot_bytes() {
  return card_cost_off<T, MM>() + (int)((GP * sizeof(T) + 15) / 16) * 16;
}
// MG: per-lane card regions are 2D slots + 16 B apart, so the 8 lanes of a
// 128-bit shared-memory phase hit distinct bank quads (a 2D x CS stride is a
// multiple of 128 B: every lane's card load would fall in the same banks)
template <typename T, int GP, int MM> __host__ __device__ constexpr int mg_lane_stride() {
  return 2 * LaneDepth<T>::D * card_slot_bytes<T, GP, MM>() + 16;
}
// bytes of one slab record: FT | place (8 B for 32-bit time, 16 B else), or
// under packed keys the key FT << GSH | place itself (4 B)
template <typename T, bool PK> __host__ __device__ constexpr int lane_rec_bytes() {
  return PK ? 4 : (sizeof(T) == 4 ? 8 : 16);
}
// offset of the memory-tracking area in a warp's shared memory
template <typename T, int GP, bool MG, int MM, bool PK = false> __host__ __device__ constexpr size_t lane_mm_off() {
  return (size_t)LaneDepth<T>::D * 5 * 32 * lane_rec_bytes<T, PK>() +
         (MG ? (size_t)32 * mg_lane_stride<T, GP, MM>() : (size_t)2 * LaneDepth<T>::D * card_slot_bytes<T, GP, MM>()) +
         (size_t)(MG ? 0 : 32 * GP * 4);
}
template <typename T, int GP, bool MG, int MM, bool PK = false>
__host__ __device__ constexpr size_t lane_smem_per_warp() {
  // ring D x 32 + stage D x 4 x 32 records, then 2D staged cards (per lane
  // in the multi-graph variant), then (base-graph launches) the packed-key
  // avail rows [32 lanes][GP] of the PK variant, then the memory state:
  // MM 1 used[d] (int64 [GP][32]); MM 2 slack[d] = cap - used - reserved
  // (int64 [GP][32]), its clamped 32-bit copy (quads [GP/4][32][4]) and the
  // CP rounds ([GP][32] u32)
  return lane_mm_off<T, GP, MG, MM, PK>() + (MM >= 1 ? (size_t)32 * GP * 8 : 0) + (MM == 2 ? (size_t)32 * GP * 8 : 0);
}

template <int BYTES> __device__ __forceinline__ void cp_async(uint32_t saddr, const void *g);
template <> __device__ __forceinline__ void cp_async<4>(uint32_t saddr, const void *g) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(saddr), "l"(g) : "memory");
}
template <> __device__ __forceinline__ void cp_async<8>(uint32_t saddr, const void *g) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(saddr), "l"(g) : "memory");
}
template <> __device__ __forceinline__ void cp_async<16>(uint32_t saddr, const void *g) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(saddr), "l"(g) : "memory");
}
// predicated form: the copy is issued iff p
template <int BYTES> __device__ __forceinline__ void cp_async_if(bool p, uint32_t saddr, const void *g);
#define FASTT_CP_ASYNC_IF(BYTES, CACHE)                                                                    \
  template <> __device__ __forceinline__ void cp_async_if<BYTES>(bool p, uint32_t saddr, const void *g) {  \
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %2, 0;\n\t@q cp.async." CACHE                       \
                 ".shared.global [%0], [%1], " #BYTES ";\n}\n" ::"r"(saddr),                                \
                 "l"(g), "r"((int)p)                                                                        \
                 : "memory");                                                                               \
  }
FASTT_CP_ASYNC_IF(4, "ca")
FASTT_CP_ASYNC_IF(8, "ca")
FASTT_CP_ASYNC_IF(16, "cg")
#undef FASTT_CP_ASYNC_IF
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N> __device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

template <typename T> struct RowLd;
template <> struct RowLd<uint32_t> {
  template <int GP>
  __device__ static void load_s(const uint32_t *row, int G, uint32_t (&c)[GP]) {  // shared memory, 16-B aligned
    if (GP >= 4) {
#pragma unroll
      for (int j = 0; j < GP / 4; j++) {
        const uint4 x = ((const uint4 *)row)[j];
        c[4 * j] = x.x;
        c[4 * j + 1] = x.y;
        c[4 * j + 2] = x.z;
        c[4 * j + 3] = x.w;
      }
    } else {
#pragma unroll
      for (int d = 0; d < GP; d++) c[d] = row[d];
    }
  }
  template <int GP>
  __device__ static void load(const uint32_t *row, int G, uint32_t (&c)[GP]) {
    if (GP >= 4 && G == GP) {
#pragma unroll
      for (int j = 0; j < GP / 4; j++) {
        const uint4 x = __ldg((const uint4 *)row + j);
        c[4 * j] = x.x;
        c[4 * j + 1] = x.y;
        c[4 * j + 2] = x.z;
        c[4 * j + 3] = x.w;
      }
    } else {
#pragma unroll
      for (int d = 0; d < GP; d++) c[d] = d < G ? __ldg(row + d) : 0u;
    }
  }
};
template <> struct RowLd<uint64_t> {
  template <int GP>
  __device__ static void load_s(const uint64_t *row, int G, uint64_t (&c)[GP]) {
    if (GP >= 2) {
#pragma unroll
      for (int j = 0; j < GP / 2; j++) {
        const ulonglong2 x = ((const ulonglong2 *)row)[j];
        c[2 * j] = x.x;
        c[2 * j + 1] = x.y;
      }
    } else {
      c[0] = row[0];
    }
  }
  template <int GP>
  __device__ static void load(const uint64_t *row, int G, uint64_t (&c)[GP]) {
    if (GP >= 2 && G == GP) {
#pragma unroll
      for (int j = 0; j < GP / 2; j++) {
        const ulonglong2 x = __ldg((const ulonglong2 *)row + j);
        c[2 * j] = x.x;
        c[2 * j + 1] = x.y;
      }
    } else {
#pragma unroll
      for (int d = 0; d < GP; d++) c[d] = d < G ? __ldg(row + d) : 0ull;
    }
  }
};

// CP devices under memory caps (Alg. 1 line 5, R9),
// one candidate per lane: repeatedly give the device with the smallest exact
// average cost (cross-multiplied, ties lowest id) the longest prefix of the
// remaining free CP ops that fits its cap, reserve that memory up front
// (slack[d] -= the prefix's mem), and drop the device; perturbation-pinned CP
// ops are excluded (free-index space).  Round r is stored as rnd[r * 32] =
// (raw CP index just past its last op) | device << 24; returns the count.
template <typename T>
__device__ __noinline__ int cp_rounds_lane(const PrepGraph *pg, const GraphConst &gc, int G, uint32_t dset, int np,
                                           const uint32_t *pp, const uint32_t *pc, uint32_t *rnd, int64_t *mv) {
  const T *costp = (const T *)pg->costp;
  const uint32_t *card = pg->card;
  const int32_t L = pg->cp_len;
  uint32_t pcs[MAXPINS], pps[MAXPINS];
  int64_t pms[MAXPINS];
  int m = 0;
  for (int k = 0; k < np; k++) {
    if (pc[k] == NONE) continue;
    const uint32_t *ci = card + (size_t)pp[k] * CARD_WORDS;
    const int64_t mk = (int64_t)(((uint64_t)ci[CW_MEMHI] << 32) | ci[CW_MEMLO]);
    int j = m++;
    while (j > 0 && pcs[j - 1] > pc[k]) {
      pcs[j] = pcs[j - 1];
      pps[j] = pps[j - 1];
      pms[j] = pms[j - 1];
      j--;
    }
    pcs[j] = pc[k];
    pps[j] = pp[k];
    pms[j] = mk;
  }
  auto raw_end = [&](int32_t f) -> int32_t {  // raw CP index just past the f-th free op (f >= 1)
    int32_t r = f - 1;
    for (int j = 0; j < m; j++)
      if ((int32_t)pcs[j] <= r) r++;
    return r + 1;
  };
  auto fp_mem = [&](int32_t f) -> int64_t {
    if (f <= 0) return 0;
    const int32_t re = raw_end(f);
    int64_t v = pg->pmem[re];
    for (int j = 0; j < m; j++)
      if ((int32_t)pcs[j] < re) v -= pms[j];
    return v;
  };
  auto fp_cost = [&](int32_t f, int d) -> int64_t {
    if (f <= 0) return 0;
    const int32_t re = raw_end(f);
    int64_t v = pg->pcost[(int64_t)re * G + d];
    for (int j = 0; j < m; j++)
      if ((int32_t)pcs[j] < re) v -= (int64_t)costp[(size_t)pps[j] * G + d];
    return v;
  };
  const int32_t Lf = L - m;
  uint32_t devs = dset;
  int32_t k = 0;
  int nr = 0;
  while (k < Lf && devs) {
    const int64_t bm = fp_mem(k), rest = fp_mem(Lf) - bm;
    int best = -1;
    int32_t tb = 0;
    int64_t Sb = 0;
    for (int d = 0; d < G; d++) {
      if (!((devs >> d) & 1u)) continue;
      const int64_t cap = gc.cap[d];
      int32_t t;
      if (rest <= cap) {
        t = Lf - k;
      } else {  // fp(k + lo) - bm <= cap < fp(k + hi) - bm
        int32_t lo = 0, hi = Lf - k;
        while (hi - lo > 1) {
          const int32_t mid = (lo + hi) >> 1;
          if (fp_mem(k + mid) - bm <= cap) lo = mid;
          else hi = mid;
        }
        t = lo;
      }
      if (t <= 0) continue;
      const int64_t S = fp_cost(k + t, d) - fp_cost(k, d);
      if (best < 0 || lt_cross((uint64_t)S, (uint64_t)tb, (uint64_t)Sb, (uint64_t)t)) {
        best = d;
        tb = t;
        Sb = S;
      }
    }
    if (best < 0) break;
    mv[best * 32] -= fp_mem(k + tb) - bm;
    rnd[nr * 32] = (uint32_t)raw_end(k + tb) | ((uint32_t)best << 24);
    devs &= ~(1u << best);
    k += tb;
    nr++;
  }
  return nr;
}

// CM: 0 = uint32 time and one link class, comm values inline in the card;
//     1 = one link class, comm per edge from pe_comm;
//     2 = several link classes (per (pred, device) comm).
// EX: G == GP (no per-device range checks).
// MG: multi-graph -- lane l simulates prepared slot q0 + l (mode 2: SPLIT and
//     rank-changing candidates, each with its own priority order, so cards
//     are staged per lane); launched with one warp per block.
// PK: packed device keys (32-bit time, one link class, base graph): the EFT
//     of device d is carried as the key (EFT << GSH) | d, so the argmin with
//     ties to the lowest device (Alg. 1 lines 12-19, R3) is a plain unsigned
//     min (3-input VIMNMX3), the cost row is pre-packed (costk = cost << GSH
//     | d), avail[d] << GSH lives in a per-lane shared-memory row so the
//     chosen device's update and the arrival on the predecessor device pa
//     (R6) are one indexed store / load instead of a select per device.
//     Exact while every key fits 32 bits: EFT <= makespan + max comm + max
//     cost at every step, so a candidate whose final makespan reaches
//     pk_lim = 2^(32-GSH) - max cost - max comm is deferred and re-run by the
//     preparation pipeline (unpacked kernels).
// MM: memory (Alg. 1 line 13, R8): 0 none; 1 per-device peak only (no caps:
//     used[d] += mem of every op placed on d); 2 finite caps -- lane-local CP
//     rounds (R9, memory reserved up front), slack[d] = cap - used - reserved
//     per lane, a device is feasible iff mem_i <= slack[d] (a CP-pinned op
//     draws on its reservation), no feasible device => INFEASIBLE.
// INS: the insertion policy (R1i; NEXT N1) -- lane l keeps, per
//     device, the device's positive-length idle slots as an array sorted by
//     start in global memory (a.gap_lane, gap_cap slots per device); EST on
//     d is the arrival when it is at or after avail[d], else the first slot
//     [a, b) ending after the arrival r with max(a, r) + w <= b (binary
//     search + short scan, as k_sim), else avail[d].  A lane whose device
//     would need more than gap_cap slots is deferred to the group kernel.
//     (base graph, no memory mode, no packed keys)
template <typename T, int GSH, int CM, bool EX, bool MG, bool PK, int MM, bool INS = false>
__global__ void __launch_bounds__(LANE_BLOCK, LANE_MINB) k_sim_lane(SimArgs a) {
  static_assert(!INS || (!MG && !PK && MM == 0), "INSERT lanes: base graph, plain keys, no memory mode");
  // slab / ring / stage record: FT | place, or the packed key (PK)
  typedef typename std::conditional<PK, uint32_t, typename Slab<T>::W>::type W;
  constexpr int GP = 1 << GSH;
  static_assert(!PK || (sizeof(T) == 4 && CM != 2 && !MG), "packed keys: 32-bit time, one link class, base graph");
  static_assert(CM != 0 || sizeof(T) == 4, "card comm values are uint32");
  const int lane = threadIdx.x & 31;
  const int64_t gwarp = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  // this lane's slab column: record of position p at col[p * 32]
  W *const col = (W *)a.slab + (size_t)gwarp * (size_t)a.slab_stride * 32 + lane;
  // shared memory of this warp: ring[D][32] (records of the last D positions)
  // and stage[D][4][32] (inline predecessors' records prefetched by cp.async)
  constexpr int D = LaneDepth<T>::D, P = D - 1;
  extern __shared__ __align__(16) unsigned char lsm[];
  unsigned char *const wsm = lsm + (threadIdx.x >> 5) * lane_smem_per_warp<T, GP, MG, MM, PK>();
  W *const ring = (W *)wsm + lane;
  W *const stage = ring + D * 32;
  const uint32_t stage_sa = (uint32_t)__cvta_generic_to_shared(stage);
  // 2D staged cards (warp-shared): the card of position u is copied at step
  // u - 2P and read at steps u - P (record prefetch) and u (compute)
  constexpr int CS = card_slot_bytes<T, GP, MM>();
  const unsigned char *const cards = wsm + (size_t)D * 5 * 32 * sizeof(W) + (MG ? (size_t)lane * mg_lane_stride<T, GP, MM>() : 0);
  const uint32_t cards_sa = (uint32_t)__cvta_generic_to_shared(cards);
  // PK: avail[d] << GSH of every lane, after the warp's cards, as device
  // pairs [d / 2][32 lanes][2] (a pair per lane is one 64-bit access; the
  // indexed access of device d by all lanes is 2-way conflicted at most)
  uint32_t *const avk = (uint32_t *)(wsm + (size_t)D * 5 * 32 * sizeof(W) + (size_t)2 * D * CS) +
                        (GP >= 2 ? 2 * lane : lane);
  auto avk_at = [&](uint32_t d) -> uint32_t & { return GP >= 2 ? avk[(d >> 1) * 64 + (d & 1)] : avk[0]; };
  // memory state (MM): mv[d * 32] = used[d] (MM 1) or slack[d] (MM 2), int64;
  // MM 2: s32 = min(slack, 2^32 - 1) as quads [d / 4][32 lanes][4] (one
  // 128-bit load per 4 devices), rnd[r * 32] = CP round r: raw CP index just
  // past the round | device << 24
  int64_t *const mv = (int64_t *)(wsm + lane_mm_off<T, GP, MG, MM, PK>()) + lane;
  uint32_t *const s32b = (uint32_t *)(wsm + lane_mm_off<T, GP, MG, MM, PK>() + (size_t)32 * GP * 8) + (GP >= 4 ? 4 * lane : lane);
  uint32_t *const rnd = (uint32_t *)(wsm + lane_mm_off<T, GP, MG, MM, PK>() + (size_t)32 * GP * 12) + lane;
  auto s32_at = [&](uint32_t d) -> uint32_t & { return GP >= 4 ? s32b[(d >> 2) * 128 + (d & 3)] : s32b[d * 32]; };
  auto clamp32 = [](int64_t v) -> uint32_t { return v >= (int64_t)0xFFFFFFFFll ? 0xFFFFFFFFu : (uint32_t)v; };
  constexpr int CO = card_cost_off<T, MM>();
  constexpr int HO = card_hdr1_off<T>();
  const bool row16 = (a.G * (int)sizeof(T)) % 16 == 0;
  // this lane's 16-B chunk of a card copy: lane 0 header (words 0-3), lane 1
  // predecessor positions (8-11), lane 2 comm (12-15, CM 0), lane 3 header
  // words 4-7 (MM), lanes C0.. the cost row (when its length is a multiple
  // of 16 B, else element-wise)
  constexpr int C0 = MM ? 4 : 3;
  const bool cc_cost = lane >= C0;
  const uint32_t cc_src = lane == 0   ? 0u
                          : lane == 1 ? 4u * CARD_HDR
                          : lane == 2 ? 4u * CW_PCOMM
                          : (MM && lane == 3) ? 16u
                                              : 16u * (lane - C0);
  const uint32_t cc_dst = lane < 3 ? 16u * lane : (MM && lane == 3) ? (uint32_t)HO : (uint32_t)CO + 16u * (lane - C0);
  const bool cc_on = lane < 2 || (lane == 2 && CM == 0) || (MM && lane == 3) ||
                     (lane >= C0 && lane - C0 < a.G * (int)sizeof(T) / 16);
  const GraphConst &gc = *a.gc;
  const int G = a.G;
  const int K = gc.K;
  // the graph (per candidate in the multi-graph variant)
  const PrepGraph *pg = MG ? a.slots : a.base;
  const uint32_t *card = pg->card;
  const T *costp = (const T *)pg->costp;
  const T *costsrc = PK ? (const T *)a.costk : costp;  // the cost rows staged with the cards
  const T *pe_comm = (const T *)pg->pe_comm;
  const uint32_t *pe_src = pg->pe_src;
  const uint32_t *posm = pg->pos;
  int32_t n = pg->n, Vraw = pg->V, cpl = pg->cp_len;
  const W *__restrict__ snap = PK ? (const W *)a.snap_key : (const W *)a.snap_rec;
  const bool cp_on = (a.flags & 1u) != 0;
  const uint32_t all = all_devices(G);
  int64_t bms = I64MAX, bidx = -1;  // this lane's best (makespan, stream index) for the sweep argmin

  // work items: a.n, or the device count of a list classified / gathered on
  // the device (n_dev)
  const int64_t nlim = a.n_dev ? ((int64_t)*a.n_dev < a.n ? (int64_t)*a.n_dev : a.n) : a.n;
  for (;;) {
    unsigned long long q0 = 0;
    if (lane == 0) q0 = atomicAdd(a.counter, 32ull);
    q0 = __shfl_sync(FULL, q0, 0);
    if ((int64_t)q0 >= nlim) break;
    const int64_t q = (int64_t)q0 + lane;
    bool active = q < nlim;
    Cand c;
    c.kind = 0;
    c.n_pins = 0;
    c.split_op = -1;
    c.dev_mask = 0;
    int64_t res_idx = -1, sidx = q;
    if (MG) {
      pg = a.slots + (active ? q : (int64_t)q0);
      card = pg->card;
      costp = (const T *)pg->costp;
      pe_comm = (const T *)pg->pe_comm;
      pe_src = pg->pe_src;
      posm = pg->pos;
      n = pg->n;
      Vraw = pg->V;
      cpl = pg->cp_len;
      if (active) {
        c = a.cands[q];
        res_idx = a.slot_result ? a.slot_result[q] : -1;
        sidx = a.slot_index ? a.slot_index[q] : q;
        if (a.slot_filter == 1 && !pg->topo) active = false;  // (the ready-set launch takes it)
      }
      if (!active) n = 0;
    } else if (active) {
      if (a.mode == 0) {
        sidx = a.first + q * a.stride;
        c = stream_cand(a.stream, sidx);
      } else if (a.mode == 1) {
        c = a.cands[q];
        res_idx = q;
      } else {  // mode 3: list ordered by BASE-prefix start step
        c = a.cands[q];
        res_idx = a.slot_result ? a.slot_result[q] : -1;
        sidx = a.slot_index[q];
      }
    }

    // ---------------------------------------------------------- validate
    int np = 0;
    uint8_t st = 0;
    bool defer = false;
    if (MG) {
      np = (active && c.kind == 1) ? c.n_pins : 0;  // (validated by the classification)
    } else if (active) {
      // (a pre-classified list holds no candidate that needs its own graph)
      defer = cand_classify<T>(c, pg, gc, a.split_mask, G, !a.preclassified, st);
      np = (st == 0 && c.kind == 1) ? c.n_pins : 0;
    }
    uint32_t pp[MAXPINS] = {NONE, NONE, NONE, NONE};
    uint32_t pdv = 0;
    if (active && !defer)
      for (int k = 0; k < np; k++) {
        pp[k] = posm[c.pin_op[k]];
        pdv |= (uint32_t)c.pin_dev[k] << (8 * k);
      }
    if (active && defer) {
      const unsigned long long k = atomicAdd(a.ndefer, 1ull);
      a.defer_q[k] = q;
    }
    if (active && !defer && st && res_idx >= 0) {
      a.out.makespan[res_idx] = I64MAX;
      a.out.status[res_idx] = st;
      if (MM && a.out.peak)
        for (int d = 0; d < G; d++) a.out.peak[res_idx * G + d] = -1;
    }
    const bool run = active && !defer && st == 0;

    // ------------------------------------------------------ prologue
    // CP devices (Alg. 1 line 5, R9) without memory caps: one
    // round over the free CP ops (perturbation-pinned CP ops excluded)
    int r_dev = -1;
    int m = 0;
    // MM 2: CP rounds (count, cursor, raw end and device of the current one)
    int nr = 0, rc = 0, rdv = -1;
    uint32_t rhi = 0;
    bool dead = false;  // MM 2: no feasible device at some step (R8)
    // INS: idle-slot counts per device, and an overflow flag (defer the lane)
    uint32_t gn[GP];
    bool ovf = false;
#pragma unroll
    for (int d = 0; d < GP; d++) gn[d] = 0;
    GapSlot<T> *const gbase =
        INS ? (GapSlot<T> *)a.gap_lane + ((size_t)gwarp * 32 + lane) * (size_t)GP * (size_t)a.gap_cap : nullptr;
    const uint32_t dmask = (MG && c.dev_mask) ? c.dev_mask : all;  // the candidate's devices (R25)
    if (MM && run) {
#pragma unroll
      for (int d = 0; d < GP; d++) mv[d * 32] = (MM == 2 && d < G) ? gc.cap[d] : 0;
    }
    if (run && cp_on && cpl > 0) {
      uint32_t pc[MAXPINS];
#pragma unroll
      for (int k = 0; k < MAXPINS; k++) {
        pc[k] = k < np ? __ldg(card + (size_t)pp[k] * CARD_WORDS + CW_CPIDX) : NONE;
        m += pc[k] != NONE;
      }
      if (MM == 2) {
        nr = cp_rounds_lane<T>(pg, gc, G, dmask, np, pp, pc, rnd, mv);
        if (nr > 0) {
          rhi = rnd[0] & 0xFFFFFFu;
          rdv = (int)(rnd[0] >> 24);
        }
      } else if (cpl - m > 0) {
        int64_t bs = 0;
        for (int d = 0; d < G; d++) {
          if (MG && !((dmask >> d) & 1u)) continue;
          int64_t s = pg->pcost[(int64_t)cpl * G + d];
#pragma unroll
          for (int k = 0; k < MAXPINS; k++)
            if (pc[k] != NONE) s -= (int64_t)costp[(size_t)pp[k] * G + d];
          if (r_dev < 0 || s < bs) {
            bs = s;
            r_dev = d;
          }
        }
      }
    }
    // BASE-prefix sharing: same ranks, same CP devices for the free CP ops,
    // no caps => the BASE schedule up to the first pinned op's step t0
    int32_t t0 = 0;
    bool share = false;
    if (!MG && run && a.snap_mode == 2 && (!MM || a.snap_used)) {
      // (caps: the same free CP list gives the base's rounds and reservations)
      share = m == 0 || (MM != 2 && a.snap_round_dev >= 0 && r_dev == a.snap_round_dev);
      if (share) {
        t0 = n;
        for (int k = 0; k < np; k++) {
          const int32_t dq = (int32_t)__ldg(a.snap_dq + pp[k]);
          t0 = dq < t0 ? dq : t0;
        }
      }
    }
    // The warp starts at lo = the smallest t0 of its candidates (0 if one of
    // them does not share): a sharing candidate started from the recorded
    // BASE state at any step <= its t0 makes the BASE decisions up to t0, so
    // all lanes may start at lo; positions before lo hold BASE records.
    int32_t lo = run ? t0 : n;
    int32_t nmax = run ? n : 0;  // steps of the warp (MG: the longest slot)
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) {
      const int32_t x = __shfl_xor_sync(FULL, lo, o);
      lo = x < lo ? x : lo;
      const int32_t y = __shfl_xor_sync(FULL, nmax, o);
      nmax = y > nmax ? y : nmax;
    }
    if (MG) lo = 0;
    if (a.stat) {  // executed op-steps (the roofline's work count)
      const uint32_t ls = __reduce_add_sync(FULL, run ? (uint32_t)(n - lo) : 0u);
      if (lane == 0 && nmax > lo) {
        atomicAdd(a.stat, (unsigned long long)(nmax - lo));
        atomicAdd(a.stat + 1, (unsigned long long)ls);
      }
    }
    T avail[GP];
    T ms = 0;
#pragma unroll
    for (int d = 0; d < GP; d++) avail[d] = 0;
    if (run && lo > 0) {  // (lo > 0 implies every running lane shares)
      const T *sa = (const T *)a.snap_avail + (size_t)lo * G;
#pragma unroll
      for (int d = 0; d < GP; d++)
        if (d < G) avail[d] = __ldg(sa + d);
      ms = __ldg((const T *)a.snap_ms + lo);
      // memory before step lo: used (MM 1), cap - used - reserved (MM 2)
      if (MM == 1)
        for (int d = 0; d < G; d++) mv[d * 32] = __ldg((const int64_t *)a.snap_used + (size_t)lo * G + d);
      if (MM == 2)
        for (int d = 0; d < G; d++) mv[d * 32] = gc.cap[d] - __ldg((const int64_t *)a.snap_ur + (size_t)lo * G + d);
    }
    if (MM == 2 && run) {
#pragma unroll
      for (int d = 0; d < GP; d++) s32_at(d) = clamp32(mv[d * 32]);
    }
    if (PK) {
#pragma unroll
      for (int d = 0; d < GP; d++) avk_at(d) = (uint32_t)avail[d] << GSH;
    }

    // the next pinned position at or after the current step (NONE: none left)
    uint32_t nxt = NONE;
#pragma unroll
    for (int k = 0; k < MAXPINS; k++)
      if (pp[k] >= (uint32_t)lo && pp[k] < nxt) nxt = pp[k];
    // ---------------------------------------------------------- main loop
    // Software pipeline over positions (all cp.async copies are predicated,
    // so the step is branch-free for every lane):
    //   step u - 2P : the card of u (header, predecessor positions, comm,
    //                 cost row) is copied into cards[u % 2D] by lanes 0..;
    //   step u - P  : the inline predecessors of u at distance > P (and
    //                 BASE records, s < lo) are copied into
    //                 stage[u % D]; one commit group per step;
    //   step u      : the others were written at most P steps earlier and
    //                 are read from the ring of the last D records.
    // A staged record was stored at least one step before its copy is issued
    // (same thread, program order).  A stage or card slot is overwritten only
    // after the step that read it has consumed the values.
    // (a record is staged iff s < max(lo, u - P); s < lo: the BASE record)
    // this lane's source row of a card copy: base + u * stride (card words or
    // the cost row), one 64-bit multiply-add per copy instead of a select of
    // two address computations
    // (PK: lane 2 copies the pre-shifted comm values comm << GSH of commk)
    const bool cc_ck = PK && CM == 0 && lane == 2;
    const char *const cc_base = cc_cost ? (const char *)costsrc + cc_src
                                : cc_ck ? (const char *)a.commk
                                        : (const char *)card + cc_src;
    const uint32_t cc_stride = cc_cost ? (uint32_t)(G * sizeof(T)) : cc_ck ? 16u : (uint32_t)(CARD_WORDS * 4);
    auto copy_card = [&](int32_t u) {
      if (MG) {  // this lane's own card: header, predecessors, comm, cost row
        if (u < n) {
          const uint32_t dst = cards_sa + (uint32_t)((u & (2 * D - 1)) * CS);
          const char *cu = (const char *)(card + (size_t)u * CARD_WORDS);
          const char *row = (const char *)(costp + (size_t)u * G);
          cp_async<16>(dst, cu);
          cp_async<16>(dst + 16, cu + 4 * CARD_HDR);
          if (CM == 0) cp_async<16>(dst + 32, cu + 4 * CW_PCOMM);
          if (MM) cp_async<16>(dst + HO, cu + 16);
          if (row16) {
            for (int j = 0; j < G * (int)sizeof(T) / 16; j++) cp_async<16>(dst + CO + 16 * j, row + 16 * j);
          } else {
            for (int j = 0; j < G; j++) cp_async<sizeof(T)>(dst + CO + j * sizeof(T), row + j * sizeof(T));
          }
        }
        return;
      }
      const uint32_t dst = cards_sa + (uint32_t)((u & (2 * D - 1)) * CS) + cc_dst;
      const char *srcp = cc_base + (size_t)(uint32_t)u * cc_stride;
      if (row16) cp_async_if<16>(cc_on && u < n, dst, srcp);
      else {
        cp_async_if<16>(cc_on && !cc_cost && u < n, dst, srcp);
        for (int j = lane; j < G; j += 32)
          cp_async_if<sizeof(T)>(u < n, cards_sa + (uint32_t)((u & (2 * D - 1)) * CS + CO + j * sizeof(T)),
                                 costsrc + (size_t)u * G + j);
      }
    };
    auto prefetch = [&](int32_t u) {  // records of step u (its card is staged)
      const unsigned char *cu = cards + (u & (2 * D - 1)) * CS;
      const uint4 hu = *(const uint4 *)cu;
      const uint32_t npu = u < n ? (hu.x & 0xFFFF) : 0u;
      if (CM == 1 && !MG)  // the inline predecessors' comm values (warp-uniform card)
        cp_async_if<sizeof(T)>((uint32_t)lane < npu && lane < 4,
                               cards_sa + (uint32_t)((u & (2 * D - 1)) * CS + 32 + (lane & 3) * sizeof(T)),
                               pe_comm + hu.y + (lane & 3));
      if (CM == 1 && MG)  // (this lane's card)
        for (uint32_t k = 0; k < npu && k < 4; k++)
          cp_async<sizeof(T)>(cards_sa + (uint32_t)((u & (2 * D - 1)) * CS + 32 + k * sizeof(T)), pe_comm + hu.y + k);
      const uint4 su = *(const uint4 *)(cu + 16);
      const uint32_t ss[4] = {su.x, su.y, su.z, su.w};
      const uint32_t sl = stage_sa + (uint32_t)((u & (D - 1)) * 4 * 32 * sizeof(W));
      const bool on = run;
      const int32_t thr = lo > u - P ? lo : u - P;
#pragma unroll
      for (int k = 0; k < 4; k++) {
        const W *gp = (int32_t)ss[k] < lo ? snap + ss[k] : col + (size_t)ss[k] * 32;
        cp_async_if<sizeof(W)>(on && (uint32_t)k < npu && (int32_t)ss[k] < thr, sl + (uint32_t)(k * 32 * sizeof(W)), gp);
      }
    };
    // record of position s < t outside the inline slots (extra predecessors)
    auto rec_at = [&](uint32_t s, int32_t t) -> W {
      if ((int32_t)s < lo) return snap[s];
      if ((int32_t)s + P >= t) return ring[(s & (D - 1)) * 32];
      return col[(size_t)s * 32];
    };
    // prologue: cards of lo .. lo+2P-1 (synchronously), records of lo .. lo+P-1
    for (int32_t u = lo; u < lo + 2 * P; u++) copy_card(u);
    cp_async_commit();
    cp_async_wait<0>();
    __syncwarp();
    for (int32_t u = lo; u < lo + P; u++) {
      prefetch(u);
      cp_async_commit();
    }
    for (int32_t t = lo; t < nmax; t++) {
      const bool live = run && !dead && (!MG || t < n);
      cp_async_wait<P - 1>();  // the group of step t - P: records of t, card of t + P
      __syncwarp();            // (cards were copied by other lanes)
      const unsigned char *cs = cards + (t & (2 * D - 1)) * CS;
      const uint4 h0 = *(const uint4 *)cs;
      const uint4 hs = *(const uint4 *)(cs + 16);
      uint4 hc = make_uint4(0, 0, 0, 0);
      if (CM == 0) hc = *(const uint4 *)(cs + 32);
      const T *cm1 = (const T *)(cs + 32);  // CM 1: staged comm values
      T cst[GP];
      RowLd<T>::template load_s<GP>((const T *)(cs + CO), G, cst);
      // the op's memory (card words 4-5, MM)
      uint32_t memlo = 0, memhi = 0;
      if (MM) {
        const uint2 mw = *(const uint2 *)(cs + HO);
        memlo = mw.x;
        memhi = mw.y;
      }
      const int64_t mem64 = (int64_t)(((uint64_t)memhi << 32) | memlo);
      bool cpf = false;  // the device is forced by a CP round (its memory is reserved)
      // (MG: a lane past its slot's last position reads a stale card)
      const uint32_t npred = (!MG || live) ? (h0.x & 0xFFFF) : 0u;
      const uint32_t src[4] = {hs.x, hs.y, hs.z, hs.w};
      // predecessor records: staged or from the ring (unused slots: garbage, masked)
      W rw[4];
      const W *stg = stage + (t & (D - 1)) * 4 * 32;
      const int32_t thr = lo > t - P ? lo : t - P;
#pragma unroll
      for (int k = 0; k < 4; k++) rw[k] = *((int32_t)src[k] < thr ? stg + k * 32 : ring + (src[k] & (D - 1)) * 32);
      prefetch(t + P);
      copy_card(t + 2 * P);
      cp_async_commit();
      T f[4];
      uint32_t p[4];
      T arrd[GP];  // CM 2: arrival per device
      T M = 0, E = 0;
      uint32_t pa = 0xFFu;
      // PK: the arrival terms in key space.  A record is the key FT << GSH |
      // place, so R_k = key_k + (c_k << GSH) orders by FT + c and carries the
      // place of predecessor k in its low bits: Mkey = max R_k gives M << GSH
      // and pa (any argmax is exact, see above); the co-located test is
      // ((key_k ^ Mkey) & (GP - 1)) == 0.  Unused slots count as key 0.
      uint32_t Mk = 0, Ek = 0, pqk = 0;
      if constexpr (PK) {
        constexpr uint32_t gmk = GP - 1;
        const uint32_t hcw[4] = {hc.x, hc.y, hc.z, hc.w};  // (commk: already << GSH)
        uint32_t rkm[4], R[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
          const bool u = (uint32_t)k < npred;
          rkm[k] = u ? (uint32_t)rw[k] : 0u;
          const uint32_t ck = CM == 0 ? hcw[k] : (u ? (uint32_t)cm1[k] << GSH : 0u);
          R[k] = rkm[k] + ck;
        }
        uint32_t Mkey = max(max(R[0], R[1]), max(R[2], R[3]));
        if (npred > 4u)  // (warp-uniform)
          for (uint32_t k = 4; k < npred; k++)
            Mkey = max(Mkey, (uint32_t)rec_at(__ldg(pe_src + h0.y + k), t) + ((uint32_t)__ldg(pe_comm + h0.y + k) << GSH));
        uint32_t Ekey = 0;
#pragma unroll
        for (int k = 0; k < 4; k++) Ekey = max(Ekey, ((rkm[k] ^ Mkey) & gmk) == 0u ? rkm[k] : R[k]);
        if (npred > 4u)
          for (uint32_t k = 4; k < npred; k++) {
            const uint32_t rk = (uint32_t)rec_at(__ldg(pe_src + h0.y + k), t);
            Ekey = max(Ekey, ((rk ^ Mkey) & gmk) == 0u ? rk : rk + ((uint32_t)__ldg(pe_comm + h0.y + k) << GSH));
          }
        Mk = Mkey & ~gmk;
        Ek = Ekey & ~gmk;
        pqk = Mkey & gmk;
      } else {
#pragma unroll
        for (int k = 0; k < 4; k++) {
          T ft;
          uint32_t pl;
          Slab<T>::decode_clean(rw[k], ft, pl);
          f[k] = (uint32_t)k < npred ? ft : (T)0;
          p[k] = (uint32_t)k < npred ? pl : 0xFFu;
        }
      }
      if (!PK && CM != 2) {
        // M = max over preds of FT + c, pa = the device of a pred attaining it,
        // E = the arrival on pa (its co-located preds contribute FT only)
        T R[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
          T cm;
          if (CM == 0) cm = (T)(k == 0 ? hc.x : k == 1 ? hc.y : k == 2 ? hc.z : hc.w);
          else cm = cm1[k];
          R[k] = (uint32_t)k < npred ? f[k] + cm : (T)0;
        }
        M = R[0];
        pa = p[0];
#pragma unroll
        for (int k = 1; k < 4; k++)
          if (R[k] > M) {
            M = R[k];
            pa = p[k];
          }
        if (npred > 4u) {  // (warp-uniform)
          for (uint32_t k = 4; k < npred; k++) {
            const W w = rec_at(__ldg(pe_src + h0.y + k), t);
            T ft;
            uint32_t pl;
            Slab<T>::decode_clean(w, ft, pl);
            const T r = ft + __ldg(pe_comm + h0.y + k);
            if (r > M) {
              M = r;
              pa = pl;
            }
          }
        }
#pragma unroll
        for (int k = 0; k < 4; k++) {
          const T v = p[k] == pa ? f[k] : R[k];
          E = v > E ? v : E;
        }
        if (npred > 4u) {
          for (uint32_t k = 4; k < npred; k++) {
            const W w = rec_at(__ldg(pe_src + h0.y + k), t);
            T ft;
            uint32_t pl;
            Slab<T>::decode_clean(w, ft, pl);
            const T v = pl == pa ? ft : ft + __ldg(pe_comm + h0.y + k);
            E = v > E ? v : E;
          }
        }
      } else if (!PK) {
        // (only live lanes: a waiting lane's records are not yet valid, and
        // here a placement indexes the link-class table)
#pragma unroll
        for (int d = 0; d < GP; d++) {
          T v = 0;
          if (live && d < G) {
#pragma unroll
            for (int k = 0; k < 4; k++)
              if ((uint32_t)k < npred) {
                const T term = p[k] == (uint32_t)d
                                   ? f[k]
                                   : f[k] + __ldg(pe_comm + (size_t)(h0.y + k) * K + gc.link_class[p[k] * G + d]);
                v = term > v ? term : v;
              }
            for (uint32_t k = 4; k < npred; k++) {
              const W w = rec_at(__ldg(pe_src + h0.y + k), t);
              T ft;
              uint32_t pl;
              Slab<T>::decode_clean(w, ft, pl);
              const T term =
                  pl == (uint32_t)d ? ft : ft + __ldg(pe_comm + (size_t)(h0.y + k) * K + gc.link_class[pl * G + d]);
              v = term > v ? term : v;
            }
          }
          arrd[d] = v;
        }
      }
      // the device forced by a perturbation pin (hard) or a CP round (Alg. 1
      // l.9-10, R9; cpf: memory reserved up front) -- rare steps: the next
      // pinned position, or a CP op while the lane has a CP device
      const bool cp_any = MM == 2 ? rc < nr : r_dev >= 0;
      auto forced_dev = [&]() -> int {
        int forced = -1;
        if ((uint32_t)t == nxt) {
          nxt = NONE;
#pragma unroll
          for (int k = 0; k < MAXPINS; k++) {
            if (pp[k] == (uint32_t)t) forced = (int)((pdv >> (8 * k)) & 0xFFu);
            else if (pp[k] > (uint32_t)t && pp[k] < nxt) nxt = pp[k];
          }
        }
        if (forced < 0 && h0.w != NONE) {
          if (MM == 2) {
            // CP ops come in CP order (positions are topological): advance
            // to the round holding raw CP index h0.w
            while (rc < nr && h0.w >= rhi) {
              rc++;
              if (rc < nr) {
                rhi = rnd[rc * 32] & 0xFFFFFFu;
                rdv = (int)(rnd[rc * 32] >> 24);
              }
            }
            if (rc < nr) forced = rdv;
          } else if (r_dev >= 0) {
            forced = r_dev;
          }
          cpf = forced >= 0;
        }
        return forced;
      };
      if constexpr (PK) {
        // keys (EFT << GSH) | d: EST = max(avail[d], arrival),
        // arrival M on every device but pa, E on pa (R6); min key = EFT
        // argmin with ties to the lowest device (Alg. 1 lines 12-19, R3)
        uint32_t av[GP];
        if (GP >= 2) {
#pragma unroll
          for (int j = 0; j < GP / 2; j++) {
            const uint2 x = *(const uint2 *)(avk + j * 64);
            av[2 * j] = x.x;
            av[2 * j + 1] = x.y;
          }
        } else {
          av[0] = avk[0];
        }
        const uint32_t pq = pqk;
        const uint32_t ap = avk_at(pq), cpa = ((const uint32_t *)(cs + CO))[pq];
        uint32_t kpa = (ap > Ek ? ap : Ek) + cpa;
        if (!EX && pq >= (uint32_t)G) kpa = 0xFFFFFFFFu;
        uint32_t key[GP];
#pragma unroll
        for (int d = 0; d < GP; d++)
          key[d] = (EX || d < G) ? (av[d] > Mk ? av[d] : Mk) + (uint32_t)cst[d] : 0xFFFFFFFFu;
        // MM 2: a device is feasible iff mem_i <= slack[d] (Alg. 1 line 13,
        // R8); infeasible keys become ~0 (the 32-bit slack copy decides when
        // the op's memory is below 2^32, exactly: slack >= 2^32 clamps to
        // 2^32 - 1 >= mem)
        uint32_t fk[GP], fkpa = kpa;
#pragma unroll
        for (int d = 0; d < GP; d++) fk[d] = key[d];
        if (MM == 2) {
          if (memhi != 0) {  // (warp-uniform)
#pragma unroll
            for (int d = 0; d < GP; d++)
              if (mv[d * 32] < mem64) fk[d] = 0xFFFFFFFFu;
            if (mv[pq * 32] < mem64) fkpa = 0xFFFFFFFFu;
          } else {
            uint32_t sv[GP];
            if (GP >= 4) {
#pragma unroll
              for (int j = 0; j < GP / 4; j++) {
                const uint4 x = *(const uint4 *)(s32b + j * 128);
                sv[4 * j] = x.x;
                sv[4 * j + 1] = x.y;
                sv[4 * j + 2] = x.z;
                sv[4 * j + 3] = x.w;
              }
            } else {
#pragma unroll
              for (int d = 0; d < GP; d++) sv[d] = s32b[d * 32];
            }
#pragma unroll
            for (int d = 0; d < GP; d++)
              if (sv[d] < memlo) fk[d] = 0xFFFFFFFFu;
            if (s32_at(pq) < memlo) fkpa = 0xFFFFFFFFu;
          }
        }
        uint32_t bk = fkpa;
#pragma unroll
        for (int d = 0; d < GP; d++) bk = fk[d] < bk ? fk[d] : bk;
        if (__any_sync(FULL, (uint32_t)t == nxt || (h0.w != NONE && cp_any))) {
          const int forced = forced_dev();
          if (forced >= 0) {  // (a CP round's device draws on its reservation)
#pragma unroll
            for (int d = 0; d < GP; d++)
              if (d == forced) bk = cpf ? key[d] : fk[d];
            const uint32_t kp = cpf ? kpa : fkpa;
            if ((uint32_t)forced == pq && kp < bk) bk = kp;
          }
        }
        const bool go = live && (MM != 2 || bk != 0xFFFFFFFFu);
        if (MM == 2 && live && !go) dead = true;  // no feasible device: INFEASIBLE
        if (go) {
          const uint32_t dc = bk & (uint32_t)(GP - 1);
          if (MM == 1) mv[dc * 32] += mem64;
          if (MM == 2 && !cpf) {
            const int64_t v = mv[dc * 32] - mem64;
            mv[dc * 32] = v;
            s32_at(dc) = clamp32(v);
          }
          const uint32_t bkc = bk & ~(uint32_t)(GP - 1);
          avk_at(bk & (uint32_t)(GP - 1)) = bkc;
          const T best = (T)(bkc >> GSH);
          ms = best > ms ? best : ms;
          // the record is the key itself: FT << GSH | device
          col[(size_t)t * 32] = bk;
          ring[(t & (D - 1)) * 32] = bk;
        }
      } else {
      // EFT per device; argmin with ties to the lowest device
      // (Alg. 1 lines 12-19, R3); devices >= G are never chosen
      T eft[GP];
      uint32_t gk[GP];  // INS: the idle slot the op would go into on d (NONE: appended)
#pragma unroll
      for (int d = 0; d < GP; d++) {
        const T arr = CM == 2 ? arrd[d] : ((uint32_t)d == pa ? E : M);
        T est = avail[d] > arr ? avail[d] : arr;
        gk[d] = NONE;
        if (INS && live && (EX || d < G) && arr < avail[d] && gn[d] > 0) {
          // R1i: the first idle slot [a, b) with max(a, r) + w <= b; slots
          // are disjoint and sorted, none ending before r can fit
          const GapSlot<T> *gl = gbase + (size_t)d * a.gap_cap;
          uint32_t lo = 0, hi = gn[d];
          while (lo < hi) {
            const uint32_t mid = (lo + hi) >> 1;
            if (gl[mid].b < arr) lo = mid + 1;
            else hi = mid;
          }
          for (uint32_t k = lo; k < gn[d]; k++) {
            const GapSlot<T> e = gl[k];
            const T tt = e.a > arr ? e.a : arr;
            if (tt + cst[d] <= e.b) {
              gk[d] = k;
              est = tt;
              break;
            }
          }
        }
        eft[d] = ((EX || d < G) && (!MG || ((dmask >> d) & 1u))) ? est + cst[d] : TT<T>::MAXV;
      }
      // MM 2: memory-feasible devices only (Alg. 1 line 13, R8)
      T feft[GP];
#pragma unroll
      for (int d = 0; d < GP; d++) {
        bool fe = true;
        if (MM == 2) fe = memhi != 0 ? mv[d * 32] >= mem64 : s32_at(d) >= memlo;
        feft[d] = fe ? eft[d] : TT<T>::MAXV;
      }
      T best = feft[0];
      int bd = 0;
#pragma unroll
      for (int d = 1; d < GP; d++)
        if (feft[d] < best) {
          best = feft[d];
          bd = d;
        }
      if (__any_sync(FULL, (uint32_t)t == nxt || (h0.w != NONE && cp_any))) {
        const int forced = forced_dev();
        if (forced >= 0) {  // (a CP round's device draws on its reservation)
#pragma unroll
          for (int d = 0; d < GP; d++)
            if (d == forced) best = cpf ? eft[d] : feft[d];
          bd = forced;
        }
      }
      const bool go = live && (MM != 2 || best != TT<T>::MAXV);
      if (MM == 2 && live && !go) dead = true;  // no feasible device: INFEASIBLE
      if (go) {
        if (MM == 1) mv[bd * 32] += mem64;
        if (MM == 2 && !cpf) {
          const int64_t v = mv[bd * 32] - mem64;
          mv[bd * 32] = v;
          s32_at(bd) = clamp32(v);
        }
        bool appended = true;
        if (INS) {
          // the chosen device's idle slots: the slot the op went into shrinks,
          // splits in two (tail shifted up) or disappears (tail shifted down);
          // an op appended after a data wait leaves a new slot [avail, ST)
          uint32_t k0 = NONE, n0 = 0;
          T av0 = 0, w0 = 0;
#pragma unroll
          for (int d = 0; d < GP; d++)
            if (d == bd) {
              k0 = gk[d];
              n0 = gn[d];
              av0 = avail[d];
              w0 = cst[d];
            }
          GapSlot<T> *gl = gbase + (size_t)bd * a.gap_cap;
          const T st0 = best - w0;
          if (k0 != NONE) {
            const GapSlot<T> e = gl[k0];
            const bool left = st0 > e.a, right = best < e.b;
            if (left && right) {
              if (n0 + 1 > (uint32_t)a.gap_cap) ovf = true;
              else {
                for (uint32_t k = n0; k > k0 + 1; k--) gl[k] = gl[k - 1];
                GapSlot<T> ne;
                ne.a = best;
                ne.b = e.b;
                gl[k0 + 1] = ne;
                gl[k0].b = st0;
                n0++;
              }
            } else if (left) {
              gl[k0].b = st0;
            } else if (right) {
              gl[k0].a = best;
            } else {
              for (uint32_t k = k0; k + 1 < n0; k++) gl[k] = gl[k + 1];
              n0--;
            }
          } else if (st0 > av0) {
            if (n0 + 1 > (uint32_t)a.gap_cap) ovf = true;
            else {
              GapSlot<T> ne;
              ne.a = av0;
              ne.b = st0;
              gl[n0++] = ne;
            }
          }
#pragma unroll
          for (int d = 0; d < GP; d++)
            if (d == bd) gn[d] = n0;
          appended = k0 == NONE;
        }
#pragma unroll
        for (int d = 0; d < GP; d++)
          if (d == bd && appended) avail[d] = best;
        ms = best > ms ? best : ms;
        W w;
        Slab<T>::make(w, best, (uint32_t)bd);
        col[(size_t)t * 32] = w;
        ring[(t & (D - 1)) * 32] = w;
      }
      }  // !PK
    }
    cp_async_wait<0>();  // (no copy may land in the stage after this candidate)

    // ------------------------------------------------------------ epilogue
    if ((PK && run && (uint32_t)ms >= a.pk_lim) || (INS && run && ovf)) {
      // a key may have wrapped / a device ran out of idle-slot capacity: re-run
      // through the preparation pipeline on the group kernel
      const unsigned long long k = atomicAdd(a.ndefer, 1ull);
      a.defer_q[k] = q;
    } else if (run) {
      if (res_idx >= 0) {
        a.out.makespan[res_idx] = dead ? I64MAX : (int64_t)ms;
        a.out.status[res_idx] = dead ? 1 : 0;
        // per-device peak (R8: the final static total; reservations are all
        // drawn by then), -1 when infeasible
        if (MM && a.out.peak)
          for (int d = 0; d < G; d++)
            a.out.peak[res_idx * G + d] = dead ? -1 : (MM == 1 ? mv[d * 32] : gc.cap[d] - mv[d * 32]);
      }
      if (!dead && ((int64_t)ms < bms || ((int64_t)ms == bms && sidx < bidx))) {
        bms = (int64_t)ms;
        bidx = sidx;
      }
    }
  }
  if (a.track_best) {
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) {
      const int64_t m2 = __shfl_xor_sync(FULL, bms, o), i2 = __shfl_xor_sync(FULL, bidx, o);
      if (i2 >= 0 && (bidx < 0 || m2 < bms || (m2 == bms && i2 < bidx))) {
        bms = m2;
        bidx = i2;
      }
    }
    if (lane == 0 && bidx >= 0) {
      const int64_t m0 = a.wbest[2 * gwarp], i0 = a.wbest[2 * gwarp + 1];
      if (i0 < 0 || bms < m0 || (bms == m0 && bidx < i0)) {
        a.wbest[2 * gwarp] = bms;
        a.wbest[2 * gwarp + 1] = bidx;
      }
    }
  }
}

}  // namespace fastt
