// k_sim_body.cuh -- the group-per-candidate DPOS simulation kernel (k_sim)
// and its CP-device rounds; included by k_sim_inst.cu, which is compiled
// once per lane-group width GSH (build.py: -DFASTT_GSH=0..5) so the
// template instances build in parallel.  See k_sim.cu for the overview.
#pragma once
#include "fastt_internal.cuh"
#include "sim_common.cuh"

namespace fastt {


#ifndef SIM_ASM_SMEM
#define SIM_ASM_SMEM 0
#endif
// 32-bit shared-memory accessors for the ready bitmap
#if SIM_ASM_SMEM
static __device__ __forceinline__ uint32_t lds32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
static __device__ __forceinline__ void sts32(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
static __device__ __forceinline__ void red_or_s(uint32_t a, uint32_t v) {
  asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
#else
extern __shared__ uint32_t smem[];
static __device__ __forceinline__ uint32_t *sptr(uint32_t a) { return (uint32_t *)__cvta_shared_to_generic(a); }
static __device__ __forceinline__ uint32_t lds32(uint32_t a) { return *sptr(a); }
static __device__ __forceinline__ void sts32(uint32_t a, uint32_t v) { *sptr(a) = v; }
static __device__ __forceinline__ void red_or_s(uint32_t a, uint32_t v) { atomicOr(sptr(a), v); }
#endif


// CP devices (Alg. 1 line 5, R9) for one candidate,
// executed by its lane group (gm = group mask, gb = first lane, d = device
// lane): repeatedly give the device with the smallest exact average cost the
// longest prefix of the remaining free CP ops that fits its memory;
// perturbation-pinned CP ops are excluded (free-index space).  Lane gb + r
// receives round r.
template <typename T>
__device__ __noinline__ void cp_rounds_g(const PrepGraph *pg, int np, const uint32_t *pp, unsigned gm, int gb, int d,
                                         int G, int64_t cap_d, uint32_t dset, uint32_t &r_lo, uint32_t &r_hi,
                                         int &r_dev, int &nrounds, uint32_t *pcp, int64_t &reserved) {
  const uint32_t *card = pg->card;
  const T *costp = (const T *)pg->costp;
  const int32_t L = pg->cp_len;
  // CP index / memory of each pinned op; the on-CP ones sorted ascending
  uint32_t pcs[MAXPINS];
  int64_t pms[MAXPINS];
  int64_t pcd[MAXPINS];  // cost on this lane's device
  int m = 0;
  for (int k = 0; k < MAXPINS; k++) {
    pcp[k] = NONE;
    pcs[k] = NONE;
    pms[k] = 0;
    pcd[k] = 0;
  }
  for (int k = 0; k < np; k++) {
    const uint32_t *ci = card + (int64_t)pp[k] * CARD_WORDS;
    pcp[k] = ci[CW_CPIDX];
    if (pcp[k] == NONE) continue;
    int j = m++;
    const int64_t mv = (int64_t)(((uint64_t)ci[CW_MEMHI] << 32) | ci[CW_MEMLO]);
    const int64_t cv = d < G ? (int64_t)costp[(int64_t)pp[k] * G + d] : 0;
    while (j > 0 && pcs[j - 1] > pcp[k]) {
      pcs[j] = pcs[j - 1];
      pms[j] = pms[j - 1];
      pcd[j] = pcd[j - 1];
      j--;
    }
    pcs[j] = pcp[k];
    pms[j] = mv;
    pcd[j] = cv;
  }
  const int32_t Lf = L - m;
  auto raw_end = [&](int32_t f) -> int32_t {  // raw index just after the f-th free op (f >= 1)
    int32_t r = f - 1;
#pragma unroll
    for (int j = 0; j < MAXPINS; j++)
      if (j < m && (int32_t)pcs[j] <= r) r++;
    return r + 1;
  };
  auto fp_mem = [&](int32_t f) -> int64_t {
    if (f <= 0) return 0;
    int32_t re = raw_end(f);
    int64_t v = pg->pmem[re];
#pragma unroll
    for (int j = 0; j < MAXPINS; j++)
      if (j < m && (int32_t)pcs[j] < re) v -= pms[j];
    return v;
  };
  auto fp_cost = [&](int32_t f) -> int64_t {  // for device d
    if (f <= 0) return 0;
    int32_t re = raw_end(f);
    int64_t v = pg->pcost[(int64_t)re * G + d];
#pragma unroll
    for (int j = 0; j < MAXPINS; j++)
      if (j < m && (int32_t)pcs[j] < re) v -= pcd[j];
    return v;
  };
  uint32_t devs = dset;  // the candidate's devices (R25)
  int32_t k = 0;
  while (k < Lf && devs) {
    int32_t t = 0;
    int64_t S = 0;
    if (d < G && ((devs >> d) & 1)) {
      int64_t bm = fp_mem(k);
      int64_t tot = fp_mem(Lf) - bm;
      if (tot <= cap_d) t = Lf - k;
      else {
        int32_t lo = 0, hi = Lf - k;
        while (hi - lo > 1) {
          int32_t mid = (lo + hi) >> 1;
          if (fp_mem(k + mid) - bm <= cap_d) lo = mid;
          else hi = mid;
        }
        t = lo;
      }
      if (t > 0) S = fp_cost(k + t) - fp_cost(k);
    }
    int best = -1;
    int32_t tb = 0;
    int64_t Sb = 0;
    for (int dd = 0; dd < G; dd++) {
      int32_t td = __shfl_sync(gm, t, gb + dd);
      int64_t Sd = __shfl_sync(gm, S, gb + dd);
      if (td > 0 && (best < 0 || lt_cross((uint64_t)Sd, (uint64_t)tb, (uint64_t)Sb, (uint64_t)td))) {
        best = dd;
        tb = td;
        Sb = Sd;
      }
    }
    if (best < 0) break;
    int64_t resv = fp_mem(k + tb) - fp_mem(k);
    if (d == nrounds) {
      r_lo = (uint32_t)k;
      r_hi = (uint32_t)(k + tb);
      r_dev = best;
    }
    if (d == best) reserved += resv;
    devs &= ~(1u << best);
    k += tb;
    nrounds++;
  }
}

// Several candidates per warp: lane group g (GP = 2^GSH lanes, GP >= G) owns
// one candidate; lane d of the group is device d.  The main loop keeps the
// warp converged (groups that finished idle) so every shuffle/vote is a
// full-warp instruction.  T: time type; MEM: track per-device memory;
// INS: insertion policy (R1i) -- lane d keeps device d's idle slots.
// FC: uint32 time and one link class -- predecessor comm values come from
// the op's card (no per-edge comm loads).
// TOPO: the priority order of the prepared graph is a topological order
// (PrepGraph::topo), so the dequeue order is the position order: the
// highest-priority op not yet dequeued has all its predecessors at higher
// priority, hence already dequeued, hence it is ready and it is the one
// popped (by induction every step pops the next position).  No ready set,
// no indegrees, no successor release; with prefix sharing the records of
// positions before t0 are read from the recorded BASE schedule in place.
template <typename T, int GSH, bool MEM, bool INS, bool FC, bool TOPO>
__global__ void __launch_bounds__(SIM_BLOCK, TOPO ? SIM_MINB_TOPO : SIM_MINB) k_sim(SimArgs a) {
  typedef typename Slab<T>::W W;
  constexpr int GP = 1 << GSH;   // lanes per candidate (>= G)
  constexpr int CPW = 32 >> GSH; // candidates per warp
  extern __shared__ uint32_t smem[];
  __shared__ int64_t s_best[SIM_BLOCK][2];      // per group leader
  __shared__ int64_t s_res[SIM_BLOCK], s_sidx[SIM_BLOCK];
  const int lane = threadIdx.x & 31;
  const int wib = threadIdx.x >> 5;
  const int grp = lane >> GSH;
  const int d = lane & (GP - 1);
  const int gb = grp << GSH;
  const unsigned gm = GP == 32 ? FULL : (((1u << GP) - 1u) << gb);
  const int lead = threadIdx.x - d;  // group leader thread (s_* index)
  const int64_t gwarp = (int64_t)blockIdx.x * (blockDim.x >> 5) + wib;
  const int64_t cslot = gwarp * CPW + grp;
  uint32_t *leaf = smem + (uint32_t)(wib * CPW + grp) * (uint32_t)a.bm_stride;
  uint32_t *summ = leaf + a.leaf_words;
  const uint32_t leaf_sa = (uint32_t)__cvta_generic_to_shared(leaf);
  const uint32_t summ_sa = (uint32_t)__cvta_generic_to_shared(summ);
  // state slabs: the CPW candidates of a warp are interleaved by position
  // ([position][candidate], 32 B per position at CPW = 4), so groups that pop
  // the same or nearby ops (they follow nearly the BASE order) share sectors
  W *const slab0 = (W *)a.slab;
  const uint32_t sb = (uint32_t)(gwarp * a.slab_stride * CPW + grp);
#define SLOT(p) (sb + (uint32_t)(p) * (uint32_t)CPW)
  const GraphConst &gc = *a.gc;
  const int G = a.G;
  const int K = gc.K;
  const int64_t cap_d = d < G ? gc.cap[d] : 0;
  const bool cp_on = (a.flags & 1u) != 0;
  const bool cap_chk = MEM && a.cap_check != 0;
  const bool lmem = MEM && a.live_mem != 0;  // liveness memory (R24)
  constexpr bool fastcomm = FC;
  static_assert(!FC || sizeof(T) == 4, "card comm values are uint32");
  // INSERT: lane d's array of device d's idle slots (sorted by start)
  GapSlot<T> *const gsl =
      INS ? (GapSlot<T> *)a.gap + ((size_t)cslot * G + (size_t)(d < G ? d : 0)) * (size_t)a.gap_stride : nullptr;
  if (d == 0) {
    s_best[lead][0] = a.track_best ? a.wbest[2 * cslot] : I64MAX;
    s_best[lead][1] = a.track_best ? a.wbest[2 * cslot + 1] : -1;
  }
  __syncwarp();

  // work items: a.n, or the device count of a list classified / gathered on
  // the device (n_dev)
  const int64_t nlim = a.n_dev ? ((int64_t)*a.n_dev < a.n ? (int64_t)*a.n_dev : a.n) : a.n;
  for (;;) {
    unsigned long long q0 = 0;
    if (lane == 0) q0 = atomicAdd(a.counter, (unsigned long long)CPW);
    q0 = __shfl_sync(FULL, q0, 0);
    if ((int64_t)q0 >= nlim) break;
    const int64_t q = (int64_t)q0 + grp;
    bool active = q < nlim;
    Cand c;
    c.kind = 0; c.n_pins = 0; c.split_op = -1;
    const PrepGraph *pg = a.base;
    int64_t res_idx = -1, sidx = q;
    if (active) {
      if (a.mode == 0) {
        sidx = a.first + q * a.stride;
        c = stream_cand(a.stream, sidx);
      } else if (a.mode == 1) {
        c = a.cands[q];
        res_idx = q;
      } else if (a.mode == 3) {  // candidate list ordered by BASE-prefix start step
        c = a.cands[q];
        res_idx = a.slot_result ? a.slot_result[q] : -1;
        sidx = a.slot_index[q];
      } else {
        c = a.cands[q];
        pg = a.slots + q;
        res_idx = a.slot_result ? a.slot_result[q] : -1;
        sidx = a.slot_index ? a.slot_index[q] : q;
        // two launches over the slots: position-order (1) / ready-set (2)
        if (a.slot_filter && (pg->topo != 0) != (a.slot_filter == 1)) active = false;
      }
    }
    if (!TOPO && active && pg->n > (int32_t)READY_SET_MAX) {  // (the bitmap covers READY_SET_MAX positions)
      active = false;
      if (a.err && d == 0) atomicOr(a.err, 1u);
    }
    const uint32_t *__restrict__ card = pg->card;
    const T *__restrict__ costp = (const T *)pg->costp;
    const T *__restrict__ pe_comm = (const T *)pg->pe_comm;
    const int32_t n = pg->n;
    const int32_t Vraw = pg->V;
    const uint32_t *__restrict__ posm = pg->pos;

    // ---------------------------------------------------------- validate
    int np = 0;
    uint8_t st = 0;
    bool defer = false;
    const uint32_t all = all_devices(G);
    const uint32_t dset = (active && c.dev_mask) ? c.dev_mask : all;  // R25
    if (active) {
      if (a.mode != 2) {
        if (c.dev_mask & ~all) st = 2;
        else if (dset != all) defer = true;  // ranks over the subset: preparation pipeline
        if (st) {
        } else if (c.kind == 0) {
        } else if (c.kind == 1) {
          np = c.n_pins;
          if (np < 1 || np > MAXPINS) st = 2;
          else {
            bool bad = false;
            for (int k = 0; k < np; k++) {
              int32_t o = c.pin_op[k];
              if (o < 0 || o >= Vraw || posm[o] == NONE || c.pin_dev[k] >= G || !((dset >> c.pin_dev[k]) & 1u))
                bad = true;
              for (int k2 = 0; k2 < k; k2++) bad |= c.pin_op[k2] == o;
            }
            if (bad) st = 2;
          }
        } else if (c.kind == 2) {
          int32_t o = c.split_op;
          if (o < 0 || o >= Vraw || posm[o] == NONE || c.split_dim > 1 ||
              !(a.split_mask[o] & (1u << c.split_dim)) || c.split_n < 2 || c.split_n > G)
            st = 2;
          else defer = true;
        } else {
          st = 2;
        }
      } else {
        np = c.kind == 1 ? c.n_pins : 0;
      }
    }
    if (st) {
      np = 0;
      defer = false;
    }
    // the candidate's pins as group-uniform arrays (positions, packed devices)
    uint32_t pp[MAXPINS] = {NONE, NONE, NONE, NONE};
    uint32_t pdv = 0;
    if (active && !defer)
      for (int k = 0; k < np; k++) {
        pp[k] = posm[c.pin_op[k]];
        pdv |= (uint32_t)c.pin_dev[k] << (8 * k);
      }
    // classify (modes 0, 1): pins that change w or c send the candidate to
    // the preparation pipeline
    {
      bool chg = false;
      if (active && !defer && a.mode != 2)
        for (int k = d; k < np; k += GP) chg |= pin_changes_ranks<T>(pg, gc, c, np, posm[c.pin_op[k]], c.pin_dev[k], G, K);
      if ((__ballot_sync(FULL, chg) & gm) != 0) defer = true;
    }
    if (active && defer && d == 0) {
      unsigned long long k = atomicAdd(a.ndefer, 1ull);
      a.defer_q[k] = q;
    }
    if (active && !defer && st && d == 0 && res_idx >= 0) {
      a.out.makespan[res_idx] = I64MAX;
      a.out.status[res_idx] = st;
    }
    if (active && !defer && st && res_idx >= 0 && a.out.peak && d < G) a.out.peak[res_idx * G + d] = -1;
    const bool run = active && !defer && st == 0;

    // ------------------------------------------------------ prologue
    int64_t used = 0, reserved = 0, peakv = 0;
    uint32_t r_lo = 0, r_hi = 0;
    int r_dev = -1, nrounds = 0;
    uint32_t pcp[MAXPINS] = {NONE, NONE, NONE, NONE};
    if (run && cp_on && pg->cp_len > 0)
      cp_rounds_g<T>(pg, np, pp, gm, gb, d, G, cap_d, dset, r_lo, r_hi, r_dev, nrounds, pcp, reserved);
    if (d == 0) {
      s_res[lead] = res_idx;
      s_sidx[lead] = sidx;
    }
    const bool want_out = run && res_idx >= 0 && a.out.place != nullptr;
    // BASE-schedule prefix sharing: with the base ranks, the base CP devices
    // for every free CP op and no memory caps, the candidate's schedule is the
    // BASE schedule until its first pinned op is dequeued (step t0), so it
    // starts from the recorded BASE state at t0 (exact)
    int32_t t0 = 0;
    bool share = false;
    if (run && !MEM && !INS && !want_out && a.snap_mode == 2 && a.mode != 2) {
      t0 = n;
      for (int k = 0; k < np; k++) {
        const int32_t dq = (int32_t)__ldg(a.snap_dq + pp[k]);
        t0 = dq < t0 ? dq : t0;
      }
      share = true;
      if (cp_on && pg->cp_len > 0) {
        int m = 0;
        for (int k = 0; k < np; k++) m += pcp[k] != NONE;
        if (m > 0) {
          // pinned CP ops change the free list: accept only one round over
          // every free CP op on the base's single-round device
          const uint32_t lo0 = __shfl_sync(gm, r_lo, gb), hi0 = __shfl_sync(gm, r_hi, gb);
          const int dv0 = __shfl_sync(gm, r_dev, gb);
          share = a.snap_round_dev >= 0 && nrounds == 1 && lo0 == 0 && (int32_t)hi0 == pg->cp_len - m &&
                  dv0 == a.snap_round_dev;
        }
      }
      if (!share) t0 = 0;  // (TOPO: a refused candidate simulates every step from its own empty state)
    }
    uint32_t top = 0;
    T avail = 0, makespan = 0;
    // INSERT: the number of idle slots before `avail` on this lane's device
    uint32_t gn = 0;
    if (run && share) {
      avail = d < G ? __ldg((const T *)a.snap_avail + (size_t)t0 * G + d) : (T)0;
      makespan = __ldg((const T *)a.snap_ms + t0);
      if (!TOPO && t0 < n) {
        const int32_t nwords = (n + 31) >> 5;
        for (int32_t w = d; w < nwords; w += GP) leaf[w] = 0;
        __syncwarp(gm);
        const W *rec0 = (const W *)a.snap_rec;
        for (int32_t p = d; p < n; p += GP) {
          const uint32_t dq = __ldg(a.snap_dq + p);
          if ((int32_t)dq < t0) {
            slab0[SLOT(p)] = rec0[p];
          } else {
            const uint32_t *cp_ = card + (size_t)p * CARD_WORDS;
            const uint32_t npr = __ldg(cp_ + CW_DEG) & 0xFFFF;
            const uint4 ps = __ldg((const uint4 *)(cp_ + CARD_HDR));
            uint32_t cnt = 0;
            if (npr > 0) cnt += (int32_t)__ldg(a.snap_dq + ps.x) >= t0;
            if (npr > 1) cnt += (int32_t)__ldg(a.snap_dq + ps.y) >= t0;
            if (npr > 2) cnt += (int32_t)__ldg(a.snap_dq + ps.z) >= t0;
            if (npr > 3) cnt += (int32_t)__ldg(a.snap_dq + ps.w) >= t0;
            if (npr > 4) {
              const uint32_t pb = __ldg(cp_ + CW_PBASE);
              for (uint32_t k = 4; k < npr; k++) cnt += (int32_t)__ldg(a.snap_dq + __ldg(pg->pe_src + pb + k)) >= t0;
            }
            Slab<T>::init(slab0, SLOT(p), cnt);
            if (cnt == 0) atomicOr(&leaf[p >> 5], 1u << (p & 31));
          }
        }
        __syncwarp(gm);
        uint32_t tb = 0;
        for (int32_t sw = d; sw < 32; sw += GP) {
          uint32_t word = 0;
          for (int b = 0; b < 32; b++) {
            const int32_t w = sw * 32 + b;
            if (w < nwords && leaf[w]) word |= 1u << b;
          }
          summ[sw] = word;
          if (word) tb |= 1u << sw;
        }
#pragma unroll
        for (int o = GP >> 1; o >= 1; o >>= 1) tb |= __shfl_xor_sync(gm, tb, o);
        top = tb;
      }
    } else if (run && !TOPO) {
      const int32_t nwords = (n + 31) >> 5;
      for (int32_t w = d; w < nwords; w += GP) leaf[w] = __ldg(pg->srcbits + w);
      for (int32_t s = d; s < 32; s += GP) summ[s] = __ldg(pg->srcsumm + s);
      top = __ldg(pg->srcsumm + 32);
      for (int32_t p = d; p < n; p += GP) Slab<T>::init(slab0, SLOT(p), __ldg(pg->npred + p));
    }
    if (a.snap_mode == 1 && run && d == 0) {
      a.snap_rounds[0] = nrounds;
      a.snap_rounds[1] = r_dev;
      a.snap_rounds[2] = (int32_t)r_lo;
      a.snap_rounds[3] = (int32_t)r_hi;
    }
    // groups of >= 4 lanes hold pin k in lane k; narrower groups keep the arrays
    uint32_t my_pos = NONE, my_pcp = NONE;
    int my_dev = 0;
    if (GP >= 4) {
      my_pos = d == 0 ? pp[0] : d == 1 ? pp[1] : d == 2 ? pp[2] : d == 3 ? pp[3] : NONE;
      my_pcp = d == 0 ? pcp[0] : d == 1 ? pcp[1] : d == 2 ? pcp[2] : d == 3 ? pcp[3] : NONE;
      my_dev = d < 4 ? (int)((pdv >> (8 * d)) & 0xFF) : 0;
    }
    __syncwarp();
    const bool dev_ok = d < G && ((dset >> d) & 1u);  // this lane's device may be used (R25)
    const bool any_pins = __any_sync(FULL, np > 0);
    const bool any_cp = __any_sync(FULL, nrounds > 0);
    const bool any_out = __any_sync(FULL, want_out);
    const int64_t ob = want_out ? res_idx * (int64_t)a.out.vmax : 0;
    const bool snap_rec_on = a.snap_mode == 1;
    // step counter; under TOPO also the position processed (each group from its t0)
    int32_t tstep = 0;
    if (TOPO) {
      int32_t lo = run ? t0 : 0x7FFFFFFF;
#pragma unroll
      for (int o = 16; o >= 1; o >>= 1) {
        const int32_t x = __shfl_xor_sync(FULL, lo, o);
        lo = x < lo ? x : lo;
      }
      tstep = lo;
    }

    // ---------------------------------------------------------- main loop
    int32_t seq = 0;
    bool infeas = false;
    const uint32_t la = leaf_sa, sa = summ_sa;  // shared-memory byte addresses
    while (TOPO ? __any_sync(FULL, run && !infeas && tstep < n) : __any_sync(FULL, top != 0)) {
      bool live;
      uint32_t i;
      int s = 0, w = 0;
      uint32_t nlw = 0, nm = 0;
      if constexpr (TOPO) {
        live = run && !infeas && tstep >= t0 && tstep < n;
        i = live ? (uint32_t)tstep : 0u;
      } else {
        live = top != 0;
        // pop: highest priority = lowest position = lowest set bit
        s = live ? __ffs(top) - 1 : 0;
        const uint32_t m = lds32(sa + 4u * s);
        const int b = m ? __ffs(m) - 1 : 0;
        w = (s << 5) + b;
        const uint32_t lw = lds32(la + 4u * w);
        i = live ? ((uint32_t)w << 5) + (__ffs(lw) - 1) : 0u;
        nlw = lw & (lw - 1);
        nm = nlw ? m : (m & (m - 1));
      }

      // round 1 (all from the op's card line): header, predecessor
      // positions and comm, this lane's successor, cost on this lane's device
      const uint32_t *cd = card + (size_t)i * CARD_WORDS;
      const uint4 h0 = __ldg((const uint4 *)cd);
      const uint4 hs = __ldg((const uint4 *)(cd + CARD_HDR));
      uint4 hc = make_uint4(0, 0, 0, 0);
      if (fastcomm) hc = __ldg((const uint4 *)(cd + CW_PCOMM));
      const T cst = __ldg(costp + (size_t)i * G + (d < G ? d : 0));
      const uint32_t s0 = TOPO ? 0u : __ldg(cd + CW_SUCC + (d < S_IN ? d : 0));
      __syncwarp();
      if constexpr (!TOPO) {
        if (live && d == 0) {
          sts32(la + 4u * w, nlw);
          sts32(sa + 4u * s, nm);
        }
        if (live && !nm) top &= top - 1;
      }
      const uint32_t npred = live ? (h0.x & 0xFFFF) : 0u;
      const uint32_t nsucc = live ? (h0.x >> 16) : 0u;
      // round 2: predecessor records, successor indegree
      const uint32_t src[4] = {hs.x, hs.y, hs.z, hs.w};
      const uint32_t cmi[4] = {hc.x, hc.y, hc.z, hc.w};
      T ft[4];
      uint32_t pl[4];
      // all four records and the successor's indegree are loaded
      // unconditionally (unused card slots hold position 0), so the loads
      // issue back to back instead of one dependent round trip each
      W rw[4];
#pragma unroll
      for (int k = 0; k < 4; k++) {
        // TOPO + sharing: positions before t0 hold the BASE records (read in place)
        const W *ad = (TOPO && share && (int32_t)src[k] < t0) ? (const W *)a.snap_rec + src[k] : slab0 + SLOT(src[k]);
        rw[k] = *ad;
      }
      const uint32_t sdeg_raw = TOPO ? 1u : Slab<T>::indeg(slab0, SLOT(s0));
#pragma unroll
      for (int k = 0; k < 4; k++) {
        T f;
        uint32_t p;
        Slab<T>::decode(rw[k], f, p);
        ft[k] = (uint32_t)k < npred ? f : (T)0;
        pl[k] = (uint32_t)k < npred ? p : (uint32_t)d;
      }
      const uint32_t sdeg = ((uint32_t)d < nsucc) ? sdeg_raw : 1u;
      // EST = max(avail[d], max_pred FT + c(pred -> i on d))   (R1, R6)
      // (INSERT: first the data-ready time r, then the idle-slot search)
      T est = INS ? (T)0 : avail;
#pragma unroll
      for (int k = 0; k < 4; k++) {
        T cm;
        if (fastcomm) cm = (T)cmi[k];
        else cm = ((uint32_t)k < npred && pl[k] != (uint32_t)d && d < G)
                      ? __ldg(pe_comm + (size_t)(h0.y + k) * K + gc.link_class[pl[k] * G + d])
                      : (T)0;
        const T term = ft[k] + (pl[k] == (uint32_t)d ? (T)0 : cm);
        est = term > est ? term : est;
      }
      if (__any_sync(FULL, npred > 4u)) {
        const uint32_t *pe_src = pg->pe_src;
        for (uint32_t k = 4; __any_sync(FULL, k < npred); k++) {
          if (k < npred) {
            T f;
            uint32_t p;
            const uint32_t q = __ldg(pe_src + h0.y + k);
            const W wq = (TOPO && share && (int32_t)q < t0) ? ((const W *)a.snap_rec)[q] : slab0[SLOT(q)];
            Slab<T>::decode(wq, f, p);
            T cm = 0;
            if (p != (uint32_t)d && d < G)
              cm = K == 1 ? __ldg(pe_comm + h0.y + k) : __ldg(pe_comm + (size_t)(h0.y + k) * K + gc.link_class[p * G + d]);
            const T term = f + cm;
            est = term > est ? term : est;
          }
        }
      }
      // INSERT (R1i): the first idle slot [ga, gb) before avail
      // with max(ga, r) + w <= gb, else the open-ended slot at avail
      // (the slots are disjoint and sorted, so no slot ending before r can
      // fit: a binary search finds the first with b >= r, then a short scan)
      uint32_t gk = NONE;
      T ga = 0, gbb = 0;
      if (INS && live && d < G && est < avail) {
        uint32_t lo = 0, hi = gn;
        while (lo < hi) {
          const uint32_t mid = (lo + hi) >> 1;
          if (gsl[mid].b < est) lo = mid + 1;
          else hi = mid;
        }
        T t = avail;
        for (uint32_t k = lo; k < gn; k++) {
          const GapSlot<T> e = gsl[k];
          const T tt = e.a > est ? e.a : est;
          if (tt + cst <= e.b) {
            gk = k;
            ga = e.a;
            gbb = e.b;
            t = tt;
            break;
          }
        }
        est = t;
      }
      const T eft = est + cst;

      // device forced by a perturbation pin (hard) or a CP pin (Alg. 1 l.9-10)
      int forced = -1;
      bool pert = false;
      if (any_pins) {
        if (GP >= 4) {
          const unsigned pm = __ballot_sync(FULL, live && my_pos == i) & gm;
          const int fd = __shfl_sync(FULL, my_dev, pm ? __ffs(pm) - 1 : lane);
          if (pm) {
            forced = fd;
            pert = true;
          }
        } else {
#pragma unroll
          for (int k = 0; k < MAXPINS; k++)
            if (live && pp[k] == i) {
              forced = (int)((pdv >> (8 * k)) & 0xFF);
              pert = true;
            }
        }
      }
      if (any_cp && __any_sync(FULL, live && h0.w != NONE)) {
        const uint32_t cpidx = h0.w;
        uint32_t below;
        if (GP >= 4) below = __popc(__ballot_sync(FULL, d < np && my_pcp < cpidx) & gm);
        else below = (pcp[0] < cpidx) + (pcp[1] < cpidx) + (pcp[2] < cpidx) + (pcp[3] < cpidx);
        const uint32_t fi = cpidx - below;
        const unsigned rm = __ballot_sync(FULL, live && forced < 0 && cpidx != NONE && d < nrounds && fi >= r_lo &&
                                                    fi < r_hi) & gm;
        const int rd = __shfl_sync(FULL, r_dev, rm ? __ffs(rm) - 1 : lane);
        if (rm) forced = rd;
      }
      int64_t mem = 0;
      if (MEM) mem = (int64_t)(((uint64_t)__ldg(cd + CW_MEMHI) << 32) | __ldg(cd + CW_MEMLO));
      bool feas = live && dev_ok && (forced < 0 || d == forced);
      if (cap_chk && (forced < 0 || pert)) feas = feas && (used + reserved + mem <= cap_d);
      // argmin EFT over feasible devices, ties -> lowest device (Alg. 1 l.12-19, R3, R8)
      const T key = feas ? eft : TT<T>::MAXV;
      T mn = key;
#pragma unroll
      for (int o = GP >> 1; o >= 1; o >>= 1) {
        const T x = __shfl_xor_sync(FULL, mn, o);
        mn = x < mn ? x : mn;
      }
      const unsigned fm = __ballot_sync(FULL, feas && key == mn) & gm;
      if (live && !fm) {
        infeas = true;
        if (!TOPO) top = 0;
      }
      const bool go = live && fm != 0;
      const int dsel = fm ? __ffs(fm) - 1 - gb : 0;
      if (snap_rec_on && go) {
        if (d < G) ((T *)a.snap_avail)[(size_t)tstep * G + d] = avail;
        if (MEM && a.snap_used && d < G) {  // memory before the step (lane kernel MM 1 / MM 2)
          ((int64_t *)a.snap_used)[(size_t)tstep * G + d] = used;
          ((int64_t *)a.snap_ur)[(size_t)tstep * G + d] = used + reserved;
        }
        if (d == 0) {
          ((T *)a.snap_ms)[tstep] = makespan;
          a.snap_dq[i] = (uint32_t)tstep;
          W rw;
          Slab<T>::make(rw, mn, (uint32_t)dsel);
          ((W *)a.snap_rec)[i] = rw;
        }
      }
      tstep++;
      if (INS) {
        // the chosen device's lane updates its idle slots: the slot the op
        // went into shrinks, splits in two (the tail of the array shifts
        // up one) or disappears (the tail shifts down); an op appended
        // after a data wait leaves a new slot [avail, ST)
        if (go && d == dsel) {
          if (gk != NONE) {
            const bool left = est > ga, right = est + cst < gbb;
            if (left && right) {
              for (uint32_t k = gn; k > gk + 1; k--) gsl[k] = gsl[k - 1];
              GapSlot<T> ne;
              ne.a = est + cst;
              ne.b = gbb;
              gsl[gk + 1] = ne;
              gsl[gk].b = est;
              gn++;
            } else if (left) {
              gsl[gk].b = est;
            } else if (right) {
              gsl[gk].a = est + cst;
            } else {
              for (uint32_t k = gk; k + 1 < gn; k++) gsl[k] = gsl[k + 1];
              gn--;
            }
          } else {
            if (est > avail) {
              GapSlot<T> ne;
              ne.a = avail;
              ne.b = est;
              gsl[gn++] = ne;
            }
            avail = mn;
          }
        }
      }
      if (go && d == dsel) {
        if (!INS) avail = mn;
        if (MEM) {
          used += mem;
          if (forced >= 0 && !pert) reserved -= mem;
          if (lmem) peakv = used > peakv ? used : peakv;
        }
      }
      if (lmem) {
        // R24: this op was the last unreleased consumer of an input -> free
        // that input's output bytes on its device; a sink frees its own
        uint32_t hw[4];
#pragma unroll
        for (int k = 0; k < 4; k++) hw[k] = (go && (uint32_t)k < npred) ? Slab<T>::hiword(slab0, SLOT(src[k])) : 256u;
        __syncwarp();
#pragma unroll
        for (int k = 0; k < 4; k++)
          if (go && (uint32_t)k < npred) {
            if (d == 0) Slab<T>::set_hiword(slab0, SLOT(src[k]), hw[k] - 256u);
            if ((hw[k] >> 8) == 1u && (uint32_t)d == pl[k]) used -= __ldg(pg->act + src[k]);
          }
        if (__any_sync(FULL, go && npred > 4u)) {
          for (uint32_t k = 4; __any_sync(FULL, go && k < npred); k++) {
            uint32_t sp = 0, w = 256u;
            if (go && k < npred) {
              sp = __ldg(pg->pe_src + h0.y + k);
              w = Slab<T>::hiword(slab0, SLOT(sp));
            }
            __syncwarp();
            if (go && k < npred) {
              if (d == 0) Slab<T>::set_hiword(slab0, SLOT(sp), w - 256u);
              if ((w >> 8) == 1u && (uint32_t)d == (w & 0xFFu)) used -= __ldg(pg->act + sp);
            }
          }
        }
        if (go && nsucc == 0 && d == dsel) used -= __ldg(pg->act + i);
      }
      if (go) makespan = mn > makespan ? mn : makespan;
      // (the indegree field of a scheduled op holds its consumer count under R24)
      if (go && d == 0) Slab<T>::sched(slab0, SLOT(i), mn, (uint32_t)dsel | (lmem ? nsucc << 8 : 0u));
      if (any_out) {
        const T stt = __shfl_sync(FULL, est, gb + dsel);
        if (go && want_out && d == 0) {
          const uint32_t u = __ldg(cd + CW_UID);
          a.out.place[ob + u] = (uint8_t)dsel;
          if (a.out.start) a.out.start[ob + u] = (int64_t)stt;
          if (a.out.deq) a.out.deq[ob + seq] = (int32_t)u;
        }
        seq++;
      }
      if constexpr (TOPO) {
        __syncwarp();
        continue;
      }
      // release successors into the ready bitmap
      uint32_t bits = 0;
      if (go && (uint32_t)d < nsucc) {
        const uint32_t dg = sdeg - 1;
        Slab<T>::set_indeg(slab0, SLOT(s0), dg);
        if (dg == 0) {
          red_or_s(la + 4u * (s0 >> 5), 1u << (s0 & 31));
          red_or_s(sa + 4u * (s0 >> 10), 1u << ((s0 >> 5) & 31));
          bits = 1u << (s0 >> 10);
        }
      }
      if (__any_sync(FULL, go && nsucc > (uint32_t)GP)) {
        for (uint32_t kk = GP + d; __any_sync(FULL, go && kk - d < nsucc); kk += GP) {
          if (go && kk < nsucc) {
            const uint32_t dst = kk < (uint32_t)S_IN ? __ldg(cd + CW_SUCC + kk) : __ldg(pg->se_dst + h0.z + kk);
            const uint32_t dg = Slab<T>::indeg(slab0, SLOT(dst)) - 1;
            Slab<T>::set_indeg(slab0, SLOT(dst), dg);
            if (dg == 0) {
              red_or_s(la + 4u * (dst >> 5), 1u << (dst & 31));
              red_or_s(sa + 4u * (dst >> 10), 1u << ((dst >> 5) & 31));
              bits |= 1u << (dst >> 10);
            }
          }
        }
      }
#pragma unroll
      for (int o = GP >> 1; o >= 1; o >>= 1) bits |= __shfl_xor_sync(FULL, bits, o);
      top |= bits;
      __syncwarp();
    }

    // ------------------------------------------------------------ epilogue
    if (snap_rec_on && run && !infeas) {
      if (d < G) ((T *)a.snap_avail)[(size_t)tstep * G + d] = avail;
      if (MEM && a.snap_used && d < G) {
        ((int64_t *)a.snap_used)[(size_t)tstep * G + d] = used;
        ((int64_t *)a.snap_ur)[(size_t)tstep * G + d] = used + reserved;
      }
      if (d == 0) ((T *)a.snap_ms)[tstep] = makespan;
    }
    if (run) {
      const int64_t ms64 = infeas ? I64MAX : (int64_t)makespan;
      const int64_t ri = s_res[lead], si = s_sidx[lead];
      if (ri >= 0) {
        if (d == 0) {
          a.out.makespan[ri] = ms64;
          a.out.status[ri] = infeas ? 1 : 0;
        }
        if (a.out.peak && d < G) a.out.peak[ri * G + d] = infeas ? -1 : (lmem ? peakv : used);
        if (infeas && a.out.place != nullptr) {
          const int64_t o2 = ri * (int64_t)a.out.vmax;
          for (int32_t u = d; u < a.out.vmax; u += GP) {
            a.out.place[o2 + u] = 0xFF;
            if (a.out.start) a.out.start[o2 + u] = -1;
            if (a.out.deq) a.out.deq[o2 + u] = -1;
          }
        }
      }
      if (d == 0 && !infeas && (ms64 < s_best[lead][0] || (ms64 == s_best[lead][0] && si < s_best[lead][1]))) {
        s_best[lead][0] = ms64;
        s_best[lead][1] = si;
      }
    }
    __syncwarp();
  }
  __syncwarp();
  if (a.track_best && d == 0) {
    a.wbest[2 * cslot] = s_best[lead][0];
    a.wbest[2 * cslot + 1] = s_best[lead][1];
  }
}

}  // namespace fastt
