// k_sim_lane.cu -- position-order DPOS simulation, one candidate per lane
// (SURVEY 8(a) S2, S5, S6, S7 for the candidates that keep the base ranks).
//
// When the prepared priority order is topological (PrepGraph::topo: every
// edge has w_i + c_ij > 0, so rank_u strictly decreases along edges, R2) the
// op dequeued at step t is the op at priority position t for EVERY candidate
// that keeps the base ranks (see k_sim.cu, TOPO).  All 32 candidates of a
// warp therefore process the same op at the same step: the op's card, cost
// row and comm values are warp-uniform loads (one transaction each), and the
// per-candidate work is lane-local -- no shuffles, no votes, no shared
// memory.  Lane l owns candidate q0 + l:
//   state   : avail[d] (Alg. 1 "avail[j]", APPEND reading R1) and the running
//             makespan in registers; the per-op record FT | place in the
//             warp's slab column [position][32 lanes] (a step's 32 stores
//             are one 256-B line).
//   EST     : with one link class the transfer time of an edge does not
//             depend on the device pair (R10), so the arrival of a
//             predecessor is FT + c on every device except its own, where it
//             is FT (R6).  Let M = max over preds of FT + c, attained by a
//             pred on device pa.  On any device d != pa the arrival is M
//             (that pred contributes M, nothing exceeds it); on pa it is
//             E = max over preds of (place == pa ? FT : FT + c).  So the
//             device loop is EST(d) = max(avail[d], d == pa ? E : M)
//             (P:571-574), EFT = EST + cost[op][d], argmin with ties to the
//             lowest device (Alg. 1 lines 12-19, R3).  Several link classes
//             (CM = 2) evaluate each (pred, device) term directly.
//   CP pins : no memory caps on this path (R8), so Alg. 1 line 5 / R9 is one
//             round: every free CP op goes to the device with the smallest
//             total cost of the free CP ops (equal counts, exact compare).
//   sharing : a candidate whose schedule provably equals the BASE schedule
//             before its first pinned op (k_sim.cu) starts at that
//             step t0 from the recorded BASE avail/makespan; records of
//             positions before t0 are read from the BASE record in place.
// Memory caps, liveness memory, INSERT, per-op outputs, SPLIT and
// rank-changing candidates stay on k_sim (group-per-candidate kernel).
#include "fastt_internal.cuh"
#include "sim_common.cuh"

namespace fastt {

template <typename T> struct RowLd;
template <> struct RowLd<uint32_t> {
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

// CM: 0 = uint32 time and one link class, comm values inline in the card;
//     1 = one link class, comm per edge from pe_comm;
//     2 = several link classes (per (pred, device) comm).
template <typename T, int GSH, int CM>
__global__ void __launch_bounds__(LANE_BLOCK, LANE_MINB) k_sim_lane(SimArgs a) {
  typedef typename Slab<T>::W W;
  constexpr int GP = 1 << GSH;
  static_assert(CM != 0 || sizeof(T) == 4, "card comm values are uint32");
  const int lane = threadIdx.x & 31;
  const int64_t gwarp = (int64_t)blockIdx.x * (LANE_BLOCK / 32) + (threadIdx.x >> 5);
  // this lane's slab column: record of position p at col[p * 32]
  W *const col = (W *)a.slab + (size_t)gwarp * (size_t)a.slab_stride * 32 + lane;
  const GraphConst &gc = *a.gc;
  const int G = a.G;
  const int K = gc.K;
  const PrepGraph *pg = a.base;
  const uint32_t *__restrict__ card = pg->card;
  const T *__restrict__ costp = (const T *)pg->costp;
  const T *__restrict__ pe_comm = (const T *)pg->pe_comm;
  const uint32_t *__restrict__ pe_src = pg->pe_src;
  const uint32_t *__restrict__ posm = pg->pos;
  const int32_t n = pg->n, Vraw = pg->V, cpl = pg->cp_len;
  const W *__restrict__ snap = (const W *)a.snap_rec;
  const bool cp_on = (a.flags & 1u) != 0;
  const uint32_t all = all_devices(G);
  int64_t bms = I64MAX, bidx = -1;  // this lane's best (makespan, stream index) for the sweep argmin

  for (;;) {
    unsigned long long q0 = 0;
    if (lane == 0) q0 = atomicAdd(a.counter, 32ull);
    q0 = __shfl_sync(FULL, q0, 0);
    if ((int64_t)q0 >= a.n) break;
    const int64_t q = (int64_t)q0 + lane;
    const bool active = q < a.n;
    Cand c;
    c.kind = 0;
    c.n_pins = 0;
    c.split_op = -1;
    c.dev_mask = 0;
    int64_t res_idx = -1, sidx = q;
    if (active) {
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
    if (active) {
      if (c.dev_mask & ~all) st = 2;
      else if (c.dev_mask && c.dev_mask != all) defer = true;  // device subset (R25): own ranks
      if (st) {
      } else if (c.kind == 0) {
      } else if (c.kind == 1) {
        np = c.n_pins;
        if (np < 1 || np > MAXPINS) st = 2;
        else {
          const uint32_t dset = c.dev_mask ? c.dev_mask : all;
          bool bad = false;
          for (int k = 0; k < np; k++) {
            const int32_t o = c.pin_op[k];
            if (o < 0 || o >= Vraw || posm[o] == NONE || c.pin_dev[k] >= G || !((dset >> c.pin_dev[k]) & 1u))
              bad = true;
            for (int k2 = 0; k2 < k; k2++) bad |= c.pin_op[k2] == o;
          }
          if (bad) st = 2;
        }
      } else if (c.kind == 2) {
        const int32_t o = c.split_op;
        if (o < 0 || o >= Vraw || posm[o] == NONE || c.split_dim > 1 || !(a.split_mask[o] & (1u << c.split_dim)) ||
            c.split_n < 2 || c.split_n > G)
          st = 2;
        else defer = true;
      } else {
        st = 2;
      }
    }
    if (st) {
      np = 0;
      defer = false;
    }
    uint32_t pp[MAXPINS] = {NONE, NONE, NONE, NONE};
    uint32_t pdv = 0;
    if (active && !defer)
      for (int k = 0; k < np; k++) {
        pp[k] = posm[c.pin_op[k]];
        pdv |= (uint32_t)c.pin_dev[k] << (8 * k);
      }
    // pins that change w or c (R5) need the candidate's own ranks
    if (active && !defer)
      for (int k = 0; k < np && !defer; k++)
        defer = pin_changes_ranks<T>(pg, gc, c, np, pp[k], c.pin_dev[k], G, K);
    if (active && defer) {
      const unsigned long long k = atomicAdd(a.ndefer, 1ull);
      a.defer_q[k] = q;
    }
    if (active && !defer && st && res_idx >= 0) {
      a.out.makespan[res_idx] = I64MAX;
      a.out.status[res_idx] = st;
    }
    const bool run = active && !defer && st == 0;

    // ------------------------------------------------------ prologue
    // CP devices (Alg. 1 line 5, R9) without memory caps: one
    // round over the free CP ops (perturbation-pinned CP ops excluded)
    int r_dev = -1;
    int m = 0;
    if (run && cp_on && cpl > 0) {
      uint32_t pc[MAXPINS];
#pragma unroll
      for (int k = 0; k < MAXPINS; k++) {
        pc[k] = k < np ? __ldg(card + (size_t)pp[k] * CARD_WORDS + CW_CPIDX) : NONE;
        m += pc[k] != NONE;
      }
      if (cpl - m > 0) {
        int64_t bs = 0;
        for (int d = 0; d < G; d++) {
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
    if (run && a.snap_mode == 2) {
      share = m == 0 || (a.snap_round_dev >= 0 && r_dev == a.snap_round_dev);
      if (share) {
        t0 = n;
        for (int k = 0; k < np; k++) {
          const int32_t dq = (int32_t)__ldg(a.snap_dq + pp[k]);
          t0 = dq < t0 ? dq : t0;
        }
      }
    }
    T avail[GP];
    T ms = 0;
#pragma unroll
    for (int d = 0; d < GP; d++) avail[d] = 0;
    if (share) {
      const T *sa = (const T *)a.snap_avail + (size_t)t0 * G;
#pragma unroll
      for (int d = 0; d < GP; d++)
        if (d < G) avail[d] = __ldg(sa + d);
      ms = __ldg((const T *)a.snap_ms + t0);
    }
    int32_t lo = run ? t0 : n;
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) {
      const int32_t x = __shfl_xor_sync(FULL, lo, o);
      lo = x < lo ? x : lo;
    }

    // ---------------------------------------------------------- main loop
    for (int32_t t = lo; t < n; t++) {
      const bool live = run && t >= t0;
      const uint32_t *cd = card + (size_t)t * CARD_WORDS;
      const uint4 h0 = __ldg((const uint4 *)cd);
      const uint4 hs = __ldg((const uint4 *)(cd + CARD_HDR));
      uint4 hc = make_uint4(0, 0, 0, 0);
      if (CM == 0) hc = __ldg((const uint4 *)(cd + CW_PCOMM));
      T cst[GP];
      RowLd<T>::template load<GP>(costp + (size_t)t * G, G, cst);
      const uint32_t npred = h0.x & 0xFFFF;
      const uint32_t src[4] = {hs.x, hs.y, hs.z, hs.w};
      // predecessor records (unused card slots hold position 0: valid address)
      W rw[4];
#pragma unroll
      for (int k = 0; k < 4; k++) rw[k] = (share && (int32_t)src[k] < t0) ? snap[src[k]] : col[(size_t)src[k] * 32];
      T f[4];
      uint32_t p[4];
#pragma unroll
      for (int k = 0; k < 4; k++) {
        T ft;
        uint32_t pl;
        Slab<T>::decode(rw[k], ft, pl);
        f[k] = (uint32_t)k < npred ? ft : (T)0;
        p[k] = (uint32_t)k < npred ? pl : 0xFFu;
      }
      T arrd[GP];  // CM 2: arrival per device
      T M = 0, E = 0;
      uint32_t pa = 0xFFu;
      if (CM != 2) {
        T R[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
          T cm;
          if (CM == 0) cm = (T)(k == 0 ? hc.x : k == 1 ? hc.y : k == 2 ? hc.z : hc.w);
          else cm = (uint32_t)k < npred ? __ldg(pe_comm + h0.y + k) : (T)0;
          R[k] = (uint32_t)k < npred ? f[k] + cm : (T)0;
        }
#pragma unroll
        for (int k = 0; k < 4; k++)
          if ((uint32_t)k < npred && (pa == 0xFFu || R[k] > M)) {
            M = R[k];
            pa = p[k];
          }
        if (npred > 4u) {  // (warp-uniform)
          for (uint32_t k = 4; k < npred; k++) {
            const uint32_t qs = __ldg(pe_src + h0.y + k);
            const W w = (share && (int32_t)qs < t0) ? snap[qs] : col[(size_t)qs * 32];
            T ft;
            uint32_t pl;
            Slab<T>::decode(w, ft, pl);
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
            const uint32_t qs = __ldg(pe_src + h0.y + k);
            const W w = (share && (int32_t)qs < t0) ? snap[qs] : col[(size_t)qs * 32];
            T ft;
            uint32_t pl;
            Slab<T>::decode(w, ft, pl);
            const T v = pl == pa ? ft : ft + __ldg(pe_comm + h0.y + k);
            E = v > E ? v : E;
          }
        }
      } else {
#pragma unroll
        for (int d = 0; d < GP; d++) {
          T v = 0;
          if (d < G) {
#pragma unroll
            for (int k = 0; k < 4; k++)
              if ((uint32_t)k < npred) {
                const T term = p[k] == (uint32_t)d
                                   ? f[k]
                                   : f[k] + __ldg(pe_comm + (size_t)(h0.y + k) * K + gc.link_class[p[k] * G + d]);
                v = term > v ? term : v;
              }
            for (uint32_t k = 4; k < npred; k++) {
              const uint32_t qs = __ldg(pe_src + h0.y + k);
              const W w = (share && (int32_t)qs < t0) ? snap[qs] : col[(size_t)qs * 32];
              T ft;
              uint32_t pl;
              Slab<T>::decode(w, ft, pl);
              const T term =
                  pl == (uint32_t)d ? ft : ft + __ldg(pe_comm + (size_t)(h0.y + k) * K + gc.link_class[pl * G + d]);
              v = term > v ? term : v;
            }
          }
          arrd[d] = v;
        }
      }
      // device forced by a perturbation pin (hard) or a CP pin (Alg. 1 l.9-10)
      int forced = -1;
#pragma unroll
      for (int k = 0; k < MAXPINS; k++)
        if (pp[k] == (uint32_t)t) forced = (int)((pdv >> (8 * k)) & 0xFFu);
      if (forced < 0 && r_dev >= 0 && h0.w != NONE) forced = r_dev;
      // argmin EFT, ties -> lowest device (Alg. 1 lines 12-19, R3)
      T best = 0;
      int bd = -1;
#pragma unroll
      for (int d = 0; d < GP; d++) {
        if (d < G) {
          const T arr = CM == 2 ? arrd[d] : ((uint32_t)d == pa ? E : M);
          const T est = avail[d] > arr ? avail[d] : arr;
          const T eft = est + cst[d];
          if ((forced < 0 || forced == d) && (bd < 0 || eft < best)) {
            best = eft;
            bd = d;
          }
        }
      }
      if (live) {
#pragma unroll
        for (int d = 0; d < GP; d++)
          if (d == bd) avail[d] = best;
        ms = best > ms ? best : ms;
        W w;
        Slab<T>::make(w, best, (uint32_t)bd);
        col[(size_t)t * 32] = w;
      }
    }

    // ------------------------------------------------------------ epilogue
    if (run) {
      if (res_idx >= 0) {
        a.out.makespan[res_idx] = (int64_t)ms;
        a.out.status[res_idx] = 0;
      }
      if ((int64_t)ms < bms || ((int64_t)ms == bms && sidx < bidx)) {
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

template <typename T, int CM>
static const void *lane_fn_t(int gshift) {
  switch (gshift) {
    case 0: return (const void *)k_sim_lane<T, 0, CM>;
    case 1: return (const void *)k_sim_lane<T, 1, CM>;
    case 2: return (const void *)k_sim_lane<T, 2, CM>;
    case 3: return (const void *)k_sim_lane<T, 3, CM>;
    case 4: return (const void *)k_sim_lane<T, 4, CM>;
    default: return (const void *)k_sim_lane<T, 5, CM>;
  }
}
static const void *lane_fn(int tbits, int gshift, int cm) {
  if (tbits == 32) {
    if (cm == 0) return lane_fn_t<uint32_t, 0>(gshift);
    return cm == 1 ? lane_fn_t<uint32_t, 1>(gshift) : lane_fn_t<uint32_t, 2>(gshift);
  }
  return cm == 2 ? lane_fn_t<uint64_t, 2>(gshift) : lane_fn_t<uint64_t, 1>(gshift);
}

int lane_comm_mode(const SimArgs &a, int tbits) {
  if (a.fastcomm && tbits == 32) return 0;
  return a.gc_K == 1 ? 1 : 2;
}

void launch_sim_lane(const SimArgs &a, int tbits, int grid, cudaStream_t st) {
  const void *f = lane_fn(tbits, a.gshift, lane_comm_mode(a, tbits));
  SimArgs aa = a;
  void *args[] = {&aa};
  cudaLaunchKernel(f, dim3(grid), dim3(LANE_BLOCK), args, 0, st);
}

int lane_occupancy(int tbits, int gshift) {
  int nb = 1 << 30, x = 0;
  for (int cm = (tbits == 32 ? 0 : 1); cm < 3; cm++) {
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&x, lane_fn(tbits, gshift, cm), LANE_BLOCK, 0);
    nb = x < nb ? x : nb;
  }
  return nb;
}

}  // namespace fastt
