// k_lane_pk.cuh -- the sweep's dominant kernel: one candidate per lane on
// the base graph with packed device keys (the
// candidates that keep the base ranks, 32-bit time, one link class).
//
// Same method as k_sim_lane (k_sim_lane_body.cuh: position order, EST/EFT,
// argmin, CP pins, BASE-prefix sharing, memory modes), restaged for B200:
//   * every position has a compact 16-B aligned "PK card" (pkc, built once
//     per base by k_pack_costs): header (in-degree, edge base, CP index),
//     the 4 inline predecessor positions, their comm << GSH, the op's memory
//     and the packed cost row (cost << GSH | d).  The cards of 8 consecutive
//     positions (a chunk) are copied into the warp's 32-card ring by ONE
//     cp.async.bulk (TMA bulk engine, SASS UBLKCP) two chunks ahead, with
//     completion on an mbarrier (expect_tx / complete_tx) waited once per
//     chunk;
//   * records are packed keys FT << GSH | device (4 B): a step's 32 records
//     are one 128-B row of the warp's slab, so the up-to-4 far predecessor
//     rows of a step are staged by ONE warp-wide 16-B cp.async (lane l copies
//     chunk l & 7 of predecessor l >> 3) P steps ahead; a predecessor before
//     the warp's start step lo is the BASE record (the same for every lane):
//     its 16-B chunk of the BASE key array is staged and word s & 3 read.
//     With the copies the issuing step writes the step's read plan (per
//     predecessor: the shared-memory address of its record, per-lane or
//     not), so the step itself reads each record with one add and one load.
// The state record rows are written by this warp with plain stores and read
// back by cp.async (the generic proxy); only the read-only cards (written by
// an earlier kernel) go through the async proxy.
//
// CPL candidates per lane (CPL = 2 for the makespan-only sweep, MM 0): a
// warp runs 32 * CPL candidates, lane l holding candidates 2l and 2l + 1 of
// its batch.  Everything a step reads once per warp -- the card, the read
// plan, the staging issue, the loop and chunk control, the forced-device
// vote -- is shared by the lane's candidates; a record row is 32 * CPL keys
// (lane l's pair adjacent: one 8-B load / store per lane and predecessor).
#pragma once
#include "fastt_internal.cuh"
#include "sim_common.cuh"
#include "k_sim_lane_body.cuh"  // cp_rounds_lane, RowLd, cp.async helpers, LANE_D

namespace fastt {

// PK card: words 0-3 header (deg, pbase, cpidx, -), 4-7 predecessor
// positions, 8-11 their comm << GSH, 12-13 mem lo/hi, 14-15 -, then the
// packed cost row padded to a multiple of 4 words
__host__ __device__ constexpr int pk_card_words(int GP) { return 16 + ((GP + 3) / 4) * 4; }
__host__ __device__ constexpr int pk_card_bytes(int GP) { return 4 * pk_card_words(GP); }

constexpr int PK_CR = 32;  // card ring slots (4 chunks of 8)
template <int GP, int MM, int CPL = 1> __host__ __device__ constexpr size_t pk_mm_off() {
  // card mbarriers [4] u64 (64 B) | ring [D][32 CPL] u32 | stage [D][4][32 CPL] u32 |
  // read plans [D][8] u32 | cards [32] | avail keys [CPL][GP/2][32][2] u32 |
  // memory state (as k_sim_lane; CPL 1)
  return (size_t)64 + (size_t)LANE_D * 32 * 4 * CPL + (size_t)LANE_D * 4 * 32 * 4 * CPL + (size_t)LANE_D * 32 +
         (size_t)PK_CR * pk_card_bytes(GP) + (size_t)32 * GP * 4 * CPL;
}
template <int GP, int MM, int CPL = 1> __host__ __device__ constexpr size_t pk_smem_per_warp() {
  return pk_mm_off<GP, MM, CPL>() + (MM >= 1 ? (size_t)32 * GP * 8 * CPL : 0) + (MM == 2 ? (size_t)32 * GP * 8 : 0);
}

__device__ __forceinline__ void mbar_init(uint32_t a, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(count) : "memory");
}
// arrive (the barrier's single expected arrival) and expect `bytes` of
// asynchronous copies (complete_tx) before the phase completes
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t a, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(a), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t a, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred done;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 done, [%0], %1;\n\t"
      "@!done bra WAIT_%=;\n}\n" ::"r"(a),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes, uint32_t mbar) {
  asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(mbar)
               : "memory");
}
__device__ __forceinline__ void cp16_if(bool p, uint32_t saddr, const void *g) {
  asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %2, 0;\n\t@q cp.async.cg.shared.global [%0], [%1], 16;\n}\n" ::"r"(
                   saddr),
               "l"(g), "r"((int)p)
               : "memory");
}

// EX: G == GP.  MM: memory mode (0 none, 1 peak, 2 caps; k_sim_lane).
// CPL: candidates per lane (2 only with MM 0).
template <int GSH, bool EX, int MM, int CPL>
__global__ void __launch_bounds__(LANE_BLOCK, CPL == 1 ? LANE_MINB : CPL == 2 ? 3 : 2) k_lane_pk(SimArgs a) {
  constexpr int GP = 1 << GSH;
  constexpr uint32_t GMK = GP - 1;
  constexpr int D = LANE_D, P = D - 1;
  constexpr int CB = pk_card_bytes(GP);
  constexpr int RW = 32 * CPL;  // keys per record row
  static_assert((D & (D - 1)) == 0 && CB % 16 == 0, "pipeline slots");
  static_assert(CPL == 1 || (CPL == 2 && MM <= 1) || (CPL == 4 && MM == 0),
                "two candidates per lane: makespan (+ peak memory); four: makespan only");
  const int lane = threadIdx.x & 31;
  int64_t gwarp = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5) + a.gwarp_off;
  if (a.lane_batches > 0) {
    // non-persistent launch: the warp's slab column block and wbest entry
    // are a slot taken from the bitmap for the warp's lifetime (at most
    // n_slab_slots warps are resident, so one is always free)
    uint32_t sl = 0;
    if (lane == 0) {
      const uint32_t nw = (uint32_t)(a.n_slab_slots + 31) >> 5;
      for (uint32_t w = (uint32_t)(gwarp % nw);; w = w + 1 == nw ? 0 : w + 1) {
        uint32_t v = a.slot_bm[w];
        bool got = false;
        while (~v) {
          const uint32_t b = __ffs(~v) - 1;
          if (w * 32 + b >= (uint32_t)a.n_slab_slots) break;
          const uint32_t old = atomicOr(&a.slot_bm[w], 1u << b);
          if (!(old & (1u << b))) {
            sl = w * 32 + b;
            got = true;
            break;
          }
          v = old | (1u << b);
        }
        if (got) break;
      }
      __threadfence();  // (the previous holder's wbest entry is visible)
    }
    gwarp = __shfl_sync(FULL, (int)sl, 0);
  }
  // this lane's slab columns (record of position p, candidate j at
  // col[p * RW + j]); row p of the warp (all RW records) starts at col0 + p * RW
  uint32_t *const col = (uint32_t *)a.slab + (size_t)gwarp * (size_t)a.slab_stride * RW + CPL * lane;
  const uint32_t *const col0 = col - CPL * lane;
  extern __shared__ __align__(16) unsigned char lsm[];
  unsigned char *const wsm = lsm + (threadIdx.x >> 5) * pk_smem_per_warp<GP, MM, CPL>();
  const uint32_t wsa = (uint32_t)__cvta_generic_to_shared(wsm);
  const uint32_t mbar_sa = wsa;                                         // card barriers [4] u64
  uint32_t *const ring = (uint32_t *)(wsm + 64) + CPL * lane;          // [D][RW]
  const uint32_t ring_sa = wsa + 64;
  const uint32_t stage_sa = ring_sa + D * 4 * RW;                       // [D][4][RW]
  uint32_t *const plan = (uint32_t *)(wsm + 64 + D * 20 * RW);          // [D][8]: per predecessor (address, lane mask)
  unsigned char *const cards = wsm + 64 + D * 20 * RW + D * 32;         // [PK_CR][CB]
  const uint32_t cards_sa = wsa + 64 + D * 20 * RW + D * 32;
  // avail keys of candidate j: [GP/2][32][2] pairs of devices per lane
  uint32_t *const avk0 = (uint32_t *)(cards + PK_CR * CB) + (GP >= 2 ? 2 * lane : lane);
  auto avk_j = [&](int j) -> uint32_t * { return avk0 + j * 32 * GP; };
  auto avk_at = [&](int j, uint32_t d) -> uint32_t & {
    return GP >= 2 ? avk_j(j)[(d >> 1) * 64 + (d & 1)] : avk_j(j)[0];
  };
  // memory state (MM >= 1) of candidate j: mv_j(j)[d * 32]
  int64_t *const mv = (int64_t *)(wsm + pk_mm_off<GP, MM, CPL>()) + lane;
  auto mv_j = [&](int j) -> int64_t * { return mv + j * 32 * GP; };
  uint32_t *const s32b =
      (uint32_t *)(wsm + pk_mm_off<GP, MM, CPL>() + (size_t)32 * GP * 8) + (GP >= 4 ? 4 * lane : lane);
  uint32_t *const rnd = (uint32_t *)(wsm + pk_mm_off<GP, MM, CPL>() + (size_t)32 * GP * 12) + lane;
  auto s32_at = [&](uint32_t d) -> uint32_t & { return GP >= 4 ? s32b[(d >> 2) * 128 + (d & 3)] : s32b[d * 32]; };
  auto clamp32 = [](int64_t v) -> uint32_t { return v >= (int64_t)0xFFFFFFFFll ? 0xFFFFFFFFu : (uint32_t)v; };
  if (lane == 0)
    for (int j = 0; j < 4; j++) mbar_init(mbar_sa + 8 * j, 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();

  const GraphConst &gc = *a.gc;
  const int G = a.G;
  const PrepGraph *pg = a.base;
  const uint32_t *card = pg->card;
  const uint32_t *costp = (const uint32_t *)pg->costp;
  const uint32_t *pe_comm = (const uint32_t *)pg->pe_comm;
  const uint32_t *pe_src = pg->pe_src;
  const uint32_t *posm = pg->pos;
  const uint32_t *pkc = a.pkc;
  const int32_t n = pg->n, cpl = pg->cp_len;
  const uint32_t *__restrict__ snap = a.snap_key;
  // (CPL 2 / 4: each BASE key twice / four times, so an aligned 8-/16-B load
  // gives it to every candidate of a lane)
  const uint32_t *__restrict__ snapx = CPL == 1 ? a.snap_key : CPL == 2 ? a.snap_key2 : a.snap_key4;
  const bool cp_on = (a.flags & 1u) != 0;
  int64_t bms = I64MAX, bidx = -1;
  uint32_t zc = 0;  // card chunks issued by this warp so far (barrier zc & 3, phase (zc >> 2) & 1)
  // this lane's part of a step's record staging: chunks (lane & 7) + 8 i,
  // i < CPL, of inline predecessor (lane >> 3)
  const int pk_k = lane >> 3, pk_c = lane & 7;

  const int64_t nlim = a.n_dev ? ((int64_t)*a.n_dev < a.n ? (int64_t)*a.n_dev : a.n) : a.n;
  for (int32_t nb = 0; a.lane_batches <= 0 || nb < a.lane_batches; nb++) {
    unsigned long long q0 = 0;
    if (lane == 0) q0 = atomicAdd(a.counter, (unsigned long long)RW);
    q0 = __shfl_sync(FULL, q0, 0);
    if ((int64_t)q0 >= nlim) break;
    // ------------------------------------------------ per-candidate state
    int64_t q[CPL], res_idx[CPL], sidx[CPL];
    bool run[CPL], dead[CPL];
    uint32_t pp[CPL][MAXPINS], pdv[CPL], nxt[CPL], ms[CPL];
    int np[CPL], r_dev[CPL], m[CPL], nr[CPL], rc[CPL], rdv[CPL];
    uint32_t rhi[CPL];
    int32_t t0[CPL];
    const uint32_t all = all_devices(G);
#pragma unroll
    for (int j = 0; j < CPL; j++) {
      q[j] = (int64_t)q0 + CPL * lane + j;
      const bool active = q[j] < nlim;
      Cand c;
      c.kind = 0;
      c.n_pins = 0;
      c.split_op = -1;
      c.dev_mask = 0;
      res_idx[j] = -1;
      sidx[j] = q[j];
      if (active) {
        if (a.mode == 0) {
          sidx[j] = a.first + q[j] * a.stride;
          c = stream_cand(a.stream, sidx[j]);
        } else if (a.mode == 1) {
          c = a.cands[q[j]];
          res_idx[j] = q[j];
        } else {  // mode 3: list ordered by BASE-prefix start step
          c = a.cands[q[j]];
          res_idx[j] = a.slot_result ? a.slot_result[q[j]] : -1;
          sidx[j] = a.slot_index[q[j]];
        }
      }
      // -------------------------------------------------------- validate
      uint8_t st = 0;
      bool defer = false;
      np[j] = 0;
      if (active) {
        defer = cand_classify<uint32_t>(c, pg, gc, a.split_mask, G, !a.preclassified, st);
        np[j] = (st == 0 && c.kind == 1) ? c.n_pins : 0;
      }
      pdv[j] = 0;
#pragma unroll
      for (int k = 0; k < MAXPINS; k++) pp[j][k] = NONE;
      if (active && !defer)
        for (int k = 0; k < np[j]; k++) {
          pp[j][k] = posm[c.pin_op[k]];
          pdv[j] |= (uint32_t)c.pin_dev[k] << (8 * k);
        }
      if (active && defer) {
        const unsigned long long k = atomicAdd(a.ndefer, 1ull);
        a.defer_q[k] = q[j];
      }
      if (active && !defer && st && res_idx[j] >= 0) {
        a.out.makespan[res_idx[j]] = I64MAX;
        a.out.status[res_idx[j]] = st;
        if (MM && a.out.peak)
          for (int d = 0; d < G; d++) a.out.peak[res_idx[j] * G + d] = -1;
      }
      run[j] = active && !defer && st == 0;

      // ---------------------------------------------------- prologue
      // CP devices (Alg. 1 line 5, R9): without caps one round of
      // the free CP ops on the device of least total cost; with caps the
      // lane-local rounds with reservations (cp_rounds_lane)
      r_dev[j] = -1;
      m[j] = 0;
      nr[j] = 0;
      rc[j] = 0;
      rdv[j] = -1;
      rhi[j] = 0;
      dead[j] = false;
      if (MM && run[j]) {
#pragma unroll
        for (int d = 0; d < GP; d++) mv_j(j)[d * 32] = (MM == 2 && d < G) ? gc.cap[d] : 0;
      }
      if (run[j] && cp_on && cpl > 0) {
        uint32_t pc[MAXPINS];
#pragma unroll
        for (int k = 0; k < MAXPINS; k++) {
          pc[k] = k < np[j] ? __ldg(card + (size_t)pp[j][k] * CARD_WORDS + CW_CPIDX) : NONE;
          m[j] += pc[k] != NONE;
        }
        if (MM == 2) {
          nr[j] = cp_rounds_lane<uint32_t>(pg, gc, G, all, np[j], pp[j], pc, rnd, mv);
          if (nr[j] > 0) {
            rhi[j] = rnd[0] & 0xFFFFFFu;
            rdv[j] = (int)(rnd[0] >> 24);
          }
        } else if (cpl - m[j] > 0) {
          int64_t bs = 0;
          for (int d = 0; d < G; d++) {
            int64_t sd = pg->pcost[(int64_t)cpl * G + d];
#pragma unroll
            for (int k = 0; k < MAXPINS; k++)
              if (pc[k] != NONE) sd -= (int64_t)costp[(size_t)pp[j][k] * G + d];
            if (r_dev[j] < 0 || sd < bs) {
              bs = sd;
              r_dev[j] = d;
            }
          }
        }
      }
      // BASE-prefix sharing (k_sim_lane): the warp starts at lo = min t0
      t0[j] = 0;
      if (run[j] && a.snap_mode == 2 && (!MM || a.snap_used)) {
        const bool share = m[j] == 0 || (MM != 2 && a.snap_round_dev >= 0 && r_dev[j] == a.snap_round_dev);
        if (share) {
          t0[j] = n;
          for (int k = 0; k < np[j]; k++) {
            const int32_t dq = (int32_t)__ldg(a.snap_dq + pp[j][k]);
            t0[j] = dq < t0[j] ? dq : t0[j];
          }
        }
      }
    }
    bool run_any = false;
    int32_t lo = n;
#pragma unroll
    for (int j = 0; j < CPL; j++) {
      run_any |= run[j];
      if (run[j] && t0[j] < lo) lo = t0[j];
    }
    const int32_t nmax = __any_sync(FULL, run_any) ? n : 0;
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) {
      const int32_t x = __shfl_xor_sync(FULL, lo, o);
      lo = x < lo ? x : lo;
    }
    if (a.stat) {
      uint32_t mine = 0;
#pragma unroll
      for (int j = 0; j < CPL; j++) mine += run[j] ? (uint32_t)(n - lo) : 0u;
      const uint32_t ls = __reduce_add_sync(FULL, mine);
      if (lane == 0 && nmax > lo) {
        atomicAdd(a.stat, (unsigned long long)(nmax - lo) * CPL);
        atomicAdd(a.stat + 1, (unsigned long long)ls);
      }
    }
#pragma unroll
    for (int j = 0; j < CPL; j++) {
      ms[j] = 0;
#pragma unroll
      for (int d = 0; d < GP; d++) avk_at(j, d) = 0;
      if (run[j] && lo > 0) {  // (lo > 0: every running lane shares)
        const uint32_t *sa = (const uint32_t *)a.snap_avail + (size_t)lo * G;
#pragma unroll
        for (int d = 0; d < GP; d++)
          if (d < G) avk_at(j, d) = __ldg(sa + d) << GSH;
        ms[j] = __ldg((const uint32_t *)a.snap_ms + lo);
        if (MM == 1)
          for (int d = 0; d < G; d++) mv_j(j)[d * 32] = __ldg((const int64_t *)a.snap_used + (size_t)lo * G + d);
        if (MM == 2)
          for (int d = 0; d < G; d++)
            mv[d * 32] = gc.cap[d] - __ldg((const int64_t *)a.snap_ur + (size_t)lo * G + d);
      }
      if (MM == 2 && run[j]) {
#pragma unroll
        for (int d = 0; d < GP; d++) s32_at(d) = clamp32(mv[d * 32]);
      }
      nxt[j] = NONE;
#pragma unroll
      for (int k = 0; k < MAXPINS; k++)
        if (pp[j][k] >= (uint32_t)lo && pp[j][k] < nxt[j]) nxt[j] = pp[j][k];
    }

    // ------------------------------------------------------ pipeline
    // records: the far predecessor rows of step u are staged at step u - P
    // (one commit group per step, waited P - 1 groups later: the group of
    // step t is complete at step t); a record of position s < u is staged
    // iff s < max(lo, u - P), else read from the ring of the last D records.
    // cards: chunk c = positions [8c, 8c + 8) is copied by one bulk copy at
    // step 8(c - 2) and waited at step 8c - P (its first card is read by the
    // staging of step 8c); chunks up to j0 + 1 (j0 = ceil(lo / 8)) are copied
    // directly here.
    const int32_t jlo = lo >> 3, j0 = (lo + 7) >> 3;
    const uint32_t z0 = zc;
    uint32_t zw = zc;
    const uint32_t lane4 = 4u * CPL * (uint32_t)lane;
    {
      const int32_t pend = min(n, 8 * (j0 + 2));
      for (int32_t u = 8 * jlo; u < pend; u++) {
        const uint32_t *src = pkc + (size_t)u * (CB / 4);
        uint32_t *dst = (uint32_t *)(cards + (u & (PK_CR - 1)) * CB);
        for (int w = lane; w < CB / 4; w += 32) dst[w] = __ldg(src + w);
      }
    }
    __syncwarp();
    // (branch-free: past the last position the card slot is stale, the
    // copy is predicated off and the plan is never read)
    auto issue = [&](int32_t u) {  // records of step u and its read plan
      const uint32_t slot = (uint32_t)u & (D - 1);
      const uint32_t *cu = (const uint32_t *)(cards + (u & (PK_CR - 1)) * CB);
      const uint32_t npu = cu[0] & 0xFFFF;
      const uint32_t s = cu[4 + pk_k];
      const int32_t thr = lo > u - P ? lo : u - P;
      const bool staged = u < n && (uint32_t)pk_k < npu && (int32_t)s < thr;
      const bool base_rec = (int32_t)s < lo;  // the BASE record: one 16-B chunk holds it
      const uint32_t row = stage_sa + (slot * 4 + (uint32_t)pk_k) * (4 * RW);
      const uint32_t sw = CPL * s;  // the BASE key's word in the CPL-fold array
#pragma unroll
      for (int i = 0; i < CPL; i++) {
        const int cc = pk_c + 8 * i;
        const uint32_t *src = base_rec ? snapx + (sw & ~3u) : col0 + (size_t)s * RW + 4 * cc;
        cp16_if(staged && (!base_rec || cc == 0), row + 16 * cc, src);
      }
      // the read plan of predecessor pk_k: its record row's address and the
      // per-lane mask (0: the BASE record, the same word(s) for every
      // candidate; the 8 lanes of a predecessor store the same pair)
      const uint32_t ad = staged ? (base_rec ? row + 4 * (sw & 3u) : row) : ring_sa + (s & (D - 1)) * (4 * RW);
      const uint32_t mk = (staged && base_rec) ? 0u : 0xFFFFFFFFu;
      *(uint2 *)(plan + slot * 8 + 2 * pk_k) = make_uint2(ad, mk);
      cp_async_commit();
    };
    auto issue_chunk = [&](int32_t c) {  // cards [8c, 8c + 8) into the card ring
      if (8 * c < n) {
        const uint32_t z = zc++;
        if (lane == 0) {
          const uint32_t cnt = (uint32_t)min(8, n - 8 * c);
          const uint32_t mb = mbar_sa + 8 * (z & 3);
          mbar_arrive_expect_tx(mb, cnt * CB);
          bulk_g2s(cards_sa + (uint32_t)(((8 * c) & (PK_CR - 1)) * CB), pkc + (size_t)(8 * c) * (CB / 4), cnt * CB, mb);
        }
      }
    };
    for (int32_t u = lo; u < lo + P; u++) issue(u);
    // a record of position s, candidate j (extra predecessors beyond the card's 4)
    auto rec_at = [&](uint32_t s, int32_t t, int j) -> uint32_t {
      if ((int32_t)s < lo) return __ldg(snap + s);
      if ((int32_t)s + P >= t) return ring[(s & (D - 1)) * RW + j];
      return col[(size_t)s * RW + j];
    };
    for (int32_t t = lo; t < nmax; t++) {
      if (((t + P) & 7) == 0) {  // the next chunk's first card is staged below
        const int32_t c = (t + P) >> 3;
        if (c >= j0 + 2 && 8 * c < n) {
          const uint32_t z = z0 + (uint32_t)(c - (j0 + 2));
          mbar_wait(mbar_sa + 8 * (z & 3), (z >> 2) & 1);
          zw = z + 1;
        }
      }
      if ((t & 7) == 0) issue_chunk((t >> 3) + 2);
      cp_async_wait<P - 1>();  // the group of step t: its staged records
      __syncwarp();            // (and the read plan other lanes wrote)
      const uint32_t *cw = (const uint32_t *)(cards + (t & (PK_CR - 1)) * CB);
      const uint4 h0 = *(const uint4 *)cw;
      const uint4 hc = *(const uint4 *)(cw + 8);  // comm << GSH (0 in unused slots)
      uint32_t cst[GP];
      RowLd<uint32_t>::template load_s<GP>(cw + 16, G, cst);
      uint32_t memlo = 0, memhi = 0;
      if (MM) {
        const uint2 mw = *(const uint2 *)(cw + 12);
        memlo = mw.x;
        memhi = mw.y;
      }
      const int64_t mem64 = (int64_t)(((uint64_t)memhi << 32) | memlo);
      const uint32_t npred = h0.x & 0xFFFF;
      uint32_t rk[CPL][4];
      {
        const uint4 pa = *(const uint4 *)(plan + (t & (D - 1)) * 8);
        const uint4 pb = *(const uint4 *)(plan + (t & (D - 1)) * 8 + 4);
        const uint32_t ad[4] = {pa.x + (lane4 & pa.y), pa.z + (lane4 & pa.w), pb.x + (lane4 & pb.y),
                                pb.z + (lane4 & pb.w)};
#pragma unroll
        for (int k = 0; k < 4; k++) {
          if (CPL == 1) {
            rk[0][k] = *(const uint32_t *)__cvta_shared_to_generic(ad[k]);
          } else if (CPL == 2) {  // (a BASE record is a doubled pair: the same key for both)
            const uint2 x = *(const uint2 *)__cvta_shared_to_generic(ad[k]);
            rk[0][k] = x.x;
            rk[CPL - 1][k] = x.y;
          } else {
            const uint4 x = *(const uint4 *)__cvta_shared_to_generic(ad[k]);
            rk[0][k] = x.x;
            rk[1 % CPL][k] = x.y;
            rk[2 % CPL][k] = x.z;
            rk[3 % CPL][k] = x.w;
          }
        }
      }
      // (the slots issue(t + P) overwrites were read at step t - 1, before
      // every lane passed this step's __syncwarp)
      issue(t + P);
      const uint32_t hcw[4] = {hc.x, hc.y, hc.z, hc.w};
      uint32_t bk[CPL], key[CPL][GP], kpa[CPL], fk[CPL][GP], fkpa[CPL];
      uint32_t pq[CPL];
#pragma unroll
      for (int j = 0; j < CPL; j++) {
        // arrival terms in key space (k_sim_lane): R_k = key_k + (c_k << GSH)
        uint32_t rkm[4], R[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
          rkm[k] = (uint32_t)k < npred ? rk[j][k] : 0u;
          R[k] = rkm[k] + hcw[k];
        }
        uint32_t Mkey = max(max(R[0], R[1]), max(R[2], R[3]));
        if (npred > 4u)  // (warp-uniform)
          for (uint32_t k = 4; k < npred; k++)
            Mkey = max(Mkey, rec_at(__ldg(pe_src + h0.y + k), t, j) + (__ldg(pe_comm + h0.y + k) << GSH));
        uint32_t Ekey = 0;
#pragma unroll
        for (int k = 0; k < 4; k++) Ekey = max(Ekey, ((rkm[k] ^ Mkey) & GMK) == 0u ? rkm[k] : R[k]);
        if (npred > 4u)
          for (uint32_t k = 4; k < npred; k++) {
            const uint32_t r = rec_at(__ldg(pe_src + h0.y + k), t, j);
            Ekey = max(Ekey, ((r ^ Mkey) & GMK) == 0u ? r : r + (__ldg(pe_comm + h0.y + k) << GSH));
          }
        const uint32_t Mk = Mkey & ~GMK, Ek = Ekey & ~GMK;
        pq[j] = Mkey & GMK;
        // keys (EFT << GSH) | d (Alg. 1 lines 12-19, R3, R6)
        uint32_t av[GP];
        if (GP >= 2) {
#pragma unroll
          for (int i = 0; i < GP / 2; i++) {
            const uint2 x = *(const uint2 *)(avk_j(j) + i * 64);
            av[2 * i] = x.x;
            av[2 * i + 1] = x.y;
          }
        } else {
          av[0] = avk_j(j)[0];
        }
        const uint32_t ap = avk_at(j, pq[j]), cpa = cw[16 + pq[j]];
        kpa[j] = (ap > Ek ? ap : Ek) + cpa;
        if (!EX && pq[j] >= (uint32_t)G) kpa[j] = 0xFFFFFFFFu;
#pragma unroll
        for (int d = 0; d < GP; d++) key[j][d] = (EX || d < G) ? (av[d] > Mk ? av[d] : Mk) + cst[d] : 0xFFFFFFFFu;
#pragma unroll
        for (int d = 0; d < GP; d++) fk[j][d] = key[j][d];
        fkpa[j] = kpa[j];
        if (MM == 2) {  // Alg. 1 line 13, R8 (k_sim_lane)
          if (memhi != 0) {
#pragma unroll
            for (int d = 0; d < GP; d++)
              if (mv[d * 32] < mem64) fk[j][d] = 0xFFFFFFFFu;
            if (mv[pq[j] * 32] < mem64) fkpa[j] = 0xFFFFFFFFu;
          } else {
            uint32_t sv[GP];
            if (GP >= 4) {
#pragma unroll
              for (int i = 0; i < GP / 4; i++) {
                const uint4 x = *(const uint4 *)(s32b + i * 128);
                sv[4 * i] = x.x;
                sv[4 * i + 1] = x.y;
                sv[4 * i + 2] = x.z;
                sv[4 * i + 3] = x.w;
              }
            } else {
#pragma unroll
              for (int d = 0; d < GP; d++) sv[d] = s32b[d * 32];
            }
#pragma unroll
            for (int d = 0; d < GP; d++)
              if (sv[d] < memlo) fk[j][d] = 0xFFFFFFFFu;
            if (s32_at(pq[j]) < memlo) fkpa[j] = 0xFFFFFFFFu;
          }
        }
        bk[j] = fkpa[j];
#pragma unroll
        for (int d = 0; d < GP; d++) bk[j] = fk[j][d] < bk[j] ? fk[j][d] : bk[j];
      }
      // the device forced by a perturbation pin (hard) or a CP round (Alg. 1
      // l.9-10, R9; cpf: memory reserved up front) -- rare steps
      bool want = false;
#pragma unroll
      for (int j = 0; j < CPL; j++) {
        const bool cp_any = MM == 2 ? rc[j] < nr[j] : r_dev[j] >= 0;
        want |= (uint32_t)t == nxt[j] || (h0.z != NONE && cp_any);
      }
      bool cpf[CPL];
#pragma unroll
      for (int j = 0; j < CPL; j++) cpf[j] = false;
      if (__any_sync(FULL, want)) {
#pragma unroll
        for (int j = 0; j < CPL; j++) {
          int forced = -1;
          if ((uint32_t)t == nxt[j]) {
            nxt[j] = NONE;
#pragma unroll
            for (int k = 0; k < MAXPINS; k++) {
              if (pp[j][k] == (uint32_t)t) forced = (int)((pdv[j] >> (8 * k)) & 0xFFu);
              else if (pp[j][k] > (uint32_t)t && pp[j][k] < nxt[j]) nxt[j] = pp[j][k];
            }
          }
          if (forced < 0 && h0.z != NONE) {
            if (MM == 2) {
              while (rc[j] < nr[j] && h0.z >= rhi[j]) {
                rc[j]++;
                if (rc[j] < nr[j]) {
                  rhi[j] = rnd[rc[j] * 32] & 0xFFFFFFu;
                  rdv[j] = (int)(rnd[rc[j] * 32] >> 24);
                }
              }
              if (rc[j] < nr[j]) forced = rdv[j];
            } else if (r_dev[j] >= 0) {
              forced = r_dev[j];
            }
            cpf[j] = forced >= 0;
          }
          if (forced >= 0) {
#pragma unroll
            for (int d = 0; d < GP; d++)
              if (d == forced) bk[j] = cpf[j] ? key[j][d] : fk[j][d];
            const uint32_t kp = cpf[j] ? kpa[j] : fkpa[j];
            if ((uint32_t)forced == pq[j] && kp < bk[j]) bk[j] = kp;
          }
        }
      }
      uint32_t rec[CPL];
#pragma unroll
      for (int j = 0; j < CPL; j++) {
        const bool live = run[j] && !dead[j];
        const bool go = live && (MM != 2 || bk[j] != 0xFFFFFFFFu);
        if (MM == 2 && live && !go) dead[j] = true;  // no feasible device: INFEASIBLE (R8)
        rec[j] = bk[j];
        if (go) {
          const uint32_t dc = bk[j] & GMK;
          if (MM == 1) mv_j(j)[dc * 32] += mem64;
          if (MM == 2 && !cpf[j]) {
            const int64_t v = mv[dc * 32] - mem64;
            mv[dc * 32] = v;
            s32_at(dc) = clamp32(v);
          }
          const uint32_t bkc = bk[j] & ~GMK;
          avk_at(j, dc) = bkc;
          ms[j] = max(ms[j], bkc >> GSH);
        }
      }
      // the record is the key FT << GSH | device (a lane that is not running
      // writes its column too: no other candidate reads it)
      if (CPL == 1) {
        if (run[0] && !dead[0]) {
          col[(size_t)t * RW] = rec[0];
          ring[(t & (D - 1)) * RW] = rec[0];
        }
      } else if (CPL == 2) {
        const uint2 r2 = make_uint2(rec[0], rec[CPL - 1]);
        *(uint2 *)(col + (size_t)t * RW) = r2;
        *(uint2 *)(ring + (t & (D - 1)) * RW) = r2;
      } else {
        const uint4 r4 = make_uint4(rec[0], rec[1 % CPL], rec[2 % CPL], rec[3 % CPL]);
        *(uint4 *)(col + (size_t)t * RW) = r4;
        *(uint4 *)(ring + (t & (D - 1)) * RW) = r4;
      }
    }
    // drain: nothing may land in the stage or card slots after this batch
    cp_async_wait<0>();
    for (uint32_t z = zw; z < zc; z++) mbar_wait(mbar_sa + 8 * (z & 3), (z >> 2) & 1);
    __syncwarp();

    // ------------------------------------------------------------ epilogue
#pragma unroll
    for (int j = 0; j < CPL; j++) {
      if (run[j] && ms[j] >= a.pk_lim) {  // a key may have wrapped: re-run unpacked
        const unsigned long long k = atomicAdd(a.ndefer, 1ull);
        a.defer_q[k] = q[j];
      } else if (run[j]) {
        if (res_idx[j] >= 0) {
          a.out.makespan[res_idx[j]] = dead[j] ? I64MAX : (int64_t)ms[j];
          a.out.status[res_idx[j]] = dead[j] ? 1 : 0;
          if (MM && a.out.peak)
            for (int d = 0; d < G; d++)
              a.out.peak[res_idx[j] * G + d] = dead[j] ? -1 : (MM == 1 ? mv_j(j)[d * 32] : gc.cap[d] - mv[d * 32]);
        }
        if (!dead[j] && ((int64_t)ms[j] < bms || ((int64_t)ms[j] == bms && sidx[j] < bidx))) {
          bms = (int64_t)ms[j];
          bidx = sidx[j];
        }
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
  if (a.lane_batches > 0) {
    __syncwarp();
    if (lane == 0) {  // release the slot
      __threadfence();
      atomicAnd(&a.slot_bm[gwarp >> 5], ~(1u << (gwarp & 31)));
    }
  }
}

}  // namespace fastt
