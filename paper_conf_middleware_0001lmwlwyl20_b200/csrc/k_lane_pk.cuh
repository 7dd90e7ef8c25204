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
template <int GP, int MM> __host__ __device__ constexpr size_t pk_mm_off() {
  // card mbarriers [4] u64 (64 B) | ring [D][32] u32 | stage [D][4][32] u32 |
  // read plans [D][8] u32 | cards [32] | avail keys [GP/2][32][2] u32 |
  // memory state (as k_sim_lane)
  return (size_t)64 + (size_t)LANE_D * 32 * 4 + (size_t)LANE_D * 4 * 32 * 4 + (size_t)LANE_D * 32 +
         (size_t)PK_CR * pk_card_bytes(GP) + (size_t)32 * GP * 4;
}
template <int GP, int MM> __host__ __device__ constexpr size_t pk_smem_per_warp() {
  return pk_mm_off<GP, MM>() + (MM >= 1 ? (size_t)32 * GP * 8 : 0) + (MM == 2 ? (size_t)32 * GP * 8 : 0);
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
template <int GSH, bool EX, int MM>
__global__ void __launch_bounds__(LANE_BLOCK, LANE_MINB) k_lane_pk(SimArgs a) {
  constexpr int GP = 1 << GSH;
  constexpr uint32_t GMK = GP - 1;
  constexpr int D = LANE_D, P = D - 1;
  constexpr int CB = pk_card_bytes(GP);
  static_assert((D & (D - 1)) == 0 && CB % 16 == 0, "pipeline slots");
  const int lane = threadIdx.x & 31;
  int64_t gwarp = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
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
  // this lane's slab column (record of position p at col[p * 32]); row p of
  // the warp (all 32 records) starts at col0 + p * 32
  uint32_t *const col = (uint32_t *)a.slab + (size_t)gwarp * (size_t)a.slab_stride * 32 + lane;
  const uint32_t *const col0 = col - lane;
  extern __shared__ __align__(16) unsigned char lsm[];
  unsigned char *const wsm = lsm + (threadIdx.x >> 5) * pk_smem_per_warp<GP, MM>();
  const uint32_t wsa = (uint32_t)__cvta_generic_to_shared(wsm);
  const uint32_t mbar_sa = wsa;                              // card barriers [4] u64
  uint32_t *const ring = (uint32_t *)(wsm + 64) + lane;     // [D][32]
  const uint32_t ring_sa = wsa + 64;
  const uint32_t stage_sa = ring_sa + D * 128;              // [D][4][32]
  uint32_t *const plan = (uint32_t *)(wsm + 64 + D * 640);  // [D][8]: per predecessor (address, lane mask)
  unsigned char *const cards = wsm + 64 + D * 672;          // [PK_CR][CB]
  const uint32_t cards_sa = wsa + 64 + D * 672;
  uint32_t *const avk = (uint32_t *)(cards + PK_CR * CB) + (GP >= 2 ? 2 * lane : lane);
  auto avk_at = [&](uint32_t d) -> uint32_t & { return GP >= 2 ? avk[(d >> 1) * 64 + (d & 1)] : avk[0]; };
  int64_t *const mv = (int64_t *)(wsm + pk_mm_off<GP, MM>()) + lane;
  uint32_t *const s32b = (uint32_t *)(wsm + pk_mm_off<GP, MM>() + (size_t)32 * GP * 8) + (GP >= 4 ? 4 * lane : lane);
  uint32_t *const rnd = (uint32_t *)(wsm + pk_mm_off<GP, MM>() + (size_t)32 * GP * 12) + lane;
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
  const bool cp_on = (a.flags & 1u) != 0;
  int64_t bms = I64MAX, bidx = -1;
  uint32_t zc = 0;  // card chunks issued by this warp so far (barrier zc & 3, phase (zc >> 2) & 1)
  // this lane's part of a step's record staging: chunk (lane & 7) of inline
  // predecessor (lane >> 3)
  const int pk_k = lane >> 3, pk_c = lane & 7;

  const int64_t nlim = a.n_dev ? ((int64_t)*a.n_dev < a.n ? (int64_t)*a.n_dev : a.n) : a.n;
  for (int32_t nb = 0; a.lane_batches <= 0 || nb < a.lane_batches; nb++) {
    unsigned long long q0 = 0;
    if (lane == 0) q0 = atomicAdd(a.counter, 32ull);
    q0 = __shfl_sync(FULL, q0, 0);
    if ((int64_t)q0 >= nlim) break;
    const int64_t q = (int64_t)q0 + lane;
    const bool active = q < nlim;
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
      defer = cand_classify<uint32_t>(c, pg, gc, a.split_mask, G, !a.preclassified, st);
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
    // CP devices (Alg. 1 line 5, R9): without caps one round of
    // the free CP ops on the device of least total cost; with caps the
    // lane-local rounds with reservations (cp_rounds_lane)
    int r_dev = -1, m = 0, nr = 0, rc = 0, rdv = -1;
    uint32_t rhi = 0;
    bool dead = false;
    const uint32_t all = all_devices(G);
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
        nr = cp_rounds_lane<uint32_t>(pg, gc, G, all, np, pp, pc, rnd, mv);
        if (nr > 0) {
          rhi = rnd[0] & 0xFFFFFFu;
          rdv = (int)(rnd[0] >> 24);
        }
      } else if (cpl - m > 0) {
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
    // BASE-prefix sharing (k_sim_lane): the warp starts at lo = min t0
    int32_t t0 = 0;
    if (run && a.snap_mode == 2 && (!MM || a.snap_used)) {
      const bool share = m == 0 || (MM != 2 && a.snap_round_dev >= 0 && r_dev == a.snap_round_dev);
      if (share) {
        t0 = n;
        for (int k = 0; k < np; k++) {
          const int32_t dq = (int32_t)__ldg(a.snap_dq + pp[k]);
          t0 = dq < t0 ? dq : t0;
        }
      }
    }
    int32_t lo = run ? t0 : n;
    const int32_t nmax = __any_sync(FULL, run) ? n : 0;
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) {
      const int32_t x = __shfl_xor_sync(FULL, lo, o);
      lo = x < lo ? x : lo;
    }
    if (a.stat) {
      const uint32_t ls = __reduce_add_sync(FULL, run ? (uint32_t)(n - lo) : 0u);
      if (lane == 0 && nmax > lo) {
        atomicAdd(a.stat, (unsigned long long)(nmax - lo));
        atomicAdd(a.stat + 1, (unsigned long long)ls);
      }
    }
    uint32_t ms = 0;
#pragma unroll
    for (int d = 0; d < GP; d++) avk_at(d) = 0;
    if (run && lo > 0) {  // (lo > 0: every running lane shares)
      const uint32_t *sa = (const uint32_t *)a.snap_avail + (size_t)lo * G;
#pragma unroll
      for (int d = 0; d < GP; d++)
        if (d < G) avk_at(d) = __ldg(sa + d) << GSH;
      ms = __ldg((const uint32_t *)a.snap_ms + lo);
      if (MM == 1)
        for (int d = 0; d < G; d++) mv[d * 32] = __ldg((const int64_t *)a.snap_used + (size_t)lo * G + d);
      if (MM == 2)
        for (int d = 0; d < G; d++) mv[d * 32] = gc.cap[d] - __ldg((const int64_t *)a.snap_ur + (size_t)lo * G + d);
    }
    if (MM == 2 && run) {
#pragma unroll
      for (int d = 0; d < GP; d++) s32_at(d) = clamp32(mv[d * 32]);
    }
    uint32_t nxt = NONE;
#pragma unroll
    for (int k = 0; k < MAXPINS; k++)
      if (pp[k] >= (uint32_t)lo && pp[k] < nxt) nxt = pp[k];

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
    const uint32_t lane4 = 4u * (uint32_t)lane;
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
      const uint32_t *src = base_rec ? snap + (s & ~3u) : col0 + (size_t)s * 32 + 4 * pk_c;
      const uint32_t row = stage_sa + (slot * 4 + (uint32_t)pk_k) * 128;
      cp16_if(staged && (!base_rec || pk_c == 0), row + 16 * pk_c, src);
      // the read plan of predecessor pk_k: its record's address for lane 0
      // and the per-lane mask (the 8 lanes of a predecessor store the same
      // pair: one broadcast store)
      const uint32_t ad = staged ? (base_rec ? row + 4 * (s & 3u) : row) : ring_sa + (s & (D - 1)) * 128;
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
    // a record of position s (extra predecessors beyond the card's 4)
    auto rec_at = [&](uint32_t s, int32_t t) -> uint32_t {
      if ((int32_t)s < lo) return __ldg(snap + s);
      if ((int32_t)s + P >= t) return ring[(s & (D - 1)) * 32];
      return col[(size_t)s * 32];
    };
    for (int32_t t = lo; t < nmax; t++) {
      const bool live = run && !dead;
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
      bool cpf = false;
      const uint32_t npred = h0.x & 0xFFFF;
      uint32_t rk[4];
      {
        const uint4 pa = *(const uint4 *)(plan + (t & (D - 1)) * 8);
        const uint4 pb = *(const uint4 *)(plan + (t & (D - 1)) * 8 + 4);
        const uint32_t ad[4] = {pa.x + (lane4 & pa.y), pa.z + (lane4 & pa.w), pb.x + (lane4 & pb.y),
                                pb.z + (lane4 & pb.w)};
#pragma unroll
        for (int k = 0; k < 4; k++) rk[k] = *(const uint32_t *)__cvta_shared_to_generic(ad[k]);
      }
      // (the slots issue(t + P) overwrites were read at step t - 1, before
      // every lane passed this step's __syncwarp)
      issue(t + P);
      // arrival terms in key space (k_sim_lane): R_k = key_k + (c_k << GSH)
      const uint32_t hcw[4] = {hc.x, hc.y, hc.z, hc.w};
      uint32_t rkm[4], R[4];
#pragma unroll
      for (int k = 0; k < 4; k++) {
        rkm[k] = (uint32_t)k < npred ? rk[k] : 0u;
        R[k] = rkm[k] + hcw[k];
      }
      uint32_t Mkey = max(max(R[0], R[1]), max(R[2], R[3]));
      if (npred > 4u)  // (warp-uniform)
        for (uint32_t k = 4; k < npred; k++)
          Mkey = max(Mkey, rec_at(__ldg(pe_src + h0.y + k), t) + (__ldg(pe_comm + h0.y + k) << GSH));
      uint32_t Ekey = 0;
#pragma unroll
      for (int k = 0; k < 4; k++) Ekey = max(Ekey, ((rkm[k] ^ Mkey) & GMK) == 0u ? rkm[k] : R[k]);
      if (npred > 4u)
        for (uint32_t k = 4; k < npred; k++) {
          const uint32_t r = rec_at(__ldg(pe_src + h0.y + k), t);
          Ekey = max(Ekey, ((r ^ Mkey) & GMK) == 0u ? r : r + (__ldg(pe_comm + h0.y + k) << GSH));
        }
      const uint32_t Mk = Mkey & ~GMK, Ek = Ekey & ~GMK, pq = Mkey & GMK;
      // keys (EFT << GSH) | d (Alg. 1 lines 12-19, R3, R6)
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
      const uint32_t ap = avk_at(pq), cpa = cw[16 + pq];
      uint32_t kpa = (ap > Ek ? ap : Ek) + cpa;
      if (!EX && pq >= (uint32_t)G) kpa = 0xFFFFFFFFu;
      uint32_t key[GP];
#pragma unroll
      for (int d = 0; d < GP; d++) key[d] = (EX || d < G) ? (av[d] > Mk ? av[d] : Mk) + cst[d] : 0xFFFFFFFFu;
      uint32_t fk[GP], fkpa = kpa;
#pragma unroll
      for (int d = 0; d < GP; d++) fk[d] = key[d];
      if (MM == 2) {  // Alg. 1 line 13, R8 (k_sim_lane)
        if (memhi != 0) {
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
      // the device forced by a perturbation pin (hard) or a CP round (Alg. 1
      // l.9-10, R9; cpf: memory reserved up front) -- rare steps
      const bool cp_any = MM == 2 ? rc < nr : r_dev >= 0;
      if (__any_sync(FULL, (uint32_t)t == nxt || (h0.z != NONE && cp_any))) {
        int forced = -1;
        if ((uint32_t)t == nxt) {
          nxt = NONE;
#pragma unroll
          for (int k = 0; k < MAXPINS; k++) {
            if (pp[k] == (uint32_t)t) forced = (int)((pdv >> (8 * k)) & 0xFFu);
            else if (pp[k] > (uint32_t)t && pp[k] < nxt) nxt = pp[k];
          }
        }
        if (forced < 0 && h0.z != NONE) {
          if (MM == 2) {
            while (rc < nr && h0.z >= rhi) {
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
        if (forced >= 0) {
#pragma unroll
          for (int d = 0; d < GP; d++)
            if (d == forced) bk = cpf ? key[d] : fk[d];
          const uint32_t kp = cpf ? kpa : fkpa;
          if ((uint32_t)forced == pq && kp < bk) bk = kp;
        }
      }
      const bool go = live && (MM != 2 || bk != 0xFFFFFFFFu);
      if (MM == 2 && live && !go) dead = true;  // no feasible device: INFEASIBLE (R8)
      if (go) {
        const uint32_t dc = bk & GMK;
        if (MM == 1) mv[dc * 32] += mem64;
        if (MM == 2 && !cpf) {
          const int64_t v = mv[dc * 32] - mem64;
          mv[dc * 32] = v;
          s32_at(dc) = clamp32(v);
        }
        const uint32_t bkc = bk & ~GMK;
        avk_at(dc) = bkc;
        ms = max(ms, bkc >> GSH);
        col[(size_t)t * 32] = bk;  // the record is the key: FT << GSH | device
        ring[(t & (D - 1)) * 32] = bk;
      }
    }
    // drain: nothing may land in the stage or card slots after this batch
    cp_async_wait<0>();
    for (uint32_t z = zw; z < zc; z++) mbar_wait(mbar_sa + 8 * (z & 3), (z >> 2) & 1);
    __syncwarp();

    // ------------------------------------------------------------ epilogue
    if (run && ms >= a.pk_lim) {  // a key may have wrapped: re-run unpacked
      const unsigned long long k = atomicAdd(a.ndefer, 1ull);
      a.defer_q[k] = q;
    } else if (run) {
      if (res_idx >= 0) {
        a.out.makespan[res_idx] = dead ? I64MAX : (int64_t)ms;
        a.out.status[res_idx] = dead ? 1 : 0;
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
  if (a.lane_batches > 0) {
    __syncwarp();
    if (lane == 0) {  // release the slot
      __threadfence();
      atomicAnd(&a.slot_bm[gwarp >> 5], ~(1u << (gwarp & 31)));
    }
  }
}

}  // namespace fastt
