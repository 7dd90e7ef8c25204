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
//             step t0; the warp starts at the smallest t0 of its lanes
//             from the recorded BASE avail/makespan, and records of
//             positions before that step are read from the BASE record.
// Memory caps, liveness memory, INSERT, per-op outputs, SPLIT and
// rank-changing candidates stay on k_sim (group-per-candidate kernel).
//
// The kernel itself is in k_sim_lane_body.cuh (instances: k_sim_lane_inst.cu).
#include "k_sim_lane_body.cuh"
#include "k_lane_pk.cuh"
#include <cstdio>
#include <cstring>

namespace fastt {

// kernel getters of the per-(GSH, MM) instance objects (k_sim_lane_inst.cu)
#define FASTT_LANE_CASE(N)                                                        \
  case N:                                                                         \
    return mm == 0 ? lane_fn_g##N##_m0(tbits, cm, exact, mg, pk)                  \
                   : mm == 1 ? lane_fn_g##N##_m1(tbits, cm, exact, mg, pk)        \
                             : lane_fn_g##N##_m2(tbits, cm, exact, mg, pk);
static const void *lane_fn(int tbits, int gshift, int cm, bool exact, bool mg, bool pk, int mm) {
  switch (gshift) {
    FASTT_LANE_CASE(0)
    FASTT_LANE_CASE(1)
    FASTT_LANE_CASE(2)
    FASTT_LANE_CASE(3)
    FASTT_LANE_CASE(4)
    default:
      FASTT_LANE_CASE(5)
  }
}
#undef FASTT_LANE_CASE

template <typename T, bool MG, int MM, bool PK> static size_t lane_smem_t(int gshift) {
  switch (gshift) {
    case 0: return lane_smem_per_warp<T, 1, MG, MM, PK>();
    case 1: return lane_smem_per_warp<T, 2, MG, MM, PK>();
    case 2: return lane_smem_per_warp<T, 4, MG, MM, PK>();
    case 3: return lane_smem_per_warp<T, 8, MG, MM, PK>();
    case 4: return lane_smem_per_warp<T, 16, MG, MM, PK>();
    default: return lane_smem_per_warp<T, 32, MG, MM, PK>();
  }
}
template <bool MG, bool PK> static size_t lane_smem_w(int tbits, int gshift, int mm) {
  if (tbits == 32)
    return mm == 0 ? lane_smem_t<uint32_t, MG, 0, PK>(gshift)
                   : mm == 1 ? lane_smem_t<uint32_t, MG, 1, PK>(gshift) : lane_smem_t<uint32_t, MG, 2, PK>(gshift);
  return mm == 0 ? lane_smem_t<uint64_t, MG, 0, false>(gshift)
                 : mm == 1 ? lane_smem_t<uint64_t, MG, 1, false>(gshift) : lane_smem_t<uint64_t, MG, 2, false>(gshift);
}
// dynamic shared memory of a block: LANE_BLOCK threads, or one warp (MG);
// pk: the packed-key variant (4-byte records)
size_t lane_smem(int tbits, int gshift, bool mg, int mm, bool pk) {
  if (mg) return lane_smem_w<true, false>(tbits, gshift, mm);
  return (LANE_BLOCK / 32) * (pk ? lane_smem_w<false, true>(tbits, gshift, mm) : lane_smem_w<false, false>(tbits, gshift, mm));
}

__global__ void k_pack_costs(const PrepGraph *pgp, int32_t n, int G, int gshift, int64_t E, uint32_t *costk,
                             uint32_t *commk, uint32_t *pkc, int pkw, unsigned long long *mx) {
  const PrepGraph &P = *pgp;
  const uint32_t *c = (const uint32_t *)P.costp;
  const uint32_t *pc = (const uint32_t *)P.pe_comm;
  uint32_t mc = 0, mm = 0;
  const int64_t NG = (int64_t)n * G;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < NG; i += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t v = c[i];
    mc = v > mc ? v : mc;
    costk[i] = (v << gshift) | (uint32_t)(i % G);
  }
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < E; i += (int64_t)gridDim.x * blockDim.x)
    mm = pc[i] > mm ? pc[i] : mm;
  // the cards' inline comm values (words 12-15, 0 in unused slots), pre-shifted
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < 4 * (int64_t)n;
       i += (int64_t)gridDim.x * blockDim.x)
    commk[i] = P.card[(i >> 2) * CARD_WORDS + CW_PCOMM + (i & 3)] << gshift;
  // compact PK cards (k_lane_pk.cuh): deg, pbase, cpidx, 0 | 4 predecessor
  // positions | their comm << gshift | mem lo, hi, 0, 0 | packed cost row
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < (int64_t)pkw * n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t p = i / pkw;
    const int w = (int)(i % pkw);
    const uint32_t *cd = P.card + p * CARD_WORDS;
    uint32_t v = 0;
    if (w == 0) v = cd[CW_DEG];
    else if (w == 1) v = cd[CW_PBASE];
    else if (w == 2) v = cd[CW_CPIDX];
    else if (w >= 4 && w < 8) v = cd[CARD_HDR + (w - 4)];
    else if (w >= 8 && w < 12) v = cd[CW_PCOMM + (w - 8)] << gshift;
    else if (w == 12) v = cd[CW_MEMLO];
    else if (w == 13) v = cd[CW_MEMHI];
    else if (w >= 16 && w - 16 < G) v = (c[p * G + (w - 16)] << gshift) | (uint32_t)(w - 16);
    pkc[i] = v;
  }
  atomicMax(mx, (unsigned long long)mc);
  atomicMax(mx + 1, (unsigned long long)mm);
}
int pk_card_words_host(int gshift) { return pk_card_words(1 << gshift); }
void launch_pack_costs(const PrepGraph *pg_dev, int32_t n, int G, int gshift, int64_t E, uint32_t *costk,
                       uint32_t *commk, uint32_t *pkc, unsigned long long *mx, cudaStream_t st) {
  k_pack_costs<<<148, 256, 0, st>>>(pg_dev, n, G, gshift, E, costk, commk, pkc, pk_card_words(1 << gshift), mx);
}

// BASE records as packed keys, and doubled (key2[2p] = key2[2p + 1] =
// key[p]) for the two-candidates-per-lane kernel
__global__ void k_snap_keys(const unsigned long long *rec, int32_t n, int gshift, uint32_t *key, uint2 *key2,
                            uint4 *key4) {
  for (int32_t p = blockIdx.x * blockDim.x + threadIdx.x; p < n; p += gridDim.x * blockDim.x) {
    const unsigned long long w = rec[p];
    const uint32_t k = ((uint32_t)w << gshift) | (uint32_t)(w >> 32);
    key[p] = k;
    key2[p] = make_uint2(k, k);
    key4[p] = make_uint4(k, k, k, k);
  }
}
void launch_snap_keys(const void *rec, int32_t n, int gshift, uint32_t *key, uint32_t *key2, uint32_t *key4,
                      cudaStream_t st) {
  if (n > 0)
    k_snap_keys<<<(n + 255) / 256, 256, 0, st>>>((const unsigned long long *)rec, n, gshift, key, (uint2 *)key2,
                                                  (uint4 *)key4);
}

int lane_comm_mode(const SimArgs &a, int tbits) {
  if (a.fastcomm && tbits == 32) return 0;
  return a.gc_K == 1 ? 1 : 2;
}

// a.lane: 1 = candidates of the base graph (LANE_BLOCK threads per block),
// 2 = prepared slots, one per lane (one warp per block; grid = warps)
// the packed-key kernel k_lane_pk (k_lane_pk.cuh) and its shared memory
static const void *lane_pk_fn(int gshift, int mm, bool exact, int cpl) {
  switch (gshift) {
    case 0: return lane_pk_fn_g0(mm, exact, cpl);
    case 1: return lane_pk_fn_g1(mm, exact, cpl);
    case 2: return lane_pk_fn_g2(mm, exact, cpl);
    case 3: return lane_pk_fn_g3(mm, exact, cpl);
    case 4: return lane_pk_fn_g4(mm, exact, cpl);
    default: return lane_pk_fn_g5(mm, exact, cpl);
  }
}
template <int GP> static size_t pk_smem_w(int mm, int cpl) {
  if (cpl == 4 && mm == 0) return pk_smem_per_warp<GP, 0, 4>();
  if (cpl >= 2 && mm <= 1) return mm == 0 ? pk_smem_per_warp<GP, 0, 2>() : pk_smem_per_warp<GP, 1, 2>();
  return mm == 0 ? pk_smem_per_warp<GP, 0>() : mm == 1 ? pk_smem_per_warp<GP, 1>() : pk_smem_per_warp<GP, 2>();
}
static size_t lane_pk_smem(int gshift, int mm, int cpl, int wpb) {
  size_t w;
  switch (gshift) {
    case 0: w = pk_smem_w<1>(mm, cpl); break;
    case 1: w = pk_smem_w<2>(mm, cpl); break;
    case 2: w = pk_smem_w<4>(mm, cpl); break;
    case 3: w = pk_smem_w<8>(mm, cpl); break;
    case 4: w = pk_smem_w<16>(mm, cpl); break;
    default: w = pk_smem_w<32>(mm, cpl); break;
  }
  return (size_t)wpb * w;
}

static const void *lane_ins_fn(int tbits, int gshift, int cm, bool exact) {
  switch (gshift) {
    case 0: return lane_ins_fn_g0(tbits, cm, exact);
    case 1: return lane_ins_fn_g1(tbits, cm, exact);
    case 2: return lane_ins_fn_g2(tbits, cm, exact);
    case 3: return lane_ins_fn_g3(tbits, cm, exact);
    case 4: return lane_ins_fn_g4(tbits, cm, exact);
    default: return lane_ins_fn_g5(tbits, cm, exact);
  }
}

void launch_sim_lane(const SimArgs &a, int tbits, int grid, cudaStream_t st) {
  const bool mg = a.lane == 2;
  const int cm = lane_comm_mode(a, tbits);
  if (a.ins) {  // INSERT (R1i): the plain-key base-graph kernel with idle-slot arrays
    const void *f = lane_ins_fn(tbits, a.gshift, cm, a.G == (1 << a.gshift));
    const size_t sm = lane_smem(tbits, a.gshift, false, 0, false);
    cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    SimArgs aa = a;
    void *args[] = {&aa};
    cudaLaunchKernel(f, dim3(grid), dim3(LANE_BLOCK), args, sm, st);
    return;
  }
  const bool pk = !mg && tbits == 32 && cm != 2 && a.costk != nullptr && a.pk_lim > 0;
  if (pk && a.pkc) {  // the base-graph sweep kernel: TMA-staged packed-key cards
    const int cpl = a.pk_cpl == 4 && a.lane_mm == 0 ? 4 : a.pk_cpl >= 2 && a.lane_mm <= 1 ? 2 : 1;
    const int wpb = a.pk_wpb > 0 ? a.pk_wpb : LANE_BLOCK / 32;
    const void *f = lane_pk_fn(a.gshift, a.lane_mm, a.G == (1 << a.gshift), cpl);
    const size_t sm = lane_pk_smem(a.gshift, a.lane_mm, cpl, wpb);
    cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    SimArgs aa = a;
    void *args[] = {&aa};
    cudaLaunchKernel(f, dim3(grid), dim3(32 * wpb), args, sm, st);
    return;
  }
  const void *f = lane_fn(tbits, a.gshift, cm, a.G == (1 << a.gshift), mg, pk, a.lane_mm);
  const size_t sm = lane_smem(tbits, a.gshift, mg, a.lane_mm, pk);
  if (mg) cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  SimArgs aa = a;
  void *args[] = {&aa};
  cudaLaunchKernel(f, dim3(grid), dim3(mg ? 32 : LANE_BLOCK), args, sm, st);
}

// resident blocks per SM of the base-graph launch of memory mode mm and
// packed keys pk (the minimum over the comm / exactness variants); sets their
// dynamic shared memory limit
int lane_occupancy(int tbits, int gshift, int mm, bool pk, int cpl, int wpb) {
  int nb = 1 << 30, x = 0;
  if (pk && tbits != 32) return 0;
  if (pk) {  // k_lane_pk (blocks of wpb warps)
    if (mm > 1) cpl = 1;
    if (mm == 1 && cpl > 2) cpl = 2;
    const size_t sm = lane_pk_smem(gshift, mm, cpl, wpb);
    for (int ex = 0; ex < 2; ex++) {
      const void *f = lane_pk_fn(gshift, mm, ex != 0, cpl);
      cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&x, f, 32 * wpb, sm);
      nb = x < nb ? x : nb;
    }
    return nb;
  }
  const size_t sm = lane_smem(tbits, gshift, false, mm, pk);
  for (int v = (tbits == 32 ? 0 : 2); v < (tbits == 32 ? 6 : 6); v++) {
    if (pk && (v >> 1) == 2) continue;  // (packed keys need one link class)
    const void *f = lane_fn(tbits, gshift, v >> 1, v & 1, false, pk, mm);
    cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&x, f, LANE_BLOCK, sm);
    nb = x < nb ? x : nb;
  }
  return nb;
}

}  // namespace fastt

namespace fastt {
// (FASTT_HOST_TRACE) registers and shared memory of a k_lane_pk instance
void lane_pk_attrs(int gshift, int mm, int cpl, char *buf, size_t len) {
  cudaFuncAttributes fa;
  for (int ex = 0; ex < 2; ex++) {
    if (cudaFuncGetAttributes(&fa, lane_pk_fn(gshift, mm, ex != 0, cpl)) != cudaSuccess) continue;
    const size_t o = strlen(buf);
    snprintf(buf + o, len - o, " [ex %d: %d regs, %zu static smem, %d max dyn smem, %zu local]", ex, fa.numRegs,
             fa.sharedSizeBytes, fa.maxDynamicSharedSizeBytes, fa.localSizeBytes);
  }
}
}  // namespace fastt
