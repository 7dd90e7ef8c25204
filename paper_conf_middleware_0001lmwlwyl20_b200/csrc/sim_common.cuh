// sim_common.cuh -- device helpers shared by the simulation kernels (k_sim.cu,
// k_sim_lane.cu): time-type traits, the per-op state record, the sweep's
// candidate stream (R21) and the rank-change classification of PIN candidates.
#pragma once
#include "fastt_internal.cuh"

namespace fastt {

#define FULL 0xFFFFFFFFu

template <typename T> struct TT;
template <> struct TT<uint32_t> {
  static constexpr uint32_t MAXV = 0xFFFFFFFFu;
  __device__ static uint32_t wmin(uint32_t v) { return __reduce_min_sync(FULL, v); }
};
template <> struct TT<uint64_t> {
  static constexpr uint64_t MAXV = ~0ull;
  __device__ static uint64_t wmin(uint64_t v) {
    uint32_t hi = (uint32_t)(v >> 32);
    uint32_t mh = __reduce_min_sync(FULL, hi);
    uint32_t lo = hi == mh ? (uint32_t)v : 0xFFFFFFFFu;
    uint32_t ml = __reduce_min_sync(FULL, lo);
    return ((uint64_t)mh << 32) | ml;
  }
};

// per-op state record in the warp's slab: FT | place:8 | indegree:24
template <typename T> struct Slab;
template <> struct Slab<uint32_t> {
  typedef unsigned long long W;
  __device__ static void init(W *s, uint32_t p, uint32_t npred) { s[p] = (unsigned long long)(npred << 8) << 32; }
  __device__ static void load(const W *s, uint32_t p, uint32_t &ft, uint32_t &plc) {
    unsigned long long w = s[p];
    ft = (uint32_t)w;
    plc = (uint32_t)(w >> 32) & 0xFF;
  }
  __device__ static void decode(const W &w, uint32_t &ft, uint32_t &plc) {
    ft = (uint32_t)w;
    plc = (uint32_t)(w >> 32) & 0xFF;
  }
  // a record written by make() / sched() without indegree bits
  __device__ static void decode_clean(const W &w, uint32_t &ft, uint32_t &plc) {
    ft = (uint32_t)w;
    plc = (uint32_t)(w >> 32);
  }
  __device__ static uint32_t indeg(const W *s, uint32_t p) {
    return (*((const uint32_t *)(s + p) + 1)) >> 8;
  }
  __device__ static void set_indeg(W *s, uint32_t p, uint32_t v) { *((uint32_t *)(s + p) + 1) = v << 8; }
  __device__ static void sched(W *s, uint32_t p, uint32_t ft, uint32_t plc) {
    s[p] = ((unsigned long long)plc << 32) | ft;
  }
  __device__ static void make(W &w, uint32_t ft, uint32_t plc) { w = ((unsigned long long)plc << 32) | ft; }
  // liveness (R24): a scheduled op keeps its unreleased-consumer count in the indegree field
  __device__ static uint32_t hiword(const W *s, uint32_t p) { return *((const uint32_t *)(s + p) + 1); }
  __device__ static void set_hiword(W *s, uint32_t p, uint32_t v) { *((uint32_t *)(s + p) + 1) = v; }
};
template <> struct Slab<uint64_t> {
  typedef ulonglong2 W;
  __device__ static void init(W *s, uint32_t p, uint32_t npred) {
    W w;
    w.x = 0;
    w.y = (unsigned long long)(npred << 8);
    s[p] = w;
  }
  __device__ static void load(const W *s, uint32_t p, uint64_t &ft, uint32_t &plc) {
    W w = s[p];
    ft = w.x;
    plc = (uint32_t)w.y & 0xFF;
  }
  __device__ static void decode(const W &w, uint64_t &ft, uint32_t &plc) {
    ft = w.x;
    plc = (uint32_t)w.y & 0xFF;
  }
  __device__ static void decode_clean(const W &w, uint64_t &ft, uint32_t &plc) {
    ft = w.x;
    plc = (uint32_t)w.y;
  }
  __device__ static uint32_t indeg(const W *s, uint32_t p) {
    return (*((const uint32_t *)(s + p) + 2)) >> 8;
  }
  __device__ static void set_indeg(W *s, uint32_t p, uint32_t v) { *((uint32_t *)(s + p) + 2) = v << 8; }
  __device__ static void sched(W *s, uint32_t p, uint64_t ft, uint32_t plc) {
    W w;
    w.x = ft;
    w.y = plc;
    s[p] = w;
  }
  __device__ static void make(W &w, uint64_t ft, uint32_t plc) {
    w.x = ft;
    w.y = plc;
  }
  __device__ static uint32_t hiword(const W *s, uint32_t p) { return *((const uint32_t *)(s + p) + 2); }
  __device__ static void set_hiword(W *s, uint32_t p, uint32_t v) { *((uint32_t *)(s + p) + 2) = v; }
};

__device__ __forceinline__ uint64_t splitmix64(uint64_t &s) {
  s += 0x9E3779B97F4A7C15ull;
  uint64_t z = s;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}



// R21: the c-th candidate of the sweep stream
__device__ inline Cand stream_cand(const StreamState &S, int64_t c) {
  Cand o;
  o.kind = 0; o.n_pins = 0; o.split_dim = 0; o.split_n = 0; o.split_op = -1;
  for (int k = 0; k < 4; k++) { o.pin_op[k] = -1; o.pin_dev[k] = 0; }
  o.dev_mask = 0;
  if (c == 0) return o;
  if (c <= S.n_split) {
    o.kind = 2;
    o.split_op = S.split_op[c - 1];
    o.split_dim = S.split_dim[c - 1];
    o.split_n = S.split_n[c - 1];
    return o;
  }
  if (c <= S.n_split + S.n_subset) {  // R25: BASE on the first k devices
    o.dev_mask = (1u << (int)(c - S.n_split)) - 1u;
    return o;
  }
  o.kind = 1;
  uint64_t st = S.seed ^ ((uint64_t)c * 0x9E3779B97F4A7C15ull);
  uint64_t x0 = splitmix64(st);
  int K = S.kmin + (int)(x0 % (uint64_t)(S.kmax - S.kmin + 1));
  if (K > S.n_live) K = S.n_live;
  o.n_pins = (uint8_t)K;
  for (int k = 0; k < K; k++) {
    uint64_t xo = splitmix64(st);
    int32_t idx = (int32_t)(xo % (uint64_t)S.n_live);
    for (;;) {
      bool taken = false;
      for (int q = 0; q < k; q++) taken |= o.pin_op[q] == S.live[idx];
      if (!taken) break;
      idx = idx + 1 == S.n_live ? 0 : idx + 1;
    }
    int32_t op = S.live[idx];
    uint64_t xd = splitmix64(st);
    o.pin_op[k] = op;
    o.pin_dev[k] = (uint8_t)((S.base_place[op] + 1 + (int)(xd % (uint64_t)(S.G - 1))) % S.G);
  }
  return o;
}

// c of an edge under allowed sets (R5), from per-class comm values
template <typename T>
__device__ __forceinline__ T c_allowed_t(const GraphConst &gc, const T *pc, int su, int tv) {
  uint32_t mask;
  if (su < 0 && tv < 0) mask = gc.offdiag_mask;
  else if (su >= 0 && tv < 0) mask = gc.row_mask[su];
  else if (su < 0) mask = gc.col_mask[tv];
  else {
    if (su == tv) return 0;
    return pc[gc.link_class[su * gc.G + tv]];
  }
  T best = 0;
  while (mask) {
    int k = __ffs(mask) - 1;
    mask &= mask - 1;
    T c = pc[k];
    best = c > best ? c : best;
  }
  return best;
}

__device__ __forceinline__ bool lt_cross(uint64_t a, uint64_t mb, uint64_t b, uint64_t ma) {
  uint64_t h1 = __umul64hi(a, mb), l1 = a * mb, h2 = __umul64hi(b, ma), l2 = b * ma;
  return h1 < h2 || (h1 == h2 && l1 < l2);
}

// A PIN candidate keeps the base ranks iff w of each pinned op and
// c of every edge touching one are unchanged under R5's allowed
// sets; otherwise it is deferred to the per-candidate preparation pipeline.
template <typename T>
static __device__ __noinline__ bool pin_changes_ranks(const PrepGraph *pg, const GraphConst &gc, const Cand &c, int np,
                                               uint32_t i, int di, int G, int K) {
  const T *costp = (const T *)pg->costp;
  const T *pe_comm = (const T *)pg->pe_comm;
  const uint32_t *posm = pg->pos;
  bool changed = false;
  T wmax = 0;
  for (int d = 0; d < G; d++) {
    T v = costp[(int64_t)i * G + d];
    wmax = v > wmax ? v : wmax;
  }
  changed |= costp[(int64_t)i * G + di] != wmax;
  const uint32_t *ci = pg->card + (int64_t)i * CARD_WORDS;
  uint32_t deg = ci[CW_DEG], pb = ci[CW_PBASE], sbb = ci[CW_SBASE];
  for (uint32_t j = 0; j < (deg & 0xFFFF) && !changed; j++) {
    uint32_t e = pb + j, o = pg->pe_src[e];
    int po = -1;
    for (int k = 0; k < np; k++)
      if (posm[c.pin_op[k]] == o) po = c.pin_dev[k];
    const T *pc = pe_comm + (int64_t)e * K;
    changed |= c_allowed_t<T>(gc, pc, -1, -1) != c_allowed_t<T>(gc, pc, po, di);
  }
  for (uint32_t j = 0; j < (deg >> 16) && !changed; j++) {
    uint32_t o = pg->se_dst[sbb + j], e = pg->se_pe[sbb + j];
    int po = -1;
    for (int k = 0; k < np; k++)
      if (posm[c.pin_op[k]] == o) po = c.pin_dev[k];
    const T *pc = pe_comm + (int64_t)e * K;
    changed |= c_allowed_t<T>(gc, pc, -1, -1) != c_allowed_t<T>(gc, pc, di, po);
  }
  return changed;
}

// Validation and classification of a candidate on the base graph (SURVEY
// 8(a) S2-S5): st = 2 for a bad specification (BADSPEC: pins out of range,
// on dead ops, on devices outside the candidate's subset or repeated; a split
// of an op or dim that is not splittable, n outside 2..G; an unknown kind),
// else 0.  Returns true iff a valid candidate needs its own prepared graph
// (the preparation pipeline): a SPLIT (SplitOperation, Alg. 2 lines 16-30),
// a proper device subset (R25: ranks over the subset), or -- when rank_test
// -- pins that change w or c under R5's allowed sets.  The single definition
// used by the pre-classification pass and the lane kernel's prologue.
template <typename T>
__device__ __forceinline__ bool cand_classify(const Cand &c, const PrepGraph *pg, const GraphConst &gc,
                                              const uint8_t *split_mask, int G, bool rank_test, uint8_t &st) {
  const uint32_t all = all_devices(G);
  const uint32_t *posm = pg->pos;
  const int32_t Vraw = pg->V;
  st = 0;
  bool defer = false;
  if (c.dev_mask & ~all) {
    st = 2;
    return false;
  }
  if (c.dev_mask && c.dev_mask != all) defer = true;  // device subset (R25): own ranks
  if (c.kind == 0) {
  } else if (c.kind == 1) {
    const int np = c.n_pins;
    if (np < 1 || np > MAXPINS) {
      st = 2;
      return false;
    }
    const uint32_t dset = c.dev_mask ? c.dev_mask : all;
    for (int k = 0; k < np; k++) {
      const int32_t o = c.pin_op[k];
      bool bad = o < 0 || o >= Vraw || posm[o] == NONE || c.pin_dev[k] >= G || !((dset >> c.pin_dev[k]) & 1u);
      for (int k2 = 0; k2 < k; k2++) bad |= c.pin_op[k2] == o;
      if (bad) {
        st = 2;
        return false;
      }
    }
    if (!defer && rank_test)
      for (int k = 0; k < np && !defer; k++)
        defer = pin_changes_ranks<T>(pg, gc, c, np, posm[c.pin_op[k]], c.pin_dev[k], G, gc.K);
  } else if (c.kind == 2) {
    const int32_t o = c.split_op;
    if (o < 0 || o >= Vraw || posm[o] == NONE || c.split_dim > 1 || !(split_mask[o] & (1u << c.split_dim)) ||
        c.split_n < 2 || c.split_n > G) {
      st = 2;
      return false;
    }
    defer = true;
  } else {
    st = 2;
    return false;
  }
  return defer;
}

}  // namespace fastt
