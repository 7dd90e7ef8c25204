// k_prep.cu -- graph preparation kernels (SURVEY 8(a) S1, S3, S4, S5, S8 helpers).
//
//   k_materialize : SplitOperation (Alg. 2 lines 16-30; R13) into a slot
//   k_rank        : rank_u with per-candidate allowed device sets (R5)
//   k_sort        : priority order (rank desc, id asc; R2/R3) by a stable CTA radix sort
//   k_cards_*     : the position-ordered PrepGraph (cards, cost table, edge arrays)
//   k_cp          : critical path (R7) and its prefix sums for the CP devices
//   k_bound       : the schedule bound that selects 32-bit time (R18)
//   k_splitlist   : Alg. 2 lines 4-5: placement-aware CP, split-eligible, sorted (R15)
#include <algorithm>
#include "fastt_internal.cuh"

namespace fastt {

#define FULL 0xFFFFFFFFu

__device__ __forceinline__ uint64_t warp_max_u64(uint64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    uint64_t x = __shfl_xor_sync(FULL, v, o);
    v = x > v ? x : v;
  }
  return v;
}
__device__ __forceinline__ uint32_t warp_min_u32(uint32_t v) { return __reduce_min_sync(FULL, v); }

// ---------------------------------------------------------------- materialize

// Bulk copy of the base raw block into every SPLIT slot (same layout, contiguous).
// (nact: device count of active slots, nullable -- slots at or past it exit)
// Words [hole_lo, hole_hi) are skipped (the cost, mem and param tables:
// split slots read a base op's from the base graph, only the overlay rows
// -- written by k_patch_split -- are their own).
__global__ void k_copy_block(const uint4 *src, uint4 *dst_base, int64_t slot_stride_words, int64_t words,
                             const Cand *cands, const uint32_t *nact, int64_t hole_lo, int64_t hole_hi) {
  if ((nact && blockIdx.y >= *nact) || cands[blockIdx.y].kind != 2) return;
  uint4 *dst = dst_base + (int64_t)blockIdx.y * slot_stride_words;
  const int64_t hole = hole_hi - hole_lo, n = words - hole;
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = k < hole_lo ? k : k + hole;
    dst[i] = src[i];
  }
}

// remove `o` from a sorted adjacency list and append `nw` (larger than every id)
__device__ void list_replace(int32_t *ids, int64_t *bytes, uint8_t *prm, uint32_t off, uint32_t cnt, int32_t o,
                             int32_t nw) {
  uint32_t j = 0;
  while (j < cnt && ids[off + j] != o) j++;
  if (j == cnt) return;
  int64_t b = bytes[off + j];
  uint8_t p = prm[off + j];
  for (; j + 1 < cnt; j++) {
    ids[off + j] = ids[off + j + 1];
    bytes[off + j] = bytes[off + j + 1];
    prm[off + j] = prm[off + j + 1];
  }
  ids[off + cnt - 1] = nw;
  bytes[off + cnt - 1] = b;
  prm[off + cnt - 1] = p;
}

__device__ __forceinline__ bool edge_cut(int dim, int p) { return dim == 0 ? !p : (bool)p; }

// One CTA per slot: apply SplitOperation to the slot's copy of the base graph.
__global__ void k_patch_split(const RawGraph *base_p, RawGraph *raws, const GraphConst *gc, const Cand *cands,
                              const uint32_t *nact) {
  if ((nact && blockIdx.x >= *nact) || cands[blockIdx.x].kind != 2) return;  // non-split slots alias the base graph: never write them
  const RawGraph &B = *base_p;
  RawGraph &R = raws[blockIdx.x];
  const Cand c = cands[blockIdx.x];
  const int G = gc->G;
  const int32_t o = c.split_op, n = c.split_n, dim = c.split_dim;
  __shared__ int32_t s_P, s_S, s_to;
  const int32_t V = B.V;
  if (threadIdx.x == 0) {
    uint32_t P = B.pred_cnt[o], S = B.succ_cnt[o];
    s_P = (int32_t)P;
    s_S = (int32_t)S;
    int64_t ecur = B.E;
    const int32_t sp0 = V, s0 = V + P, con0 = V + P + n;
    const uint32_t po = B.pred_off[o], so = B.succ_off[o];
    // split nodes: pre -> sp_a -> s_k
    for (uint32_t a = 0; a < P; a++) {
      int32_t pre = B.pred_src[po + a];
      int64_t b = B.pred_bytes[po + a];
      uint8_t p = B.pred_param[po + a];
      int32_t sp = sp0 + a;
      list_replace(R.succ_dst, R.succ_bytes, R.succ_param, R.succ_off[pre], R.succ_cnt[pre], o, sp);
      R.pred_off[sp] = (uint32_t)ecur;
      R.pred_cnt[sp] = 1;
      R.pred_src[ecur] = pre; R.pred_bytes[ecur] = b; R.pred_param[ecur] = p;
      ecur++;
      int64_t cc = gc->copy_fs ? ceil_div64(b * gc->copy_fs, 1000000) : 0;
      for (int d = 0; d < G; d++) R.cost[(int64_t)sp * G + d] = cc;
      R.mem[sp] = 0; R.param[sp] = 0; R.split_mask[sp] = 0; R.alive[sp] = 1;
    }
    // successor lists of split nodes (s_0..s_{n-1}) live in a block after
    int64_t ecur_s = ecur;  // succ side uses the same slot numbering on its own arrays
    for (uint32_t a = 0; a < P; a++) {
      int32_t sp = sp0 + a;
      int64_t b = B.pred_bytes[po + a];
      uint8_t p = B.pred_param[po + a];
      R.succ_off[sp] = (uint32_t)ecur_s;
      R.succ_cnt[sp] = n;
      for (int k = 0; k < n; k++) {
        R.succ_dst[ecur_s] = s0 + k;
        R.succ_bytes[ecur_s] = edge_cut(dim, p) ? part_bytes(b, n, k) : b;
        R.succ_param[ecur_s] = p;
        ecur_s++;
      }
    }
    // sub-ops s_k: preds = sp_0..sp_{P-1}, succs = con_0..con_{S-1}
    for (int k = 0; k < n; k++) {
      int32_t s = s0 + k;
      R.pred_off[s] = (uint32_t)ecur;
      R.pred_cnt[s] = P;
      for (uint32_t a = 0; a < P; a++) {
        int64_t b = B.pred_bytes[po + a];
        uint8_t p = B.pred_param[po + a];
        R.pred_src[ecur] = sp0 + a;
        R.pred_bytes[ecur] = edge_cut(dim, p) ? part_bytes(b, n, k) : b;
        R.pred_param[ecur] = p;
        ecur++;
      }
      R.succ_off[s] = (uint32_t)ecur_s;
      R.succ_cnt[s] = S;
      for (uint32_t a = 0; a < S; a++) {
        int64_t b = B.succ_bytes[so + a];
        R.succ_dst[ecur_s] = con0 + a;
        R.succ_bytes[ecur_s] = part_bytes(b, n, k);
        R.succ_param[ecur_s] = B.succ_param[so + a];
        ecur_s++;
      }
      for (int d = 0; d < G; d++) R.cost[(int64_t)s * G + d] = ceil_div64(B.cost[(int64_t)o * G + d], n);
      int64_t act = B.mem[o] - B.param[o];
      int64_t prm = dim == 0 ? B.param[o] : part_bytes(B.param[o], n, k);
      R.mem[s] = part_bytes(act, n, k) + prm;
      R.param[s] = prm;
      R.split_mask[s] = 0;
      R.alive[s] = 1;
    }
    // concat nodes: s_k -> con_b -> suc
    for (uint32_t a = 0; a < S; a++) {
      int32_t suc = B.succ_dst[so + a];
      int64_t b = B.succ_bytes[so + a];
      uint8_t p = B.succ_param[so + a];
      int32_t con = con0 + a;
      list_replace(R.pred_src, R.pred_bytes, R.pred_param, R.pred_off[suc], R.pred_cnt[suc], o, con);
      R.pred_off[con] = (uint32_t)ecur;
      R.pred_cnt[con] = n;
      for (int k = 0; k < n; k++) {
        R.pred_src[ecur] = s0 + k;
        R.pred_bytes[ecur] = part_bytes(b, n, k);
        R.pred_param[ecur] = p;
        ecur++;
      }
      R.succ_off[con] = (uint32_t)ecur_s;
      R.succ_cnt[con] = 1;
      R.succ_dst[ecur_s] = suc; R.succ_bytes[ecur_s] = b; R.succ_param[ecur_s] = p;
      ecur_s++;
      int64_t cc = gc->copy_fs ? ceil_div64(b * gc->copy_fs, 1000000) : 0;
      for (int d = 0; d < G; d++) R.cost[(int64_t)con * G + d] = cc;
      R.mem[con] = 0; R.param[con] = 0; R.split_mask[con] = 0; R.alive[con] = 1;
    }
    // Alg. 2 line 28: remove op and its edges
    R.alive[o] = 0;
    R.pred_cnt[o] = 0;
    R.succ_cnt[o] = 0;
    for (int d = 0; d < G; d++) R.cost[(int64_t)o * G + d] = 0;
    R.mem[o] = 0; R.param[o] = 0; R.split_mask[o] = 0;
    R.V = V + P + n + S;
    R.n_live = B.n_live - 1 + P + n + S;
    R.E = ecur > ecur_s ? ecur : ecur_s;
    R.H = B.H;
    R.ov_o = o;
    R.ov_base = V;
    R.ov_P = (int32_t)P;
    R.ov_n = n;
    R.ov_S = (int32_t)S;
    s_to = -1;
  }
  __syncthreads();
  // find o in the base topo order (parallel search)
  for (int32_t t = threadIdx.x; t < B.n_live; t += blockDim.x)
    if (B.topo[t] == o) s_to = t;
  __syncthreads();
  const int32_t P = s_P, S = s_S, to = s_to, ins = P + n + S;
  // new topo: base[0..to) ++ [sp.., s.., con..] ++ base(to..]
  const int32_t nl = B.n_live - 1 + ins;
  for (int32_t t = threadIdx.x; t < nl; t += blockDim.x) {
    int32_t v;
    if (t < to) v = B.topo[t];
    else if (t < to + ins) v = V + (t - to);
    else v = B.topo[t - ins + 1];
    R.topo[t] = v;
  }
}

// host-visible entry points used by the ABI (declared in the .cpp)
void launch_copy_block(const void *src, void *dst, int64_t slot_stride_bytes, int64_t bytes, const Cand *cands,
                       int nslots, cudaStream_t st, const uint32_t *nact, int64_t hole_lo, int64_t hole_hi) {
  int64_t words = (bytes + 15) / 16;
  const int64_t copied = words - (hole_hi - hole_lo) / 16;
  dim3 grid((unsigned)((copied + 255) / 256 > 1024 ? 1024 : (copied + 255) / 256), (unsigned)nslots);
  k_copy_block<<<grid, 256, 0, st>>>((const uint4 *)src, (uint4 *)dst, slot_stride_bytes / 16, words, cands, nact,
                                     hole_lo / 16, hole_hi / 16);
}
void launch_patch_split(const RawGraph *base, RawGraph *raws, const GraphConst *gc, const Cand *cands, int nslots,
                        cudaStream_t st, const uint32_t *nact) {
  k_patch_split<<<nslots, 256, 0, st>>>(base, raws, gc, cands, nact);
}

// ----------------------------------------------------------------- ranks

// link classes over the device pairs (s, t), s in S, t in T, s != t
__device__ __forceinline__ uint32_t class_mask(const GraphConst &gc, uint32_t S, uint32_t T) {
  uint32_t m = 0;
  for (uint32_t a = S; a; a &= a - 1) {
    const int s = __ffs(a) - 1;
    for (uint32_t b = T & ~(1u << s); b; b &= b - 1) m |= 1u << gc.link_class[s * gc.G + (__ffs(b) - 1)];
  }
  return m;
}

// c_ij of P:544-547 with the allowed sets of R5: a pinned endpoint's device,
// else the candidate's device set dset (R25; offm = class_mask(dset, dset))
__device__ __forceinline__ int64_t c_allowed(const GraphConst &gc, int64_t bytes, int su, int tv, uint32_t dset,
                                             uint32_t offm) {
  const bool full = dset == all_devices(gc.G);
  uint32_t mask;
  if (su < 0 && tv < 0) mask = offm;
  else if (su >= 0 && tv < 0) mask = full ? gc.row_mask[su] : class_mask(gc, 1u << su, dset);
  else if (su < 0) mask = full ? gc.col_mask[tv] : class_mask(gc, dset, 1u << tv);
  else {
    if (su == tv) return 0;
    return comm_class(gc, bytes, gc.link_class[su * gc.G + tv]);
  }
  int64_t best = 0;
  while (mask) {
    int k = __ffs(mask) - 1;
    mask &= mask - 1;
    int64_t c = comm_class(gc, bytes, k);
    best = c > best ? c : best;
  }
  return best;
}

__device__ __forceinline__ int pin_of(int32_t u, const int32_t *po, const int32_t *pd, int np) {
  int r = -1;
#pragma unroll
  for (int k = 0; k < MAXPINS; k++)
    if (k < np && po[k] == u) r = pd[k];
  return r;
}

// rank of one op u evaluated by one lane: w_u over the allowed
// devices + max over successors of (c_uv + rank_v)
__device__ __forceinline__ void rank_one(const RawGraph &R, const int64_t *cost, const GraphConst &gc, uint64_t *rank,
                                         int32_t u, const int32_t *po, const int32_t *pd, int np, uint32_t dset,
                                         uint32_t offm) {
  const int G = gc.G;
  const int pu = pin_of(u, po, pd, np);
  int64_t w = 0;
  if (pu >= 0) w = cost[(int64_t)u * G + pu];
  else
    for (int d = 0; d < G; d++) {
      const int64_t c = cost[(int64_t)u * G + d];
      w = ((dset >> d) & 1u) && c > w ? c : w;
    }
  const uint32_t off = R.succ_off[u], cnt_s = R.succ_cnt[u];
  uint64_t best = 0;
  for (uint32_t j = 0; j < cnt_s; j++) {
    const int32_t s = R.succ_dst[off + j];
    const uint64_t v =
        (uint64_t)c_allowed(gc, R.succ_bytes[off + j], pu, pin_of(s, po, pd, np), dset, offm) + rank[s];
    best = v > best ? v : best;
  }
  rank[u] = (uint64_t)w + best;
}

// One warp per slot: rank_u level by level (increasing height: every
// successor of an op sits on a lower level); the ops of a level are
// independent, one lane each.  A split slot inserts its concat nodes before
// level h(o), its sub-ops with level h(o) and its split nodes after it.
// the level records of a base graph (LvlRec): one thread per level-order index
__global__ void k_lvlrec(const RawGraph *rp, const GraphConst *gcp, int32_t n_live, LvlRec *out) {
  const RawGraph R = *rp;
  const GraphConst &gc = *gcp;
  const int G = gc.G;
  const uint32_t all = all_devices(G);
  for (int32_t q = blockIdx.x * blockDim.x + threadIdx.x; q < n_live; q += gridDim.x * blockDim.x) {
    LvlRec r;
    const int32_t u = R.lvl_ops[q];
    r.u = R.alive[u] ? u : -1;
    r.ns = (int32_t)R.succ_cnt[u];
    int64_t w = 0;
    for (int d = 0; d < G; d++) {
      const int64_t c = R.cost[(int64_t)u * G + d];
      w = c > w ? c : w;
    }
    r.w = w;
    const uint32_t so = R.succ_off[u];
#pragma unroll
    for (int k = 0; k < 4; k++) {
      const bool ok = k < r.ns;
      r.s[k] = ok ? R.succ_dst[so + k] : -1;
      r.c[k] = ok ? c_allowed(gc, R.succ_bytes[so + k], -1, -1, all, gc.offdiag_mask) : 0;
    }
    out[q] = r;
  }
}
void launch_lvlrec(const RawGraph *raw, const GraphConst *gc, int32_t n_live, LvlRec *out, cudaStream_t st) {
  if (n_live > 0) k_lvlrec<<<(n_live + 255) / 256, 256, 0, st>>>(raw, gc, n_live, out);
}

__global__ void k_rank(const RawGraph *raws, PrepGraph *pgs, const GraphConst *gcp, const Cand *cands, int nslots,
                       const uint64_t *base_rank, const uint32_t *nact, const int64_t *base_cost,
                       const LvlRec *lrec) {
  const int lane = threadIdx.x & 31;
  const int slot = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (slot >= nslots || (nact && (uint32_t)slot >= *nact)) return;
  // by value: the rank stores cannot alias the descriptor, so its pointers
  // stay in registers instead of being re-loaded after every store
  const RawGraph R = raws[slot];
  PrepGraph &P = pgs[slot];
  const GraphConst &gc = *gcp;
  int32_t po[MAXPINS], pd[MAXPINS];
  int np = 0;
  uint32_t dset = all_devices(gc.G);
  if (cands) {
    Cand c = cands[slot];
    if (c.kind == 1) {
      np = c.n_pins;
      for (int k = 0; k < MAXPINS; k++) { po[k] = c.pin_op[k]; pd[k] = c.pin_dev[k]; }
    }
    if (c.dev_mask) dset = c.dev_mask;  // R25
  }
  for (int k = np; k < MAXPINS; k++) { po[k] = -1; pd[k] = -1; }
  const uint32_t offm = dset == all_devices(gc.G) ? gc.offdiag_mask : class_mask(gc, dset, dset);
  uint64_t *rank = P.rank;
  for (int32_t u = lane; u < R.V; u += 32) rank[u] = ~0ull;
  __syncwarp();
  const bool split = R.ov_P >= 0;
  const int32_t ho = split ? R.height[R.ov_o] : -1;
  int32_t lev0 = 0;
  if (split && base_rank && cands && cands[slot].kind == 2 && cands[slot].dev_mask == 0) {
    // an op below the split op's height has no path to it: its descendants,
    // their costs and edges are the base graph's, and so is its rank_u
    const int32_t hi = R.lvl_off[ho];
    for (int32_t q = lane; q < hi; q += 32) {
      const int32_t u = R.lvl_ops[q];
      if (R.alive[u]) rank[u] = base_rank[u];
    }
    __syncwarp();
    lev0 = ho;
  }
  // Fast path (lrec): a level above the split op's (every level of a PIN
  // slot) reads one base record per op -- its w and the first 4 successors'
  // c are the base graph's unless the op or that successor is pinned, or the
  // op is a predecessor of the split op (its successor list now holds a
  // split node): those take rank_one on the slot's lists, as do successors
  // past the 4th (from the slot's lists, unchanged for these ops) and the
  // ops past a level's first 32.
  const bool fast = lrec != nullptr && dset == all_devices(gc.G);
  int32_t opre[8];
  int32_t nopre = 0;
  if (fast && split) {
    nopre = R.ov_P <= 8 ? R.ov_P : -1;
    for (int k = 0; k < 8; k++)  // (split node a's single predecessor is the split op's a-th)
      opre[k] = k < nopre ? R.pred_src[R.pred_off[R.ov_base + k]] : -1;
  }
  for (int32_t lev = lev0; lev <= R.H; lev++) {
    if (fast && !(split && lev == ho) && nopre >= 0) {
      const int32_t lo = R.lvl_off[lev], cnt = R.lvl_off[lev + 1] - lo;
      if (lane < cnt) {
        const LvlRec r = lrec[lo + lane];
        const int32_t u = r.u;
        const bool skip = u < 0 || (split && u == R.ov_o);  // (dead)
        bool own = false;
#pragma unroll
        for (int k = 0; k < MAXPINS; k++) own |= k < np && (po[k] == u || po[k] == r.s[0] || po[k] == r.s[1] ||
                                                           po[k] == r.s[2] || po[k] == r.s[3]);
#pragma unroll
        for (int a = 0; a < 8; a++) own |= opre[a] == u;
        if (!skip && !own) {
          uint64_t best = 0;
#pragma unroll
          for (int k = 0; k < 4; k++) {
            const uint64_t v = k < r.ns ? (uint64_t)r.c[k] + rank[r.s[k]] : 0;
            best = v > best ? v : best;
          }
          if (r.ns > 4) {  // the rest from the slot's lists (they hold the split node already)
            const uint32_t off = R.succ_off[u];
            for (int32_t j = 4; j < r.ns; j++) {
              const int32_t sj = R.succ_dst[off + j];
              const uint64_t v =
                  (uint64_t)c_allowed(gc, R.succ_bytes[off + j], -1, pin_of(sj, po, pd, np), dset, offm) + rank[sj];
              best = v > best ? v : best;
            }
          }
          rank[u] = (uint64_t)r.w + best;
        } else if (!skip) {
          rank_one(R, split && base_cost && u < R.ov_base ? base_cost : R.cost, gc, rank, u, po, pd, np, dset, offm);
        }
      }
      for (int32_t q = lane + 32; q < cnt; q += 32) {
        const int32_t u = R.lvl_ops[lo + q];
        if (R.alive[u])
          rank_one(R, split && base_cost && u < R.ov_base ? base_cost : R.cost, gc, rank, u, po, pd, np, dset, offm);
      }
      __syncwarp();
      continue;
    }
    for (int phase = 0; phase < 3; phase++) {
      // phase 0: concat nodes (label 4h(o)-2), 1: the level (+ sub-ops at h(o)), 2: split nodes (4h(o)+2)
      int32_t lo, cnt;
      const int32_t *list = nullptr;
      if (phase == 1) {
        lo = R.lvl_off[lev];
        cnt = R.lvl_off[lev + 1] - lo;
        list = R.lvl_ops + lo;
      } else {
        if (!split || lev != ho) continue;
        lo = phase == 0 ? R.ov_base + R.ov_P + R.ov_n : R.ov_base;
        cnt = phase == 0 ? R.ov_S : R.ov_P;
      }
      const int32_t extra = (phase == 1 && split && lev == ho) ? R.ov_n : 0;
      for (int32_t q = lane; q < cnt + extra; q += 32) {
        int32_t u = q < cnt ? (list ? list[q] : lo + q) : R.ov_base + R.ov_P + (q - cnt);
        if (R.alive[u]) rank_one(R, split && base_cost && u < R.ov_base ? base_cost : R.cost, gc, rank, u, po, pd, np,
                                 dset, offm);
      }
      __syncwarp();
    }
  }
}

void launch_rank(const RawGraph *raws, PrepGraph *pgs, const GraphConst *gc, const Cand *cands, int nslots, int G,
                 cudaStream_t st, const uint64_t *base_rank, const uint32_t *nact, const int64_t *base_cost,
                 const LvlRec *lvlrec) {
  (void)G;
  int warps_per_block = 4;
  int blocks = (nslots + warps_per_block - 1) / warps_per_block;
  k_rank<<<blocks, warps_per_block * 32, 0, st>>>(raws, pgs, gc, cands, nslots, base_rank, nact, base_cost, lvlrec);
}

__device__ uint32_t cta_exscan(uint32_t v, uint32_t *total, uint32_t *s_w);

// Heights (edges on the longest path to a sink) and the per-height op lists of
// a base graph: a frontier peel from the sinks (one CTA), then a counting sort.
__global__ void __launch_bounds__(1024) k_heights(RawGraph *Rp, int32_t *scratch, int64_t vcap) {
  RawGraph &R = *Rp;
  int32_t *rem = scratch, *fa = scratch + vcap, *fb = scratch + 2 * vcap;
  __shared__ int32_t s_na, s_nb, s_H;
  __shared__ uint32_t s_w[33];
  const int tid = threadIdx.x;
  if (tid == 0) { s_na = 0; s_nb = 0; s_H = -1; }  // H = -1: no live op
  __syncthreads();
  for (int32_t u = tid; u < R.V; u += blockDim.x) {
    R.height[u] = -1;
    rem[u] = (int32_t)R.succ_cnt[u];
    if (R.alive[u] && R.succ_cnt[u] == 0) {
      R.height[u] = 0;
      fa[atomicAdd(&s_na, 1)] = u;
    }
  }
  __syncthreads();
  int32_t lev = 0;
  int32_t *cur = fa, *nxt = fb;
  while (true) {
    const int32_t nc = s_na;
    if (nc == 0) break;
    for (int32_t k = tid; k < nc; k += blockDim.x) {
      const int32_t u = cur[k];
      for (uint32_t j = 0; j < R.pred_cnt[u]; j++) {
        const int32_t p = R.pred_src[R.pred_off[u] + j];
        if (atomicSub(&rem[p], 1) == 1) {
          R.height[p] = lev + 1;
          nxt[atomicAdd(&s_nb, 1)] = p;
        }
      }
    }
    __syncthreads();
    if (tid == 0) {
      s_na = s_nb;
      s_nb = 0;
      s_H = lev;
    }
    int32_t *t = cur; cur = nxt; nxt = t;
    lev++;
    __syncthreads();
  }
  const int32_t H = s_H;
  // counting sort by height: counts -> exclusive offsets -> scatter
  for (int32_t h = tid; h <= H + 1; h += blockDim.x) R.lvl_off[h] = 0;
  __syncthreads();
  for (int32_t u = tid; u < R.V; u += blockDim.x)
    if (R.height[u] >= 0) atomicAdd(&R.lvl_off[R.height[u] + 1], 1);
  __syncthreads();
  uint32_t run = 0;
  for (int32_t t0 = 0; t0 <= H + 1; t0 += blockDim.x) {
    const int32_t h = t0 + tid;
    const uint32_t v = h <= H + 1 ? (uint32_t)R.lvl_off[h] : 0u;
    uint32_t tot;
    const uint32_t pre = cta_exscan(v, &tot, s_w);
    if (h <= H + 1) R.lvl_off[h] = (int32_t)(run + pre + v);  // inclusive: lvl_off[h] = end of level h-1
    run += tot;
  }
  __syncthreads();
  // lvl_off[h] now holds the start of level h (level counts were shifted by one)
  for (int32_t h = tid; h <= H; h += blockDim.x) rem[h] = R.lvl_off[h];
  __syncthreads();
  for (int32_t u = tid; u < R.V; u += blockDim.x)
    if (R.height[u] >= 0) R.lvl_ops[atomicAdd(&rem[R.height[u]], 1)] = u;
  if (tid == 0) R.H = H;
}

void launch_heights(RawGraph *raw_dev, int32_t *scratch, int64_t vcap, cudaStream_t st) {
  k_heights<<<1, 1024, 0, st>>>(raw_dev, scratch, vcap);
}

// ------------------------------------------------------------- radix sort

constexpr int SORT_T = 512;

// CTA exclusive scan of one value per thread; returns the prefix, *total = sum
__device__ uint32_t cta_exscan(uint32_t v, uint32_t *total, uint32_t *s_w) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_w[w] = x;
  __syncthreads();
  if (w == 0) {
    uint32_t t = lane < nw ? s_w[lane] : 0;
    uint32_t tt = t;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(FULL, tt, o);
      if (lane >= o) tt += y;
    }
    if (lane < nw) s_w[lane] = tt - t;
    if (lane == 31) s_w[32] = tt;
  }
  __syncthreads();
  uint32_t r = s_w[w] + x - v;
  *total = s_w[32];
  __syncthreads();
  return r;
}

// cta_exscan on a 64-bit word: two independent 32-bit counters scanned in
// one pass (half the barriers), valid while each half's CTA total stays
// below 2^32 (no carry crosses into the high half).
__device__ uint64_t cta_exscan64(uint64_t v, uint64_t *total, uint64_t *s_w) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  uint64_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint64_t y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_w[w] = x;
  __syncthreads();
  if (w == 0) {
    uint64_t t = lane < nw ? s_w[lane] : 0;
    uint64_t tt = t;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint64_t y = __shfl_up_sync(FULL, tt, o);
      if (lane >= o) tt += y;
    }
    if (lane < nw) s_w[lane] = tt - t;
    if (lane == 31) s_w[32] = tt;
  }
  __syncthreads();
  uint64_t r = s_w[w] + x - v;
  *total = s_w[32];
  __syncthreads();
  return r;
}

// One CTA per slot: order live ops by (rank desc, uid asc) with a stable LSD
// radix sort of key = (2^key_bits - 1 - rank) over values initially in uid order.
template <typename KT>  // key type: uint32_t when key_bits <= 32 (half the key traffic), else uint64_t
__global__ void __launch_bounds__(SORT_T) k_sort(PrepGraph *pgs, const RawGraph *raws, int key_bits,
                                                 const uint32_t *nact) {
  if (nact && blockIdx.x >= *nact) return;
  PrepGraph &P = pgs[blockIdx.x];
  const RawGraph &R = raws[blockIdx.x];
  __shared__ uint32_t s_w[33];
  __shared__ uint32_t s_base[256], s_tot[256], s_cst[256];
  __shared__ uint32_t s_cnt[SORT_T / 32][257];
  __shared__ KT s_k[SORT_T];  // a chunk in digit order (coalesced write-out)
  __shared__ uint32_t s_v[SORT_T];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const uint64_t maxk = key_bits >= 64 ? ~0ull : ((1ull << key_bits) - 1);
  // compaction of live uids in ascending order
  uint32_t run = 0;
  for (int32_t t0 = 0; t0 < R.V; t0 += SORT_T) {
    int32_t u = t0 + tid;
    uint32_t live = (u < R.V && R.alive[u]) ? 1u : 0u;
    uint32_t tot;
    uint32_t pre = cta_exscan(live, &tot, s_w);
    if (live) {
      ((KT *)P.key0)[run + pre] = (KT)(maxk - P.rank[u]);
      P.val0[run + pre] = (uint32_t)u;
    }
    run += tot;
  }
  const int32_t n = (int32_t)run;
  if (tid == 0) P.n = n;
  KT *kin = (KT *)P.key0, *kout = (KT *)P.key1;
  uint32_t *vin = P.val0, *vout = P.val1;
  const unsigned lt = (1u << lane) - 1;
  for (int sh = 0; sh < key_bits; sh += 8) {
    for (int d = tid; d < 256; d += SORT_T) s_base[d] = 0;
    __syncthreads();
    for (int32_t i = tid; i < n; i += SORT_T) atomicAdd(&s_base[(kin[i] >> sh) & 255], 1u);
    __syncthreads();
    if (wid == 0) {
      // exclusive scan of 256 digit counts by one warp (8 per lane)
      uint32_t loc[8], s = 0;
#pragma unroll
      for (int q = 0; q < 8; q++) { loc[q] = s_base[lane * 8 + q]; s += loc[q]; }
      uint32_t x = s;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(FULL, x, o);
        if (lane >= o) x += y;
      }
      uint32_t e = x - s;
#pragma unroll
      for (int q = 0; q < 8; q++) { s_base[lane * 8 + q] = e; e += loc[q]; }
    }
    __syncthreads();
    for (int32_t t0 = 0; t0 < n; t0 += SORT_T) {
      for (int q = tid; q < (SORT_T / 32) * 257; q += SORT_T) (&s_cnt[0][0])[q] = 0;
      __syncthreads();
      int32_t i = t0 + tid;
      bool valid = i < n;
      KT k = valid ? kin[i] : (KT)0;
      uint32_t v = valid ? vin[i] : 0;
      uint32_t dg = valid ? (uint32_t)((k >> sh) & 255) : 256u;
      unsigned peers = __match_any_sync(FULL, dg);
      uint32_t rk = __popc(peers & lt);
      if (rk == 0) s_cnt[wid][dg] = __popc(peers);
      __syncthreads();
      if (tid < 256) {
        uint32_t r = 0;
        for (int w = 0; w < SORT_T / 32; w++) {
          uint32_t c = s_cnt[w][tid];
          s_cnt[w][tid] = r;
          r += c;
        }
        s_tot[tid] = r;
      }
      __syncthreads();
      if (wid == 0) {  // the chunk's digit starts: exclusive scan of s_tot (8 per lane)
        uint32_t loc[8], sm = 0;
#pragma unroll
        for (int q = 0; q < 8; q++) { loc[q] = s_tot[lane * 8 + q]; sm += loc[q]; }
        uint32_t x = sm;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t y = __shfl_up_sync(FULL, x, o);
          if (lane >= o) x += y;
        }
        uint32_t e = x - sm;
#pragma unroll
        for (int q = 0; q < 8; q++) { s_cst[lane * 8 + q] = e; e += loc[q]; }
      }
      __syncthreads();
      // stable within the chunk: digit, then warp, then lane
      if (valid) {
        const uint32_t l = s_cst[dg] + s_cnt[wid][dg] + rk;
        s_k[l] = k;
        s_v[l] = v;
      }
      __syncthreads();
      // write-out in chunk order: a digit's keys land contiguously
      if (i < n) {
        const KT kk = s_k[tid];
        const uint32_t d = (uint32_t)((kk >> sh) & 255);
        const uint32_t dst = s_base[d] + ((uint32_t)tid - s_cst[d]);
        kout[dst] = kk;
        vout[dst] = s_v[tid];
      }
      __syncthreads();
      if (tid < 256) s_base[tid] += s_tot[tid];
      __syncthreads();
    }
    KT *tk = kin; kin = kout; kout = tk;
    uint32_t *tv = vin; vin = vout; vout = tv;
  }
  // positions
  for (int32_t u = tid; u < R.V; u += SORT_T) P.pos[u] = NONE;
  __syncthreads();
  for (int32_t p = tid; p < n; p += SORT_T) {
    uint32_t u = vin[p];
    P.uid[p] = u;
    P.pos[u] = (uint32_t)p;
  }
}

void launch_sort(PrepGraph *pgs, const RawGraph *raws, int nslots, int key_bits, int max_n, cudaStream_t st,
                 const uint32_t *nact) {
  (void)max_n;
  if (key_bits <= 32) k_sort<uint32_t><<<nslots, SORT_T, 0, st>>>(pgs, raws, key_bits, nact);
  else k_sort<uint64_t><<<nslots, SORT_T, 0, st>>>(pgs, raws, key_bits, nact);
}

// ----------------------------------------------------------------- cards

// One CTA per slot: degree scans in position order + card headers.
__global__ void __launch_bounds__(SORT_T) k_cards_hdr(const RawGraph *raws, PrepGraph *pgs, const uint32_t *nact,
                                                      const int64_t *base_mem, const int64_t *base_param) {
  if (nact && blockIdx.x >= *nact) return;
  const RawGraph R = raws[blockIdx.x];  // (by value: see k_rank)
  // (a split slot's base-op memory from the base graph: see k_copy_block)
  const bool bm = base_mem && R.ov_P >= 0;
  PrepGraph &P = pgs[blockIdx.x];
  __shared__ uint64_t s_w[33];
  const int32_t n = P.n;
  uint32_t runp = 0, runs = 0;
  for (int32_t w = threadIdx.x; w < (n + 31) / 32; w += blockDim.x) P.srcbits[w] = 0;
  if (threadIdx.x == 0) P.topo = 1;  // cleared by k_cards_edges on a backward edge
  __syncthreads();
  for (int32_t t0 = 0; t0 < n; t0 += blockDim.x) {
    int32_t p = t0 + threadIdx.x;
    uint32_t u = p < n ? P.uid[p] : 0;
    uint32_t np_ = p < n ? R.pred_cnt[u] : 0, ns_ = p < n ? R.succ_cnt[u] : 0;
    // both degree scans in one pass: degrees < 2^16 (CW_DEG), so a chunk's
    // half-totals stay below 2^26
    uint64_t tot2;
    const uint64_t b2 = cta_exscan64((uint64_t)np_ | ((uint64_t)ns_ << 32), &tot2, s_w);
    const uint32_t bp = (uint32_t)b2, bs = (uint32_t)(b2 >> 32);
    const uint32_t totp = (uint32_t)tot2, tots = (uint32_t)(tot2 >> 32);
    if (p < n) {
      uint32_t *c = P.card + (int64_t)p * CARD_WORDS;
      const bool fb = bm && (int32_t)u < R.ov_base;
      const int64_t mu = fb ? base_mem[u] : R.mem[u], pu = fb ? base_param[u] : R.param[u];
      const uint64_t m = (uint64_t)mu;
      // the header words 0-7 (CW_DEG .. CW_FLAGS) as two 16-B stores
      static_assert(CW_DEG == 0 && CW_PBASE == 1 && CW_SBASE == 2 && CW_CPIDX == 3 && CW_MEMLO == 4 &&
                        CW_MEMHI == 5 && CW_UID == 6 && CW_FLAGS == 7, "card header layout");
      *(uint4 *)c = make_uint4(np_ | (ns_ << 16), runp + bp, runs + bs, NONE);
      *(uint4 *)(c + 4) = make_uint4((uint32_t)m, (uint32_t)(m >> 32), u, 0u);
      P.act[p] = mu - pu;
      P.npred[p] = np_;
      if (np_ == 0) atomicOr(&P.srcbits[p >> 5], 1u << (p & 31));
    }
    runp += totp;
    runs += tots;
  }
  if (threadIdx.x == 0) P.E = runp;
  __syncthreads();
  // summary level of the source bitmap (read by the simulator's prologue)
  if (threadIdx.x < 32) {
    const int32_t nw = (n + 31) / 32;
    uint32_t sw = 0;
    for (int b = 0; b < 32; b++) {
      int32_t w = (int32_t)threadIdx.x * 32 + b;
      if (w < nw && P.srcbits[w]) sw |= 1u << b;
    }
    P.srcsumm[threadIdx.x] = sw;
    unsigned top = __ballot_sync(0xFFFFFFFFu, sw != 0);
    if (threadIdx.x == 0) P.srcsumm[32] = top;
  }
}

// One thread per position: the cost row, the predecessor edge arrays and
// the inline predecessor entries of the card (words 8-15); clears P.topo on
// an edge that does not go from a lower to a higher position.
template <typename T>
__global__ void k_cards_pred(const RawGraph *raws, PrepGraph *pgs, const GraphConst *gcp, const uint32_t *nact,
                             const int64_t *base_cost) {
  const int slot = blockIdx.y;
  if (nact && (uint32_t)slot >= *nact) return;
  const RawGraph R = raws[slot];  // (by value: see k_rank)
  PrepGraph &P = pgs[slot];
  const GraphConst &gc = *gcp;
  const int G = gc.G, K = gc.K;
  const int32_t n = P.n;
  T *costp = (T *)P.costp;
  T *pec = (T *)P.pe_comm;
  bool back = false;
  for (int32_t p = blockIdx.x * blockDim.x + threadIdx.x; p < n; p += gridDim.x * blockDim.x) {
    uint32_t *c = P.card + (int64_t)p * CARD_WORDS;
    const uint32_t u = P.uid[p];
    const uint2 dp = *(const uint2 *)c;  // CW_DEG, CW_PBASE (k_cards_hdr)
    const uint32_t np_ = dp.x & 0xFFFF, pb = dp.y;
    const int64_t *cr = base_cost && R.ov_P >= 0 && (int32_t)u < R.ov_base ? base_cost : R.cost;  // (see k_copy_block)
    if (sizeof(T) == 4 && (G & 3) == 0) {  // 16-B stores of the row (4 devices each)
      for (int d = 0; d < G; d += 4) {
        const longlong2 a = *(const longlong2 *)(cr + (int64_t)u * G + d);
        const longlong2 b = *(const longlong2 *)(cr + (int64_t)u * G + d + 2);
        *(uint4 *)(costp + (int64_t)p * G + d) = make_uint4((uint32_t)a.x, (uint32_t)a.y, (uint32_t)b.x, (uint32_t)b.y);
      }
    } else {
      for (int d = 0; d < G; d++) costp[(int64_t)p * G + d] = (T)cr[(int64_t)u * G + d];
    }
    const uint32_t po = R.pred_off[u];
    uint32_t inl[P_IN] = {0, 0, 0, 0}, icm[P_IN] = {0, 0, 0, 0};  // unused slots hold position 0
#pragma unroll
    for (int j = 0; j < P_IN; j++)
      if ((uint32_t)j < np_) {
        const int32_t s = R.pred_src[po + j];
        const int64_t b = R.pred_bytes[po + j];
        const uint32_t sp = P.pos[s];
        P.pe_src[pb + j] = sp;
        back |= sp >= (uint32_t)p;
        for (int k = 0; k < K; k++) pec[(int64_t)(pb + j) * K + k] = (T)comm_class(gc, b, k);
        inl[j] = sp;
        icm[j] = (uint32_t)comm_class(gc, b, 0);  // used only for uint32 time, one class
      }
    for (uint32_t j = P_IN; j < np_; j++) {
      const int32_t s = R.pred_src[po + j];
      const int64_t b = R.pred_bytes[po + j];
      const uint32_t sp = P.pos[s];
      P.pe_src[pb + j] = sp;
      back |= sp >= (uint32_t)p;
      for (int k = 0; k < K; k++) pec[(int64_t)(pb + j) * K + k] = (T)comm_class(gc, b, k);
    }
    *(uint4 *)(c + CARD_HDR) = make_uint4(inl[0], inl[1], inl[2], inl[3]);
    *(uint4 *)(c + CW_PCOMM) = make_uint4(icm[0], icm[1], icm[2], icm[3]);
  }
  if (__syncthreads_or(back) && threadIdx.x == 0) P.topo = 0;  // the priority order is not topological
}

// One warp per position: successor edge arrays and inline successor entries
// (words 16-31).  Only the ready-set simulator and the PIN classification
// read them, so slots whose order is topological are skipped unless `all`.
__global__ void k_cards_succ(const RawGraph *raws, PrepGraph *pgs, int all, const uint32_t *nact) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int slot = blockIdx.y;
  if (nact && (uint32_t)slot >= *nact) return;
  const RawGraph R = raws[slot];  // (by value: see k_rank)
  PrepGraph &P = pgs[slot];
  if (!all && P.topo) return;
  const int32_t n = P.n;
  for (int64_t p = gw; p < n; p += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    uint32_t *c = P.card + p * CARD_WORDS;
    const uint32_t u = P.uid[p];
    const uint32_t ns_ = c[CW_DEG] >> 16, sb = c[CW_SBASE];
    const uint32_t so = R.succ_off[u];
    for (uint32_t j = lane; j < ns_; j += 32) {
      int32_t d = R.succ_dst[so + j];
      uint32_t dp = P.pos[d];
      P.se_dst[sb + j] = dp;
      // index of edge (u -> d) within d's predecessor list
      uint32_t dpo = R.pred_off[d], dcnt = R.pred_cnt[d], q = 0;
      while (q < dcnt && R.pred_src[dpo + q] != (int32_t)u) q++;
      P.se_pe[sb + j] = P.card[(int64_t)dp * CARD_WORDS + CW_PBASE] + q;
      if (j < S_IN) c[CW_SUCC + j] = dp;
    }
    // unused inline slots hold position 0 so the simulator may load them speculatively
    if (lane >= ns_ && lane < S_IN) c[CW_SUCC + lane] = 0;
  }
}

void launch_cards(const RawGraph *raws, PrepGraph *pgs, const GraphConst *gc, int nslots, int max_n, int G, int K,
                  int tbits, cudaStream_t st, bool succ_all, const uint32_t *nact, const int64_t *base_cost,
                  const int64_t *base_mem, const int64_t *base_param) {
  (void)G; (void)K;
  k_cards_hdr<<<nslots, SORT_T, 0, st>>>(raws, pgs, nact, base_mem, base_param);
  dim3 gp((unsigned)std::max(1, std::min((max_n + 255) / 256, 1024)), nslots);
  if (tbits == 32) k_cards_pred<uint32_t><<<gp, 256, 0, st>>>(raws, pgs, gc, nact, base_cost);
  else k_cards_pred<uint64_t><<<gp, 256, 0, st>>>(raws, pgs, gc, nact, base_cost);
  int blocks = (max_n * 32 + 255) / 256;
  if (blocks > 2048) blocks = 2048;
  // (only the rare non-topological slots do work unless succ_all: a full-width
  // grid per slot cost ~3.5 ms per 4k-slot wave in empty blocks alone)
  if (!succ_all && nslots > 1 && blocks > 32) blocks = 32;
  if (blocks < 1) blocks = 1;
  k_cards_succ<<<dim3(blocks, nslots), 256, 0, st>>>(raws, pgs, succ_all ? 1 : 0, nact);
}

// -------------------------------------------------------------------- CP

// One warp per slot: the critical path (R4, R7) -- the highest-priority entry
// op, then repeatedly the successor of highest priority (= lowest position) --
// and its prefix sums of memory and per-device cost (for R9).
template <typename T>
__global__ void k_cp(const RawGraph *raws, PrepGraph *pgs, int nslots, int G, const uint32_t *nact) {
  const int lane = threadIdx.x & 31;
  const int slot = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (slot >= nslots || (nact && (uint32_t)slot >= *nact)) return;
  const RawGraph R = raws[slot];  // (by value: see k_rank)
  PrepGraph &P = pgs[slot];
  const int32_t n = P.n;
  const T *costp = (const T *)P.costp;
  if (n == 0) {
    if (lane == 0) { P.cp_len = 0; P.pmem[0] = 0; }
    if (lane < G) P.pcost[lane] = 0;
    return;
  }
  // first source position
  uint32_t cur = NONE;
  for (int32_t w0 = 0; w0 < (n + 31) / 32 && cur == NONE; w0 += 32) {
    uint32_t word = (w0 + lane) < (n + 31) / 32 ? P.srcbits[w0 + lane] : 0;
    unsigned b = __ballot_sync(FULL, word != 0);
    if (b) {
      int l = __ffs(b) - 1;
      uint32_t wv = __shfl_sync(FULL, word, l);
      cur = (uint32_t)(w0 + l) * 32 + (__ffs(wv) - 1);
    }
  }
  int64_t accm = 0, accc = 0;
  // the walk's arrays in registers: its stores would otherwise force the
  // PrepGraph pointers to be re-loaded on every step of the chain
  uint32_t *const card = P.card, *const cpl = P.cp;
  const uint32_t *const pos = P.pos;
  int64_t *const pmem = P.pmem, *const pcost = P.pcost;
  if (lane == 0) pmem[0] = 0;
  if (lane < G) pcost[lane] = 0;
  int32_t len = 0;
  while (cur != NONE) {
    const uint32_t *c = card + (int64_t)cur * CARD_WORDS;
    uint32_t deg = c[CW_DEG];
    int64_t m = (int64_t)(((uint64_t)c[CW_MEMHI] << 32) | c[CW_MEMLO]);
    const uint32_t uid = c[CW_UID];
    if (lane == 0) {
      cpl[len] = cur;
      card[(int64_t)cur * CARD_WORDS + CW_CPIDX] = (uint32_t)len;
    }
    accm += m;
    if (lane < G) accc += (int64_t)costp[(int64_t)cur * G + lane];
    len++;
    if (lane == 0) pmem[len] = accm;
    if (lane < G) pcost[(int64_t)len * G + lane] = accc;
    // successors from the raw lists (the card's successor part is built
    // only where the ready-set simulator needs it)
    const uint32_t ns_ = deg >> 16, so = R.succ_off[uid];
    uint32_t best = NONE;
    for (uint32_t j = lane; j < ns_; j += 32) {
      const uint32_t d = pos[R.succ_dst[so + j]];
      best = d < best ? d : best;
    }
    best = warp_min_u32(best);
    cur = ns_ ? best : NONE;
  }
  if (lane == 0) P.cp_len = len;
}

void launch_cp(const RawGraph *raws, PrepGraph *pgs, int nslots, int G, int tbits, cudaStream_t st,
               const uint32_t *nact) {
  int blocks = (nslots + 3) / 4;
  if (tbits == 32) k_cp<uint32_t><<<blocks, 128, 0, st>>>(raws, pgs, nslots, G, nact);
  else k_cp<uint64_t><<<blocks, 128, 0, st>>>(raws, pgs, nslots, G, nact);
}

// ----------------------------------------------------------------- bound

// out[0] += sum over live ops of (max cost + max over in-edges of max_k comm)
// out[1]  = max over splittable ops of the largest split overlay increment.
__device__ __forceinline__ int64_t maxcomm_all(const GraphConst &gc, int64_t b) {
  int64_t m = 0;
  for (int k = 0; k < gc.K; k++) {
    int64_t c = comm_class(gc, b, k);
    m = c > m ? c : m;
  }
  return gc.G > 1 ? m : 0;
}

__global__ void k_bound(const RawGraph *rp, const GraphConst *gcp, unsigned long long *out) {
  const RawGraph &R = *rp;
  const GraphConst &gc = *gcp;
  const int G = gc.G;
  unsigned long long sum = 0, mx = 0;
  for (int32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < R.V; u += gridDim.x * blockDim.x) {
    if (!R.alive[u]) continue;
    int64_t mc = 0;
    for (int d = 0; d < G; d++) mc = R.cost[(int64_t)u * G + d] > mc ? R.cost[(int64_t)u * G + d] : mc;
    int64_t mi = 0, sin = 0, smaxin = 0;
    for (uint32_t j = 0; j < R.pred_cnt[u]; j++) {
      int64_t b = R.pred_bytes[R.pred_off[u] + j];
      int64_t c = maxcomm_all(gc, b);
      mi = c > mi ? c : mi;
      sin += c + (gc.copy_fs ? ceil_div64(b * gc.copy_fs, 1000000) : 0);
    }
    smaxin = mi;
    sum += (unsigned long long)(mc + mi);
    if (R.split_mask[u]) {
      int64_t sout = 0;
      for (uint32_t j = 0; j < R.succ_cnt[u]; j++) {
        int64_t b = R.succ_bytes[R.succ_off[u] + j];
        sout += maxcomm_all(gc, b) + (gc.copy_fs ? ceil_div64(b * gc.copy_fs, 1000000) : 0);
      }
      unsigned long long ex = (unsigned long long)(sin + mc + (G - 1) + (int64_t)G * smaxin + sout);
      mx = ex > mx ? ex : mx;
    }
  }
  atomicAdd(&out[0], sum);
  atomicMax(&out[1], mx);
}

void launch_bound(const RawGraph *raw, const GraphConst *gc, int G, unsigned long long *out, cudaStream_t st) {
  (void)G;
  k_bound<<<148, 256, 0, st>>>(raw, gc, out);
}

// ------------------------------------------------------------ split list

// Alg. 2 lines 4-5 (R15) for placement S: rank'(i) = cost[i][S(i)] +
// max_succ (comm(b, S(i), S(j)) + rank'(j)); CP by R7 on rank'; keep ops
// with a splittable dimension; sort by cost on the assigned device desc, id asc.
__global__ void k_splitlist(const RawGraph *rp, const GraphConst *gcp, const uint8_t *place, int32_t *list,
                            int32_t *nlist, int64_t *rk, int32_t *cp) {
  const RawGraph &R = *rp;
  const GraphConst &gc = *gcp;
  const int lane = threadIdx.x & 31;
  const int G = gc.G;
  const int32_t nl = R.n_live;
  for (int32_t base = nl - 1; base >= 0; base -= 32) {
    int32_t tl = base - lane;
    int32_t mine = tl >= 0 ? R.topo[tl] : -1;
    int cnt = base + 1 < 32 ? base + 1 : 32;
    for (int q = 0; q < cnt; q++) {
      int32_t u = __shfl_sync(FULL, mine, q);
      int su = place[u];
      uint32_t off = R.succ_off[u], cs = R.succ_cnt[u];
      uint64_t best = 0;
      for (uint32_t j0 = 0; j0 < cs; j0 += 32) {
        uint64_t v = 0;
        if (j0 + lane < cs) {
          int32_t s = R.succ_dst[off + j0 + lane];
          int64_t b = R.succ_bytes[off + j0 + lane];
          int ts = place[s];
          int64_t cm = su == ts ? 0 : comm_class(gc, b, gc.link_class[su * G + ts]);
          v = (uint64_t)(cm + rk[s]);
        }
        v = warp_max_u64(v);
        best = v > best ? v : best;
      }
      if (lane == 0) rk[u] = R.cost[(int64_t)u * G + su] + (int64_t)best;
      __syncwarp();
    }
  }
  if (lane != 0) return;
  // sources: max (rank', -id)
  int32_t cur = -1;
  for (int32_t u = 0; u < R.V; u++) {
    if (!R.alive[u] || R.pred_cnt[u] != 0) continue;
    if (cur < 0 || rk[u] > rk[cur] || (rk[u] == rk[cur] && u < cur)) cur = u;
  }
  int32_t len = 0;
  while (cur >= 0) {
    cp[len++] = cur;
    int32_t nxt = -1;
    for (uint32_t j = 0; j < R.succ_cnt[cur]; j++) {
      int32_t s = R.succ_dst[R.succ_off[cur] + j];
      if (nxt < 0 || rk[s] > rk[nxt] || (rk[s] == rk[nxt] && s < nxt)) nxt = s;
    }
    cur = nxt;
  }
  int32_t m = 0;
  for (int32_t q = 0; q < len; q++)
    if (R.split_mask[cp[q]]) list[m++] = cp[q];
  for (int32_t a = 1; a < m; a++) {
    int32_t x = list[a];
    int64_t cx = R.cost[(int64_t)x * G + place[x]];
    int32_t b = a;
    while (b > 0) {
      int32_t y = list[b - 1];
      int64_t cy = R.cost[(int64_t)y * G + place[y]];
      if (cy > cx || (cy == cx && y < x)) break;
      list[b] = y;
      b--;
    }
    list[b] = x;
  }
  *nlist = m;
}

void launch_splitlist(const RawGraph *raw, const GraphConst *gc, const uint8_t *place, int32_t *list, int32_t *nlist,
                      int64_t *scratch_rank, int32_t *scratch_cp, int G, cudaStream_t st) {
  (void)G;
  k_splitlist<<<1, 32, 0, st>>>(raw, gc, place, list, nlist, scratch_rank, scratch_cp);
}

}  // namespace fastt
