// k_sim.cu -- batched DPOS list-scheduling simulation.
//
// Persistent kernel; a warp holds 32/GP candidates, one per group of GP
// lanes (GP = the device count rounded up to a power of two; lane d of a
// group is device d).  Work is fetched from a global counter.  Per candidate:
//   prologue : decode (stream R21 / list), validate, classify (do its ranks
//              equal the base ranks? else defer to the per-candidate
//              preparation pipeline), CP-device rounds (R9),
//              ready-set bitmap from the source bitmap, indegrees into the
//              candidate's slab.
//   loop     : pop the max-priority ready op = find-first-set over the
//              position bitmap (2 levels in smem + 1 in a register);
//              loads from the op's 128-B card (predecessor positions and
//              comm, successors) + the cost row, then the predecessor
//              records; lane d forms EST(d) = max(avail[d], max_pred FT +
//              comm) (R1, R6), EFT = EST + cost; memory-feasible
//              argmin over the group with ties to the lowest device
//              (Alg. 1 lines 12-19, R3, R8); CP pins (lines 9-10) and
//              perturbation pins override it; release successors
//              (indegree in the slab) into the bitmap.
//   epilogue : makespan = max FT (R16), peak memory per device, outputs,
//              per-slot best (makespan, index) for the sweep argmin (S7).
// Time arithmetic runs in T = uint32 when the load-time bound proves every
// schedule fits (R18), else uint64; results are identical.
//
// The kernel itself is in k_sim_body.cuh (instances: k_sim_inst.cu).
#include "fastt_internal.cuh"
#include "sim_common.cuh"

namespace fastt {


__global__ void k_candgen(StreamState S, int64_t first, int64_t n, const int64_t *idx_list, int64_t stride,
                          Cand *out, int64_t *out_index) {
  for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x) {
    int64_t c = idx_list ? first + idx_list[q] * stride : first + q;
    out[q] = stream_cand(S, c);
    if (out_index) out_index[q] = c;
  }
}

void launch_candgen(const StreamState &s, int64_t first, int64_t n, Cand *out, cudaStream_t st) {
  if (n <= 0) return;
  int blocks = (int)((n + 255) / 256 < 4096 ? (n + 255) / 256 : 4096);
  k_candgen<<<blocks, 256, 0, st>>>(s, first, n, nullptr, 1, out, nullptr);
}
void launch_candgen_idx(const StreamState &s, int64_t first, int64_t stride, const int64_t *qlist, int64_t n,
                        Cand *out, int64_t *out_index, cudaStream_t st) {
  if (n <= 0) return;
  int blocks = (int)((n + 255) / 256 < 4096 ? (n + 255) / 256 : 4096);
  k_candgen<<<blocks, 256, 0, st>>>(s, first, n, qlist, stride, out, out_index);
}

// kernel getters of the per-GSH instance objects (k_sim_inst.cu)
static const void *sim_fn(int tbits, int gshift, bool mem, bool ins = false, bool fc = false, bool topo = false) {
  switch (gshift) {
    case 0: return sim_fn_g0(tbits, mem, ins, fc, topo);
    case 1: return sim_fn_g1(tbits, mem, ins, fc, topo);
    case 2: return sim_fn_g2(tbits, mem, ins, fc, topo);
    case 3: return sim_fn_g3(tbits, mem, ins, fc, topo);
    case 4: return sim_fn_g4(tbits, mem, ins, fc, topo);
    default: return sim_fn_g5(tbits, mem, ins, fc, topo);
  }
}

void launch_sim(const SimArgs &a, int tbits, int grid, int block, size_t smem, cudaStream_t st) {
  if (a.lane) {
    launch_sim_lane(a, tbits, grid, st);
    return;
  }
  if (a.ins && grid > a.ins_grid) grid = a.ins_grid;  // INSERT slot arrays exist for ins_grid blocks
  const void *f = sim_fn(tbits, a.gshift, a.need_mem != 0, a.ins != 0, a.fastcomm != 0, a.topo != 0);
  SimArgs aa = a;
  void *args[] = {&aa};
  cudaLaunchKernel(f, dim3(grid), dim3(block), args, smem, st);
}

int sim_occupancy(int tbits, int gshift, int block, size_t smem, bool topo) {
  int nb = 1 << 30, x = 0;
  for (int v = 0; v < 8; v++) {
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&x, sim_fn(tbits, gshift, v & 1, (v >> 2) & 1, (v >> 1) & 1, topo),
                                                  block, smem);
    nb = x < nb ? x : nb;
  }
  return nb;
}
cudaError_t sim_set_smem(int tbits, int gshift, size_t smem) {
  for (int v = 0; v < 8; v++) {
    cudaError_t e = cudaFuncSetAttribute(sim_fn(tbits, gshift, v & 1, (v >> 1) & 1, v >> 2, false),
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

// ------------------------------------------------- start-step bucketing
// Key of a candidate for prefix sharing: the BASE dequeue step of its first
// pinned op (n for BASE, 0 otherwise).  Candidates are bucket-sorted by it so
// the lane groups of a warp start at similar steps.
template <typename T>
__global__ void k_t0_keys(int from_stream, StreamState S, int64_t first, int64_t stride, const Cand *list, int64_t n,
                          const uint32_t *pos, const uint32_t *snap_dq, int32_t nops, int32_t vraw, int G, Cand *out,
                          int64_t *oidx, uint32_t *key, T0Classify cl, uint32_t defer_key) {
  for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x) {
    Cand c;
    int64_t ix;
    if (from_stream) {
      ix = first + q * stride;
      c = stream_cand(S, ix);
    } else {
      ix = q;
      c = list[q];
    }
    uint32_t k = 0;
    if (c.kind == 0) k = (uint32_t)nops;
    else if (c.kind == 1 && c.n_pins >= 1 && c.n_pins <= MAXPINS) {
      k = (uint32_t)nops;
      for (int j = 0; j < c.n_pins; j++) {
        const int32_t o = c.pin_op[j];
        if (o < 0 || o >= vraw || pos[o] == NONE || c.pin_dev[j] >= G) {
          k = 0;
          break;
        }
        const uint32_t t = snap_dq[pos[o]];
        k = t < k ? t : k;
      }
    }
    if (cl.on) {
      uint8_t st;
      if (cand_classify<T>(c, cl.pg, *cl.gc, cl.split_mask, G, true, st)) k = defer_key;
    }
    out[q] = c;
    oidx[q] = ix;
    key[q] = k;
  }
}

__global__ void k_bucket_hist(const uint32_t *key, int64_t n, int shift, uint32_t *hist) {
  for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(&hist[key[q] >> shift], 1u);
}

// exclusive scan of nb <= 1024 bucket counts, in place (one block of 1024);
// nlast (nullable) receives the offset of bucket nb - 1
__global__ void k_bucket_scan(uint32_t *hist, int nb, uint32_t *nlast) {
  __shared__ uint32_t sw[33];
  const int t = threadIdx.x, lane = t & 31, w = t >> 5;
  uint32_t v = t < nb ? hist[t] : 0, x = v;
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) sw[w] = x;
  __syncthreads();
  if (w == 0) {
    uint32_t z = sw[lane], zz = z;
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(FULL, zz, o);
      if (lane >= o) zz += y;
    }
    sw[lane] = zz - z;
  }
  __syncthreads();
  if (t < nb) hist[t] = sw[w] + x - v;
  if (nlast && t == nb - 1) *nlast = sw[w] + x - v;
}

__global__ void k_bucket_scatter(const uint32_t *key, const Cand *in, const int64_t *iidx, int64_t n, int shift,
                                 int nb, uint32_t *cursor, Cand *out, int64_t *oidx, int64_t *ores) {
  for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x) {
    // ascending start step = longest remaining simulation first
    const uint32_t b = key[q] >> shift;
    const uint32_t dst = atomicAdd(&cursor[b], 1u);
    out[dst] = in[q];
    oidx[dst] = iidx[q];
    if (ores) ores[dst] = iidx[q];
  }
  (void)nb;
}

void launch_t0_sort(int from_stream, const StreamState &S, int64_t first, int64_t stride, const Cand *list, int64_t n,
                    const uint32_t *pos, const uint32_t *snap_dq, int32_t nops, int32_t vraw, int G, Cand *tmp_c,
                    int64_t *tmp_i, uint32_t *key, uint32_t *hist, Cand *out_c, int64_t *out_i, int64_t *out_res,
                    cudaStream_t st, T0Classify cl) {
  if (n <= 0) return;
  int shift = 0;
  while ((nops >> shift) >= 1023) shift++;
  int nb = (nops >> shift) + 1;
  // classified lists: one more bucket (index nb) at the tail for the deferred
  const uint32_t defer_key = (uint32_t)nb << shift;
  if (cl.on) nb++;
  const int blocks = (int)((n + 255) / 256 < 2048 ? (n + 255) / 256 : 2048);
  if (cl.tbits == 64)
    k_t0_keys<uint64_t><<<blocks, 256, 0, st>>>(from_stream, S, first, stride, list, n, pos, snap_dq, nops, vraw, G,
                                                tmp_c, tmp_i, key, cl, defer_key);
  else
    k_t0_keys<uint32_t><<<blocks, 256, 0, st>>>(from_stream, S, first, stride, list, n, pos, snap_dq, nops, vraw, G,
                                                tmp_c, tmp_i, key, cl, defer_key);
  cudaMemsetAsync(hist, 0, sizeof(uint32_t) * 1024, st);
  k_bucket_hist<<<blocks, 256, 0, st>>>(key, n, shift, hist);
  k_bucket_scan<<<1, 1024, 0, st>>>(hist, nb, cl.on ? cl.n_main : nullptr);
  k_bucket_scatter<<<blocks, 256, 0, st>>>(key, tmp_c, tmp_i, n, shift, nb, hist, out_c, out_i, out_res);
}

// the deferred tail of a classified sorted list: entries [*n_main + off,
// *n_main + off + cap) into the preparation slots; *nslot = their count
__global__ void k_gather_tail(const Cand *src, const int64_t *sidx, const int64_t *sres, const uint32_t *n_main,
                              int64_t n, int64_t off, int cap, Cand *dst, int64_t *didx, int64_t *dres, uint32_t *nslot) {
  const int64_t base = (int64_t)*n_main + off;
  int64_t cnt = n - base;
  cnt = cnt < 0 ? 0 : (cnt > cap ? cap : cnt);
  if (blockIdx.x == 0 && threadIdx.x == 0) *nslot = (uint32_t)cnt;
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < cnt; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t q = base + k;
    dst[k] = src[q];
    if (didx) didx[k] = sidx[q];
    if (dres) dres[k] = sres ? sres[q] : -1;
  }
}
void launch_gather_tail(const Cand *src, const int64_t *sidx, const int64_t *sres, const uint32_t *n_main, int64_t n,
                        int64_t off, int cap, Cand *dst, int64_t *didx, int64_t *dres, uint32_t *nslot,
                        cudaStream_t st) {
  const int blocks = (cap + 255) / 256 < 1024 ? (cap + 255) / 256 : 1024;
  k_gather_tail<<<blocks > 0 ? blocks : 1, 256, 0, st>>>(src, sidx, sres, n_main, n, off, cap, dst, didx, dres, nslot);
}
// ------------------------------------------------- device deferral loop
__global__ void k_defer_setup(DeferBlock *b, int64_t n, int cap, int src, int do_tail, int results, const Cand *cands,
                              StreamState ss, int64_t first, int64_t stride) {
  b->n = n;
  b->cap = cap;
  b->src = src;
  b->do_tail = do_tail;
  b->results = results;
  b->cands = cands;
  b->ss = ss;
  b->first = first;
  b->stride = stride;
}
void launch_defer_setup(DeferBlock *blk, int64_t n, int cap, int src, int do_tail, int results, const Cand *cands,
                        const StreamState &ss, int64_t first, int64_t stride, cudaStream_t st) {
  k_defer_setup<<<1, 1, 0, st>>>(blk, n, cap, src, do_tail, results, cands, ss, first, stride);
}
// the loop's entry: the tail past the arena (the arena held [n_main, n_main
// + cap)) and the deferral count; the WHILE condition = any work left
__global__ void k_defer_begin(DeferBlock *b, const uint32_t *n_main, const unsigned long long *ndefer,
                              cudaGraphConditionalHandle h) {
  b->n_main = b->do_tail ? (int64_t)*n_main : -1;
  b->tail_lo = b->do_tail ? b->n_main + b->cap : b->n;
  if (b->tail_lo > b->n) b->tail_lo = b->n;
  b->n_defer = (int64_t)*ndefer;
  b->total = (b->n - b->tail_lo) + b->n_defer;
  b->phase = b->tail_lo < b->n ? 0 : 1;
  b->off = 0;
  b->nact = 0;
  cudaGraphSetConditional(h, b->total > 0 ? 1u : 0u);
}
void launch_defer_begin(DeferBlock *blk, const uint32_t *n_main, const unsigned long long *ndefer,
                        cudaGraphConditionalHandle h, cudaStream_t st) {
  k_defer_begin<<<1, 1, 0, st>>>(blk, n_main, ndefer, h);
}
// one round: the next at most cap entries; the condition = entries left after it
__global__ void k_defer_plan(DeferBlock *b, cudaGraphConditionalHandle h) {
  int64_t lo, cnt;
  if (b->phase == 0) {
    lo = b->tail_lo + b->off;
    cnt = b->n - lo;
  } else {
    lo = b->off;
    cnt = b->n_defer - lo;
  }
  if (cnt > b->cap) cnt = b->cap;
  if (cnt < 0) cnt = 0;
  b->q_lo = lo;
  b->q_cnt = cnt;
  b->q_phase = b->phase;
  b->nact = (uint32_t)cnt;
  b->off += cnt;
  bool more;
  if (b->phase == 0) {
    if (b->tail_lo + b->off >= b->n) {  // the tail is done: the deferral queue next
      b->phase = 1;
      b->off = 0;
      more = b->n_defer > 0;
    } else {
      more = true;
    }
  } else {
    more = b->off < b->n_defer;
  }
  cudaGraphSetConditional(h, more ? 1u : 0u);
}
void launch_defer_plan(DeferBlock *blk, cudaGraphConditionalHandle h, cudaStream_t st) {
  k_defer_plan<<<1, 1, 0, st>>>(blk, h);
}
// the round's candidates into the preparation slots (phase 0: sorted
// positions; phase 1: defer_q entries of the sorted list, the candidate list
// or the stream)
__global__ void k_defer_gather(const DeferBlock *b, const Cand *srt_c, const int64_t *srt_i, const int64_t *srt_res,
                               const int64_t *defer_q, Cand *dst, int64_t *didx, int64_t *dres) {
  const int64_t cnt = b->q_cnt, lo = b->q_lo;
  const bool tail = b->q_phase == 0;
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < cnt; k += (int64_t)gridDim.x * blockDim.x) {
    Cand c;
    int64_t sidx, res;
    if (tail || b->src == 0) {
      const int64_t q = tail ? lo + k : defer_q[lo + k];
      c = srt_c[q];
      sidx = srt_i[q];
      res = srt_res ? srt_res[q] : -1;
    } else if (b->src == 1) {
      const int64_t q = defer_q[lo + k];
      c = b->cands[q];
      sidx = q;
      res = q;
    } else {
      const int64_t q = defer_q[lo + k];
      sidx = b->first + q * b->stride;
      c = stream_cand(b->ss, sidx);
      res = -1;
    }
    dst[k] = c;
    if (didx) didx[k] = sidx;
    if (dres) dres[k] = res;
  }
}
void launch_defer_gather(const DeferBlock *blk, int cap, const Cand *srt_c, const int64_t *srt_i,
                         const int64_t *srt_res, const int64_t *defer_q, Cand *dst, int64_t *didx, int64_t *dres,
                         cudaStream_t st) {
  const int blocks = (cap + 255) / 256 < 1024 ? (cap + 255) / 256 : 1024;
  k_defer_gather<<<blocks > 0 ? blocks : 1, 256, 0, st>>>(blk, srt_c, srt_i, srt_res, defer_q, dst, didx, dres);
}
// per-warp best pairs (makespan, index) := (INT64_MAX, -1)
__global__ void k_init_best(int64_t *wb, int64_t nw) {
  for (int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; w < nw; w += (int64_t)gridDim.x * blockDim.x) {
    wb[2 * w] = I64MAX;
    wb[2 * w + 1] = -1;
  }
}
void launch_init_best(int64_t *wb, int64_t nw, cudaStream_t st) {
  if (nw > 0) k_init_best<<<(int)((nw + 255) / 256 < 1024 ? (nw + 255) / 256 : 1024), 256, 0, st>>>(wb, nw);
}

__global__ void k_gather_sorted(const Cand *src, const int64_t *sidx, const int64_t *sres, const int64_t *qs, int64_t n,
                                Cand *dst, int64_t *didx, int64_t *dres) {
  int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= n) return;
  const int64_t q = qs[k];
  dst[k] = src[q];
  if (didx) didx[k] = sidx[q];
  if (dres) dres[k] = sres ? sres[q] : -1;
}
void launch_gather_sorted(const Cand *src, const int64_t *sidx, const int64_t *sres, const int64_t *qs, int64_t n,
                          Cand *dst, int64_t *didx, int64_t *dres, cudaStream_t st) {
  if (n <= 0) return;
  k_gather_sorted<<<(unsigned)((n + 127) / 128), 128, 0, st>>>(src, sidx, sres, qs, n, dst, didx, dres);
}

// ------------------------------------------------------------------ argmin

// lexicographic min over per-warp (makespan, index) pairs (R3)
__global__ void k_argmin(const int64_t *wb, int64_t nw, int64_t *best) {
  __shared__ int64_t sm[32], si[32];
  int64_t bm = I64MAX, bi = -1;
  for (int64_t w = threadIdx.x; w < nw; w += blockDim.x) {
    int64_t m = wb[2 * w], i = wb[2 * w + 1];
    if (i >= 0 && (m < bm || (m == bm && (bi < 0 || i < bi)))) { bm = m; bi = i; }
  }
  for (int o = 16; o > 0; o >>= 1) {
    int64_t m = __shfl_xor_sync(FULL, bm, o), i = __shfl_xor_sync(FULL, bi, o);
    if (i >= 0 && (m < bm || (m == bm && (bi < 0 || i < bi)))) { bm = m; bi = i; }
  }
  if ((threadIdx.x & 31) == 0) { sm[threadIdx.x >> 5] = bm; si[threadIdx.x >> 5] = bi; }
  __syncthreads();
  if (threadIdx.x < 32) {
    int nw2 = blockDim.x >> 5;
    bm = threadIdx.x < nw2 ? sm[threadIdx.x] : I64MAX;
    bi = threadIdx.x < nw2 ? si[threadIdx.x] : -1;
    for (int o = 16; o > 0; o >>= 1) {
      int64_t m = __shfl_xor_sync(FULL, bm, o), i = __shfl_xor_sync(FULL, bi, o);
      if (i >= 0 && (m < bm || (m == bm && (bi < 0 || i < bi)))) { bm = m; bi = i; }
    }
    if (threadIdx.x == 0) { best[0] = bi >= 0 ? bm : I64MAX; best[1] = bi; }
  }
}

void launch_argmin(const int64_t *wbest, int64_t nwarps, int64_t *best_dev, cudaStream_t st) {
  k_argmin<<<1, 1024, 0, st>>>(wbest, nwarps, best_dev);
}

__global__ void k_fill_i64(int64_t *p, int64_t n, int64_t v) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) p[i] = v;
}
__global__ void k_iota_i64(int64_t *p, int64_t n) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) p[k] = k;
}
void launch_iota_i64(int64_t *p, int64_t n, cudaStream_t st) {
  if (n > 0) k_iota_i64<<<(int)((n + 255) / 256 < 1024 ? (n + 255) / 256 : 1024), 256, 0, st>>>(p, n);
}
void launch_fill_i64(int64_t *p, int64_t n, int64_t v, cudaStream_t st) {
  if (n <= 0) return;
  int blocks = (int)((n + 255) / 256 < 4096 ? (n + 255) / 256 : 4096);
  k_fill_i64<<<blocks, 256, 0, st>>>(p, n, v);
}

// ------------------------------------------------------------------- order

// Execution order list A (Alg. 1 line 23, R17): ops sorted by (start asc,
// dequeue seq asc) = a stable LSD radix sort by start of the dequeue list.
// One CTA per result.
constexpr int ORD_T = 1024;
__global__ void __launch_bounds__(ORD_T) k_order(const int32_t *deq, const int64_t *start, int32_t *order,
                                                  const int64_t *results, int64_t vmax, int key_bits, uint64_t *k0,
                                                  uint64_t *k1, uint32_t *v0, uint32_t *v1) {
  __shared__ uint32_t s_base[256], s_tot[256];
  __shared__ uint32_t s_cnt[ORD_T / 32][257];
  __shared__ int32_t s_n;
  const int64_t r = results ? results[blockIdx.x] : blockIdx.x;
  const int32_t *dq = deq + r * vmax;
  const int64_t *stt = start + r * vmax;
  int32_t *ord = order + r * vmax;
  uint64_t *kin = k0 + blockIdx.x * vmax, *kout = k1 + blockIdx.x * vmax;
  uint32_t *vin = v0 + blockIdx.x * vmax, *vout = v1 + blockIdx.x * vmax;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  if (tid == 0) s_n = 0;
  __syncthreads();
  // n = number of dequeued ops (prefix of non-negative entries)
  for (int64_t k = tid; k < vmax; k += ORD_T)
    if (dq[k] >= 0 && (k + 1 == vmax || dq[k + 1] < 0)) s_n = (int32_t)(k + 1);
  __syncthreads();
  const int32_t n = s_n;
  for (int32_t k = tid; k < n; k += ORD_T) {
    uint32_t u = (uint32_t)dq[k];
    kin[k] = (uint64_t)stt[u];
    vin[k] = u;
  }
  __syncthreads();
  const unsigned lt = (1u << lane) - 1;
  for (int sh = 0; sh < key_bits; sh += 8) {
    for (int d = tid; d < 256; d += ORD_T) s_base[d] = 0;
    __syncthreads();
    for (int32_t i = tid; i < n; i += ORD_T) atomicAdd(&s_base[(kin[i] >> sh) & 255], 1u);
    __syncthreads();
    if (wid == 0) {
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
    for (int32_t t0 = 0; t0 < n; t0 += ORD_T) {
      for (int q = tid; q < (ORD_T / 32) * 257; q += ORD_T) (&s_cnt[0][0])[q] = 0;
      __syncthreads();
      int32_t i = t0 + tid;
      bool valid = i < n;
      uint64_t k = valid ? kin[i] : 0;
      uint32_t v = valid ? vin[i] : 0;
      uint32_t dg = valid ? (uint32_t)((k >> sh) & 255) : 256u;
      unsigned peers = __match_any_sync(FULL, dg);
      uint32_t rk = __popc(peers & lt);
      if (rk == 0) s_cnt[wid][dg] = __popc(peers);
      __syncthreads();
      if (tid < 256) {
        uint32_t rr = 0;
        for (int w = 0; w < ORD_T / 32; w++) {
          uint32_t c = s_cnt[w][tid];
          s_cnt[w][tid] = rr;
          rr += c;
        }
        s_tot[tid] = rr;
      }
      __syncthreads();
      if (valid) {
        uint32_t dst = s_base[dg] + s_cnt[wid][dg] + rk;
        kout[dst] = k;
        vout[dst] = v;
      }
      __syncthreads();
      if (tid < 256) s_base[tid] += s_tot[tid];
      __syncthreads();
    }
    uint64_t *tk = kin; kin = kout; kout = tk;
    uint32_t *tv = vin; vin = vout; vout = tv;
  }
  for (int64_t k = tid; k < vmax; k += ORD_T) ord[k] = k < n ? (int32_t)vin[k] : -1;
}

void launch_order_chunk(const int32_t *deq, const int64_t *start, int32_t *order, const int64_t *results, int64_t n,
                        int64_t vmax, int key_bits, uint64_t *k0, uint64_t *k1, uint32_t *v0, uint32_t *v1,
                        cudaStream_t st) {
  if (n <= 0) return;
  k_order<<<(unsigned)n, ORD_T, 0, st>>>(deq, start, order, results, vmax, key_bits, k0, k1, v0, v1);
}

// slot setup for the preparation pipeline: SPLIT slots use their own raw
// copy, every other slot reads the base raw graph in place
__global__ void k_slot_setup(const Cand *cands, const RawGraph *tmpl, const RawGraph *base, RawGraph *raws,
                             int nslots) {
  int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= nslots) return;
  raws[k] = cands[k].kind == 2 ? tmpl[k] : *base;
}
void launch_slot_setup(const Cand *cands, const RawGraph *tmpl, const RawGraph *base, RawGraph *raws, int nslots,
                       cudaStream_t st) {
  k_slot_setup<<<(nslots + 127) / 128, 128, 0, st>>>(cands, tmpl, base, raws, nslots);
}

__global__ void k_gather_cands(const Cand *src, const int64_t *idx, int64_t n, Cand *dst, int64_t *res) {
  int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= n) return;
  dst[k] = src[idx[k]];
  if (res) res[k] = idx[k];
}
void launch_gather_cands(const Cand *src, const int64_t *idx, int64_t n, Cand *dst, int64_t *res, cudaStream_t st) {
  if (n <= 0) return;
  k_gather_cands<<<(unsigned)((n + 127) / 128), 128, 0, st>>>(src, idx, n, dst, res);
}

}  // namespace fastt
