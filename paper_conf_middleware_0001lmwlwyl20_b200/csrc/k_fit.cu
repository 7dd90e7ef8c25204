// k_fit.cu -- communication cost-model fit.
//
// "To build the communication cost model, we gather tensors across the same
// source-destination device pairs into one group.  For each group, we use
// linear regression to obtain a linear model: tensor size vs. transfer
// time.".  Reading R26: per ordered pair (s, t), the least-squares
// line time = alpha + beta * bytes with alpha, beta >= 0, reported as the
// nearest integers (halves up) in the units of the library's model R10:
// alpha in ns, beta in fs/byte.
//
// Two kernels:
//   k_fit_sums  -- one pass over the samples (HBM-bound): per block, exact
//                  integer moment sums per pair (n, Sb, St in 64 bits, Sbb and
//                  Sbt in 128 bits) in shared memory, then added into the
//                  global sums.  Integer addition is associative, so the sums
//                  are exact whatever the order.
//   k_fit_solve -- one thread per pair: the constrained normal equations in
//                  exact 128/256-bit integer arithmetic.
// Envelope (samples checked in k_fit_sums, the count on the host): bytes and
// time in [0, 2^40), fewer than 2^24 samples, so Sb, St < 2^64 and
// Sbb, Sbt < 2^104; every intermediate of the solve fits 256 bits and both
// results fit 64 bits.
#include <algorithm>

#include "fastt_internal.cuh"

namespace fastt {

typedef unsigned long long u64;
typedef unsigned __int128 u128;

struct FitSums {  // per pair, in global memory
  u64 n, sb, st, sbb_lo, sbb_hi, sbt_lo, sbt_hi, pad;
};

__device__ __forceinline__ void add128(u64 *lo, u64 *hi, u128 x) {
  const u64 xl = (u64)x;
  u64 xh = (u64)(x >> 64);
  const u64 old = atomicAdd(lo, xl);
  if (old + xl < old) xh += 1;  // carry out of the low word
  if (xh) atomicAdd(hi, xh);
}

__global__ void k_fit_sums(int G, int64_t n, const uint8_t *src, const uint8_t *dst, const int64_t *bytes,
                           const int64_t *tns, FitSums *out, unsigned *err) {
  extern __shared__ u64 sh[];  // [7][G*G]
  const int P = G * G;
  for (int k = threadIdx.x; k < 7 * P; k += blockDim.x) sh[k] = 0;
  __syncthreads();
  u64 *s_n = sh, *s_b = sh + P, *s_t = sh + 2 * P, *s_bbl = sh + 3 * P, *s_bbh = sh + 4 * P, *s_btl = sh + 5 * P,
      *s_bth = sh + 6 * P;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int s = src[i], d = dst[i];
    const int64_t bi = bytes[i], ti = tns[i];
    if (s >= G || d >= G || s == d || bi < 0 || ti < 0 || bi >= (1ll << 40) || ti >= (1ll << 40)) {
      atomicOr(err, 1u);  // outside R26's envelope: the call fails with EINVAL
      continue;
    }
    const int p = s * G + d;
    const u64 b = (u64)bi, t = (u64)ti;
    atomicAdd(&s_n[p], 1ull);
    atomicAdd(&s_b[p], b);
    atomicAdd(&s_t[p], t);
    add128(&s_bbl[p], &s_bbh[p], (u128)b * b);
    add128(&s_btl[p], &s_bth[p], (u128)b * t);
  }
  __syncthreads();
  for (int p = threadIdx.x; p < P; p += blockDim.x) {
    if (!s_n[p]) continue;
    FitSums &o = out[p];
    atomicAdd(&o.n, s_n[p]);
    atomicAdd(&o.sb, s_b[p]);
    atomicAdd(&o.st, s_t[p]);
    add128(&o.sbb_lo, &o.sbb_hi, ((u128)s_bbh[p] << 64) | s_bbl[p]);
    add128(&o.sbt_lo, &o.sbt_hi, ((u128)s_bth[p] << 64) | s_btl[p]);
  }
}

// ------------------------------------------------ 256-bit helpers (solve)
struct U256 {
  u128 hi, lo;
};
__device__ __forceinline__ U256 mul_128_64(u128 x, u64 y) {  // x < 2^128, y < 2^64
  const u128 p0 = (u128)(u64)x * y, p1 = (u128)(u64)(x >> 64) * y;
  U256 r;
  r.lo = p0 + (p1 << 64);
  r.hi = (p1 >> 64) + (r.lo < p0 ? 1 : 0);
  return r;
}
__device__ __forceinline__ bool lt256(const U256 &a, const U256 &b) { return a.hi < b.hi || (a.hi == b.hi && a.lo < b.lo); }
__device__ __forceinline__ U256 sub256(const U256 &a, const U256 &b) {  // a >= b
  U256 r;
  r.lo = a.lo - b.lo;
  r.hi = a.hi - b.hi - (a.lo < b.lo ? 1 : 0);
  return r;
}
__device__ __forceinline__ U256 shl256(u128 x, int s) {  // x << s, 0 <= s < 128
  U256 r;
  r.lo = x << s;
  r.hi = s ? x >> (128 - s) : 0;
  return r;
}
// nearest integer of num / den, halves up; the quotient must fit 64 bits
__device__ u64 divround(U256 num, u128 den) {
  u64 q = 0;
  for (int s = 63; s >= 0; s--) {
    const U256 d = shl256(den, s);
    if (!lt256(num, d)) {
      num = sub256(num, d);
      q |= 1ull << s;
    }
  }
  // remainder num.lo < den: round up iff 2 * rem >= den
  return q + (num.lo >= den - num.lo ? 1 : 0);
}
__device__ __forceinline__ u64 divround128(u128 num, u128 den) {
  const u128 q = num / den, r = num - q * den;
  return (u64)q + (r >= den - r ? 1 : 0);
}

__global__ void k_fit_solve(int G, const FitSums *sums, int64_t *alpha, int64_t *beta, int64_t *count) {
  const int p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= G * G) return;
  const FitSums S = sums[p];
  int64_t a = 0, b = 0;
  if (S.n > 0) {
    const u128 sbb = ((u128)S.sbb_hi << 64) | S.sbb_lo, sbt = ((u128)S.sbt_hi << 64) | S.sbt_lo;
    const u128 den = (u128)S.n * sbb - (u128)S.sb * S.sb;  // >= 0 (Cauchy-Schwarz)
    const u128 nbt = (u128)S.n * sbt, bt = (u128)S.sb * S.st;
    if (den == 0 || nbt < bt) {
      // no spread in bytes, or the b = 0 face (slope numerator < 0): mean time
      a = (int64_t)divround128(S.st, S.n);
    } else {
      const U256 A1 = mul_128_64(sbb, S.st), A2 = mul_128_64(sbt, S.sb);
      if (lt256(A1, A2)) {
        // the a = 0 face: slope = Sbt / Sbb
        b = (int64_t)divround128(sbt * 1000000u, sbb);
      } else {
        // interior: a = (Sbb St - Sb Sbt) / den, slope = (n Sbt - Sb St) / den
        a = (int64_t)divround(sub256(A1, A2), den);
        b = (int64_t)divround(mul_128_64(nbt - bt, 1000000ull), den);
      }
    }
  }
  const int s = p / G, t = p % G;
  alpha[p] = s == t ? 0 : a;
  beta[p] = s == t ? 0 : b;
  if (count) count[p] = (int64_t)S.n;
}

void launch_fit(int G, int64_t n, const uint8_t *src, const uint8_t *dst, const int64_t *bytes, const int64_t *tns,
                void *sums, unsigned *err, int64_t *alpha, int64_t *beta, int64_t *count, int sms, cudaStream_t st) {
  const int P = G * G;
  const size_t smem = (size_t)7 * P * sizeof(u64);
  cudaFuncSetAttribute(k_fit_sums, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaMemsetAsync(sums, 0, sizeof(FitSums) * P, st);
  cudaMemsetAsync(err, 0, sizeof(unsigned), st);
  int64_t blocks = (n + 255) / 256;
  if (blocks > 4 * (int64_t)sms) blocks = 4 * (int64_t)sms;
  if (blocks > 0) k_fit_sums<<<(unsigned)blocks, 256, smem, st>>>(G, n, src, dst, bytes, tns, (FitSums *)sums, err);
  k_fit_solve<<<(P + 127) / 128, 128, 0, st>>>(G, (const FitSums *)sums, alpha, beta, count);
}
size_t fit_sums_bytes(int G) { return sizeof(FitSums) * (size_t)G * G; }

// ------------------------------------------------ computation cost table
// "execution time of a (sub-)operation on a device, using the operation's
// name and device as the key": per (op, device) entry the sum and
// count of its samples (64-bit integer atomics: exact, order-independent),
// then the mean rounded to the nearest ns, halves up: q + (2r >= cnt).
__global__ void k_cost_sums(int32_t V, int G, int64_t n, const int32_t *op, const uint8_t *dev, const int64_t *tns,
                            u64 *sum, u64 *cnt, unsigned *err) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t o = op[i];
    const int d = dev[i];
    const int64_t t = tns[i];
    if (o < 0 || o >= V || d >= G || t < 0 || t >= (1ll << 40)) {
      atomicOr(err, 1u);
      continue;
    }
    const int64_t e = (int64_t)o * G + d;
    atomicAdd(&sum[e], (u64)t);
    atomicAdd(&cnt[e], 1ull);
  }
}
__global__ void k_cost_final(int64_t ne, const u64 *sum, const u64 *cnt, int64_t *cost) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < ne; e += (int64_t)gridDim.x * blockDim.x) {
    const u64 c = cnt[e], s = sum[e];
    cost[e] = c ? (int64_t)(s / c + (2 * (s % c) >= c ? 1 : 0)) : 0;  // (unknown: 0)
  }
}
void launch_cost_table(int32_t V, int G, int64_t n, const int32_t *op, const uint8_t *dev, const int64_t *tns,
                       void *scratch, unsigned *err, int64_t *cost, int sms, cudaStream_t st) {
  const int64_t ne = (int64_t)V * G;
  u64 *sum = (u64 *)scratch, *cnt = sum + ne;
  cudaMemsetAsync(scratch, 0, sizeof(u64) * 2 * ne, st);
  if (n > 0) {
    const int blocks = (int)std::min<int64_t>((n + 255) / 256, (int64_t)sms * 8);
    k_cost_sums<<<blocks, 256, 0, st>>>(V, G, n, op, dev, tns, sum, cnt, err);
  }
  k_cost_final<<<(int)std::min<int64_t>((ne + 255) / 256, (int64_t)sms * 8), 256, 0, st>>>(ne, sum, cnt, cost);
}

}  // namespace fastt
