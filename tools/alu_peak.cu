// alu_peak.cu -- measured int32 throughput of the SM pipes the lane kernel
// issues on (B200, sm_100a): the roofline denominator of bench.py's "alu"
// bound.  Each kernel runs 8 independent dependency chains per thread, 16
// warps per SM on every SM, and reports SASS lane-instructions per second
// (CUDA events, best of 5).  ptxas fuses chains of one op into 3-input
// forms (IADD3 / VIMNMX3 do two ops), so every chain alternates two op kinds
// that have no fused form -- one SASS instruction per PTX op (checked with
// cuobjdump -sass: 512 + 512 per kernel body):
//   minxor : min.u32 + xor.b32    (VIMNMX + LOP3: both on the ALU pipe)
//   addxor : add.u32 + xor.b32    (ptxas emits IMAD.IADD on the FMA pipe + LOP3)
//   madxor : mad.lo.u32 + xor.b32 (IMAD on the FMA pipe + LOP3 on the ALU pipe)
// alu_pipe_tops = minxor (the integer ALU pipe alone); issue_tops = the best
// mixed ALU + FMA rate (the warp-issue limit, one instruction per SMSP per clock).
// Build & run: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o alu_peak alu_peak.cu && ./alu_peak
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int ITERS = 4096;
constexpr int CH = 8;

template <int KIND>
__global__ void __launch_bounds__(512) k_pipe(uint32_t *out, uint32_t seed) {
  uint32_t a[CH], b = seed ^ threadIdx.x, c = seed * 3u + blockIdx.x;
#pragma unroll
  for (int j = 0; j < CH; j++) a[j] = seed + j * 7u + threadIdx.x;
  for (int it = 0; it < ITERS; it++) {
#pragma unroll
    for (int j = 0; j < CH; j++) {
      if (KIND == 0) asm volatile("{ min.u32 %0, %0, %1; xor.b32 %0, %0, %2; }" : "+r"(a[j]) : "r"(b), "r"(c));
      if (KIND == 1) asm volatile("{ add.u32 %0, %0, %1; xor.b32 %0, %0, %2; }" : "+r"(a[j]) : "r"(b), "r"(c));
      if (KIND == 2) asm volatile("{ mad.lo.u32 %0, %0, %1, %2; xor.b32 %0, %0, %1; }" : "+r"(a[j]) : "r"(b), "r"(c));
    }
  }
  uint32_t s = 0;
#pragma unroll
  for (int j = 0; j < CH; j++) s ^= a[j];
  if (s == 0x12345678u) out[0] = s;  // keep the chains alive
}

template <int KIND> static double run(int sms, int ops_per_inst) {
  uint32_t *out;
  cudaMalloc(&out, 4);
  const int block = 512, grid = sms;  // 16 warps per SM
  k_pipe<KIND><<<grid, block>>>(out, 1);
  cudaDeviceSynchronize();
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  double best = 0;
  for (int r = 0; r < 5; r++) {
    cudaEventRecord(e0);
    for (int k = 0; k < 10; k++) k_pipe<KIND><<<grid, block>>>(out, 1 + k);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    const double lane_ops = 10.0 * grid * block * (double)ITERS * CH * ops_per_inst;
    const double v = lane_ops / (ms / 1000.0);
    best = v > best ? v : best;
  }
  cudaFree(out);
  return best;
}

int main() {
  cudaDeviceProp p;
  cudaGetDeviceProperties(&p, 0);
  const int sms = p.multiProcessorCount;
  const double mx = run<0>(sms, 2), ax = run<1>(sms, 2), fx = run<2>(sms, 2);
  int clk_khz = 0;
  cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
  printf("{\"gpu\": \"%s\", \"sms\": %d, \"warps_per_sm\": 16, \"chains_per_thread\": %d, "
         "\"unit\": \"T lane-instructions/s\", \"minxor\": %.4f, \"addxor\": %.4f, \"madxor\": %.4f, "
         "\"alu_pipe_tops\": %.4f, \"issue_tops\": %.4f, \"rated_clock_mhz\": %.1f}\n",
         p.name, sms, CH, mx / 1e12, ax / 1e12, fx / 1e12, mx / 1e12, (ax > fx ? ax : fx) / 1e12, clk_khz / 1000.0);
  return 0;
}
