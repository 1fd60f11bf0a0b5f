// tp_roof.cu -- the measured INT32 issue roof ("Issue roof = measured INT32
// throughput (bench microbenchmark of SHF/LOP3/IADD at 148 SMs)").  The low-bitwidth decoders
// are bound by integer instruction issue, not by HBM (SURVEY finding 4, App. C.4; the paper's
// DFOR is "bounded by shared memory bandwidth"), so their roofline denominator is
// the rate at which the SMs retire the instructions the decode consists of: funnel shifts
// (SHF), masks (LOP3), adds (IADD3) -- the ALU pipe -- and IMAD on the FMA pipe.
//
// One kernel, every SM full (8 CTAs x 256 threads), 8 independent dependency chains per thread
// (enough ILP to cover the 4-cycle ALU latency), every operation inline PTX whose operands
// change per iteration so ptxas can neither fold nor merge them (checked in the SASS: one SHF /
// LOP3 / IADD3 / IMAD per PTX op).  Three-register forms: 0 SHF, 1 LOP3, 2 IADD3, 3 IMAD,
// 4 SHF+LOP3+IADD3 (ALU pipe), 5 LOP3 / IMAD alternating (ALU + FMA pipes); two-register +
// immediate forms: 6 SHF, 7 LOP3, 8 IMAD, 9 LOP3 / SHF / IMAD mixed over both pipes (the
// per-SMSP issue limit of one warp instruction per cycle).
#include <cuda_runtime.h>

#include <atomic>
#include <cstdint>

#include "tilepack.h"

namespace tp {
extern std::atomic<uint64_t> g_launches;
}

namespace {

constexpr int ROOF_THREADS = 256, ROOF_CTAS_PER_SM = 8, ROOF_CHAINS = 8, ROOF_UNROLL = 16;

__device__ __forceinline__ uint32_t op_shf(uint32_t a, uint32_t b, uint32_t s) {
  uint32_t d;
  asm volatile("shf.r.wrap.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(s));
  return d;
}
__device__ __forceinline__ uint32_t op_lop3(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  return d;
}
// three addends: one IADD3 (a two-operand add may be issued as IMAD on the FMA pipe)
__device__ __forceinline__ uint32_t op_add(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  asm volatile("{\n\t.reg .u32 t;\n\tadd.u32 t, %1, %2;\n\tadd.u32 %0, t, %3;\n\t}" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  return d;
}
// two-register forms (an immediate third operand): the per-SMSP register-read budget
// halves the rate of three-register ALU / FMA instructions (B300_MICROARCH.md: FFMA imm-form
// rt_SMSP = 1 vs 2), and the decoders' shifts and masks mostly take compile-time immediates
__device__ __forceinline__ uint32_t op_shf_imm(uint32_t a, uint32_t b) {
  uint32_t d;
  asm volatile("shf.r.wrap.b32 %0, %1, %2, 7;" : "=r"(d) : "r"(a), "r"(b));
  return d;
}
__device__ __forceinline__ uint32_t op_lop3_imm(uint32_t a, uint32_t b) {
  uint32_t d;
  asm volatile("lop3.b32 %0, %1, %2, 0x0f0f0f0f, 0x6a;" : "=r"(d) : "r"(a), "r"(b));
  return d;
}
__device__ __forceinline__ uint32_t op_mad_imm(uint32_t a, uint32_t b) {
  uint32_t d;
  asm volatile("mad.lo.u32 %0, %1, 0x9E3779B1, %2;" : "=r"(d) : "r"(a), "r"(b));
  return d;
}
__device__ __forceinline__ uint32_t op_mad(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  return d;
}

template <int KIND>
__global__ void __launch_bounds__(ROOF_THREADS) k_int_roof(uint32_t iters, uint32_t seed, uint32_t* sink) {
  uint32_t a[ROOF_CHAINS];
#pragma unroll
  for (int c = 0; c < ROOF_CHAINS; ++c) a[c] = seed * (threadIdx.x + 1u) + (uint32_t)c * 0x9E3779B9u;
  uint32_t k = seed ^ blockIdx.x;
  for (uint32_t it = 0; it < iters; ++it) {
#pragma unroll
    for (int u = 0; u < ROOF_UNROLL; ++u) {
#pragma unroll
      for (int c = 0; c < ROOF_CHAINS; ++c) {
        const uint32_t o = a[(c + 1) % ROOF_CHAINS];  // the previous value of a neighbour chain
        if (KIND == 0) a[c] = op_shf(a[c], o, k);
        else if (KIND == 1) a[c] = op_lop3(a[c], o, k);
        else if (KIND == 2) a[c] = op_add(a[c], o, k);
        else if (KIND == 3) a[c] = op_mad(a[c], o, k);
        else if (KIND == 4) a[c] = (u % 3 == 0) ? op_shf(a[c], o, k) : (u % 3 == 1) ? op_lop3(a[c], o, k) : op_add(a[c], o, k);
        else if (KIND == 5) a[c] = (c & 1) ? op_mad(a[c], o, k) : op_lop3(a[c], o, k);
        else if (KIND == 6) a[c] = op_shf_imm(a[c], o);
        else if (KIND == 7) a[c] = op_lop3_imm(a[c], o);
        else if (KIND == 8) a[c] = op_mad_imm(a[c], o);
        else a[c] = (c & 1) ? op_mad_imm(a[c], o) : (c & 2) ? op_shf_imm(a[c], o) : op_lop3_imm(a[c], o);
      }
    }
    k += 0x61C88647u;
    if (KIND >= 6) a[0] ^= k;  // a loop-carried value in the immediate-form chains
  }
  uint32_t r = 0;
#pragma unroll
  for (int c = 0; c < ROOF_CHAINS; ++c) r ^= a[c];
  if (r == 0x12345678u) sink[0] = r;  // keeps the chains live; practically never stored
}

}  // namespace

extern "C" {

tp_status tp_bench_int_roof(int kind, uint32_t iters, uint32_t* d_sink, uint64_t* warp_insts, void* stream) {
  if (kind < 0 || kind > 9 || !d_sink || !warp_insts || iters == 0) return TP_EINVAL;
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int grid = sms * ROOF_CTAS_PER_SM;
  auto s = (cudaStream_t)stream;
  switch (kind) {
    case 0: k_int_roof<0><<<grid, ROOF_THREADS, 0, s>>>(iters, 12345u, d_sink); break;
    case 1: k_int_roof<1><<<grid, ROOF_THREADS, 0, s>>>(iters, 12345u, d_sink); break;
    case 2: k_int_roof<2><<<grid, ROOF_THREADS, 0, s>>>(iters, 12345u, d_sink); break;
    case 3: k_int_roof<3><<<grid, ROOF_THREADS, 0, s>>>(iters, 12345u, d_sink); break;
    case 4: k_int_roof<4><<<grid, ROOF_THREADS, 0, s>>>(iters, 12345u, d_sink); break;
    case 5: k_int_roof<5><<<grid, ROOF_THREADS, 0, s>>>(iters, 12345u, d_sink); break;
    case 6: k_int_roof<6><<<grid, ROOF_THREADS, 0, s>>>(iters, 12345u, d_sink); break;
    case 7: k_int_roof<7><<<grid, ROOF_THREADS, 0, s>>>(iters, 12345u, d_sink); break;
    case 8: k_int_roof<8><<<grid, ROOF_THREADS, 0, s>>>(iters, 12345u, d_sink); break;
    default: k_int_roof<9><<<grid, ROOF_THREADS, 0, s>>>(iters, 12345u, d_sink); break;
  }
  tp::g_launches.fetch_add(1, std::memory_order_relaxed);
  *warp_insts = (uint64_t)grid * (ROOF_THREADS / 32) * iters * ROOF_UNROLL * ROOF_CHAINS;
  return cudaGetLastError() == cudaSuccess ? TP_OK : TP_ECUDA;
}

}  // extern "C"
