// tp_cascaded.cu -- the CASCADING decompression baseline of the paper (P:462-549,
// P:1403-1417): the same GPU-FOR / GPU-DFOR / GPU-RFOR bytes, decoded one layer at a time,
// every layer a separate kernel that reads its input from and writes its output to global
// memory (the ablation behind "tile-based decompression is 2.6x / 4x / 8x
// faster").  Not a hot path: it exists to be measured against tp_decode.
//
//   FOR+BitPack        (2 passes): unpack bits -> add reference
//   Delta+FOR+BitPack  (3 passes): unpack bits -> add reference -> per-tile prefix sum
//   RLE+FOR+BitPack    (8 passes): unpack values -> add reference -> unpack run lengths ->
//                                  add reference -> scan lengths -> scatter run marks ->
//                                  scan marks -> gather values   (+1 zero fill of the marks)
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstring>

#include "tilepack.h"

namespace tp {
extern std::atomic<uint64_t> g_launches;
// tile-pipeline decode -> global (tp_kernels.cu); raw: packed offsets of FOR / DFOR blocks
tp_status decode_global_impl(const tp_column* dcol, int32_t* d_out, bool raw, void* stream);
}

namespace tpc {

constexpr unsigned FULL = 0xffffffffu;

// bitwidth byte j of the bitwidth words at w (R2); word offset of miniblock j when every
// earlier miniblock is full (32 entries at b_i bits = b_i words)
__device__ __forceinline__ uint32_t bw_byte(const uint32_t* w, uint32_t j) {
  return min((w[j >> 2] >> (8u * (j & 3u))) & 255u, 32u);
}
__device__ __forceinline__ uint32_t mb_offset(const uint32_t* w, uint32_t j) {  // sum of bytes [0, j)
  uint32_t off = 0;
  for (uint32_t q = 0; q < (j >> 2); ++q) off += (w[q] * 0x01010101u) >> 24;
  const uint32_t low = w[j >> 2] & ((1u << (8u * (j & 3u))) - 1u);
  return off + ((low * 0x01010101u) >> 24);
}
__device__ __forceinline__ uint32_t field(const uint32_t* mb, uint32_t idx, uint32_t b) {
  const uint32_t p = idx * b;
  const uint64_t win = (uint64_t)mb[p >> 5] | ((uint64_t)mb[(p >> 5) + 1] << 32);  // Alg. 1 line 15
  return (uint32_t)((win >> (p & 31u)) & ((b >= 32) ? 0xffffffffull : ((1ull << b) - 1)));
}

// pass "unpack bit-packing" of 128-entry FOR blocks: E[i] = packed offset of slot i
__global__ void k_unpack_blocks(const uint32_t* __restrict__ starts, const uint32_t* __restrict__ data,
                                uint64_t nslots, uint32_t* __restrict__ E) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nslots;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t* blk = data + starts[i >> 7];
    const uint32_t j = (uint32_t)(i >> 5) & 3u;
    E[i] = field(blk + 2 + mb_offset(blk + 1, j), (uint32_t)i & 31u, bw_byte(blk + 1, j));
  }
}
// pass "add the frame of reference": X[i] = E[i] + ref(block of i); 16-byte vector accesses,
// the reference read once per 4 values (n4 = n rounded down to 4; the tail is done by thread 0)
__global__ void k_add_ref_blocks(const uint32_t* __restrict__ starts, const uint32_t* __restrict__ data,
                                 const uint32_t* __restrict__ E, uint64_t n, uint32_t* __restrict__ X) {
  const uint64_t n4 = n >> 2;
  for (uint64_t q = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; q < n4; q += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t ref = data[starts[q >> 5]];  // 4 values never straddle a 128-value block
    uint4 v = reinterpret_cast<const uint4*>(E)[q];
    v.x += ref; v.y += ref; v.z += ref; v.w += ref;
    reinterpret_cast<uint4*>(X)[q] = v;
  }
  if (blockIdx.x == 0 && threadIdx.x < (n & 3)) {
    const uint64_t i = (n & ~uint64_t(3)) + threadIdx.x;
    X[i] = E[i] + data[starts[i >> 7]];
  }
}
// DFOR pass "delta decode": one warp per 512-slot tile, coalesced chunks of 32 slots, warp scan
__global__ void k_tile_prefix(const uint32_t* __restrict__ starts, const uint32_t* __restrict__ data,
                              const uint32_t* __restrict__ D, uint64_t n, uint64_t ntiles, int32_t* __restrict__ out) {
  const uint32_t lane = threadIdx.x & 31u;
  for (uint64_t t = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; t < ntiles;
       t += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    uint32_t carry = data[starts[4 * t] - 1];  // the tile's first value
    for (uint32_t k = 0; k < 16; ++k) {
      const uint64_t s = 512 * t + 32 * k + lane;
      const uint32_t d = s < n ? D[s] : 0u;  // slots >= n only feed rows >= n
      uint32_t incl = d;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, incl, o);
        if (lane >= (uint32_t)o) incl += y;
      }
      if (s < n) out[s] = (int32_t)(carry + incl - d);
      carry += __shfl_sync(FULL, incl, 31);
    }
  }
}
// RFOR stream pass "unpack": E[512k + i] = packed entry i of stream block k (i < r_k)
__global__ void k_unpack_stream(const uint32_t* __restrict__ starts, const uint32_t* __restrict__ data,
                                uint64_t nrb, uint32_t* __restrict__ E) {
  for (uint64_t s = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; s < 512 * nrb;
       s += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t* blk = data + starts[s >> 9];
    const uint32_t i = (uint32_t)s & 511u, r = blk[0];
    if (i < r) {
      const uint32_t j = i >> 5;
      E[s] = field(blk + 6 + mb_offset(blk + 2, j), i & 31u, bw_byte(blk + 2, j));
    }
  }
}
// RFOR stream pass "add reference"
__global__ void k_add_ref_stream(const uint32_t* __restrict__ starts, const uint32_t* __restrict__ data,
                                 uint64_t nrb, uint32_t* __restrict__ E) {
  for (uint64_t s = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; s < 512 * nrb;
       s += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t* blk = data + starts[s >> 9];
    if (((uint32_t)s & 511u) < blk[0]) E[s] += blk[1];
  }
}
// RLE pass 1 (scan): S[512k + i] = exclusive prefix of the run lengths of block k
__global__ void k_scan_lengths(const uint32_t* __restrict__ startsL, const uint32_t* __restrict__ dataL,
                               const uint32_t* __restrict__ L, uint64_t nrb, uint32_t* __restrict__ S) {
  const uint32_t lane = threadIdx.x & 31u;
  for (uint64_t k = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; k < nrb;
       k += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    const uint32_t r = dataL[startsL[k]];
    uint32_t carry = 0;
    for (uint32_t q = 0; 32 * q < r; ++q) {
      const uint32_t i = 32 * q + lane;
      const uint32_t l = i < r ? L[512 * k + i] : 0u;
      uint32_t incl = l;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, incl, o);
        if (lane >= (uint32_t)o) incl += y;
      }
      if (i < r) S[512 * k + i] = carry + incl - l;
      carry += __shfl_sync(FULL, incl, 31);
    }
  }
}
// RLE pass 2 (scatter): M[512k + S_i] = i + 1
__global__ void k_scatter_marks(const uint32_t* __restrict__ startsL, const uint32_t* __restrict__ dataL,
                                const uint32_t* __restrict__ S, uint64_t nrb, uint32_t* __restrict__ M) {
  for (uint64_t s = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; s < 512 * nrb;
       s += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t k = s >> 9;
    const uint32_t i = (uint32_t)s & 511u;
    if (i < dataL[startsL[k]]) M[512 * k + S[s]] = i + 1;
  }
}
// RLE pass 3 (scan): inclusive max-scan of the marks -> run index of every row (in place)
__global__ void k_scan_marks(uint64_t nrb, uint32_t* __restrict__ M) {
  const uint32_t lane = threadIdx.x & 31u;
  for (uint64_t k = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; k < nrb;
       k += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    uint32_t carry = 0;
    for (uint32_t q = 0; q < 16; ++q) {
      uint32_t incl = M[512 * k + 32 * q + lane];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, incl, o);
        if (lane >= (uint32_t)o) incl = max(incl, y);
      }
      incl = max(incl, carry);
      M[512 * k + 32 * q + lane] = incl;
      carry = __shfl_sync(FULL, incl, 31);
    }
  }
}
// RLE pass 4 (gather): out[row] = V[run index of row]
__global__ void k_gather(const uint32_t* __restrict__ V, const uint32_t* __restrict__ M, uint64_t n,
                         int32_t* __restrict__ out) {
  for (uint64_t row = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; row < n;
       row += (uint64_t)gridDim.x * blockDim.x)
    out[row] = (int32_t)V[(row & ~uint64_t(511)) + M[row] - 1];
}

static int grid() {
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (sms <= 0) sms = 148;
  }
  return sms * 8;
}

static tp_status done(int launches) {
  tp::g_launches.fetch_add(launches);
  return cudaGetLastError() == cudaSuccess ? TP_OK : TP_ECUDA;
}

}  // namespace tpc

using namespace tpc;

extern "C" {

uint64_t tp_cascaded_workspace_words(const tp_column* c) {
  if (!c) return 0;
  if (c->scheme == TP_RFOR) return 4 * 512 * c->num_blocks;  // values, lengths, starts, marks
  return 128 * c->num_blocks;                                 // unpacked offsets / deltas
}

tp_status tp_decode_cascaded(const tp_column* c, int32_t* d_out, uint32_t* d_work, void* stream) {
  if (!c || !d_out || !d_work || c->scheme == TP_FORNM || c->scheme == TP_NONE) return TP_EINVAL;
  if (c->n == 0) return TP_OK;
  if (c->n >= (1ull << 32)) return TP_EUNSUPPORTED;
  cudaStream_t s = (cudaStream_t)stream;
  const int G = grid();
  const uint64_t nb = c->num_blocks, n = c->n;
  uint32_t* out = reinterpret_cast<uint32_t*>(d_out);
  // the bit-unpacking pass is the optimised tile decoder itself, writing the packed offsets
  // (no reference) to global memory: the cascade then pays only for its extra layers
  if (c->scheme == TP_FOR) {
    tp_status st = tp::decode_global_impl(c, reinterpret_cast<int32_t*>(d_work), true, stream);
    if (st != TP_OK) return st;
    k_add_ref_blocks<<<G, 256, 0, s>>>(c->starts0, c->data0, d_work, n, out);
    return done(1);
  }
  if (c->scheme == TP_DFOR) {
    tp_status st = tp::decode_global_impl(c, reinterpret_cast<int32_t*>(d_work), true, stream);
    if (st != TP_OK) return st;
    k_add_ref_blocks<<<G, 256, 0, s>>>(c->starts0, c->data0, d_work, n, d_work);
    k_tile_prefix<<<G, 256, 0, s>>>(c->starts0, c->data0, d_work, n, (n + 511) / 512, d_out);
    return done(2);
  }
  if (c->scheme != TP_RFOR) return TP_EINVAL;
  uint32_t* V = d_work;
  uint32_t* L = V + 512 * nb;
  uint32_t* S = L + 512 * nb;
  uint32_t* M = S + 512 * nb;
  k_unpack_stream<<<G, 256, 0, s>>>(c->starts0, c->data0, nb, V);
  k_add_ref_stream<<<G, 256, 0, s>>>(c->starts0, c->data0, nb, V);
  k_unpack_stream<<<G, 256, 0, s>>>(c->starts1, c->data1, nb, L);
  k_add_ref_stream<<<G, 256, 0, s>>>(c->starts1, c->data1, nb, L);
  k_scan_lengths<<<G, 256, 0, s>>>(c->starts1, c->data1, L, nb, S);
  cudaMemsetAsync(M, 0, 512 * nb * sizeof(uint32_t), s);
  k_scatter_marks<<<G, 256, 0, s>>>(c->starts1, c->data1, S, nb, M);
  k_scan_marks<<<G, 256, 0, s>>>(nb, M);
  k_gather<<<G, 256, 0, s>>>(V, M, n, d_out);
  return done(8);
}

}  // extern "C"
