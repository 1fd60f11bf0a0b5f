// tp_encode.cu -- the tile-parallel GPU encoder: GPU-FOR, GPU-DFOR,
// GPU-RFOR and the GPU-* scheme choice computed from a DEVICE column, byte-identical to the
// host encoder (tp_host.cpp) and to the oracle (readings R1-R20).
//
// The paper encodes on the CPU once (250M values in 1.2 / 1.3 / 2.2 s on 6 vCPUs);
// every 512-row tile is encoded independently, so the only
// cross-tile dependency is the word offset of each tile in the output -- an exclusive prefix
// sum of tile sizes.  One pass over HBM:
//   * persistent CTAs of 8 warps take 8-tile chunks (4096 rows) in order from an atomic
//     counter; warp w loads tile w of the chunk (coalesced 16-byte loads) into shared memory;
//   * the warp plans its tile: FOR blocks of 128 (ref = signed min, R4; per-miniblock
//     bitwidth = bit length of the OR of the offsets, == bit length of the max, R3; neutral
//     pads, R8), DFOR delta slots (R12, R13: slot s = x[s+1] - x[s], pads neutral), RFOR runs
//     (R17, R18: values / lengths of the maximal runs inside the 512-row block, each stream
//     FOR-packed into 16 tight miniblocks of 32 entries);
//   * the chunk's word count is published and its base offset found by a decoupled look-back
//     over the preceding chunks' status words (single-pass scan; no second read of the input);
//   * the warp writes block_starts, headers and the packed words: lane t builds output word t
//     from the <= ceil(32/b)+1 entries whose bits fall into it (LSB-first, R1), so the stores
//     are coalesced and need no atomics.
// A "sizes" instantiation runs the three plans on each tile and only accumulates the stream
// word counts (GPU-*: P:1206-1217, ties FOR < DFOR < RFOR, R20).
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <climits>
#include <cstring>

#include "tilepack.h"
#include "tp_device.cuh"

namespace tp {
extern std::atomic<uint64_t> g_launches;
}

namespace tp {
namespace enc {

constexpr int EW = 8;                                  // warps per CTA = tiles per chunk
constexpr int ETHREADS = 32 * EW;
constexpr uint32_t CHUNK_ROWS = EW * TILE_ROWS;        // 4096 rows per chunk
constexpr uint64_t ST_AGG = 1ull << 62, ST_INC = 2ull << 62, ST_VAL = (1ull << 62) - 1;
constexpr int MODE_SIZES = 0;                          // SCHEME template value: all three plans, counts only

// workspace (u64 words): [0] chunk counter, [1..2] stream totals, [3..4] max tile words,
// [5] overflow flag, [6..9] sizes mode: FOR, DFOR, RFOR values, RFOR lengths; then the
// look-back status words, two per chunk (stream 0, stream 1)
constexpr int W_CTR = 0, W_TOT = 1, W_MTW = 3, W_OVF = 5, W_SIZES = 6, W_STATUS = 16;

// per-warp plan of one stream of the current tile
struct Plan {
  int32_t ref[4];     // FOR / DFOR: per block; RFOR: [0]
  uint32_t b[16];     // bitwidth of each miniblock (0 for absent ones)
  uint32_t off[17];   // exclusive prefix of the miniblocks' data words; off[16] = total
  uint32_t cnt[16];   // entries per miniblock (RFOR; FOR / DFOR: valid entries)
  uint32_t words;     // the tile's words in this stream
};
struct WarpHdr {
  Plan p[2];
  uint32_t r;         // RFOR run count
  uint32_t m;         // rows of the tile
};
// per-warp arrays (words): X (values), then DFOR deltas / RFOR V, S, L
template <int SCHEME>
__host__ __device__ constexpr int n_arrays() { return SCHEME == TP_FOR ? 1 : SCHEME == TP_DFOR ? 2 : 4; }
constexpr uint32_t HDR_WORDS = (sizeof(WarpHdr) + 15) / 16 * 4;

__device__ __forceinline__ uint32_t bitlen(uint32_t u) { return u ? 32u - __clz(u) : 0u; }

// exclusive prefix of x over lanes 0..15 (lanes 16..31 get garbage); total in *tot
__device__ __forceinline__ uint32_t excl16(uint32_t x, uint32_t lane, uint32_t* tot) {
  uint32_t s = x;
#pragma unroll
  for (int d = 1; d < 16; d <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, s, d);
    if ((lane & 15u) >= (uint32_t)d) s += y;
  }
  *tot = __shfl_sync(FULL, s, 15);
  return s - x;
}

// FOR-plan the nblk blocks of 128 slots of src (slots >= nvalid are neutral pads, R8 / R13)
__device__ void plan_for_blocks(const int32_t* src, uint32_t nvalid, uint32_t nblk, Plan& P, uint32_t lane,
                                uint32_t extra_words) {
#pragma unroll 1
  for (uint32_t k = 0; k < nblk; ++k) {
    const uint32_t s0 = 128u * k + 4u * lane;
    const int4 q = *reinterpret_cast<const int4*>(src + s0);
    const int32_t v[4] = {q.x, q.y, q.z, q.w};
    int32_t mn = INT_MAX;
#pragma unroll
    for (int j = 0; j < 4; ++j)
      if (s0 + j < nvalid) mn = min(mn, v[j]);
    mn = __reduce_min_sync(FULL, mn);
    const int32_t ref = 128u * k < nvalid ? mn : 0;  // a block of pads only: ref 0 (R14)
    uint32_t o = 0u;
#pragma unroll
    for (int j = 0; j < 4; ++j)
      if (s0 + j < nvalid) o |= (uint32_t)v[j] - (uint32_t)ref;  // offsets mod 2^32 (R4)
    o |= __shfl_xor_sync(FULL, o, 1);
    o |= __shfl_xor_sync(FULL, o, 2);
    o |= __shfl_xor_sync(FULL, o, 4);
    if ((lane & 7u) == 0) {
      const uint32_t j = 4u * k + (lane >> 3);
      P.b[j] = bitlen(o);  // bit length of the OR == bit length of the max (R3)
      const uint32_t lo = 32u * j;
      P.cnt[j] = nvalid > lo ? min(32u, nvalid - lo) : 0u;
    }
    if (lane == 0) P.ref[k] = ref;
  }
  __syncwarp();
  const uint32_t bj = lane < 16 && (lane >> 2) < nblk ? P.b[lane] : 0u;
  uint32_t tot;
  const uint32_t ex = excl16(bj, lane, &tot);  // full miniblocks: b words each
  if (lane < 16) {
    P.off[lane] = ex;
    if (lane >= 4 * nblk) { P.b[lane] = 0u; P.cnt[lane] = 0u; }
  }
  if (lane == 0) {
    P.off[16] = tot;
    P.words = extra_words + 2u * nblk + tot;
  }
  __syncwarp();
}

// FOR-plan one RFOR stream block of r entries (16 tight miniblocks of 32, R17)
__device__ void plan_rfor_stream(const int32_t* src, uint32_t r, Plan& P, uint32_t lane) {
  int32_t mn = INT_MAX;
  for (uint32_t i = lane; i < r; i += 32) mn = min(mn, src[i]);
  mn = __reduce_min_sync(FULL, mn);
  const int32_t ref = mn;
  uint32_t my_b = 0u;
#pragma unroll 1
  for (uint32_t q = 0; q < 16; ++q) {
    if (32u * q >= r) break;  // warp-uniform
    const uint32_t i = 32u * q + lane;
    const uint32_t u = i < r ? (uint32_t)src[i] - (uint32_t)ref : 0u;
    const uint32_t o = __reduce_or_sync(FULL, u);
    if (lane == q) my_b = bitlen(o);
  }
  const uint32_t cnt = lane < 16 ? (r > 32u * lane ? min(32u, r - 32u * lane) : 0u) : 0u;
  const uint32_t wq = (cnt * my_b + 31u) >> 5;  // tight: ceil(cnt * b / 32) words
  uint32_t tot;
  const uint32_t ex = excl16(wq, lane, &tot);
  if (lane < 16) {
    P.b[lane] = my_b;
    P.cnt[lane] = cnt;
    P.off[lane] = ex;
  }
  if (lane == 0) {
    P.ref[0] = ref;
    P.off[16] = tot;
    P.words = 6u + tot;
  }
  __syncwarp();
}

// runs of the tile (R18): V[idx] = value, S[idx] = start row, L[idx] = length; returns r
__device__ uint32_t find_runs(const int32_t* X, uint32_t m, int32_t* V, int32_t* S, int32_t* L, uint32_t lane) {
  uint32_t base = 0u;
  const uint32_t lt = (1u << lane) - 1u;
#pragma unroll 1
  for (uint32_t q = 0; q < 16; ++q) {
    if (32u * q >= m) break;
    const uint32_t row = 32u * q + lane;
    const bool f = row < m && (row == 0 || X[row] != X[row - 1]);
    const uint32_t bal = __ballot_sync(FULL, f);
    if (f) {
      const uint32_t idx = base + __popc(bal & lt);
      V[idx] = X[row];
      S[idx] = (int32_t)row;
    }
    base += __popc(bal);
  }
  __syncwarp();
  for (uint32_t i = lane; i < base; i += 32) L[i] = (i + 1 < base ? S[i + 1] : (int32_t)m) - S[i];
  __syncwarp();
  return base;
}

// output word w of miniblock j (entries src[0..cnt), bitwidth b, reference ref): the OR of
// every entry whose bit range [i b, i b + b) meets [32 w, 32 w + 32) (R1)
__device__ __forceinline__ uint32_t pack_word(const int32_t* src, uint32_t cnt, uint32_t b, uint32_t w,
                                              int32_t ref) {
  const uint32_t bit0 = 32u * w;
  uint32_t i = bit0 / b;
  const uint32_t iend = min(cnt, (bit0 + 31u) / b + 1u);
  uint32_t word = 0u;
  for (; i < iend; ++i) {
    const uint32_t u = (uint32_t)src[i] - (uint32_t)ref;
    const int p = (int)(i * b) - (int)bit0;
    word |= p >= 0 ? (u << p) : (u >> (-p));
  }
  return word;
}

// last miniblock j with off[j] <= t (t < off[16]): its data holds word t
__device__ __forceinline__ uint32_t find_mb(const uint32_t* off, uint32_t t) {
  uint32_t lo = 0;
#pragma unroll
  for (uint32_t step = 8; step > 0; step >>= 1)
    if (off[lo + step] <= t) lo += step;
  return lo;
}

// write one tile's FOR / DFOR blocks (data base B, first block index blk0)
__device__ void write_for_tile(const int32_t* src, const Plan& P, uint32_t nblk, bool dfor, int32_t first,
                               uint64_t B, uint64_t blk0, uint32_t* starts, uint32_t* data, uint32_t lane) {
  const uint64_t d0 = B + (dfor ? 1u : 0u);
  if (dfor && lane == 0) data[B] = (uint32_t)first;  // first value of the tile
  if (lane < nblk) {
    const uint64_t bs = d0 + 2u * lane + P.off[4 * lane];
    starts[blk0 + lane] = (uint32_t)bs;
    data[bs] = (uint32_t)P.ref[lane];
    data[bs + 1] = P.b[4 * lane] | P.b[4 * lane + 1] << 8 | P.b[4 * lane + 2] << 16 | P.b[4 * lane + 3] << 24;
  }
  const uint32_t tot = P.off[16];
  for (uint32_t t = lane; t < tot; t += 32) {
    const uint32_t j = find_mb(P.off, t);
    const uint32_t k = j >> 2;
    data[d0 + 2u * (k + 1u) + t] = pack_word(src + 32u * j, P.cnt[j], P.b[j], t - P.off[j], P.ref[k]);
  }
}

// write one RFOR stream block at B
__device__ void write_rfor_stream(const int32_t* src, const Plan& P, uint32_t r, uint64_t B, uint64_t blk,
                                  uint32_t* starts, uint32_t* data, uint32_t lane) {
  if (lane == 0) {
    starts[blk] = (uint32_t)B;
    data[B] = r;
    data[B + 1] = (uint32_t)P.ref[0];
  }
  if (lane >= 2 && lane < 6) {
    const uint32_t q = lane - 2;
    data[B + lane] = P.b[4 * q] | P.b[4 * q + 1] << 8 | P.b[4 * q + 2] << 16 | P.b[4 * q + 3] << 24;
  }
  const uint32_t tot = P.off[16];
  for (uint32_t t = lane; t < tot; t += 32) {
    const uint32_t j = find_mb(P.off, t);
    data[B + 6u + t] = pack_word(src + 32u * j, P.cnt[j], P.b[j], t - P.off[j], P.ref[0]);
  }
}

// ---- decoupled look-back (stream s): exclusive prefix of chunk c's words
__device__ __forceinline__ uint64_t ld_status(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_status(unsigned long long* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ uint64_t look_back(unsigned long long* status, uint32_t c, uint64_t agg, uint32_t lane) {
  if (c == 0) {
    if (lane == 0) st_status(status, ST_INC | agg);
    return 0;
  }
  if (lane == 0) st_status(status + c, ST_AGG | agg);
  uint64_t excl = 0;
  int64_t pos = (int64_t)c - 1;  // highest chunk of the window
  while (true) {
    const int64_t i = pos - (int64_t)lane;
    uint64_t v = i >= 0 ? ld_status(status + i) : ST_INC;  // before chunk 0: prefix 0
    while (__any_sync(FULL, (v >> 62) == 0)) {
      if ((v >> 62) == 0) {
        __nanosleep(32);
        v = ld_status(status + i);
      }
    }
    const uint32_t inc = __ballot_sync(FULL, (v >> 62) == 2);
    const uint32_t stop = inc ? __ffs(inc) - 1 : 32u;  // nearest chunk with an inclusive prefix
    uint64_t x = lane <= stop ? (v & ST_VAL) : 0;
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) x += __shfl_xor_sync(FULL, x, d);
    excl += x;
    if (inc) break;
    pos -= 32;
  }
  if (lane == 0) st_status(status + c, ST_INC | (excl + agg));
  return excl;
}

// ------------------------------------------------------------------ the kernel
template <int SCHEME>
struct EncArgs {
  const int32_t* x;
  uint32_t n, ntiles, nchunks, nblocks;  // nblocks: block_starts entries - 1 (stream 0)
  uint32_t* starts0;
  uint32_t* data0;
  uint32_t* starts1;
  uint32_t* data1;
  uint64_t cap0, cap1;        // data capacity (words, without guards)
  unsigned long long* work;
};

template <int SCHEME>
__global__ void __launch_bounds__(ETHREADS) k_encode(const __grid_constant__ EncArgs<SCHEME> A) {
  extern __shared__ __align__(16) uint32_t esm[];
  constexpr bool SIZES = SCHEME == MODE_SIZES;
  constexpr int NA = SIZES ? 4 : n_arrays<SCHEME>();
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31u;
  __shared__ uint32_t s_chunk;
  __shared__ uint32_t s_words[2][EW];
  __shared__ unsigned long long s_base[2], s_agg[2];
  WarpHdr& H = *reinterpret_cast<WarpHdr*>(esm + warp * (HDR_WORDS + NA * 512u));
  int32_t* X = reinterpret_cast<int32_t*>(esm + warp * (HDR_WORDS + NA * 512u) + HDR_WORDS);
  int32_t* A1 = X + 512;  // DFOR deltas / RFOR values
  int32_t* A2 = X + 1024; // RFOR run starts
  int32_t* A3 = X + 1536; // RFOR run lengths
  unsigned long long* work = A.work;

  while (true) {
    if (threadIdx.x == 0) s_chunk = (uint32_t)atomicAdd(work + W_CTR, 1ull);
    __syncthreads();
    const uint32_t c = s_chunk;
    if (c >= A.nchunks) break;
    const uint32_t t = c * EW + warp;  // this warp's tile
    const bool has = t < A.ntiles;
    const uint32_t r0 = t * TILE_ROWS;
    const uint32_t m = has ? min((uint32_t)TILE_ROWS, A.n - r0) : 0u;
    uint32_t w0 = 0u, w1 = 0u, wf = 0u, wd = 0u, wv = 0u, wl = 0u;
    if (has) {
      // ---- stage the tile (coalesced 16-byte loads; the tail row by row)
      if (m == TILE_ROWS) {
        const int4* src = reinterpret_cast<const int4*>(A.x + r0);
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const int4 q = __ldcs(src + 32 * k + lane);
          *reinterpret_cast<int4*>(X + 128 * k + 4 * lane) = q;
        }
      } else {
        for (uint32_t i = lane; i < TILE_ROWS; i += 32) X[i] = i < m ? __ldcs(A.x + r0 + i) : 0;
      }
      __syncwarp();
      const uint32_t nblk = (m + 127u) >> 7;
      if (SIZES || SCHEME == TP_FOR) {
        plan_for_blocks(X, m, nblk, H.p[0], lane, 0u);
        wf = H.p[0].words;
      }
      if (SIZES || SCHEME == TP_DFOR) {
        for (uint32_t s = lane; s < TILE_ROWS; s += 32)  // delta slots (R12, R13)
          A1[s] = s + 1 < m ? (int32_t)((uint32_t)X[s + 1] - (uint32_t)X[s]) : 0;
        __syncwarp();
        plan_for_blocks(A1, m - 1u, nblk, H.p[0], lane, 1u);
        wd = H.p[0].words;
      }
      if (SIZES || SCHEME == TP_RFOR) {
        const uint32_t r = find_runs(X, m, A1, A2, A3, lane);
        if (lane == 0) H.r = r;
        plan_rfor_stream(A1, r, H.p[0], lane);
        plan_rfor_stream(A3, r, H.p[1], lane);
        wv = H.p[0].words;
        wl = H.p[1].words;
      }
      w0 = SCHEME == TP_FOR ? wf : SCHEME == TP_DFOR ? wd : wv;
      w1 = SCHEME == TP_RFOR ? wl : 0u;
    }
    if (SIZES) {
      // counts only: one atomic per warp and scheme stream
      if (lane == 0 && has) {
        atomicAdd(work + W_SIZES + 0, (unsigned long long)wf);
        atomicAdd(work + W_SIZES + 1, (unsigned long long)wd);
        atomicAdd(work + W_SIZES + 2, (unsigned long long)wv);
        atomicAdd(work + W_SIZES + 3, (unsigned long long)wl);
      }
      __syncthreads();
      continue;
    }
    if (lane == 0) {
      s_words[0][warp] = w0;
      s_words[1][warp] = w1;
    }
    if (SCHEME != TP_RFOR && threadIdx.x == 0) s_base[1] = s_agg[1] = 0;
    __syncthreads();
    // ---- chunk offsets: warp 0 (stream 0) and warp 1 (stream 1, RFOR) look back
    constexpr int NS = SCHEME == TP_RFOR ? 2 : 1;
    if (warp < NS) {
      const uint32_t mine = lane < EW ? s_words[warp][lane] : 0u;
      uint64_t agg = mine, mx = mine;
#pragma unroll
      for (int d = 16; d > 0; d >>= 1) {
        agg += __shfl_xor_sync(FULL, agg, d);
        mx = max(mx, (uint64_t)__shfl_xor_sync(FULL, (uint32_t)mx, d));
      }
      const uint64_t base = look_back(work + W_STATUS + (uint64_t)warp * A.nchunks, c, agg, lane);
      if (lane == 0) {
        s_base[warp] = base;
        s_agg[warp] = agg;
        atomicMax(work + W_MTW + warp, (unsigned long long)mx);
        const uint64_t cap = warp == 0 ? A.cap0 : A.cap1;
        if (base + agg > cap) atomicOr(work + W_OVF, 1ull);
        if (c == A.nchunks - 1) work[W_TOT + warp] = base + agg;
      }
    }
    __syncthreads();
    // ---- write: block_starts, headers, packed words
    const bool ovf = s_base[0] + s_agg[0] > A.cap0 || (SCHEME == TP_RFOR && s_base[1] + s_agg[1] > A.cap1);
    if (has && !ovf) {
      uint64_t B0 = s_base[0], B1 = s_base[1];
      for (uint32_t w = 0; w < warp; ++w) {
        B0 += s_words[0][w];
        B1 += s_words[1][w];
      }
      const uint32_t nblk = (m + 127u) >> 7;
      if (SCHEME == TP_FOR) {
        write_for_tile(X, H.p[0], nblk, false, 0, B0, 4ull * t, A.starts0, A.data0, lane);
      } else if (SCHEME == TP_DFOR) {
        write_for_tile(A1, H.p[0], nblk, true, X[0], B0, 4ull * t, A.starts0, A.data0, lane);
      } else {
        write_rfor_stream(A1, H.p[0], H.r, B0, t, A.starts0, A.data0, lane);
        write_rfor_stream(A3, H.p[1], H.r, B1, t, A.starts1, A.data1, lane);
      }
      if (t == A.ntiles - 1) {  // the column's end: last block_starts entry + zero guards (R6, R9)
        const uint64_t e0 = B0 + w0, e1 = B1 + w1;
        if (lane < TP_GUARD_WORDS) {
          A.data0[e0 + lane] = 0u;
          A.starts0[A.nblocks + 1 + lane] = 0u;
          if (SCHEME == TP_RFOR) {
            A.data1[e1 + lane] = 0u;
            A.starts1[A.nblocks + 1 + lane] = 0u;
          }
        }
        if (lane == 0) {
          A.starts0[A.nblocks] = (uint32_t)e0;
          if (SCHEME == TP_RFOR) A.starts1[A.nblocks] = (uint32_t)e1;
        }
      }
    }
    __syncthreads();  // shared arrays are reused by the next chunk
  }
}

// "None": the plain column padded to whole 32-row miniblocks, block_starts = 512 k
__global__ void k_encode_none(const int32_t* __restrict__ x, uint64_t n, uint64_t words, uint64_t nb,
                              uint32_t* __restrict__ starts, uint32_t* __restrict__ data) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < words + TP_GUARD_WORDS; i += stride)
    data[i] = i < n ? (uint32_t)x[i] : 0u;
  for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nb + 1 + TP_GUARD_WORDS; k += stride)
    starts[k] = k < nb ? (uint32_t)(k * TILE_ROWS) : k == nb ? (uint32_t)words : 0u;
}

static int g_enc_sms = 0;
template <class K>
static int enc_grid(K kernel, size_t smem) {
  if (g_enc_sms == 0) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_enc_sms, cudaDevAttrMultiProcessorCount, dev);
    if (g_enc_sms <= 0) g_enc_sms = 148;
  }
  cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, ETHREADS, smem);
  return g_enc_sms * std::max(1, occ);
}

static uint64_t nchunks_of(uint64_t n) { return (n + CHUNK_ROWS - 1) / CHUNK_ROWS; }

template <int SCHEME>
static tp_status launch_encode(const EncArgs<SCHEME>& a, void* stream) {
  constexpr int NA = SCHEME == MODE_SIZES ? 4 : n_arrays<SCHEME>();
  const size_t smem = (size_t)EW * (HDR_WORDS + NA * 512u) * 4u;
  const int grid = std::max(1, std::min<int>(enc_grid(k_encode<SCHEME>, smem), (int)a.nchunks));
  k_encode<SCHEME><<<grid, ETHREADS, smem, (cudaStream_t)stream>>>(a);
  tp::g_launches.fetch_add(1, std::memory_order_relaxed);
  return cudaGetLastError() == cudaSuccess ? TP_OK : TP_ECUDA;
}

static uint64_t nblocks_of(int scheme, uint64_t n) {
  return scheme == TP_FOR || scheme == TP_DFOR ? (n + 127) / 128 : (n + TILE_ROWS - 1) / TILE_ROWS;
}

}  // namespace enc
}  // namespace tp

using namespace tp;
using namespace tp::enc;

extern "C" {

uint64_t tp_gpu_encode_workspace_bytes(uint64_t n) { return 8u * (W_STATUS + 2u * nchunks_of(n)); }

tp_status tp_gpu_encode_bound(int scheme, uint64_t n, uint64_t* num_blocks, uint64_t* words0, uint64_t* words1) {
  if (scheme < TP_FOR || scheme > TP_NONE) return TP_EINVAL;
  if (n >= (1ull << 32)) return TP_EUNSUPPORTED;
  const uint64_t nb = nblocks_of(scheme, n), nt = (n + TILE_ROWS - 1) / TILE_ROWS;
  uint64_t w0 = 0, w1 = 0;
  if (scheme == TP_FOR) w0 = nb * (2 + 128);
  else if (scheme == TP_DFOR) w0 = nt + nb * (2 + 128);
  else if (scheme == TP_RFOR) w0 = w1 = nb * (6 + 512);
  else w0 = (n + 31) / 32 * 32;
  if (num_blocks) *num_blocks = nb;
  if (words0) *words0 = w0;
  if (words1) *words1 = w1;
  return TP_OK;
}

tp_status tp_gpu_encode_sizes(const int32_t* d_x, uint64_t n, void* d_work, uint64_t* words4, void* stream) {
  if ((n && !d_x) || !d_work || !words4) return TP_EINVAL;
  if (n >= (1ull << 32)) return TP_EUNSUPPORTED;
  if (reinterpret_cast<uintptr_t>(d_x) & 15u) return TP_EINVAL;
  memset(words4, 0, 4 * sizeof(uint64_t));
  if (n == 0) return TP_OK;
  auto* work = reinterpret_cast<unsigned long long*>(d_work);
  if (cudaMemsetAsync(work, 0, 8u * W_STATUS, (cudaStream_t)stream) != cudaSuccess) return TP_ECUDA;
  EncArgs<MODE_SIZES> a{};
  a.x = d_x;
  a.n = (uint32_t)n;
  a.ntiles = (uint32_t)((n + TILE_ROWS - 1) / TILE_ROWS);
  a.nchunks = (uint32_t)nchunks_of(n);
  a.work = work;
  tp_status st = launch_encode(a, stream);
  if (st != TP_OK) return st;
  unsigned long long h[4];
  if (cudaMemcpyAsync(h, work + W_SIZES, sizeof(h), cudaMemcpyDeviceToHost, (cudaStream_t)stream) != cudaSuccess ||
      cudaStreamSynchronize((cudaStream_t)stream) != cudaSuccess)
    return TP_ECUDA;
  for (int i = 0; i < 4; ++i) words4[i] = h[i];
  return TP_OK;
}

tp_status tp_gpu_choose_scheme(const int32_t* d_x, uint64_t n, void* d_work, int* scheme, uint64_t* bytes,
                               void* stream) {
  if (!scheme) return TP_EINVAL;
  uint64_t w[4];
  tp_status st = tp_gpu_encode_sizes(d_x, n, d_work, w, stream);
  if (st != TP_OK) return st;
  const uint64_t nb128 = (n + 127) / 128, nb512 = (n + TILE_ROWS - 1) / TILE_ROWS;
  const uint64_t b[3] = {4 * (3 + nb128 + 1 + w[0]), 4 * (3 + nb128 + 1 + w[1]),
                         4 * (3 + 2 * (nb512 + 1) + w[2] + w[3])};
  int best = TP_FOR;
  for (int s = TP_DFOR; s <= TP_RFOR; ++s)  // ties -> FOR < DFOR < RFOR (R20)
    if (b[s - 1] < b[best - 1]) best = s;
  *scheme = best;
  if (bytes) *bytes = b[best - 1];
  return TP_OK;
}

tp_status tp_gpu_encode_launch(int scheme, const int32_t* d_x, uint64_t n, uint32_t* d_starts0, uint32_t* d_data0,
                               uint64_t cap0, uint32_t* d_starts1, uint32_t* d_data1, uint64_t cap1, void* d_work,
                               void* stream) {
  if (scheme < TP_FOR || scheme > TP_NONE || (n && !d_x) || !d_starts0 || !d_data0 || !d_work) return TP_EINVAL;
  if (scheme == TP_RFOR && (!d_starts1 || !d_data1)) return TP_EINVAL;
  if (n >= (1ull << 32)) return TP_EUNSUPPORTED;
  if (reinterpret_cast<uintptr_t>(d_x) & 15u) return TP_EINVAL;
  auto* work = reinterpret_cast<unsigned long long*>(d_work);
  cudaStream_t s = (cudaStream_t)stream;
  const uint64_t nb = nblocks_of(scheme, n);
  if (cudaMemsetAsync(work, 0, tp_gpu_encode_workspace_bytes(n), s) != cudaSuccess) return TP_ECUDA;
  if (scheme == TP_NONE) {
    const uint64_t words = (n + 31) / 32 * 32;
    if (words > cap0) return TP_ESIZE;
    k_encode_none<<<1184, 256, 0, s>>>(d_x, n, words, nb, d_starts0, d_data0);
    tp::g_launches.fetch_add(1, std::memory_order_relaxed);
    if (cudaGetLastError() != cudaSuccess) return TP_ECUDA;
    const unsigned long long h[5] = {words, 0, TILE_ROWS, 0, 0};
    return cudaMemcpyAsync(work + W_TOT, h, sizeof(h), cudaMemcpyHostToDevice, s) == cudaSuccess ? TP_OK : TP_ECUDA;
  }
  if (n == 0) {  // no tiles: block_starts = {0} + guards, data = guards
    if (cudaMemsetAsync(d_starts0, 0, 4 * (1 + TP_GUARD_WORDS), s) != cudaSuccess ||
        cudaMemsetAsync(d_data0, 0, 4 * TP_GUARD_WORDS, s) != cudaSuccess)
      return TP_ECUDA;
    if (scheme == TP_RFOR && (cudaMemsetAsync(d_starts1, 0, 4 * (1 + TP_GUARD_WORDS), s) != cudaSuccess ||
                              cudaMemsetAsync(d_data1, 0, 4 * TP_GUARD_WORDS, s) != cudaSuccess))
      return TP_ECUDA;
    return TP_OK;
  }
  auto fill = [&](auto& a) {
    a.x = d_x;
    a.n = (uint32_t)n;
    a.ntiles = (uint32_t)((n + TILE_ROWS - 1) / TILE_ROWS);
    a.nchunks = (uint32_t)nchunks_of(n);
    a.nblocks = (uint32_t)nb;
    a.starts0 = d_starts0; a.data0 = d_data0; a.cap0 = cap0;
    a.starts1 = d_starts1; a.data1 = d_data1; a.cap1 = cap1;
    a.work = work;
  };
  if (scheme == TP_FOR) { EncArgs<TP_FOR> a{}; fill(a); return launch_encode(a, stream); }
  if (scheme == TP_DFOR) { EncArgs<TP_DFOR> a{}; fill(a); return launch_encode(a, stream); }
  EncArgs<TP_RFOR> a{};
  fill(a);
  return launch_encode(a, stream);
}

tp_status tp_gpu_encode_result(int scheme, uint64_t n, const uint32_t* d_starts0, const uint32_t* d_data0,
                               const uint32_t* d_starts1, const uint32_t* d_data1, const void* d_work,
                               tp_column* out, void* stream) {
  if (scheme < TP_FOR || scheme > TP_NONE || !d_work || !out) return TP_EINVAL;
  unsigned long long h[5] = {0, 0, 0, 0, 0};
  if (n > 0 && cudaMemcpyAsync(h, reinterpret_cast<const unsigned long long*>(d_work) + W_TOT, sizeof(h),
                               cudaMemcpyDeviceToHost, (cudaStream_t)stream) != cudaSuccess)
    return TP_ECUDA;
  if (cudaStreamSynchronize((cudaStream_t)stream) != cudaSuccess) return TP_ECUDA;
  if (h[4]) return TP_ESIZE;
  if (h[0] >= (1ull << 32) || h[1] >= (1ull << 32)) return TP_EUNSUPPORTED;
  memset(out, 0, sizeof(*out));
  out->scheme = (uint32_t)scheme;
  out->n = n;
  out->num_blocks = nblocks_of(scheme, n);
  const bool rf = scheme == TP_RFOR;
  out->block_size = scheme == TP_FOR || scheme == TP_DFOR ? 128u : TILE_ROWS;
  out->miniblock_count = scheme == TP_FOR || scheme == TP_DFOR ? 4u : rf ? 16u : 1u;
  out->tile_blocks = scheme == TP_FOR || scheme == TP_DFOR ? 4u : 1u;
  out->starts0 = d_starts0; out->data0 = d_data0; out->words0 = h[0];
  if (rf) { out->starts1 = d_starts1; out->data1 = d_data1; out->words1 = h[1]; }
  out->max_tile_words0 = (uint32_t)h[2];
  out->max_tile_words1 = (uint32_t)h[3];
  return TP_OK;
}

tp_status tp_gpu_encode(int scheme, const int32_t* d_x, uint64_t n, uint32_t* d_starts0, uint32_t* d_data0,
                        uint64_t cap0, uint32_t* d_starts1, uint32_t* d_data1, uint64_t cap1, void* d_work,
                        tp_column* out, void* stream) {
  tp_status st = tp_gpu_encode_launch(scheme, d_x, n, d_starts0, d_data0, cap0, d_starts1, d_data1, cap1, d_work,
                                      stream);
  if (st != TP_OK) return st;
  return tp_gpu_encode_result(scheme, n, d_starts0, d_data0, d_starts1, d_data1, d_work, out, stream);
}

}  // extern "C"
