// tp_encode.cu -- the tile-parallel GPU encoder: GPU-FOR, GPU-DFOR,
// GPU-RFOR and the GPU-* scheme choice computed from a DEVICE column, byte-identical to the
// host encoder (tp_host.cpp) and to the oracle (readings R1-R20).
//
// The paper encodes on the CPU once (250M values in 1.2 / 1.3 / 2.2 s on 6 vCPUs);
// every 512-row tile is encoded independently, so the only
// cross-tile dependency is the word offset of each tile in the output -- an exclusive prefix
// sum of tile sizes.  One pass over HBM:
//   * persistent CTAs of 8 warps take chunks in order from an atomic counter (chunk_rows():
//     FOR / DFOR 16384 rows = 8 warps x 2 tiles x 2 sub-rounds, RFOR and the sizes pass 8192
//     rows = 8 warps x 2 tiles); each warp loads its tiles (coalesced 16-byte loads) into
//     shared memory;
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

constexpr int EW = 8;                                  // warps per CTA
constexpr int ETHREADS = 32 * EW;
constexpr uint64_t ST_AGG = 1ull << 62, ST_INC = 2ull << 62, ST_VAL = (1ull << 62) - 1;
constexpr int MODE_SIZES = 0;                          // SCHEME template value: all three plans, counts only

// tiles per warp: 2 (lane l owns miniblock l & 15 of tile l >> 4, the decoder's mapping)
__host__ __device__ constexpr int tpw_of(int) { return 2; }
constexpr uint32_t STG_TILE = 528;
// RFOR / sizes: three regions per warp -- X (the 2 staged tiles, then the value stream's
// output staging), V (run values of both tiles, then the run-length stream's staging), L
// (run lengths); a tile's stream output <= 6 + 512 words, staged at tile * RF_STG
constexpr uint32_t RF_REGION = 1040, RF_STG = 520;
// sub-rounds per chunk: FOR / DFOR warps stage and pack 2 x 2 tiles before the chunk's
// look-back (halves the look-back waits per row, measured); RFOR packs from registers after it
#ifndef TP_ENC_KS
#define TP_ENC_KS 2
#endif
__host__ __device__ constexpr int ks_of(int scheme) { return scheme == TP_FOR || scheme == TP_DFOR ? TP_ENC_KS : 1; }
__host__ __device__ constexpr uint32_t chunk_rows(int scheme) {
  return EW * tpw_of(scheme) * ks_of(scheme) * TILE_ROWS;
}
// per-warp shared words: FOR / DFOR per sub-round the two staged tiles, re-used in place as
// the output staging (2 x 528 >= 2 x (1 + 4 (2 + 128)) words) + 16 relative block starts;
// RFOR / sizes: X, run starts S, V, L
__host__ __device__ constexpr uint32_t warp_words(int scheme) {
  return scheme == TP_FOR || scheme == TP_DFOR ? 1056u * ks_of(scheme) + 16u : 3u * RF_REGION;
}

// workspace (u64 words): [0] chunk counter, [1..2] stream totals, [3..4] max tile words,
// [5] overflow flag, [6..9] sizes mode: FOR, DFOR, RFOR values, RFOR lengths; then the
// look-back status words, two per chunk (stream 0, stream 1)
constexpr int W_CTR = 0, W_TOT = 1, W_MTW = 3, W_OVF = 5, W_SIZES = 6, W_STATUS = 16;

__device__ __forceinline__ uint32_t bitlen(uint32_t u) { return u ? 32u - __clz(u) : 0u; }

// shared layout of staged rows: miniblock-major (32 words per 32-row miniblock), the 16-byte
// chunk q of miniblock mb at chunk q ^ (mb & 7), so that 8 lanes reading chunk q of 8
// consecutive miniblocks hit 8 distinct bank groups (conflict-free 128-bit loads)
__device__ __forceinline__ uint32_t xs(uint32_t r) {
  const uint32_t mb = r >> 5;
  return (mb << 5) | ((((r >> 2) & 7u) ^ (mb & 7u)) << 2) | (r & 3u);
}
__device__ __forceinline__ void load_mb(const uint32_t* X, uint32_t mb, uint32_t (&v)[32]) {
  const uint32_t* b = X + 32u * mb;
  const uint32_t sw = mb & 7u;
#pragma unroll
  for (int q = 0; q < 8; ++q) {
    const uint4 t = *reinterpret_cast<const uint4*>(b + 4u * ((uint32_t)q ^ sw));
    v[4 * q] = t.x; v[4 * q + 1] = t.y; v[4 * q + 2] = t.z; v[4 * q + 3] = t.w;
  }
}

// segmented (16-lane) exclusive prefix of x; *tot = the segment's total
__device__ __forceinline__ uint32_t excl16(uint32_t x, uint32_t lane, uint32_t* tot) {
  uint32_t s = x;
#pragma unroll
  for (int d = 1; d < 16; d <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, s, d);
    if ((lane & 15u) >= (uint32_t)d) s += y;
  }
  *tot = __shfl_sync(FULL, s, (lane & 16u) | 15u);
  return s - x;
}
// bitwidth word of the 4 miniblocks j .. j+3 (R2), valid in lanes with j % 4 == 0
__device__ __forceinline__ uint32_t bw_word(uint32_t b, uint32_t lane) {
  const uint32_t b1 = __shfl_down_sync(FULL, b, 1), b2 = __shfl_down_sync(FULL, b, 2),
                 b3 = __shfl_down_sync(FULL, b, 3);
  return b | b1 << 8 | b2 << 16 | b3 << 24;
}

// ---- bit packing of one 32-entry miniblock at compile-time bitwidth B (the inverse of
// Alg. 1 lines 12-17: entry i at stream bits [i B, i B + B), LSB-first, R1); stores words
// [0, nw) of the packed miniblock (nw = B for FOR, ceil(cnt B / 32) for the tight RFOR
// miniblocks, R17).  Entries must already be < 2^B.
template <int B>
__device__ __forceinline__ void pack_fixed(const uint32_t (&u)[32], uint32_t* dst, uint32_t nw) {
  if constexpr (B > 0) {
#pragma unroll
    for (int k = 0; k < B; ++k) {
      uint32_t w = 0u;
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        const int p = i * B - 32 * k;
        if (p > -B && p < 32) w |= p >= 0 ? (u[i] << p) : (u[i] >> (-p));
      }
      if ((uint32_t)k < nw) dst[k] = w;
    }
  }
}
#define TP_PCASE(B) \
  case B:           \
    pack_fixed<B>(u, dst, nw); break;
// warp-cooperative dispatch: the specialised routine runs once per distinct bitwidth among
// the lanes (as the decoder's unpack_mb)
__device__ __forceinline__ void pack_mb(const uint32_t (&u)[32], uint32_t b, uint32_t* dst, uint32_t nw) {
  uint32_t todo = FULL;
  do {
    const uint32_t bl = __shfl_sync(FULL, b, __ffs(todo) - 1);
    const bool mine = b == bl;
    todo &= ~__ballot_sync(FULL, mine);
    if (mine) {
      switch (bl) {
        TP_PCASE(0) TP_PCASE(1) TP_PCASE(2) TP_PCASE(3) TP_PCASE(4) TP_PCASE(5) TP_PCASE(6) TP_PCASE(7)
        TP_PCASE(8) TP_PCASE(9) TP_PCASE(10) TP_PCASE(11) TP_PCASE(12) TP_PCASE(13) TP_PCASE(14) TP_PCASE(15)
        TP_PCASE(16) TP_PCASE(17) TP_PCASE(18) TP_PCASE(19) TP_PCASE(20) TP_PCASE(21) TP_PCASE(22) TP_PCASE(23)
        TP_PCASE(24) TP_PCASE(25) TP_PCASE(26) TP_PCASE(27) TP_PCASE(28) TP_PCASE(29) TP_PCASE(30) TP_PCASE(31)
        default: pack_fixed<32>(u, dst, nw); break;
      }
    }
  } while (todo);
}
#undef TP_PCASE

// ---- FOR plan of the lane's miniblock j of a tile whose slots >= nvalid are neutral pads
// (R8 / R13): block reference = signed min over the block's real slots (R4; 0 for a block of
// pads only, R14), bitwidth = bit length of the OR of the offsets (== of the max, R3).
// v: the slots; on return u = offsets (pads 0), b = bitwidth, ref = the block's reference.
__device__ __forceinline__ void plan_for_mb(const uint32_t (&v)[32], uint32_t j, uint32_t nvalid,
                                            uint32_t (&u)[32], uint32_t& b, int32_t& ref) {
  const uint32_t lo = 32u * j;
  const uint32_t cnt = nvalid > lo ? min(32u, nvalid - lo) : 0u;
  int32_t mn = INT_MAX;
#pragma unroll
  for (int i = 0; i < 32; ++i)
    if ((uint32_t)i < cnt) mn = min(mn, (int32_t)v[i]);
  mn = min(mn, __shfl_xor_sync(FULL, mn, 1));
  mn = min(mn, __shfl_xor_sync(FULL, mn, 2));
  ref = 128u * (j >> 2) < nvalid ? mn : 0;
  uint32_t o = 0u;
#pragma unroll
  for (int i = 0; i < 32; ++i) {
    u[i] = (uint32_t)i < cnt ? v[i] - (uint32_t)ref : 0u;  // mod 2^32 (R4)
    o |= u[i];
  }
  b = bitlen(o);
}

// runs of the lane's tile (R18), lane j = miniblock j (rows 32 j .. 32 j + 31 of the tile,
// values v): the lane marks the rows of its miniblock that start a run (32-bit mask), a
// 16-lane scan of the mark counts numbers the runs, and the lane writes its runs' values
// (read back from the staged rows X, xs layout, tile base row xrow0) and lengths (up to the
// next start -- in its mask, else the first start of a later miniblock, a 16-lane suffix
// min) to Vt[xs(e)], Lt[xs(e)].  Returns r (uniform over the 16 lanes).
__device__ __forceinline__ uint32_t runs_mb(const uint32_t (&v)[32], const uint32_t* X, uint32_t xrow0, uint32_t j,
                                            uint32_t m, uint32_t* Vt, uint32_t* Lt, uint32_t lane) {
  const uint32_t row0 = 32u * j;
  const uint32_t prev = __shfl_up_sync(FULL, v[31], 1);  // the previous miniblock's last row
  uint32_t mask = 0u;
#pragma unroll
  for (int i = 0; i < 32; ++i) {
    const uint32_t pv = i ? v[i - 1] : prev;
    const bool f = row0 + i < m && ((i == 0 && j == 0) || v[i] != pv);
    mask |= (uint32_t)f << i;
  }
  uint32_t r;
  uint32_t e = excl16(__popc(mask), lane, &r);
  uint32_t s = mask ? row0 + __ffs(mask) - 1u : m;  // first start at or after this miniblock
#pragma unroll
  for (int d = 1; d < 16; d <<= 1) {
    const uint32_t y = __shfl_down_sync(FULL, s, d);
    if ((lane & 15u) + d < 16u) s = min(s, y);
  }
  uint32_t nf = __shfl_down_sync(FULL, s, 1);  // first start after this miniblock
  if ((lane & 15u) == 15u) nf = m;
  uint32_t mm = mask;
  while (mm) {
    const uint32_t i = __ffs(mm) - 1u;
    mm &= mm - 1u;
    const uint32_t end = mm ? row0 + __ffs(mm) - 1u : nf;
    Vt[xs(e)] = X[xs(xrow0 + row0 + i)];
    Lt[xs(e)] = end - (row0 + i);
    ++e;
  }
  return r;
}

// RFOR plan of the lane's miniblock j (16 tight miniblocks of 32 entries, R17) of the stream
// whose entries sit in A (xs layout), r entries
__device__ __forceinline__ void plan_rfor_mb(const uint32_t* A, uint32_t j, uint32_t r, uint32_t (&u)[32],
                                             uint32_t& b, int32_t& ref, uint32_t& cnt) {
  uint32_t v[32];
  load_mb(A, j, v);
  cnt = r > 32u * j ? min(32u, r - 32u * j) : 0u;
  int32_t mn = INT_MAX;
#pragma unroll
  for (int i = 0; i < 32; ++i)
    if ((uint32_t)i < cnt) mn = min(mn, (int32_t)v[i]);
#pragma unroll
  for (int d = 1; d < 16; d <<= 1) mn = min(mn, __shfl_xor_sync(FULL, mn, d));
  ref = mn;
  uint32_t o = 0u;
#pragma unroll
  for (int i = 0; i < 32; ++i) {
    u[i] = (uint32_t)i < cnt ? v[i] - (uint32_t)ref : 0u;
    o |= u[i];
  }
  b = bitlen(o);
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
  uint32_t n, ntiles, nchunks, nblocks;  // nblocks: block_starts entries - 1
  uint32_t* starts0;
  uint32_t* data0;
  uint32_t* starts1;
  uint32_t* data1;
  uint64_t cap0, cap1;        // data capacity (words, without guards)
  unsigned long long* work;
};

template <int SCHEME>
__global__ void __launch_bounds__(ETHREADS, 3) k_encode(const __grid_constant__ EncArgs<SCHEME> A) {
  extern __shared__ __align__(16) uint32_t esm[];
  constexpr bool SIZES = SCHEME == MODE_SIZES;
  constexpr bool RF = SCHEME == TP_RFOR;
  constexpr int TPW = tpw_of(SCHEME);   // tiles per warp and sub-round (2)
  constexpr int KS = ks_of(SCHEME);     // sub-rounds per chunk (staged side by side)
  constexpr int TW = TPW * KS;          // tiles per warp and chunk
  constexpr bool DF = SCHEME == TP_DFOR;
  constexpr int NS = RF ? 2 : 1;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31u;
  const uint32_t seg = lane >> 4, j = lane & 15u;
  __shared__ uint32_t s_chunk;
  __shared__ uint32_t s_words[2][EW * 2 * TP_ENC_KS];
  __shared__ unsigned long long s_base[2], s_agg[2];
  uint32_t* Xw = esm + warp * warp_words(SCHEME);
  uint32_t* bsr = Xw + KS * 1056u;  // FOR / DFOR: block starts relative to their tile, 4 per tile
  unsigned long long* work = A.work;

  while (true) {
    if (threadIdx.x == 0) s_chunk = (uint32_t)atomicAdd(work + W_CTR, 1ull);
    __syncthreads();
    const uint32_t c = s_chunk;
    if (c >= A.nchunks) break;
    const uint32_t t0 = (c * EW + warp) * TW;  // this warp's first tile
    uint32_t u[32];
    uint32_t b = 0u, P = 0u, nw = 0u;  // bitwidth, data-word offset, words of the lane's miniblock
    int32_t ref = 0;
    uint32_t my_t = t0, r = 0u;
#pragma unroll 1
    for (uint32_t p = 0; p < (uint32_t)KS; ++p) {
      uint32_t* X = Xw + p * (RF || SIZES ? 0u : 1056u);
      const uint32_t tp0 = t0 + p * TPW;
      const uint32_t r0 = tp0 * TILE_ROWS;
      const uint32_t mrows = tp0 < A.ntiles ? min((uint32_t)(TPW * TILE_ROWS), A.n - r0) : 0u;
      // ---- stage the 2 tiles (coalesced 16-byte loads, miniblock-major swizzled rows)
      if (mrows == TPW * TILE_ROWS) {
        const int4* src = reinterpret_cast<const int4*>(A.x + r0);
        int4 q[4 * TPW];
#pragma unroll
        for (int k = 0; k < 4 * TPW; ++k) q[k] = __ldcs(src + 32 * k + lane);
#pragma unroll
        for (int k = 0; k < 4 * TPW; ++k) *reinterpret_cast<int4*>(X + xs(128u * k + 4u * lane)) = q[k];
      } else if (mrows > 0) {
        for (uint32_t rr = lane; rr < TPW * TILE_ROWS; rr += 32)
          X[xs(rr)] = rr < mrows ? (uint32_t)A.x[r0 + rr] : 0u;
      }
      __syncwarp();
      // the lane's tile and miniblock
      my_t = tp0 + seg;
      const uint32_t m = my_t < A.ntiles ? min((uint32_t)TILE_ROWS, A.n - my_t * TILE_ROWS) : 0u;
      const uint32_t nblk = (m + 127u) >> 7;
      uint32_t v[32];
      load_mb(X, 16u * seg + j, v);
      uint32_t tw = 0u, wf = 0u, wd = 0u;
      if (SIZES || SCHEME == TP_FOR) {
        plan_for_mb(v, j, m, u, b, ref);
        const uint32_t bj = (j >> 2) < nblk ? b : 0u;
        uint32_t tot;
        P = excl16(bj, lane, &tot);
        nw = bj;
        tw = 2u * nblk + tot;
        wf = tw;
      }
      if (SIZES || RF) {
        // runs of the tile (before the DFOR plan below rewrites v)
        uint32_t* V = Xw + RF_REGION;
        uint32_t* L = Xw + 2u * RF_REGION;
        r = runs_mb(v, X, 512u * seg, j, m, V + 512u * seg, L + 512u * seg, lane);
      }
      if (SIZES || DF) {
        const uint32_t first = v[0];
        // delta slots (R12, R13): slot s = x[s+1] - x[s] for s < m - 1, neutral pads after
        const uint32_t nxt = __shfl_down_sync(FULL, v[0], 1);
#pragma unroll
        for (int i = 0; i < 31; ++i) v[i] = v[i + 1] - v[i];
        v[31] = nxt - v[31];
        plan_for_mb(v, j, m ? m - 1u : 0u, u, b, ref);
        const uint32_t bj = (j >> 2) < nblk ? b : 0u;
        uint32_t tot;
        P = excl16(bj, lane, &tot);
        nw = bj;
        tw = m > 0 ? 1u + 2u * nblk + tot : 0u;  // first value + blocks (no tile: no words)
        wd = tw;
        if (DF) v[0] = first;
      }
      if (SCHEME == TP_FOR || DF) {
        __syncwarp();  // every lane holds its rows: the staged tiles become the output staging
        uint32_t* stg = X + seg * STG_TILE;
        const uint32_t blk = j >> 2, d0 = DF ? 1u : 0u;
        const uint32_t bw = bw_word(b, lane);  // (warp-collective: outside the per-tile branch)
        if (m > 0) {
          if (DF && j == 0) stg[0] = v[0];  // first value of the tile
          if ((j & 3u) == 0 && blk < nblk) {
            const uint32_t bs = d0 + 2u * blk + P;  // header of block blk (P = its first mb's offset)
            stg[bs] = (uint32_t)ref;
            stg[bs + 1] = bw;
            bsr[4u * (p * TPW + seg) + blk] = bs;
          }
        }
        // one call site for every lane (warp-collective dispatch); nw = 0 past the column's end
        pack_mb(u, nw, stg + d0 + 2u * (blk + 1u) + P, nw);
        if (j == 0) s_words[0][TW * warp + p * TPW + seg] = tw;
      }
      if (SIZES || RF) {
        // the two streams (R17): plan (and, encoding, pack into the staging) the value stream,
        // then the run-length stream; stream s of tile seg staged at region s, seg * RF_STG
        __syncwarp();
        uint32_t wst[2];
#pragma unroll 1
        for (uint32_t sidx = 0; sidx < 2; ++sidx) {
          const uint32_t* E = Xw + (1u + sidx) * RF_REGION + 512u * seg;
          uint32_t cnt;
          plan_rfor_mb(E, j, r, u, b, ref, cnt);
          nw = (cnt * b + 31u) >> 5;  // tight: ceil(cnt b / 32) words
          uint32_t tot;
          P = excl16(nw, lane, &tot);
          wst[sidx] = m > 0 ? 6u + tot : 0u;
          if (RF) {
            __syncwarp();  // the region being staged into is read no more
            uint32_t* stg = Xw + sidx * RF_REGION + seg * RF_STG;
            const uint32_t bw = bw_word(b, lane);
            if (m > 0) {
              if (j == 0) { stg[0] = r; stg[1] = (uint32_t)ref; }
              if ((j & 3u) == 0) stg[2 + (j >> 2)] = bw;
            }
            pack_mb(u, m > 0 ? b : 0u, stg + 6 + P, m > 0 ? nw : 0u);
            if (j == 0) s_words[sidx][TPW * warp + seg] = wst[sidx];
          }
        }
        if (SIZES) {
          // one atomic per warp and scheme stream: both tiles' words
          const uint32_t fv = __shfl_sync(FULL, wf, 0) + __shfl_sync(FULL, wf, 16);
          const uint32_t dv = __shfl_sync(FULL, wd, 0) + __shfl_sync(FULL, wd, 16);
          const uint32_t vv = __shfl_sync(FULL, wst[0], 0) + __shfl_sync(FULL, wst[0], 16);
          const uint32_t lv = __shfl_sync(FULL, wst[1], 0) + __shfl_sync(FULL, wst[1], 16);
          if (lane == 0 && mrows > 0) {
            atomicAdd(work + W_SIZES + 0, (unsigned long long)fv);
            atomicAdd(work + W_SIZES + 1, (unsigned long long)dv);
            atomicAdd(work + W_SIZES + 2, (unsigned long long)vv);
            atomicAdd(work + W_SIZES + 3, (unsigned long long)lv);
          }
        }
      }
    }
    if (SIZES) {
      __syncthreads();
      continue;
    }
    // ---- the chunk's offsets by look-back (warp s: stream s)
    __syncthreads();
    constexpr int NT = EW * TW;
    if (warp < NS) {
      uint64_t agg = 0;
      uint32_t mx = 0u;
      for (uint32_t k = lane; k < (uint32_t)NT; k += 32) {
        agg += s_words[warp][k];
        mx = max(mx, s_words[warp][k]);
      }
#pragma unroll
      for (int d = 16; d > 0; d >>= 1) {
        agg += __shfl_xor_sync(FULL, agg, d);
        mx = max(mx, __shfl_xor_sync(FULL, mx, d));
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
    if (!RF && threadIdx.x == 0) s_base[1] = s_agg[1] = 0;
    __syncthreads();
    const bool ovf = s_base[0] + s_agg[0] > A.cap0 || (RF && s_base[1] + s_agg[1] > A.cap1);
    if (t0 < A.ntiles && !ovf) {
      uint64_t e[2];
#pragma unroll 1
      for (uint32_t sidx = 0; sidx < (uint32_t)NS; ++sidx) {
        uint32_t* data = sidx ? A.data1 : A.data0;
        uint32_t* starts = sidx ? A.starts1 : A.starts0;
        // the warp's base word: the chunk base + the earlier tiles of the chunk
        uint64_t B = s_base[sidx];
        for (uint32_t k = 0; k < TW * warp; ++k) B += s_words[sidx][k];
        // block_starts (lane 4 tl + blk: block blk of the warp's tile tl; RFOR: lane tl), then
        // the staged words of the warp's tiles, coalesced
        uint64_t off = 0, my_off = 0;
        const uint32_t tl = RF ? lane : lane >> 2, blk = RF ? 0u : lane & 3u;
#pragma unroll 1
        for (uint32_t k = 0; k < (uint32_t)TW; ++k) {
          if (k == tl) my_off = off;
          off += s_words[sidx][TW * warp + k];
        }
        const uint32_t t = t0 + tl;
        if (tl < (uint32_t)TW && t < A.ntiles) {
          if (RF) {
            starts[t] = (uint32_t)(B + my_off);
          } else {
            const uint32_t mt = min((uint32_t)TILE_ROWS, A.n - t * TILE_ROWS);
            if (blk < ((mt + 127u) >> 7)) starts[4ull * t + blk] = (uint32_t)(B + my_off + bsr[lane]);
          }
        }
        uint64_t o = B;
#pragma unroll 1
        for (uint32_t k = 0; k < (uint32_t)TW; ++k) {
          const uint32_t wk = s_words[sidx][TW * warp + k];
          const uint32_t* src = RF ? Xw + sidx * RF_REGION + k * RF_STG : Xw + (k / TPW) * 1056u + (k % TPW) * STG_TILE;
          for (uint32_t i = lane; i < wk; i += 32) data[o + i] = src[i];
          o += wk;
        }
        e[sidx] = o;
      }
      // the column's end: last block_starts entry + zero guards (R6, R9)
      if (t0 + TW >= A.ntiles) {
#pragma unroll 1
        for (uint32_t sidx = 0; sidx < (uint32_t)NS; ++sidx) {
          uint32_t* data = sidx ? A.data1 : A.data0;
          uint32_t* starts = sidx ? A.starts1 : A.starts0;
          if (lane < TP_GUARD_WORDS) {
            data[e[sidx] + lane] = 0u;
            starts[A.nblocks + 1 + lane] = 0u;
          }
          if (lane == 0) starts[A.nblocks] = (uint32_t)e[sidx];
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

static uint64_t nchunks_of(uint64_t n, int scheme = MODE_SIZES) {
  return (n + chunk_rows(scheme) - 1) / chunk_rows(scheme);
}

template <int SCHEME>
static tp_status launch_encode(const EncArgs<SCHEME>& a, void* stream) {
  const size_t smem = (size_t)EW * warp_words(SCHEME) * 4u;
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
    a.nchunks = (uint32_t)nchunks_of(n, scheme);
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
