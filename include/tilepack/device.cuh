/*
 * tilepack/device.cuh -- the paper's device-side decode functions for USER kernels:
 * LoadBitPack / LoadDBitPack / LoadRBitPack, usable "directly in user's CUDA
 * code" in place of a plain tile load ("replace BlockLoad ... by just changing a
 * single line of code").  Header-only, no dependency on libtilepack.so: a user kernel includes
 * this file (and tilepack.h for the column struct) and decodes tiles of columns that were
 * encoded by tp_encode / tp_gpu_encode (byte formats: DESIGN.md "Formats", readings R1-R19).
 *
 *   __shared__ uint32_t smem[TP_TILE_SMEM_WORDS];
 *   int32_t items[ITEMS];
 *   tp_load_for<BLOCK_THREADS, ITEMS>(col, tile, items, smem);   // GPU-FOR
 *   tp_load_dfor<BLOCK_THREADS, ITEMS>(col, tile, items, smem);  // GPU-DFOR
 *   tp_load_rfor<BLOCK_THREADS, ITEMS>(col, tile, items, smem);  // GPU-RFOR
 *
 * Contract (every function):
 *   - called by ALL threads of a block of BLOCK_THREADS threads (they synchronise with
 *     __syncthreads); BLOCK_THREADS * ITEMS == 512, the tile of D = 4 blocks of 128
 *      = one RFOR block;
 *   - `col` is a tp_column whose pointers are DEVICE pointers (starts/data arrays with the
 *     TP_GUARD_WORDS zero guard words of include/tilepack.h); `tile` < ceil(n / 512);
 *   - items[k] of thread t = row 512 * tile + k * BLOCK_THREADS + t (the striped arrangement of
 *     Crystal's BlockLoad, which these calls replace); rows >= n are left unchanged -- the
 *     caller masks them (tp_tile_rows gives the tile's valid rows);
 *   - `smem` is TP_TILE_SMEM_WORDS words of the block's shared memory, free on entry, reusable
 *     after the call returns (the call ends with __syncthreads);
 *   - the tile's compressed words are read from global memory ONCE, coalesced, into smem
 *     (tile-based decompression), and decoded from there;
 *   - integer arithmetic mod 2^32 (R4); bitwidth bytes > 32 are used as 32 (tp_validate on
 *     the host checks a column).
 */
#ifndef TILEPACK_DEVICE_CUH
#define TILEPACK_DEVICE_CUH

#include <stdint.h>

#include "../tilepack.h"

#define TP_TILE_SMEM_WORDS 2624u

/* valid rows of tile `tile` of an n-row column (512 except at the end) */
__device__ __forceinline__ uint32_t tp_tile_rows(const tp_column& col, uint32_t tile) {
  const uint64_t r0 = (uint64_t)tile * 512u;
  return r0 >= col.n ? 0u : (uint32_t)(col.n - r0 < 512u ? col.n - r0 : 512u);
}

namespace tp_dev {

/* value at stream bits [p, p + b) of the words at w, LSB-first (Alg. 1 lines 15-17, R1) */
__device__ __forceinline__ uint32_t field(const uint32_t* w, uint32_t p, uint32_t b) {
  const uint64_t win = (uint64_t)w[p >> 5] | ((uint64_t)w[(p >> 5) + 1] << 32);
  return (uint32_t)((win >> (p & 31u)) & (b >= 32u ? 0xffffffffull : ((1ull << b) - 1ull)));
}
__device__ __forceinline__ uint32_t bw_byte(uint32_t bw, uint32_t j) {  /* R2, R3, R5 */
  const uint32_t b = (bw >> (8u * j)) & 255u;
  return b > 32u ? 32u : b;
}

/* copy words [lo, hi) of src (+ 2 guard words: Alg. 1 line 15 reads data[s + 1]) into dst,
 * coalesced over the block */
template <int BT>
__device__ __forceinline__ void stage(const uint32_t* __restrict__ src, uint32_t lo, uint32_t hi, uint32_t* dst) {
  for (uint32_t i = threadIdx.x; i < hi - lo + 2u; i += BT) dst[i] = src[lo + i];
}

/* entry e of a 128-entry FOR block staged at blk: [ref][bitwidth word][4 miniblocks] (Fig. 3,
 * Alg. 1: miniblock j = e / 32 starts 2 + sum of the earlier bitwidths words into the block) */
__device__ __forceinline__ uint32_t for_entry(const uint32_t* blk, uint32_t e) {
  const uint32_t bw = blk[1], j = e >> 5;
  uint32_t off = 2u;
  for (uint32_t q = 0; q < j; ++q) off += bw_byte(bw, q);
  const uint32_t b = bw_byte(bw, j);
  return blk[0] + field(blk + off, (e & 31u) * b, b);
}

/* entry e of an RFOR stream block staged at blk: [r][ref][4 bitwidth words][16 miniblocks of
 * 32 entries], every miniblock before the last non-empty one full (layout B, R17) */
__device__ __forceinline__ uint32_t rfor_entry(const uint32_t* blk, uint32_t e) {
  const uint32_t j = e >> 5;
  uint32_t off = 6u;
  for (uint32_t q = 0; q < j; ++q) off += bw_byte(blk[2 + (q >> 2)], q & 3u);
  const uint32_t b = bw_byte(blk[2 + (j >> 2)], j & 3u);
  return blk[1] + field(blk + off, (e & 31u) * b, b);
}

/* block-wide exclusive scan of v[0..512) in place (mod 2^32); returns nothing, ends synced.
 * Each thread scans 512 / BT contiguous entries, the chunk totals are scanned by warp 0. */
template <int BT>
__device__ __forceinline__ void block_exclusive_scan512(uint32_t* v, uint32_t* tmp) {
  constexpr uint32_t PER = 512u / BT;
  const uint32_t t = threadIdx.x;
  uint32_t run = 0u;
  for (uint32_t i = 0; i < PER; ++i) {
    const uint32_t x = v[t * PER + i];
    v[t * PER + i] = run;
    run += x;
  }
  tmp[t] = run;
  __syncthreads();
  if (t < 32u) {  /* exclusive scan of the BT chunk totals (BT <= 512) */
    constexpr uint32_t PW = (BT + 31u) / 32u;
    uint32_t s = 0u;
    for (uint32_t i = 0; i < PW; ++i) s += (t * PW + i < (uint32_t)BT) ? tmp[t * PW + i] : 0u;
    uint32_t incl = s;
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
      if (t >= (uint32_t)d) incl += y;
    }
    uint32_t base = incl - s;
    for (uint32_t i = 0; i < PW; ++i) {
      if (t * PW + i < (uint32_t)BT) {
        const uint32_t x = tmp[t * PW + i];
        tmp[t * PW + i] = base;
        base += x;
      }
    }
  }
  __syncthreads();
  const uint32_t add = tmp[t];
  for (uint32_t i = 0; i < PER; ++i) v[t * PER + i] += add;
  __syncthreads();
}

}  // namespace tp_dev

/* GPU-FOR tile load (LoadBitPack): Algorithm 1 per item from the
 * tile's 4 blocks staged once in shared memory. */
template <int BLOCK_THREADS, int ITEMS>
__device__ void tp_load_for(const tp_column& col, uint32_t tile, int32_t (&items)[ITEMS], uint32_t* smem) {
  static_assert(BLOCK_THREADS * ITEMS == 512, "a tile is 512 rows: BLOCK_THREADS * ITEMS == 512");
  const uint32_t b0 = 4u * tile, b1 = b0 + 4u < col.num_blocks ? b0 + 4u : (uint32_t)col.num_blocks;
  uint32_t* st = smem;      /* the tile's 5 block_starts */
  uint32_t* w = smem + 8;   /* its words */
  if (threadIdx.x <= b1 - b0) st[threadIdx.x] = col.starts0[b0 + threadIdx.x];
  __syncthreads();
  const uint32_t lo = st[0];
  tp_dev::stage<BLOCK_THREADS>(col.data0, lo, st[b1 - b0], w);
  __syncthreads();
  const uint32_t rows = tp_tile_rows(col, tile);
#pragma unroll
  for (int k = 0; k < ITEMS; ++k) {
    const uint32_t r = (uint32_t)k * BLOCK_THREADS + threadIdx.x;
    if (r < rows) items[k] = (int32_t)tp_dev::for_entry(w + (st[r >> 7] - lo), r & 127u);
  }
  __syncthreads();
}

/* GPU-DFOR tile load (LoadDBitPack): the tile's 512 delta slots (Alg. 1 per slot,
 * slot s = x[s+1] - x[s], neutral pads, R13), a block-wide exclusive prefix sum,
 * plus the tile's first value data[starts[4 tile] - 1] (Fig. 6). */
template <int BLOCK_THREADS, int ITEMS>
__device__ void tp_load_dfor(const tp_column& col, uint32_t tile, int32_t (&items)[ITEMS], uint32_t* smem) {
  static_assert(BLOCK_THREADS * ITEMS == 512, "a tile is 512 rows: BLOCK_THREADS * ITEMS == 512");
  const uint32_t b0 = 4u * tile, b1 = b0 + 4u < col.num_blocks ? b0 + 4u : (uint32_t)col.num_blocks;
  uint32_t* st = smem;          /* 5 block_starts */
  uint32_t* D = smem + 8;       /* 512 slots -> prefix sums */
  uint32_t* tmp = D + 512;      /* scan scratch (BLOCK_THREADS words) */
  uint32_t* w = tmp + 512;      /* the tile's words, first value included */
  if (threadIdx.x <= b1 - b0) st[threadIdx.x] = col.starts0[b0 + threadIdx.x];
  __syncthreads();
  const uint32_t lo = st[0] - 1u;  /* the tile's first value */
  /* the tile ends where the next tile's first value starts (or at the column's last word) */
  const uint32_t hi = b1 < col.num_blocks ? st[b1 - b0] - 1u : st[b1 - b0];
  tp_dev::stage<BLOCK_THREADS>(col.data0, lo, hi, w);
  __syncthreads();
  const uint32_t nblk = b1 - b0;
  for (uint32_t s = threadIdx.x; s < 512u; s += BLOCK_THREADS)
    D[s] = (s >> 7) < nblk ? tp_dev::for_entry(w + (st[s >> 7] - lo), s & 127u) : 0u;
  __syncthreads();
  tp_dev::block_exclusive_scan512<BLOCK_THREADS>(D, tmp);
  const uint32_t first = w[0], rows = tp_tile_rows(col, tile);
#pragma unroll
  for (int k = 0; k < ITEMS; ++k) {
    const uint32_t r = (uint32_t)k * BLOCK_THREADS + threadIdx.x;
    if (r < rows) items[k] = (int32_t)(first + D[r]);
  }
  __syncthreads();
}

/* GPU-RFOR tile load (LoadRBitPack): unpack the block's r run values and run
 * lengths (FOR on both arrays), exclusive scan of the lengths = run start rows
 * (the prefix sums of [18]), then each item's run = the last start at or before its row
 * (a binary search over the starts; any algorithm equal to repeat(V, L) per R19). */
template <int BLOCK_THREADS, int ITEMS>
__device__ void tp_load_rfor(const tp_column& col, uint32_t tile, int32_t (&items)[ITEMS], uint32_t* smem) {
  static_assert(BLOCK_THREADS * ITEMS == 512, "a tile is 512 rows: BLOCK_THREADS * ITEMS == 512");
  uint32_t* st = smem;          /* [v0, v1, l0, l1]: the two stream blocks' word ranges */
  uint32_t* S = smem + 8;       /* run starts (512) */
  uint32_t* V = S + 512;        /* run values (512) */
  uint32_t* tmp = V + 512;      /* scan scratch */
  uint32_t* wv = tmp + 512;     /* value stream block (<= 518 + 2 words) */
  uint32_t* wl = wv + 528;      /* run-length stream block */
  if (threadIdx.x < 2u) st[threadIdx.x] = col.starts0[tile + threadIdx.x];
  else if (threadIdx.x < 4u) st[threadIdx.x] = col.starts1[tile + threadIdx.x - 2u];
  __syncthreads();
  tp_dev::stage<BLOCK_THREADS>(col.data0, st[0], st[1], wv);
  tp_dev::stage<BLOCK_THREADS>(col.data1, st[2], st[3], wl);
  __syncthreads();
  const uint32_t r = wv[0] < 512u ? wv[0] : 512u;  /* run count */
  for (uint32_t e = threadIdx.x; e < 512u; e += BLOCK_THREADS) {
    S[e] = e < r ? tp_dev::rfor_entry(wl, e) : 0u;
    V[e] = e < r ? tp_dev::rfor_entry(wv, e) : 0u;
  }
  __syncthreads();
  tp_dev::block_exclusive_scan512<BLOCK_THREADS>(S, tmp);  /* lengths -> start rows */
  const uint32_t rows = tp_tile_rows(col, tile);
#pragma unroll
  for (int k = 0; k < ITEMS; ++k) {
    const uint32_t q = (uint32_t)k * BLOCK_THREADS + threadIdx.x;
    if (q < rows) {
      uint32_t a = 0u, b = r;  /* the largest run index with S[run] <= q */
      while (b - a > 1u) {
        const uint32_t m = (a + b) >> 1;
        if (S[m] <= q) a = m; else b = m;
      }
      items[k] = (int32_t)V[a];
    }
  }
  __syncthreads();
}

#endif /* TILEPACK_DEVICE_CUH */
