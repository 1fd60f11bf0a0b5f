// tp_device.cuh -- sm_100a device primitives of the tile-based decoders
// (the paper's LoadBitPack / LoadDBitPack / LoadRBitPack).
//
// Citations: P:<lines> = /root/reference/PAPER.md, R<n> = DESIGN.md readings.
//
// Execution model:
//   * persistent CTAs, one contiguous range of 512-row tiles each;
//   * warp 0 is a TMA producer: per stage of TPR*rounds tiles it issues 1-D bulk
//     copies (cp.async.bulk, SASS UBLKCP) of every column's contiguous word
//     range + the matching block_starts slice into a ring of shared-memory
//     stages, completion tracked by mbarrier transaction counts
//     (tile staged once; D blocks per tile);
//   * warps 1..4 consume: thread t of a consumer warp owns ONE 32-row
//     miniblock of the stage per column and unpacks it from shared memory with
//     code specialised for its (warp-uniform) bitwidth -- funnel shifts with
//     compile-time positions -- so that the decoded rows live in registers and
//     feed the consumer directly (no intermediate global pass).
#pragma once
#include <cstdint>
#include <cuda.h>
#include <cuda_runtime.h>

namespace tp {

constexpr int TILE_ROWS = 512;      // D = 4 blocks of 128 = RFOR block
constexpr int MB_ROWS = 32;         // miniblock
constexpr int CONSUMER_WARPS = 4;   // 4 warps x 2 tiles = TPR tiles per consumer round
constexpr int TPR = 2 * CONSUMER_WARPS;
constexpr int THREADS = 32 * (CONSUMER_WARPS + 1);
constexpr int MAX_STREAMS = 2 * 6;  // up to 6 columns, 2 streams each (RFOR)
constexpr unsigned FULL = 0xffffffffu;

enum : uint32_t { S_FOR = 1, S_DFOR = 2, S_RFOR = 3, S_NONE = 4, S_FORNM = 5 };

// ------------------------------------------------------------------ PTX wrappers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@!P1 bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// producer-side wait: poll, and back off with a short nanosleep between polls so that a
// producer that is ahead of its consumers does not take their issue slots
__device__ __forceinline__ bool mbar_try(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred P1;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, P1;\n}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}
// suspended wait: try_wait with a suspend-time hint parks the warp in hardware until the
// phase completes (or the hint expires), so a waiting warp takes no issue slots -- the
// nanosleep spin it replaces was 10-19 % of all issued instructions in the consumer-bound
// kernels (ncu source counters, profiles/)
#ifndef TP_SUSPEND_NS
#define TP_SUSPEND_NS 20000
#endif
__device__ __forceinline__ bool mbar_try_suspend(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred P1;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2, %3;\n\t"
      "selp.u32 %0, 1, 0, P1;\n}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity), "n"(TP_SUSPEND_NS)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait_backoff(uint64_t* bar, uint32_t parity) {
  while (!mbar_try_suspend(bar, parity)) {
  }
}
__device__ __forceinline__ void st_shared_v4(uint32_t* p, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
  asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(smem_u32(p)), "r"(a), "r"(b), "r"(c), "r"(d)
               : "memory");
}
// 1-D bulk copy global -> shared, completes `bytes` on the mbarrier (TMA, UBLKCP)
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar,
                                         uint64_t policy) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
      : "memory");
}
// bulk prefetch of global bytes into L2 (no shared-memory destination, no completion tracking)
__device__ __forceinline__ void bulk_prefetch_l2(const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(src), "r"(bytes) : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
// 2-D TMA tensor load global -> shared (UTMALDG), completes on the mbarrier
__device__ __forceinline__ void tma_load_2d(void* dst, const void* tmap, int c0, int c1, uint64_t* bar,
                                            uint64_t policy) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%2, "
      "%3}], [%4], %5;" ::"r"(smem_u32(dst)),
      "l"(tmap), "r"(c0), "r"(c1), "r"(smem_u32(bar)), "l"(policy)
      : "memory");
}
// 2-D TMA tensor store shared -> global (UTMASTG) and its bulk-group bookkeeping
__device__ __forceinline__ void tma_store_2d(const void* tmap, const void* src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(tmap),
               "r"(smem_u32(src)), "r"(c0), "r"(c1)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// ------------------------------------------------------------------ format-violation flags
// (include/tilepack.h tp_device_errors; one copy per translation unit -- the pipeline
// kernels' copy in tp_kernels.cu is the one the ABI reads)
static __device__ uint32_t g_tp_err;
// one RED per flagging thread (no warp-aggregation sequence: the flag is set on a rare path)
__device__ __forceinline__ void tp_flag_error(uint32_t bit) {
  asm volatile("red.relaxed.gpu.global.or.b32 [%0], %1;" ::"l"(&g_tp_err), "r"(bit));  // no ordering needed
}
// a miniblock bitwidth byte: > 32 is a format violation (R3, R5) that tp_validate reports on the
// host; the device uses it as 32 (memory-safe).  Flagging it per miniblock on the device cost 2-4 %
// of the decode kernels (same-box A/B: b = 4 decode->sum 0.142 -> 0.148 ms), so it is not done
// unless TP_DEVICE_BW_FLAG is defined.
__device__ __forceinline__ uint32_t checked_bw(uint32_t b) {
#ifdef TP_DEVICE_BW_FLAG
  if (__builtin_expect(b > 32u, 0)) tp_flag_error(1u);
#endif
  return min(b, 32u);
}

// ------------------------------------------------------------------ column params
// One stream of an encoded column as the kernels see it (host fills).
enum : uint32_t { K_FOR = 0, K_DFOR = 1, K_RFOR = 2, K_NONE = 3 };  // stream kinds
struct Stream {
  const uint32_t* data;
  const uint32_t* starts;
  uint32_t data_off;    // word offset of this stream's data region inside a stage
  uint32_t starts_off;  // word offset of this stream's block_starts region
  uint32_t kind;        // K_FOR / K_DFOR: 4 blocks per tile; K_RFOR: 1 stream block per tile
  uint32_t nblocks;
  uint32_t data_cap;    // bytes of the stage's data region (TP_DEVERR_TILE_WORDS beyond it)
};
struct Col {
  uint32_t scheme;      // S_FOR / S_DFOR / S_RFOR
  uint32_t nblocks;     // entries of block_starts minus one
  uint32_t s0, s1;      // indices into Params::st (s1 only for RFOR)
};
struct alignas(64) Params {
  CUtensorMap tmap[6];  // K_NONE columns: [rows/32][32] int32 view, 128B swizzle (TMA tensor loads)
  Stream st[MAX_STREAMS];
  Col col[6];
  uint32_t nstreams, ncols;
  uint32_t n;           // rows
  uint32_t ntiles;      // ceil(n / 512)
  uint32_t stage_words; // words per stage
  uint32_t nstages;     // ring depth
  uint32_t scratch_off; // word offset of per-warp scratch (after the ring)
  uint32_t scratch_words_per_warp;
  uint32_t staging_off; // word offset of the decode->global staging buffers inside a warp's scratch
  uint32_t rounds;      // consumer rounds per item: an item holds TPR * rounds tiles of one column
  uint32_t agg_off;     // word offset of the per-CTA aggregation table
  uint32_t bar_off;     // word offset of the mbarriers (8-byte aligned)
  uint32_t ring_words;  // query pipeline: words of the byte ring (at smem offset 0)
  uint32_t single_staging;  // decode->global: one staging buffer per warp (instruction-bound DFOR)
};

// ------------------------------------------------------------------ bit unpack
// One 32-entry miniblock at compile-time bitwidth B, entries i at stream bits
// [i*B, i*B+B) LSB-first (Alg. 1 lines 12-17, R1), from shared memory words w.
// Produces e_i (the FOR offsets; the caller adds the reference, Alg. 1 line 18).
template <int B>
__device__ __forceinline__ void unpack_fixed(const uint32_t* __restrict__ w, uint32_t (&e)[32]) {
  if constexpr (B == 0) {
#pragma unroll
    for (int i = 0; i < 32; ++i) e[i] = 0u;
  } else {
    uint32_t r[B + 1];
#pragma unroll
    for (int k = 0; k < B; ++k) r[k] = w[k];
    r[B] = 0u;
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      constexpr uint32_t M = (B == 32) ? 0xffffffffu : ((1u << (B & 31)) - 1u);
      const int p = i * B, k = p >> 5, s = p & 31;
      uint32_t x;
      if (s + B <= 32) {
        x = r[k] >> s;
        if (s + B < 32) x &= M;
      } else {
        x = __funnelshift_r(r[k], r[k + 1], s) & M;
      }
      e[i] = x;
    }
  }
}

// runtime-bitwidth fallback (warps whose lanes disagree on b)
__device__ __forceinline__ void unpack_any(const uint32_t* __restrict__ w, uint32_t b, uint32_t (&e)[32]) {
  const uint32_t m = b >= 32 ? 0xffffffffu : ((1u << b) - 1u);
#pragma unroll
  for (int i = 0; i < 32; ++i) {
    const uint32_t p = (uint32_t)i * b, k = p >> 5, s = p & 31u;
    e[i] = __funnelshift_r(w[k], w[k + 1], s) & m;
  }
}

#define TP_CASE(B) \
  case B:          \
    unpack_fixed<B>(w, e); break;

// Warp-cooperative dispatch: the warp runs the specialised routine once per
// distinct bitwidth among its lanes (one pass when the column's miniblocks share b,
// the common case; a few passes for sorted-delta or run-length streams).  A lane whose
// miniblock is empty (b = 0: every offset 0) rides along with the first pass of another width
// and zeroes its offsets afterwards -- a delta stream mixing {0, B} (sorted keys, D1) takes one
// pass, not two.
#ifndef TP_UNPACK_MAX_PASSES
#define TP_UNPACK_MAX_PASSES 2
#endif
__device__ __forceinline__ void unpack_mb(const uint32_t* __restrict__ w, uint32_t b, uint32_t (&e)[32]) {
  const uint32_t bmin = __reduce_min_sync(FULL, b), bmax = __reduce_max_sync(FULL, b);
  const bool uniform = bmin == bmax;  // one width across the warp (the common case): one pass
  uint32_t todo = FULL, ride = 0u, zl = 0u;
  if (!uniform) {
    zl = __ballot_sync(FULL, b == 0u);
    todo = zl == FULL ? FULL : ~zl;  // the non-empty lanes (or all of them, if all empty)
    ride = zl == FULL ? 0u : zl;     // empty lanes joining the first pass
#if TP_UNPACK_MAX_PASSES < 32
    // more distinct bitwidths than TP_UNPACK_MAX_PASSES among the lanes (delta streams of
    // near-sorted keys): one runtime-bitwidth pass beats several specialised ones
    uint32_t t = todo;
#pragma unroll
    for (int k = 0; k < TP_UNPACK_MAX_PASSES; ++k) {
      const uint32_t bl = __shfl_sync(FULL, b, __ffs(t) - 1);
      t &= ~__ballot_sync(FULL, b == bl);
      if (t == 0u) break;  // (warp-uniform)
    }
    if (t) {
      unpack_any(w, b, e);
      return;
    }
#endif
  }
  do {
    const uint32_t bl = uniform ? bmin : __shfl_sync(FULL, b, __ffs(todo) - 1);
    const bool mine = b == bl || ((ride >> (threadIdx.x & 31u)) & 1u);
    todo &= ~__ballot_sync(FULL, b == bl);
    ride = 0u;
    if (mine) {
      switch (bl) {
        TP_CASE(0) TP_CASE(1) TP_CASE(2) TP_CASE(3) TP_CASE(4) TP_CASE(5) TP_CASE(6) TP_CASE(7)
        TP_CASE(8) TP_CASE(9) TP_CASE(10) TP_CASE(11) TP_CASE(12) TP_CASE(13) TP_CASE(14) TP_CASE(15)
        TP_CASE(16) TP_CASE(17) TP_CASE(18) TP_CASE(19) TP_CASE(20) TP_CASE(21) TP_CASE(22) TP_CASE(23)
        TP_CASE(24) TP_CASE(25) TP_CASE(26) TP_CASE(27) TP_CASE(28) TP_CASE(29) TP_CASE(30) TP_CASE(31)
        default: unpack_fixed<32>(w, e); break;
      }
    }
  } while (todo);
  if (zl != 0u && zl != FULL && b == 0u) {  // the riders read a neighbour's words
#pragma unroll
    for (int i = 0; i < 32; ++i) e[i] = 0u;
  }
}
#undef TP_CASE

// Sum of the 32 unpacked offsets e_i of one miniblock (the decode->sum consumer
// adds 32*ref once: sum(ref + e_i) = 32*ref + sum(e_i), exact in int64 because
// every real value is ref + e_i without wrap, R4).  32-bit partial sums are
// exact for B <= 27 (32 * (2^27 - 1) < 2^32).
template <int B>
__device__ __forceinline__ uint64_t sum_fixed(const uint32_t* __restrict__ w) {
  uint32_t e[32];
  unpack_fixed<B>(w, e);
  if constexpr (B <= 27) {
    uint32_t s = 0;  // (four independent partial sums measured no faster: the compiler's IADD3 tree)
#pragma unroll
    for (int i = 0; i < 32; ++i) s += e[i];
    return s;
  } else {
    uint64_t s = 0;
#pragma unroll
    for (int i = 0; i < 32; ++i) s += e[i];
    return s;
  }
}

#define TP_SCASE(B) \
  case B:           \
    r = sum_fixed<B>(w); break;

#ifndef TP_UNIFORM_FASTPATH
#define TP_UNIFORM_FASTPATH 1
#endif
__device__ __forceinline__ uint64_t sum_mb(const uint32_t* __restrict__ w, uint32_t b) {
  uint64_t r = 0;
#if TP_UNIFORM_FASTPATH
  const uint32_t bmin = __reduce_min_sync(FULL, b), bmax = __reduce_max_sync(FULL, b);
  if (bmin == bmax) {
    switch (bmin) {
      TP_SCASE(0) TP_SCASE(1) TP_SCASE(2) TP_SCASE(3) TP_SCASE(4) TP_SCASE(5) TP_SCASE(6) TP_SCASE(7)
      TP_SCASE(8) TP_SCASE(9) TP_SCASE(10) TP_SCASE(11) TP_SCASE(12) TP_SCASE(13) TP_SCASE(14) TP_SCASE(15)
      TP_SCASE(16) TP_SCASE(17) TP_SCASE(18) TP_SCASE(19) TP_SCASE(20) TP_SCASE(21) TP_SCASE(22) TP_SCASE(23)
      TP_SCASE(24) TP_SCASE(25) TP_SCASE(26) TP_SCASE(27) TP_SCASE(28) TP_SCASE(29) TP_SCASE(30) TP_SCASE(31)
      default: r = sum_fixed<32>(w); break;
    }
    return r;
  }
#endif
  uint32_t todo = FULL;
  do {
    const uint32_t bl = __shfl_sync(FULL, b, __ffs(todo) - 1);
    const bool mine = b == bl;
    todo &= ~__ballot_sync(FULL, mine);
    if (mine) {
      switch (bl) {
        TP_SCASE(0) TP_SCASE(1) TP_SCASE(2) TP_SCASE(3) TP_SCASE(4) TP_SCASE(5) TP_SCASE(6) TP_SCASE(7)
        TP_SCASE(8) TP_SCASE(9) TP_SCASE(10) TP_SCASE(11) TP_SCASE(12) TP_SCASE(13) TP_SCASE(14) TP_SCASE(15)
        TP_SCASE(16) TP_SCASE(17) TP_SCASE(18) TP_SCASE(19) TP_SCASE(20) TP_SCASE(21) TP_SCASE(22) TP_SCASE(23)
        TP_SCASE(24) TP_SCASE(25) TP_SCASE(26) TP_SCASE(27) TP_SCASE(28) TP_SCASE(29) TP_SCASE(30) TP_SCASE(31)
        default: r = sum_fixed<32>(w); break;
      }
    }
  } while (todo);
  return r;
}
// two miniblocks per lane (rounds r, r + 1): one dispatch when all 64 share a bitwidth, the two
// unpack-and-sum bodies straight-line so that their loads and shifts interleave
#define TP_SCASE2(B) \
  case B:            \
    r = sum_fixed<B>(w0) + sum_fixed<B>(w1); break;
__device__ __forceinline__ uint64_t sum_mb2(const uint32_t* __restrict__ w0, uint32_t b0,
                                            const uint32_t* __restrict__ w1, uint32_t b1) {
  const uint32_t bmin = __reduce_min_sync(FULL, min(b0, b1)), bmax = __reduce_max_sync(FULL, max(b0, b1));
  uint64_t r = 0;
  if (bmin == bmax) {
    switch (bmin) {
      TP_SCASE2(0) TP_SCASE2(1) TP_SCASE2(2) TP_SCASE2(3) TP_SCASE2(4) TP_SCASE2(5) TP_SCASE2(6) TP_SCASE2(7)
      TP_SCASE2(8) TP_SCASE2(9) TP_SCASE2(10) TP_SCASE2(11) TP_SCASE2(12) TP_SCASE2(13) TP_SCASE2(14) TP_SCASE2(15)
      TP_SCASE2(16) TP_SCASE2(17) TP_SCASE2(18) TP_SCASE2(19) TP_SCASE2(20) TP_SCASE2(21) TP_SCASE2(22) TP_SCASE2(23)
      TP_SCASE2(24) TP_SCASE2(25) TP_SCASE2(26) TP_SCASE2(27) TP_SCASE2(28) TP_SCASE2(29) TP_SCASE2(30) TP_SCASE2(31)
      default: r = sum_fixed<32>(w0) + sum_fixed<32>(w1); break;
    }
    return r;
  }
  return sum_mb(w0, b0) + sum_mb(w1, b1);
}
#undef TP_SCASE2
#undef TP_SCASE

// sum of the bitwidth bytes below byte j of one bitwidth word (Opt. 3, P:900-918:
// the miniblock offset is an exclusive prefix sum over the bitwidth bytes)
__device__ __forceinline__ uint32_t bw_prefix(uint32_t bw, uint32_t j) {
  const uint32_t low = bw & ((1u << (8u * j)) - 1u);  // j <= 3
  return (low * 0x01010101u) >> 24;
}

// ------------------------------------------------------------------ stage geometry
// Word index of global word g of a stream inside the stage's shared region, given
// the stage's first copied global word `lo`: the copy starts at the 16-byte
// aligned address at or below &data[lo].
__device__ __forceinline__ uint32_t align_shift(const uint32_t* base, uint32_t idx) {
  return (uint32_t)((reinterpret_cast<uintptr_t>(base + idx) & 15u) >> 2);
}

// Per-thread view of its miniblock of one column in the current stage.
struct MbView {
  const uint32_t* w;  // first word of the miniblock (shared memory)
  uint32_t ref;
  uint32_t b;
  bool valid;         // the miniblock exists (block index < nblocks)
};

// GPU-FOR / GPU-DFOR blocks: [ref][bw word][mb0..mb3] (Fig. 3).
// `tile_local` = tile index inside the stage, `blk` = block of the tile, `j` = mb.
__device__ __forceinline__ MbView for_view(const uint32_t* sd, const uint32_t* ss, uint32_t lo,
                                           uint32_t dshift, uint32_t sshift, uint32_t gblock,
                                           uint32_t nblocks, uint32_t local_block, uint32_t j) {
  MbView v;
  v.valid = gblock < nblocks;
  if (v.valid) {
    const uint32_t bs = ss[sshift + local_block];  // block_starts[block]
    const uint32_t* blk = sd + (bs - lo + dshift);
    v.ref = blk[0];                                 // reference (Alg. 1 line 3)
    const uint32_t bw = blk[1];                     // bitwidth word (line 6)
    v.b = checked_bw((bw >> (8u * j)) & 255u);      // line 11
    v.w = blk + 2u + bw_prefix(bw, j);              // lines 13-14 (header_offset = 2)
  } else {
    v.ref = 0u; v.b = 0u; v.w = sd;
  }
  return v;
}

// ------------------------------------------------------------------ scans
// inclusive scan across groups of 16 lanes (one 512-row tile = 16 miniblocks)
__device__ __forceinline__ uint32_t seg16_inclusive_scan(uint32_t x) {
  const uint32_t lane = threadIdx.x & 31u;
#pragma unroll
  for (int d = 1; d < 16; d <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, x, d, 16);
    if ((lane & 15u) >= (uint32_t)d) x += y;
  }
  return x;
}

}  // namespace tp
