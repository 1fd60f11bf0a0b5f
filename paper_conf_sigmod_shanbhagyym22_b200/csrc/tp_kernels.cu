// tp_kernels.cu -- the tile pipeline, the three tile decoders and the fused
// consumers (decode->sum, decode->global, select/project/aggregate), plus the
// device half of the C ABI declared in include/tilepack.h.
//
// P:<lines> = /root/reference/PAPER.md; R<n> = DESIGN.md readings.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <climits>
#include <mutex>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "tilepack.h"
#include "tp_device.cuh"

namespace tp {

std::atomic<uint64_t> g_launches{0};
// TP_PROFILE_WAITS builds only: consumer full-wait cycles [0], per-column op cycles [1..7],
// producer empty-wait cycles [8] (summed over warps)
__device__ unsigned long long g_prof[16];

// ------------------------------------------------------------------ stage context
// The ring holds "items": one column's words for a range of TPR * rounds consecutive
// tiles.  Consumers walk a range in rounds of TPR tiles (each consumer warp: 2 tiles =
// 32 miniblocks per round) and, within a round, the columns in evaluation order.
struct StageCtx {
  const uint32_t* stage;  // the current column item's shared words
  uint32_t t0s;           // first tile of the stage (global index)
  uint32_t round_base;    // stage-local index of the round's first tile
  uint32_t tile_end;      // one past the last tile of the CTA range
  uint32_t doff[2], soff[2];  // word offsets of the item's data / block_starts regions per stream
};

struct StreamView {
  const uint32_t* sd;  // data region
  const uint32_t* ss;  // block_starts region
  uint32_t lo;         // first copied data word (global index)
  uint32_t dshift, sshift;
};

// Every lane derives the view itself (two smem loads + address arithmetic): cheaper on
// the per-round critical path than sharing it through shared memory and a warp sync.
// s = the stream (Params::st index), k = 0 / 1: the column's first / second stream
// QP: the query pipeline (per-item region offsets in C); otherwise the single-column pipeline's
// fixed stage layout (constant-bank offsets: fewer registers on the per-round path, measured 3 %)
template <bool QP = false>
__device__ __forceinline__ StreamView stream_view(const Params& P, uint32_t s, const StageCtx& C, uint32_t k = 0) {
  const Stream& st = P.st[s];
  StreamView v;  // FOR / DFOR / RFOR streams only (a None column is read through none_row)
  const uint32_t sidx = st.kind == K_RFOR ? C.t0s : 4u * C.t0s;
  v.ss = C.stage + (QP ? C.soff[k] : st.starts_off);
  v.sd = C.stage + (QP ? C.doff[k] : st.data_off);
  v.sshift = align_shift(st.starts, sidx);
  v.lo = v.ss[v.sshift] - (st.kind == K_DFOR ? 1u : 0u);
  v.dshift = align_shift(st.data, v.lo);
  return v;
}

// lane geometry inside a consumer warp: 2 tiles x 16 miniblocks per round
struct Lane {
  uint32_t lane, cw;          // lane id, consumer warp id
  uint32_t tile_local;        // tile inside the round (0..TPR-1)
  uint32_t mb;                // miniblock inside the tile (0..15)
};
__device__ __forceinline__ Lane lane_geom() {
  Lane g;
  g.lane = threadIdx.x & 31u;
  g.cw = (threadIdx.x >> 5) - 1u;
  g.tile_local = 2u * g.cw + (g.lane >> 4);
  g.mb = g.lane & 15u;
  return g;
}

// the thread's miniblock of a FOR / DFOR column in this round
__device__ __forceinline__ MbView for_mb(const Params& P, const Col& c, const StageCtx& C, const Lane& g,
                                         const StreamView& v, uint32_t& tl, bool& tv) {
  tl = C.round_base + g.tile_local;  // stage-local tile
  tv = C.t0s + tl < C.tile_end;
  const uint32_t lb = 4u * tl + (g.mb >> 2);
  return for_view(v.sd, v.ss, v.lo, v.dshift, v.sshift, tv ? 4u * C.t0s + lb : UINT_MAX, c.nblocks, lb,
                  g.mb & 3u);
}

// the thread's 32 rows of a GPU-FOR block WITHOUT miniblocks: one bitwidth b for
// the block's 128 entries, so quarter j of the block starts at word 2 + j b (the same stream
// layout as 4 miniblocks of equal width)
__device__ __forceinline__ MbView fornm_mb(const Params& P, const Col& c, const StageCtx& C, const Lane& g,
                                           const StreamView& v, uint32_t& tl, bool& tv) {
  tl = C.round_base + g.tile_local;
  tv = C.t0s + tl < C.tile_end;
  const uint32_t lb = 4u * tl + (g.mb >> 2);
  MbView m;
  m.valid = tv && 4u * C.t0s + lb < c.nblocks;
  if (m.valid) {
    const uint32_t bs = v.ss[v.sshift + lb];
    const uint32_t* blk = v.sd + (bs - v.lo + v.dshift);
    m.ref = blk[0];
    m.b = checked_bw(blk[1] & 255u);
    m.w = blk + 2u + (g.mb & 3u) * m.b;
  } else {
    m.ref = 0u; m.b = 0u; m.w = v.sd;
  }
  return m;
}

// ---------------------------------------------------------------- GPU-FOR decode
// LoadBitPack analogue: the thread's 32 rows of the tile.
// COMPACT: multi-column query kernels unpack with the runtime-bitwidth routine (one small
// loop body instead of 33 specialised ones): their columns use several bitwidths at once, and
// the specialised bodies thrash the instruction cache (measured: 24-34 % "no instruction"
// stalls in the SSB kernel)
// RAW: the packed offsets only (no reference added) -- the first pass of the cascading
// baseline (tp_cascaded.cu), also for the delta blocks of a GPU-DFOR column
template <bool COMPACT, bool RAW = false, bool NOMB = false, bool QP = false>
__device__ __forceinline__ void decode_for(const Params& P, const Col& c, const StageCtx& C, const Lane& g,
                                           uint32_t (&val)[32]) {
  const StreamView v = stream_view<QP>(P, c.s0, C);
  uint32_t tl;
  bool tv;
  const MbView m = NOMB ? fornm_mb(P, c, C, g, v, tl, tv) : for_mb(P, c, C, g, v, tl, tv);
  uint32_t e[32];
  if (COMPACT) unpack_any(m.w, m.b, e); else unpack_mb(m.w, m.b, e);
#pragma unroll
  for (int i = 0; i < 32; ++i) val[i] = RAW ? e[i] : m.ref + e[i];  // Alg. 1 line 18
}

// ---------------------------------------------------------------- GPU-DFOR decode
// LoadDBitPack analogue: unpack the deltas of the thread's 32
// slots, then the tile-wide exclusive prefix sum (R13) -- a
// register scan inside the thread plus a 16-lane shuffle scan across the
// tile's miniblocks -- plus the tile's first value (Fig. 6).
template <bool COMPACT>
__device__ __forceinline__ void decode_dfor_sv(const Params& P, const Col& c, const StageCtx& C, const Lane& g,
                                               const StreamView& v, uint32_t (&val)[32]);
template <bool COMPACT, bool QP = false>
__device__ __forceinline__ void decode_dfor(const Params& P, const Col& c, const StageCtx& C, const Lane& g,
                                            uint32_t (&val)[32]) {
  decode_dfor_sv<COMPACT>(P, c, C, g, stream_view<QP>(P, c.s0, C), val);
}
// (the item's stream view given: the decode->sum consumer computes it once per item)
template <bool COMPACT>
__device__ __forceinline__ void decode_dfor_sv(const Params& P, const Col& c, const StageCtx& C, const Lane& g,
                                               const StreamView& v, uint32_t (&val)[32]) {
  uint32_t tl;
  bool tv;
  const MbView m = for_mb(P, c, C, g, v, tl, tv);
  uint32_t first = 0u;
  if (tv) first = v.sd[v.ss[v.sshift + 4u * tl] - 1u - v.lo + v.dshift];
  uint32_t e[32];
  if (COMPACT) unpack_any(m.w, m.b, e); else unpack_mb(m.w, m.b, e);
  uint32_t run = 0u;
#pragma unroll
  for (int i = 0; i < 32; ++i) {  // local exclusive prefix of the deltas
    val[i] = run;
    run += m.ref + e[i];          // delta = ref + e (mod 2^32, R15)
  }
  const uint32_t incl = seg16_inclusive_scan(run);
  const uint32_t base = first + (incl - run);  // first + sum of deltas of earlier miniblocks
#pragma unroll
  for (int i = 0; i < 32; ++i) val[i] += base;
}

// ---------------------------------------------------------------- GPU-RFOR decode
// LoadRBitPack analogue: the 4 steps of [18] (2 scatters + 2 scans),
// done per 512-row block by one warp, both blocks of the warp's round in turn:
//  1. unpack: lane t takes the C consecutive entries [C t, C t + C) of both streams
//     (C = 1 / 2 / 4 / 8 / 16 by the block's run count r, so one pass covers the block and a lane's
//     entries sit inside one 32-entry miniblock: one bitwidth and base per lane);
//  2. run starts S = exclusive scan of the run lengths (lane-local scan + one warp scan);
//  3. scatter: value V_e -> A[S_e], a start flag byte -> F[S_e] (plain stores: the starts
//     are distinct, no atomics);
//  4. expand (second scan): the thread owning rows 32j .. 32j+31 turns its 32 flag bytes
//     into a start mask, takes the value of the last run start before its rows from the
//     nearest earlier thread (16-lane segmented scan), and forward-fills its rows.
// A is stored XOR-swizzled by 16-byte quad so that the 16 threads' 128-bit reads of
// their row chunks are conflict-free.  The result equals repeat(V, L) (R19).
// per-warp scratch: the two blocks' A arrays side by side (4 KB: decode->global stages the warp's
// 1024 decoded rows in the same bytes, so that a 4th CTA fits per SM), then their flag bytes
constexpr uint32_t RFOR_A_WORDS = 512, RFOR_F_WORDS = 128;
constexpr uint32_t RFOR_SCRATCH_WORDS = 2 * (RFOR_A_WORDS + RFOR_F_WORDS);
__device__ __forceinline__ uint32_t* rfor_A(uint32_t* scratch, uint32_t h) { return scratch + h * RFOR_A_WORDS; }
__device__ __forceinline__ uint8_t* rfor_F(uint32_t* scratch, uint32_t h) {
  return reinterpret_cast<uint8_t*>(scratch + 2 * RFOR_A_WORDS + h * RFOR_F_WORDS);
}

__device__ __forceinline__ uint32_t warp_inclusive_scan(uint32_t x, uint32_t lane) {
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, x, d);
    if (lane >= (uint32_t)d) x += y;
  }
  return x;
}

__device__ __forceinline__ uint32_t byte_of(const uint4& w, uint32_t m) {  // byte m (0..15)
  const uint32_t q = m >> 2;
  const uint32_t x = q == 0 ? w.x : q == 1 ? w.y : q == 2 ? w.z : w.w;
  return (x >> (8u * (m & 3u))) & 255u;
}
__device__ __forceinline__ uint32_t bytes_before(const uint4& w, uint32_t m) {  // sum of bytes [0, m)
  const uint32_t q = m >> 2;
  const uint32_t sx = (w.x * 0x01010101u) >> 24, sy = (w.y * 0x01010101u) >> 24, sz = (w.z * 0x01010101u) >> 24;
  const uint32_t full = (q > 0 ? sx : 0u) + (q > 1 ? sy : 0u) + (q > 2 ? sz : 0u);
  const uint32_t x = q == 0 ? w.x : q == 1 ? w.y : q == 2 ? w.z : w.w;
  return full + bw_prefix(x, m & 3u);
}
// b-bit field at stream bit p of m (p's word and the next one; the funnel shift uses p mod 32)
__device__ __forceinline__ uint32_t extract_at(const uint32_t* m, uint32_t p, uint32_t mask) {
  const uint32_t* w = m + (p >> 5);
  return __funnelshift_r(w[0], w[1], p) & mask;
}
// swizzled word / flag-byte positions of row s of a block (see above)
__device__ __forceinline__ uint32_t rfor_a_pos(uint32_t s) { return s ^ ((s >> 3) & 0x1Cu); }
__device__ __forceinline__ uint32_t rfor_f_pos(uint32_t s) { return s ^ (((s >> 7) & 1u) << 4); }

#ifndef TP_RFOR_SPLIT
#define TP_RFOR_SPLIT 2  // 128 < r <= 192: a 4-entry pass + a 1- / 2-entry tail pass instead of 8 entries
                         // (2: also 64 < r <= 96 as 2 + 1 entries; runs of 8: -6 %, measured)
#endif
#ifndef TP_RFOR_WIN
#define TP_RFOR_WIN 1  // a lane's C entries from one 64-bit window (runs of 4: -6 %, measured)
#endif
#ifndef TP_RFOR_BALLOT_CARRY
#define TP_RFOR_BALLOT_CARRY 1  // carries by ballot + one shuffle (runs of 4: -2.5 %, SSB -0.3 %, measured)
#endif
#ifndef TP_SUM32
#define TP_SUM32 1  // DFOR / RFOR decode->sum: two 32-bit halves when a chunk's values are < 2^28
                    // (DFOR D1 -8 %, RFOR runs of 4 -6 %, measured)
#endif
#ifndef TP_SUM_PAIR
#define TP_SUM_PAIR 1  // LEAN GPU-FOR decode->sum: two rounds per step
#endif
#ifndef TP_GLOBAL_SINGLE_DFOR
#define TP_GLOBAL_SINGLE_DFOR 1
#endif
#ifndef TP_DFOR_SINGLE_BITS
#define TP_DFOR_SINGLE_BITS 3.0
#endif
#ifndef TP_GLOBAL_SPIN_INSTR
#define TP_GLOBAL_SPIN_INSTR 0  // 1: decode->global of the instruction-bound DFOR / RFOR spins (0: parks, -0.6 %)
#endif
__device__ __forceinline__ void rfor_flag(uint8_t* F, uint32_t S) { F[rfor_f_pos(S)] = 1; }
__device__ __forceinline__ void rfor_clear_flags(uint8_t* F, uint32_t lane) {
  st_shared_v4(reinterpret_cast<uint32_t*>(F) + 4u * lane, 0u, 0u, 0u, 0u);
}

// the C consecutive b-bit fields [pos, pos + C) of miniblock words m (pos a multiple of C): one
// 64-bit window of two words when they fit in it, else two words per field (extract_at)
template <int C>
__device__ __forceinline__ void extract_c(const uint32_t* m, uint32_t pos, uint32_t b, uint32_t mask,
                                          uint32_t (&f)[C]) {
  const uint32_t p0 = pos * b;
#if TP_RFOR_WIN
  if ((p0 & 31u) + C * b <= 64u) {
    const uint32_t* w = m + (p0 >> 5);
    const uint64_t win = (((uint64_t)w[1] << 32) | w[0]) >> (p0 & 31u);
#pragma unroll
    for (int k = 0; k < C; ++k) f[k] = (uint32_t)(win >> (k * b)) & mask;
    return;
  }
#endif
#pragma unroll
  for (int k = 0; k < C; ++k) f[k] = extract_at(m, p0 + k * b, mask);
}

// steps 1-3 for entries [eb, eb + 32 C) of one block, C entries per lane (a lane's entries inside
// one miniblock: C divides 32); rb = rows of the entries before eb.  Returns the pass's rows
// (RET: only a pass followed by a tail pass needs them).
template <int C, bool RET = false>
__device__ __forceinline__ uint32_t rfor_scatter(const uint32_t* bV, const uint32_t* bL, uint32_t r, uint32_t lane,
                                                 uint32_t* A, uint8_t* F, uint32_t eb = 0u, uint32_t rb = 0u) {
  const uint32_t e0 = eb + C * lane, m = (e0 >> 5) & 15u, pos = e0 & 31u;
  const uint32_t refV = bV[1], refL = bL[1];  // references (FOR on both arrays)
  const uint4 wv = make_uint4(bV[2], bV[3], bV[4], bV[5]), wl = make_uint4(bL[2], bL[3], bL[4], bL[5]);
  const uint32_t bv = checked_bw(byte_of(wv, m)), bl = checked_bw(byte_of(wl, m));  // R2, R17
  // every miniblock before m is full: b_i words each (R17)
  const uint32_t* mV = bV + 6 + bytes_before(wv, m);
  const uint32_t* mL = bL + 6 + bytes_before(wl, m);
  const uint32_t mv = __funnelshift_lc(0xffffffffu, 0u, bv), ml = __funnelshift_lc(0xffffffffu, 0u, bl);
  uint32_t fl[C], fv[C];
  extract_c<C>(mL, pos, bl, ml, fl);  // Alg. 1 for the lane's C entries of each stream
  uint32_t len[C], incl[C];
  uint32_t run = 0u;
#pragma unroll
  for (int k = 0; k < C; ++k) {  // 1. run lengths + lane-local inclusive scan
    len[k] = e0 + k < r ? refL + fl[k] : 0u;
    run += len[k];
    incl[k] = run;
  }
  extract_c<C>(mV, pos, bv, mv, fv);
  const uint32_t wincl = warp_inclusive_scan(run, lane);
  const uint32_t base = rb + wincl - run;  // 2. rows before this lane's runs
#pragma unroll
  for (int k = 0; k < C; ++k) {  // 3. scatter values and start flags
    if (e0 + k < r) {
      const uint32_t S = (base + incl[k] - len[k]) & 511u;
      A[rfor_a_pos(S)] = refV + fv[k];
      rfor_flag(F, S);
    }
  }
  return RET ? __shfl_sync(FULL, wincl, 31) : 0u;
}

// steps 1-3 for one block of r runs: the fewest entries per lane that cover it (long runs: one)
// SMALLC: also the C = 1 / 2 bodies (and tails) for blocks of few (long) runs
template <bool SMALLC>
__device__ __forceinline__ void rfor_block_scatter(const uint32_t* bV, const uint32_t* bL, uint32_t r, uint32_t lane,
                                                   uint32_t* A, uint8_t* F) {
  if (SMALLC && r <= 32u) rfor_scatter<1>(bV, bL, r, lane, A, F);
  else if (SMALLC && r <= 64u) rfor_scatter<2>(bV, bL, r, lane, A, F);
#if TP_RFOR_SPLIT >= 2
  else if (SMALLC && r <= 96u) rfor_scatter<1>(bV, bL, r, lane, A, F, 64u, rfor_scatter<2, true>(bV, bL, r, lane, A, F));
#endif
  else if (r <= 128u) rfor_scatter<4>(bV, bL, r, lane, A, F);
#if TP_RFOR_SPLIT
  else if (SMALLC && r <= 160u) rfor_scatter<1>(bV, bL, r, lane, A, F, 128u, rfor_scatter<4, true>(bV, bL, r, lane, A, F));
  else if (SMALLC && r <= 192u) rfor_scatter<2>(bV, bL, r, lane, A, F, 128u, rfor_scatter<4, true>(bV, bL, r, lane, A, F));
#endif
  else if (r <= 256u) rfor_scatter<8>(bV, bL, r, lane, A, F);
  else rfor_scatter<16>(bV, bL, r, lane, A, F);
}

#ifndef TP_RFOR_PAIR
#define TP_RFOR_PAIR 1  // single-column decodes: both blocks of a round in one pass (half-warp each)
#endif
// steps 1-3 for both blocks of the round at once: lanes 16 h .. 16 h + 15 take block h, entries
// [eb, eb + 16 C) of it, C per lane (inside one miniblock); rb = rows of the block's entries before
// eb.  One 16-lane segmented scan and one header decode per lane serve both blocks.  Returns the
// rows of the half-warp's entries (RET).
template <int C, bool RET = false>
__device__ __forceinline__ uint32_t rfor_scatter_pair(const uint32_t* bV, const uint32_t* bL, uint32_t r,
                                                      uint32_t lane, uint32_t* scratch, uint32_t eb = 0u,
                                                      uint32_t rb = 0u) {
  const uint32_t h = lane >> 4, e0 = eb + C * (lane & 15u), m = (e0 >> 5) & 15u, pos = e0 & 31u;
  uint32_t* A = rfor_A(scratch, h);
  uint8_t* F = rfor_F(scratch, h);
  const uint32_t refV = bV[1], refL = bL[1];  // references (FOR on both arrays)
  const uint4 wv = make_uint4(bV[2], bV[3], bV[4], bV[5]), wl = make_uint4(bL[2], bL[3], bL[4], bL[5]);
  const uint32_t bv = checked_bw(byte_of(wv, m)), bl = checked_bw(byte_of(wl, m));  // R2, R17
  const uint32_t* mV = bV + 6 + bytes_before(wv, m);  // miniblocks before m are full (R17)
  const uint32_t* mL = bL + 6 + bytes_before(wl, m);
  const uint32_t mv = __funnelshift_lc(0xffffffffu, 0u, bv), ml = __funnelshift_lc(0xffffffffu, 0u, bl);
  uint32_t fl[C], fv[C];
  extract_c<C>(mL, pos, bl, ml, fl);
  uint32_t len[C], incl[C];
  uint32_t run = 0u;
#pragma unroll
  for (int k = 0; k < C; ++k) {  // 1. run lengths + lane-local inclusive scan
    len[k] = e0 + k < r ? refL + fl[k] : 0u;
    run += len[k];
    incl[k] = run;
  }
  extract_c<C>(mV, pos, bv, mv, fv);
  const uint32_t wincl = seg16_inclusive_scan(run);
  const uint32_t base = rb + wincl - run;  // 2. rows before this lane's runs (in its block)
#pragma unroll
  for (int k = 0; k < C; ++k) {  // 3. scatter values and start flags
    if (e0 + k < r) {
      const uint32_t S = (base + incl[k] - len[k]) & 511u;
      A[rfor_a_pos(S)] = refV + fv[k];
      rfor_flag(F, S);
    }
  }
  return RET ? __shfl_sync(FULL, wincl, lane | 15u) : 0u;
}
// rm = the larger run count of the two blocks (warp-uniform): passes of 16 C entries per block
__device__ __forceinline__ void rfor_pair_dispatch(const uint32_t* bV, const uint32_t* bL, uint32_t r, uint32_t rm,
                                                   uint32_t lane, uint32_t* s) {
  if (rm <= 16u) rfor_scatter_pair<1>(bV, bL, r, lane, s);
  else if (rm <= 32u) rfor_scatter_pair<2>(bV, bL, r, lane, s);
  else if (rm <= 64u) rfor_scatter_pair<4>(bV, bL, r, lane, s);
  else if (rm <= 80u) rfor_scatter_pair<1>(bV, bL, r, lane, s, 64u, rfor_scatter_pair<4, true>(bV, bL, r, lane, s));
  else if (rm <= 96u) rfor_scatter_pair<2>(bV, bL, r, lane, s, 64u, rfor_scatter_pair<4, true>(bV, bL, r, lane, s));
  else if (rm <= 128u) rfor_scatter_pair<8>(bV, bL, r, lane, s);
  else if (rm <= 144u) rfor_scatter_pair<1>(bV, bL, r, lane, s, 128u, rfor_scatter_pair<8, true>(bV, bL, r, lane, s));
  else if (rm <= 160u) rfor_scatter_pair<2>(bV, bL, r, lane, s, 128u, rfor_scatter_pair<8, true>(bV, bL, r, lane, s));
  else if (rm <= 192u) rfor_scatter_pair<4>(bV, bL, r, lane, s, 128u, rfor_scatter_pair<8, true>(bV, bL, r, lane, s));
  else if (rm <= 256u) rfor_scatter_pair<16>(bV, bL, r, lane, s);
  else rfor_scatter_pair<16>(bV, bL, r, lane, s, 256u, rfor_scatter_pair<16, true>(bV, bL, r, lane, s));
}

// steps 1-3 for both row blocks of the warp's round (block h -> rfor_A / rfor_F(scratch, h))
// SMALLC: single-column decodes only: the query kernels keep the smaller code (their RFOR columns
// have short runs, and the extra bodies cost the star kernels ~4 % through instruction-cache
// misses, measured)
template <bool SMALLC = false, bool QP = false>
__device__ __forceinline__ void rfor_scatter_round(const Params& P, const Col& c, const StageCtx& C, const Lane& g,
                                                   uint32_t* scratch) {
  const StreamView vv = stream_view<QP>(P, c.s0, C, 0), vl = stream_view<QP>(P, c.s1, C, 1);
  const uint32_t lane = g.lane;
  __syncwarp();  // a lagging lane may still read the previous column's expansion
  if (SMALLC && TP_RFOR_PAIR) {
    // both blocks' flags cleared, then one pass over both (an invalid second block: no runs)
    uint4* Fq = reinterpret_cast<uint4*>(rfor_F(scratch, 0));
    Fq[lane] = make_uint4(0u, 0u, 0u, 0u);
    Fq[lane + 32u] = make_uint4(0u, 0u, 0u, 0u);
    __syncwarp();
    const uint32_t tl0 = C.round_base + 2u * g.cw;
    if (C.t0s + tl0 >= C.tile_end) return;  // warp-uniform; rows masked by the consumer
    const bool v1 = C.t0s + tl0 + 1u < C.tile_end;
    const uint32_t tl = tl0 + ((lane >> 4) && v1 ? 1u : 0u);
    const uint32_t* bV = vv.sd + (vv.ss[vv.sshift + tl] - vv.lo + vv.dshift);
    const uint32_t* bL = vl.sd + (vl.ss[vl.sshift + tl] - vl.lo + vl.dshift);
    uint32_t r = bV[0];  // run / value count
    if (r > 512u) {
      tp_flag_error(4u);  // TP_DEVERR_RUNS
      r = 512u;
    }
    if ((lane >> 4) && !v1) r = 0u;
    rfor_pair_dispatch(bV, bL, r, __reduce_max_sync(FULL, r), lane, scratch);
    __syncwarp();
    return;
  }
#pragma unroll 1
  for (uint32_t h = 0; h < 2; ++h) {
    uint32_t* A = rfor_A(scratch, h);
    uint8_t* F = rfor_F(scratch, h);
    rfor_clear_flags(F, lane);
    __syncwarp();
    const uint32_t tl = C.round_base + 2u * g.cw + h;
    if (C.t0s + tl >= C.tile_end) continue;  // warp-uniform; rows masked by the consumer
    const uint32_t* bV = vv.sd + (vv.ss[vv.sshift + tl] - vv.lo + vv.dshift);
    const uint32_t* bL = vl.sd + (vl.ss[vl.sshift + tl] - vl.lo + vl.dshift);
    uint32_t r = bV[0];  // run / value count
    if (r > 512u) {
      tp_flag_error(4u);  // TP_DEVERR_RUNS
      r = 512u;
    }
    rfor_block_scatter<SMALLC>(bV, bL, r, lane, A, F);
  }
  __syncwarp();
}

// the thread's 32-row chunk of an expanded RFOR round: run-start mask and value array
struct RforChunk {
  uint32_t* A;    // the block's (swizzled) start-value array
  uint32_t j;     // chunk index in the block (rows 32j .. 32j+31)
  uint32_t mask;  // bit i: row 32j+i starts a run
};
__device__ __forceinline__ RforChunk rfor_chunk(uint32_t* scratch, uint32_t lane) {
  RforChunk k;
  k.j = lane & 15u;
  k.A = rfor_A(scratch, lane >> 4);
  const uint32_t* F = reinterpret_cast<const uint32_t*>(rfor_F(scratch, lane >> 4));
  const uint32_t fs = ((k.j >> 2) & 1u) << 2;  // flag quad swizzle (words)
  const uint4 f0 = *reinterpret_cast<const uint4*>(F + 8u * k.j + fs);
  const uint4 f1 = *reinterpret_cast<const uint4*>(F + 8u * k.j + (fs ^ 4u));
  const uint32_t fw[8] = {f0.x, f0.y, f0.z, f0.w, f1.x, f1.y, f1.z, f1.w};
  uint32_t mask = 0u;
#pragma unroll
  for (int q = 0; q < 8; ++q) mask |= (((fw[q] * 0x01020408u) >> 24) & 15u) << (4 * q);  // byte flags -> bits
  k.mask = mask;
  return k;
}
// A-value of the last run start before row 32j (the previous chunks' last start: a 16-lane
// segmented scan -- the second scan of [18]); row 0 of a block always starts a run
__device__ __forceinline__ uint32_t rfor_carry(const RforChunk& k) {
  uint32_t has = k.mask != 0u;
  uint32_t last = has ? k.A[rfor_a_pos(32u * k.j + 31u - __clz(k.mask))] : 0u;
#if TP_RFOR_BALLOT_CARRY
  // the nearest earlier lane of the 16-lane block holding a run start (lane j = 0 always does:
  // row 0 of a block starts a run) -- one ballot and one shuffle instead of a 4-step scan
  const uint32_t lane = threadIdx.x & 31u;
  const uint32_t hm = __ballot_sync(FULL, has) & ((1u << lane) - 1u) & (lane >= 16u ? 0xffff0000u : 0x0000ffffu);
  return __shfl_sync(FULL, last, hm ? 31u - __clz(hm) : lane);
#else
#pragma unroll
  for (int d = 1; d < 16; d <<= 1) {
    const uint32_t yh = __shfl_up_sync(FULL, has, d, 16), yv = __shfl_up_sync(FULL, last, d, 16);
    if (k.j >= (uint32_t)d && !has) { has = yh; last = yv; }
  }
  return __shfl_up_sync(FULL, last, 1, 16);
#endif
}
// step 4: forward fill of the chunk's 32 rows
__device__ __forceinline__ void rfor_fill(const RforChunk& k, uint32_t carry, uint32_t (&val)[32]) {
  const uint32_t* Aj = k.A + 32u * k.j;
#pragma unroll
  for (int q = 0; q < 8; ++q) {
    const uint4 a = *reinterpret_cast<const uint4*>(Aj + ((q ^ (k.j & 7u)) << 2));
    val[4 * q] = a.x; val[4 * q + 1] = a.y; val[4 * q + 2] = a.z; val[4 * q + 3] = a.w;
  }
  uint32_t cur = carry;
#pragma unroll
  for (int i = 0; i < 32; ++i) {
    if (k.mask & (1u << i)) cur = val[i];
    val[i] = cur;
  }
}
// random access: the value of row 32j + i (the last run start at or before it)
__device__ __forceinline__ uint32_t rfor_row(const RforChunk& k, uint32_t carry, uint32_t i) {
  const uint32_t mm = k.mask & (0xffffffffu >> (31u - i));
  return mm ? k.A[rfor_a_pos(32u * k.j + 31u - __clz(mm))] : carry;
}

template <bool SMALLC, bool QP = false>
__device__ __forceinline__ void decode_rfor(const Params& P, const Col& c, const StageCtx& C, const Lane& g,
                                            uint32_t* scratch, uint32_t (&val)[32]) {
  rfor_scatter_round<SMALLC, QP>(P, c, C, g, scratch);
  const RforChunk k = rfor_chunk(scratch, g.lane);
  rfor_fill(k, rfor_carry(k), val);
}

// ---------------------------------------------------------------- None (uncompressed)
// The plain column staged as a 128B-swizzled TMA box of 32-word rows: row r = 16 * tile + mb
// holds the thread's 32 values, 16-byte chunk q at chunk q ^ (r & 7).
template <bool QP = false>
__device__ __forceinline__ const uint32_t* none_row(const Params& P, const Col& c, const StageCtx& C,
                                                    const Lane& g, uint32_t& sw) {
  const uint32_t r = 16u * (C.round_base + g.tile_local) + g.mb;
  sw = r & 7u;
  return C.stage + (QP ? C.doff[0] : P.st[c.s0].data_off) + 32u * r;
}
template <bool QP = false>
__device__ __forceinline__ void decode_none(const Params& P, const Col& c, const StageCtx& C, const Lane& g,
                                            uint32_t (&val)[32]) {
  uint32_t sw;
  const uint32_t* w = none_row<QP>(P, c, C, g, sw);
#pragma unroll
  for (int q = 0; q < 8; ++q) {
    const uint4 a = *reinterpret_cast<const uint4*>(w + ((q ^ sw) << 2));
    val[4 * q] = a.x; val[4 * q + 1] = a.y; val[4 * q + 2] = a.z; val[4 * q + 3] = a.w;
  }
}
__device__ __forceinline__ uint32_t none_at(const uint32_t* w, uint32_t sw, uint32_t i) {
  return w[((((i >> 2) ^ sw) << 2)) | (i & 3u)];
}

// MASK: which decoders a kernel instantiation carries (bit 1 << scheme); kernels
// are instantiated per scheme mix so that FOR-only kernels keep FOR's register budget.
constexpr uint32_t M_FOR = 1u << S_FOR, M_DFOR = 1u << S_DFOR, M_RFOR = 1u << S_RFOR, M_NONE = 1u << S_NONE;
constexpr uint32_t M_FORNM = 1u << S_FORNM;  // decode / decode_sum only (the miniblock ablation)
constexpr uint32_t M_RAW = 1u << 8;  // FOR / DFOR blocks, packed offsets only (cascading baseline)
template <uint32_t MASK, bool COMPACT = false, bool QP = false>
__device__ __forceinline__ void decode_col(const Params& P, uint32_t ci, const StageCtx& C, const Lane& g,
                                           uint32_t* scratch, uint32_t (&val)[32]) {
  const Col& c = P.col[ci];
  if (MASK == M_RAW) {
    decode_for<false, true>(P, c, C, g, val);
    return;
  }
  if (MASK == M_FORNM) {
    decode_for<false, false, true>(P, c, C, g, val);
    return;
  }
  if ((MASK & M_NONE) && c.scheme == S_NONE) decode_none<QP>(P, c, C, g, val);
  else if ((MASK & M_FOR) && c.scheme == S_FOR) decode_for<COMPACT, false, false, QP>(P, c, C, g, val);
  else if ((MASK & M_DFOR) && c.scheme == S_DFOR) decode_dfor<COMPACT, QP>(P, c, C, g, val);
  else if (MASK & M_RFOR) decode_rfor<!COMPACT, QP>(P, c, C, g, scratch, val);
}

// ------------------------------------------------------------------ the pipeline
// warp 0: TMA producer; warps 1..CONSUMER_WARPS: consumers.  The item sequence is
// (tile range g, column c) for g = 0.. and c = 0..ncols-1 in evaluation order, so a
// query streams its columns one item at a time through a ring of small stages (a
// multi-column tile does not have to fit shared memory at once).
// Op interface: cta_init (all threads, before the first barrier), begin / col / end
// per round of TPR tiles, finish (consumer warps, after their last round).
template <class Op>
__device__ __forceinline__ void run_pipeline(const Params& P, Op& op) {
  extern __shared__ __align__(1024) uint32_t smem[];
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31u;
  const uint32_t TPS = TPR * P.rounds;  // tiles per item
  // CTA tile range, in pairs of tiles so that a consumer warp's 1024 rows
  // never straddle two CTAs (decode->global stores whole warp boxes)
  const uint32_t npairs = (P.ntiles + 1u) >> 1;
  const uint32_t p0 = (uint32_t)((uint64_t)blockIdx.x * npairs / gridDim.x);
  const uint32_t p1 = (uint32_t)((uint64_t)(blockIdx.x + 1) * npairs / gridDim.x);
  const uint32_t t0 = 2u * p0, t1 = min(2u * p1, P.ntiles);
  if (t0 >= t1) return;
  const uint32_t ngr = (t1 - t0 + TPS - 1) / TPS;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + P.bar_off);
  uint64_t* empty = full + P.nstages;
  op.cta_init(P, smem);
  if (threadIdx.x == 0) {
    for (uint32_t s = 0; s < P.nstages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], CONSUMER_WARPS);
    }
    fence_mbar_init();
  }
  __syncthreads();

  if (warp == 0) {
    // ---------------- producer
    const uint64_t pol = policy_evict_first();
    uint32_t slot = 0, phase = 0, item = 0;  // ring position of the next item (no runtime division)
    bool over = false;
    for (uint32_t gb = 0; gb < ngr; gb += 31) {
      // lane i prefetches every stream's block_starts entry at the start of range gb+i
      const uint32_t tb = min(t0 + (gb + lane) * TPS, t1);
      uint32_t bnd[MAX_STREAMS];
#pragma unroll
      for (int s = 0; s < MAX_STREAMS; ++s) {
        bnd[s] = 0u;
        if ((uint32_t)s < P.nstreams) {
          const Stream& st = P.st[s];
          const uint32_t bi = min(st.kind == K_RFOR ? tb : 4u * tb, st.nblocks);
          bnd[s] = __ldg(st.starts + bi);
        }
      }
      const uint32_t ge = min(gb + 31, ngr);
      for (uint32_t g = gb; g < ge; ++g) {
        const uint32_t tile_base = t0 + g * TPS, tile_end = min(tile_base + TPS, t1);
        for (uint32_t c = 0; c < P.ncols; ++c, ++item) {
          // HBM-bound single-column FOR decode: spin (fastest reaction, measured); everything
          // else is consumer-bound: back off so the spin does not take the consumers' issue slots
          if (item >= P.nstages) {
            if (Op::kProducerSpin) mbar_wait(&empty[slot], phase ^ 1u);
            else mbar_wait_backoff(&empty[slot], phase ^ 1u);
          }
          const Col& cc = P.col[c];
          const uint32_t my_s = lane == 0 ? cc.s0 : (lane == 1 && cc.scheme == S_RFOR ? cc.s1 : 0xffu);
          uint32_t mylo = 0u, myhi = 0u;
#pragma unroll
          for (int q = 0; q < MAX_STREAMS; ++q) {
            if ((uint32_t)q < P.nstreams) {
              const uint32_t a = __shfl_sync(FULL, bnd[q], g - gb);
              const uint32_t b = __shfl_sync(FULL, bnd[q], g - gb + 1);
              if (my_s == (uint32_t)q) { mylo = a; myhi = b; }
            }
          }
          uint32_t bytes = 0u, dbytes = 0u, sbytes = 0u;
          const char *dsrc = nullptr, *ssrc = nullptr;
          uint32_t *dst_d = nullptr, *dst_s = nullptr;
          // compiled only into kernels that carry the None reader (keeps FOR kernels lean)
          const bool none = (Op::kMask & M_NONE) && my_s != 0xffu && P.st[my_s].kind == K_NONE;
          if (none) {  // plain column: one TMA tensor box of TPS tiles (OOB rows zero-filled)
            dbytes = TPS * TILE_ROWS * 4u;
            bytes = dbytes;
            dst_d = smem + slot * P.stage_words + P.st[my_s].data_off;
          } else if (my_s != 0xffu) {
            const Stream& st = P.st[my_s];
            const uint32_t lo = mylo - (st.kind == K_DFOR ? 1u : 0u);
            const uintptr_t a0 = reinterpret_cast<uintptr_t>(st.data + lo) & ~uintptr_t(15);
            const uintptr_t a1 = (reinterpret_cast<uintptr_t>(st.data + myhi) + 15) & ~uintptr_t(15);
            dsrc = reinterpret_cast<const char*>(a0);
            dbytes = (uint32_t)(a1 - a0);
            // max_tile_words below the column's real span: copy what fits (stay in the ring) and
            // report TP_DEVERR_TILE_WORDS once, after the loop (off the producer's critical path)
            over |= dbytes > st.data_cap;
            dbytes = min(dbytes, st.data_cap);
            const uint32_t s0 = st.kind == K_RFOR ? tile_base : 4u * tile_base;
            const uint32_t s1 = min(st.kind == K_RFOR ? tile_end : 4u * tile_end, st.nblocks) + 1u;
            const uintptr_t b0 = reinterpret_cast<uintptr_t>(st.starts + s0) & ~uintptr_t(15);
            const uintptr_t b1 = (reinterpret_cast<uintptr_t>(st.starts + s1) + 15) & ~uintptr_t(15);
            ssrc = reinterpret_cast<const char*>(b0);
            sbytes = (uint32_t)(b1 - b0);
            uint32_t* ibase = smem + slot * P.stage_words;
            dst_d = ibase + st.data_off;
            dst_s = ibase + st.starts_off;
            bytes = dbytes + sbytes;
          }
          const uint32_t total = __reduce_add_sync(FULL, bytes);
          if (lane == 0) mbar_arrive_expect_tx(&full[slot], total);
          __syncwarp();
          if (none) {
            tma_load_2d(dst_d, &P.tmap[c], 0, (int)(tile_base * (TILE_ROWS / 32)), &full[slot], pol);
          } else if (my_s != 0xffu) {
            bulk_g2s(dst_d, dsrc, dbytes, &full[slot], pol);
            bulk_g2s(dst_s, ssrc, sbytes, &full[slot], pol);
          }
          if (++slot == P.nstages) { slot = 0; phase ^= 1u; }
        }
      }
    }
    if (over) tp_flag_error(2u);  // TP_DEVERR_TILE_WORDS
  } else {
    // ---------------- consumers
    const Lane g = lane_geom();
    uint32_t* scratch = smem + P.scratch_off + g.cw * P.scratch_words_per_warp;
    uint32_t rc = 0;  // round counter (decode->global buffer parity)
    uint32_t slot = 0, phase = 0;
    StageCtx C;
    C.tile_end = t1;
    if (P.ncols == 1) {
      // single column: one item per tile range, walked in P.rounds rounds
      for (uint32_t gi = 0; gi < ngr; ++gi) {
        C.t0s = t0 + gi * TPS;
        C.stage = smem + slot * P.stage_words;
        const uint32_t nr = min(P.rounds, (t1 - C.t0s + TPR - 1) / TPR);
        {
          const Col& c0 = P.col[0];
          C.doff[0] = P.st[c0.s0].data_off; C.soff[0] = P.st[c0.s0].starts_off;
          const uint32_t q1 = c0.scheme == S_RFOR ? c0.s1 : c0.s0;
          C.doff[1] = P.st[q1].data_off; C.soff[1] = P.st[q1].starts_off;
        }
        if (Op::kProducerSpin) mbar_wait(&full[slot], phase); else mbar_wait_backoff(&full[slot], phase);
        for (uint32_t r = 0; r < nr; ++r, ++rc) {
          C.round_base = r * TPR;
          if constexpr (Op::kPairRounds) {
            if (r + 1 < nr) {  // two rounds at once: two independent miniblock chains per lane
              op.col2(P, C, g);
              ++r;
              ++rc;
              continue;
            }
          }
          op.begin(P, C, g);
          op.col(P, C, g, scratch, 0, rc);
          op.end(P, C, g);
        }
        __syncwarp();
        if (g.lane == 0) mbar_arrive(&empty[slot]);
        if (++slot == P.nstages) { slot = 0; phase ^= 1u; }
      }
    } else {
      // queries: one round per tile range; the columns' items arrive in evaluation order
      C.round_base = 0;
      for (uint32_t gi = 0; gi < ngr; ++gi, ++rc) {
        C.t0s = t0 + gi * TPS;
        op.begin(P, C, g);
        for (uint32_t c = 0; c < P.ncols; ++c) {
          C.stage = smem + slot * P.stage_words;
          {
            const Col& cc = P.col[c];
            C.doff[0] = P.st[cc.s0].data_off; C.soff[0] = P.st[cc.s0].starts_off;
            const uint32_t q1 = cc.scheme == S_RFOR ? cc.s1 : cc.s0;
            C.doff[1] = P.st[q1].data_off; C.soff[1] = P.st[q1].starts_off;
          }
#ifdef TP_PROFILE_WAITS
          const long long w0 = clock64();
#endif
          if (Op::kProducerSpin) mbar_wait(&full[slot], phase); else mbar_wait_backoff(&full[slot], phase);
#ifdef TP_PROFILE_WAITS
          const long long w1 = clock64();
#endif
          op.col(P, C, g, scratch, c, rc);
          __syncwarp();
#ifdef TP_PROFILE_WAITS
          if (g.lane == 0) {
            atomicAdd(&g_prof[0], (unsigned long long)(w1 - w0));
            atomicAdd(&g_prof[1 + min(c, 6u)], (unsigned long long)(clock64() - w1));
          }
#endif
          if (g.lane == 0) mbar_arrive(&empty[slot]);
          if (++slot == P.nstages) { slot = 0; phase ^= 1u; }
        }
        op.end(P, C, g);
      }
    }
    op.finish(P, g, smem);
  }
}

// ------------------------------------------------------------------ the query pipeline
// Multi-column operators (select / project / aggregate, star queries) stream one item per column
// of each range of TPR tiles, in evaluation order.  The items of one query differ in size by up
// to 10x (a 5.7-bit RFOR date column next to a 24-bit FOR price), so the ring is a BYTE ring:
// the producer places each item at the next free 16-byte aligned offset (wrapping to the ring
// start when it does not fit at the end; a None box 1024-byte aligned) and reclaims space as the
// consumers release items, oldest first.  QNS item slots carry each item's mbarriers and layout
// {ring offset, block_starts offset of stream 0, data / block_starts offsets of stream 1}.
// The bytes in flight are the ring's whatever the column mix (fixed slots sized for the widest
// column held two items of an SSB query).  An operator may keep an item until the end of its
// round (Op::col returns false); the host must then size the ring for every item in between.
constexpr uint32_t QNS = 16;
#ifndef TP_QUERY_PREFETCH
#define TP_QUERY_PREFETCH 0  // rounds the query producer prefetches into L2 ahead of the ring (1 / 2 /
                             // 4 measured: no change on SSB SF20 -- off)
#endif
#ifndef TP_QPROD_SPIN
#define TP_QPROD_SPIN 0
#endif

// lane `src`'s boundary of stream q (warp-uniform q): a jump to the one shuffle instead of one
// shuffle pair per stream of the query (the producer's per-item cost sits on the ring's refill
// path: 24 dependent shuffles per item at 12 streams)
__device__ __forceinline__ uint32_t bnd_of(const uint32_t (&bnd)[MAX_STREAMS], uint32_t q, uint32_t src) {
  switch (q) {
#define TP_BCASE(K) \
  case K: return __shfl_sync(FULL, bnd[K], src);
    TP_BCASE(0) TP_BCASE(1) TP_BCASE(2) TP_BCASE(3) TP_BCASE(4) TP_BCASE(5)
    TP_BCASE(6) TP_BCASE(7) TP_BCASE(8) TP_BCASE(9) TP_BCASE(10)
#undef TP_BCASE
    default: return __shfl_sync(FULL, bnd[MAX_STREAMS - 1], src);
  }
}

template <class Op>
__device__ __forceinline__ void run_query_pipeline(const Params& P, Op& op) {
  extern __shared__ __align__(1024) uint32_t smem[];
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31u;
  const uint32_t npairs = (P.ntiles + 1u) >> 1;
  const uint32_t p0 = (uint32_t)((uint64_t)blockIdx.x * npairs / gridDim.x);
  const uint32_t p1 = (uint32_t)((uint64_t)(blockIdx.x + 1) * npairs / gridDim.x);
  const uint32_t t0 = 2u * p0, t1 = min(2u * p1, P.ntiles);
  if (t0 >= t1) return;
  const uint32_t ngr = (t1 - t0 + TPR - 1) / TPR;
  const uint32_t RW = P.ring_words;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + P.bar_off);
  uint64_t* empty = full + QNS;
  uint32_t* meta = reinterpret_cast<uint32_t*>(empty + QNS);  // 4 words per slot
  op.cta_init(P, smem);
  if (threadIdx.x == 0) {
    for (uint32_t s = 0; s < QNS; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], CONSUMER_WARPS);
    }
    fence_mbar_init();
  }
  __syncthreads();

  if (warp == 0) {
    // ---------------- producer
    const uint64_t pol = policy_evict_first();
    uint32_t head = 0;    // virtual word offset of the next allocation (monotonic)
    uint32_t oldest = 0;  // the oldest item not yet seen released
    uint32_t vst = 0;     // lane s < QNS: virtual start of the item in slot s
    uint32_t item = 0;
    for (uint32_t gb = 0; gb < ngr; gb += 31) {
      const uint32_t tb = min(t0 + (gb + lane) * TPR, t1);
      uint32_t bnd[MAX_STREAMS];
#pragma unroll
      for (int q = 0; q < MAX_STREAMS; ++q) {
        bnd[q] = 0u;
        if ((uint32_t)q < P.nstreams) {
          const Stream& st = P.st[q];
          bnd[q] = __ldg(st.starts + min(st.kind == K_RFOR ? tb : 4u * tb, st.nblocks));
        }
      }
      const uint32_t ge = min(gb + 31, ngr);
      for (uint32_t g = gb; g < ge; ++g) {
        const uint32_t tile_base = t0 + g * TPR, tile_end = min(tile_base + TPR, t1);
#if TP_QUERY_PREFETCH
        // the ring holds about one round of a multi-column query: run TP_QUERY_PREFETCH rounds
        // ahead in L2 (bulk prefetches of every stream's words), so that the ring's TMA copies
        // are served from L2 rather than HBM (measured: consumers spun on data 15-20 % of their
        // instructions without it)
        if (g + TP_QUERY_PREFETCH < ge) {
          const uint32_t rel = g + TP_QUERY_PREFETCH - gb;
#pragma unroll
          for (int q = 0; q < MAX_STREAMS; ++q) {
            if ((uint32_t)q < P.nstreams) {
              const uint32_t a = __shfl_sync(FULL, bnd[q], rel), b = __shfl_sync(FULL, bnd[q], rel + 1);
              if (lane == (uint32_t)q && b > a) {
                const uintptr_t a0 = reinterpret_cast<uintptr_t>(P.st[q].data + a) & ~uintptr_t(15);
                const uintptr_t a1 = (reinterpret_cast<uintptr_t>(P.st[q].data + b) + 15) & ~uintptr_t(15);
                bulk_prefetch_l2(reinterpret_cast<const void*>(a0), (uint32_t)(a1 - a0));
              }
            }
          }
        }
#endif
        for (uint32_t c = 0; c < P.ncols; ++c, ++item) {
          const Col& cc = P.col[c];
          const bool rfor = cc.scheme == S_RFOR;
          const uint32_t my_s = lane == 0 ? cc.s0 : (lane == 1 && rfor ? cc.s1 : 0xffu);
          uint32_t mylo = bnd_of(bnd, cc.s0, g - gb), myhi = bnd_of(bnd, cc.s0, g - gb + 1);
          if (rfor) {  // (column-uniform)
            const uint32_t lo1 = bnd_of(bnd, cc.s1, g - gb), hi1 = bnd_of(bnd, cc.s1, g - gb + 1);
            if (lane == 1) { mylo = lo1; myhi = hi1; }
          }
          const bool none = (Op::kMask & M_NONE) && cc.scheme == S_NONE;  // column-uniform
          uint32_t dbytes = 0u, sbytes = 0u, dwords = 0u, swords = 0u;
          const char *dsrc = nullptr, *ssrc = nullptr;
          if (none) {
            dwords = lane == 0 ? TPR * TILE_ROWS : 0u;  // one TMA tensor box (OOB rows zero-filled)
            dbytes = 4u * dwords;
          } else if (my_s != 0xffu) {
            const Stream& st = P.st[my_s];
            const uint32_t lo = mylo - (st.kind == K_DFOR ? 1u : 0u);
            const uintptr_t a0 = reinterpret_cast<uintptr_t>(st.data + lo) & ~uintptr_t(15);
            const uintptr_t a1 = (reinterpret_cast<uintptr_t>(st.data + myhi) + 15) & ~uintptr_t(15);
            dsrc = reinterpret_cast<const char*>(a0);
            dbytes = (uint32_t)(a1 - a0);
            const uint32_t s0 = st.kind == K_RFOR ? tile_base : 4u * tile_base;
            const uint32_t s1 = min(st.kind == K_RFOR ? tile_end : 4u * tile_end, st.nblocks) + 1u;
            const uintptr_t b0 = reinterpret_cast<uintptr_t>(st.starts + s0) & ~uintptr_t(15);
            const uintptr_t b1 = (reinterpret_cast<uintptr_t>(st.starts + s1) + 15) & ~uintptr_t(15);
            ssrc = reinterpret_cast<const char*>(b0);
            sbytes = (uint32_t)(b1 - b0);
            swords = sbytes >> 2;
            dwords = (dbytes >> 2) + 4u;  // + the unpack's over-read (Alg. 1 line 15 reads word k + 1)
          }
          if (__shfl_sync(FULL, dwords + swords, 0) + __shfl_sync(FULL, dwords + swords, 1) > RW) {
            // a malformed column (a tile longer than max_tile_words says) must not outgrow the
            // ring: copy what fits (the host sized the ring for the largest legitimate item)
            tp_flag_error(2u);  // TP_DEVERR_TILE_WORDS
            if (my_s != 0xffu && !none) {
              dbytes = min(dbytes, 4u * ((RW >> 1) - swords - 8u) & ~15u);
              dwords = (dbytes >> 2) + 4u;
            }
          }
          const uint32_t rw0 = __shfl_sync(FULL, dwords + swords, 0);
          const uint32_t rw1 = __shfl_sync(FULL, dwords + swords, 1);
          const uint32_t need = rw0 + rw1;  // multiples of 4 words
          uint32_t hd = none ? (head + 255u) & ~255u : head;
          if (hd % RW + need > RW) hd += RW - hd % RW;  // does not fit before the ring's end: wrap
          // reclaim: the slot's previous item, and every item still holding the space needed
#ifdef TP_PROFILE_WAITS
          const long long pw0 = clock64();
#endif
          while (item - oldest >= QNS || (oldest < item && hd + need > __shfl_sync(FULL, vst, oldest % QNS) + RW)) {
#if TP_QPROD_SPIN
            mbar_wait(&empty[oldest % QNS], (oldest / QNS) & 1u);
#else
            mbar_wait_backoff(&empty[oldest % QNS], (oldest / QNS) & 1u);
#endif
            ++oldest;
          }
#ifdef TP_PROFILE_WAITS
          if (lane == 0) atomicAdd(&g_prof[8], (unsigned long long)(clock64() - pw0));
#endif
          const uint32_t slot = item % QNS;
          if (lane == slot) vst = hd;
          head = hd + need;
          const uint32_t off = hd % RW;
          const uint32_t dw0 = __shfl_sync(FULL, dwords, 0), dw1 = __shfl_sync(FULL, dwords, 1);
          if (lane == 0)  // stream 0: data at 0, block_starts at dw0; stream 1: data at rw0, starts after it
            *reinterpret_cast<uint4*>(meta + 4u * slot) = make_uint4(off, dw0, rw0, rw0 + dw1);
          const uint32_t total = __reduce_add_sync(FULL, dbytes + sbytes);
          if (lane == 0) mbar_arrive_expect_tx(&full[slot], total);
          __syncwarp();
          uint32_t* dst = smem + off + (lane == 1 ? rw0 : 0u);
          if (none) {
            if (lane == 0) tma_load_2d(dst, &P.tmap[c], 0, (int)(tile_base * (TILE_ROWS / 32)), &full[slot], pol);
          } else if (my_s != 0xffu) {
            bulk_g2s(dst, dsrc, dbytes, &full[slot], pol);
            bulk_g2s(dst + dwords, ssrc, sbytes, &full[slot], pol);
          }
        }
      }
    }
  } else {
    // ---------------- consumers
    const Lane g = lane_geom();
    uint32_t* scratch = smem + P.scratch_off + g.cw * P.scratch_words_per_warp;
    uint32_t item = 0;
    StageCtx C;
    C.tile_end = t1;
    C.round_base = 0;
    for (uint32_t gi = 0; gi < ngr; ++gi) {
      C.t0s = t0 + gi * TPR;
      op.begin(P, C, g);
      uint32_t held = 0xffffffffu;
      for (uint32_t c = 0; c < P.ncols; ++c, ++item) {
        const uint32_t slot = item % QNS;
#ifdef TP_PROFILE_WAITS
        const long long w0 = clock64();
#endif
        mbar_wait_backoff(&full[slot], (item / QNS) & 1u);
#ifdef TP_PROFILE_WAITS
        const long long w1 = clock64();
#endif
        const uint4 mt = *reinterpret_cast<const uint4*>(meta + 4u * slot);
        C.stage = smem + mt.x;
        C.doff[0] = 0u; C.soff[0] = mt.y; C.doff[1] = mt.z; C.soff[1] = mt.w;
        const bool rel = op.col(P, C, g, scratch, c, gi);
        __syncwarp();
#ifdef TP_PROFILE_WAITS
        if (g.lane == 0) {
          atomicAdd(&g_prof[0], (unsigned long long)(w1 - w0));
          atomicAdd(&g_prof[1 + min(c, 6u)], (unsigned long long)(clock64() - w1));
        }
#endif
        if (rel) {
          if (g.lane == 0) mbar_arrive(&empty[slot]);
        } else {
          held = slot;
        }
      }
      op.end(P, C, g);
      if (held != 0xffffffffu) {
        __syncwarp();
        if (g.lane == 0) mbar_arrive(&empty[held]);
      }
    }
    op.finish(P, g, smem);
  }
}

// named barrier over the consumer warps only
__device__ __forceinline__ void consumers_sync() {
  asm volatile("bar.sync 1, %0;" ::"n"(CONSUMER_WARPS * 32) : "memory");
}

#ifndef TP_SPARSE_LANE_MAX
#define TP_SPARSE_LANE_MAX 8  // ... and (FOR filters / measures) the busiest lane's alive rows
#endif
#ifndef TP_RFOR_SPARSE_MAX
#define TP_RFOR_SPARSE_MAX 64  // (<= 64: up to two alive rows per lane; 64 vs 32: q3.1 -5 %, measured)
#endif
#ifndef TP_SPARSE_MAX
#define TP_SPARSE_MAX 512  // alive rows (of a warp's 1024) at or below which a column goes sparse
                           // (512 / 8 measured best over the 13 SSB queries at SF20)
#endif
#ifndef TP_QUERY_COMPACT
#define TP_QUERY_COMPACT true
#endif

// ------------------------------------------------------------------ consumers
__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t x) {
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) x += __shfl_xor_sync(FULL, x, d);
  return x;
}

__device__ __forceinline__ uint32_t valid_rows(const Params& P, const StageCtx& C, const Lane& g) {
  const uint32_t tile = C.t0s + C.round_base + g.tile_local;
  const uint32_t row0 = tile * TILE_ROWS + g.mb * MB_ROWS;
  if (tile >= C.tile_end || row0 >= P.n) return 0u;
  const uint32_t nrows = P.n - row0;
  return nrows >= 32u ? 0xffffffffu : ((1u << nrows) - 1u);
}

struct OpBase {
  static constexpr bool kProducerSpin = false;
  static constexpr bool kPairRounds = false;  // single-column: col2() takes rounds r and r + 1 together
  static constexpr uint32_t kMask = ~0u;  // scheme mix the kernel carries (M_*)
  __device__ void cta_init(const Params&, uint32_t*) {}
  __device__ void begin(const Params&, const StageCtx&, const Lane&) {}
  __device__ void end(const Params&, const StageCtx&, const Lane&) {}
};

// decode -> sum (decode-only microbenchmark).  LEAN (FOR below ~12 bits, where the
// kernel is instruction-bound): the stream view once per item and a CTA-uniform full-round
// test instead of a per-lane row mask + vote (measured -3..-10 % at b <= 12; at b = 16, where
// HBM binds, the plain variant is 2.7 % faster, so it keeps it)
template <uint32_t MASK, bool LEAN = false>
struct SumOp : OpBase {
  static constexpr uint32_t kMask = MASK;
  static constexpr bool kProducerSpin = MASK == M_FOR || MASK == M_FORNM;
  static constexpr bool kPairRounds = TP_SUM_PAIR && LEAN && MASK == M_FOR;
  unsigned long long* out;
  uint64_t acc;
  uint32_t sv_t0s = 0xffffffffu;  // the item whose stream view is cached (FOR)
  StreamView sv;
  // LEAN GPU-FOR, rounds r and r + 1 of the item (C.round_base = round r): the lane's two
  // miniblocks' views and unpacks are independent chains the scheduler interleaves
  __device__ void col2(const Params& P, StageCtx& C, const Lane& g) {
    const Col& c = P.col[0];
    if (C.t0s != sv_t0s) {
      sv = stream_view(P, c.s0, C);
      sv_t0s = C.t0s;
    }
    uint32_t tl;
    bool tv;
    const MbView m0 = for_mb(P, c, C, g, sv, tl, tv);
    C.round_base += TPR;
    const MbView m1 = for_mb(P, c, C, g, sv, tl, tv);
    const uint32_t tend = C.t0s + C.round_base + TPR;  // the end of the second round
    C.round_base -= TPR;
    const bool full = tend <= C.tile_end && (uint64_t)tend * TILE_ROWS <= P.n;  // (CTA-uniform)
    if (full) {
      acc += sum_mb2(m0.w, m0.b, m1.w, m1.b) + (uint64_t)((int64_t)(int32_t)m0.ref * 32) +
             (uint64_t)((int64_t)(int32_t)m1.ref * 32);
    } else {
      for (int h = 0; h < 2; ++h) {
        C.round_base += h * TPR;
        const MbView m = h ? m1 : m0;
        const uint32_t alive = valid_rows(P, C, g);
        C.round_base -= h * TPR;
        uint32_t e[32];
        unpack_mb(m.w, m.b, e);
#pragma unroll
        for (int i = 0; i < 32; ++i)
          if (alive & (1u << i)) acc += (uint64_t)(int64_t)(int32_t)(m.ref + e[i]);
      }
    }
  }
  __device__ void col(const Params& P, const StageCtx& C, const Lane& g, uint32_t* scratch, uint32_t, uint32_t) {
    const Col& c = P.col[0];
    if (MASK == M_FOR || MASK == M_FORNM) {
      MbView m;
      uint32_t alive;
      bool full;
      if constexpr (LEAN) {
        // per-item work once per item, not once per round (low bitwidths are instruction-bound)
        if (C.t0s != sv_t0s) {
          sv = stream_view(P, c.s0, C);
          sv_t0s = C.t0s;
        }
        uint32_t tl;
        bool tv;
        m = for_mb(P, c, C, g, sv, tl, tv);
        // a round whose TPR tiles are all inside the CTA range needs no row mask (CTA-uniform)
        const uint32_t tend = C.t0s + C.round_base + TPR;
        const bool full_round = tend <= C.tile_end && (uint64_t)tend * TILE_ROWS <= P.n;
        alive = full_round ? 0xffffffffu : valid_rows(P, C, g);
        full = full_round || __all_sync(FULL, alive == 0xffffffffu);
      } else {
        alive = valid_rows(P, C, g);
        const StreamView v = stream_view(P, c.s0, C);
        uint32_t tl;
        bool tv;
        m = MASK == M_FORNM ? fornm_mb(P, c, C, g, v, tl, tv) : for_mb(P, c, C, g, v, tl, tv);
        full = __all_sync(FULL, alive == 0xffffffffu);
      }
      // the branch must be warp-uniform: both sides run warp-collective dispatch code
      if (full) {
        const uint64_t se = sum_mb(m.w, m.b);
        acc += se + (uint64_t)((int64_t)(int32_t)m.ref * 32);
      } else {
        uint32_t e[32];
        unpack_mb(m.w, m.b, e);
#pragma unroll
        for (int i = 0; i < 32; ++i)
          if (alive & (1u << i)) acc += (uint64_t)(int64_t)(int32_t)(m.ref + e[i]);
      }
    } else {
      uint32_t alive;
      uint32_t val[32];
      if constexpr (LEAN && MASK == M_DFOR) {
        // GPU-DFOR is instruction-bound too: the stream view once per item, the CTA-uniform
        // full-round test
        if (C.t0s != sv_t0s) {
          sv = stream_view(P, c.s0, C);
          sv_t0s = C.t0s;
        }
        const uint32_t tend = C.t0s + C.round_base + TPR;
        const bool full_round = tend <= C.tile_end && (uint64_t)tend * TILE_ROWS <= P.n;
        alive = full_round ? 0xffffffffu : valid_rows(P, C, g);
        decode_dfor_sv<false>(P, c, C, g, sv, val);
      } else {
        alive = valid_rows(P, C, g);
        decode_col<MASK>(P, 0, C, g, scratch, val);
      }
      if (alive == 0xffffffffu) {  // per-lane branch, no collectives inside
        bool done = false;
        if constexpr (TP_SUM32 && (MASK == M_RFOR || MASK == M_DFOR)) {
          // decoded values below 2^28 (their OR says so: run values, keys of a 2^28 domain) sum
          // exactly in two 32-bit halves of 16 -- one add per value instead of a 64-bit add and
          // a sign count
          uint32_t o = 0u;
#pragma unroll
          for (int i = 0; i < 32; ++i) o |= val[i];
          if ((o >> 28) == 0u) {
            uint32_t sa = 0u, sb = 0u;
#pragma unroll
            for (int i = 0; i < 16; ++i) {
              sa += val[i];
              sb += val[16 + i];
            }
            acc += (uint64_t)sa + sb;
            done = true;
          }
        }
        if (!done) {
          uint64_t lo = 0;
          uint32_t neg = 0;
#pragma unroll
          for (int i = 0; i < 32; ++i) {  // sum(sext v) = sum(zext v) - 2^32 * #negative
            lo += val[i];
            neg += val[i] >> 31;
          }
          acc += lo - ((uint64_t)neg << 32);
        }
      } else {
#pragma unroll
        for (int i = 0; i < 32; ++i)
          if (alive & (1u << i)) acc += (uint64_t)(int64_t)(int32_t)val[i];
      }
    }
  }
  __device__ void finish(const Params&, const Lane& g, uint32_t*) {
    const uint64_t s = warp_sum_u64(acc);
    if (g.lane == 0) atomicAdd(out, (unsigned long long)s);
  }
};

// decode -> global (Fig. 7a mode): the warp's 1024 rows go to a
// 128B-swizzled 4 KB shared buffer (conflict-free 16-byte stores) and leave by
// one TMA tensor store; the partial last miniblock (n % 32 rows) is stored directly.
template <uint32_t MASK>
struct GlobalOp : OpBase {
  static constexpr uint32_t kMask = MASK;
  // HBM-bound (decoded rows are written back); the instruction-bound DFOR / RFOR expansions
  // may park their waiting warps instead (TP_GLOBAL_SPIN_INSTR 0)
  static constexpr bool kProducerSpin = TP_GLOBAL_SPIN_INSTR || (MASK != M_RFOR && MASK != M_DFOR);
  const CUtensorMap* tmap;
  int32_t* out;
  uint32_t full_rows32;  // n / 32: rows of the [n/32][32] tensor
  __device__ void col(const Params& P, const StageCtx& C, const Lane& g, uint32_t* scratch, uint32_t,
                      uint32_t rc) {
    // RFOR: the rows are staged in the expansion's own A arrays (1024-byte aligned: the host aligns
    // the scratch), so the previous round's store must have read them before this round expands
    constexpr bool OVERLAY = MASK == M_RFOR;
    // GPU-DFOR of more than a few bits / int (instruction-bound): one staging buffer, so that a
    // 4th CTA fits per SM (host's choice, warp-uniform)
    const bool SINGLE = MASK == M_DFOR && P.single_staging;
    if (OVERLAY) {
      if (g.lane == 0) bulk_wait_read<0>();
      __syncwarp();
    }
    uint32_t val[32];
    decode_col<MASK>(P, 0, C, g, scratch, val);
    const uint32_t pair_tile = C.t0s + C.round_base + 2u * g.cw;
    if (pair_tile >= C.tile_end) return;  // warp-uniform
    uint32_t* buf;
    if (OVERLAY) {
      buf = scratch;
      __syncwarp();  // every lane has read its chunk of A
    } else {
      buf = scratch + P.staging_off;
      buf = reinterpret_cast<uint32_t*>((reinterpret_cast<uintptr_t>(buf) + 1023) & ~uintptr_t(1023));
      if (SINGLE) {
        if (g.lane == 0) bulk_wait_read<0>();  // the previous store is done reading the buffer
      } else {
        buf += (rc & 1u) * 1024u;
        if (g.lane == 0) bulk_wait_read<1>();  // the store issued from this buffer earlier is done reading it
      }
      __syncwarp();
    }
    const uint32_t l = g.lane;
#pragma unroll
    for (uint32_t q = 0; q < 8; ++q) {
      st_shared_v4(buf + l * 32u + ((q ^ (l & 7u)) << 2), val[4 * q], val[4 * q + 1], val[4 * q + 2],
                   val[4 * q + 3]);
    }
    fence_proxy_async_smem();
    __syncwarp();
    const uint32_t mb0 = pair_tile * 16u;
    if (g.lane == 0 && mb0 < full_rows32) {
      tma_store_2d(tmap, buf, 0, (int)mb0);
      bulk_commit();
    }
    const uint32_t mym = mb0 + l;
    if (mym == full_rows32 && (P.n & 31u)) {  // the partial last miniblock
#pragma unroll
      for (int i = 0; i < 32; ++i)
        if (mym * 32u + i < P.n) out[mym * 32u + i] = (int32_t)val[i];
    }
  }
  __device__ void finish(const Params&, const Lane& g, uint32_t*) {
    if (g.lane == 0) bulk_wait_all();
    __syncwarp();
  }
};

// select / project / aggregate over up to 6 columns.  The host hands
// the columns over in evaluation order: predicate-only columns, then the projection
// operands a and b, so that at most two decoded miniblocks are live at a time.
struct SelectArgs {
  int32_t lo[TP_MAX_COLS], hi[TP_MAX_COLS];  // per column (evaluation order)
  uint32_t npred;                            // columns [0, npred) are predicate-only
  int proj;                                  // TP_PROJ_*
  uint32_t has_a, has_b;                     // column npred is a, npred+1 is b
};

template <uint32_t MASK>
struct SelectOp : OpBase {
  static constexpr uint32_t kMask = MASK;
  const SelectArgs* A;
  unsigned long long* out;
  uint64_t acc;
  uint32_t alive;
  uint32_t va[32];
  __device__ void begin(const Params& P, const StageCtx& C, const Lane& g) { alive = valid_rows(P, C, g); }
  __device__ bool col(const Params& P, const StageCtx& C, const Lane& g, uint32_t* scratch, uint32_t c, uint32_t) {
    if (!__any_sync(FULL, alive != 0u)) return true;  // nothing survives in this warp's rows
    uint32_t v[32];
    decode_col<MASK, TP_QUERY_COMPACT, true>(P, c, C, g, scratch, v);
    const int32_t l = A->lo[c], h = A->hi[c];
#pragma unroll
    for (int i = 0; i < 32; ++i)
      if ((int32_t)v[i] < l || (int32_t)v[i] > h) alive &= ~(1u << i);
    if (A->has_a && c == A->npred) {
      if (A->has_b) {
#pragma unroll
        for (int i = 0; i < 32; ++i) va[i] = v[i];
      } else {
#pragma unroll
        for (int i = 0; i < 32; ++i)
          if (alive & (1u << i)) acc += (uint64_t)(int64_t)(int32_t)v[i];
      }
    } else if (A->has_b && c == A->npred + 1) {
      const bool mul = A->proj == TP_PROJ_MUL;
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        if (alive & (1u << i)) {
          const int64_t xa = (int32_t)va[i], xb = (int32_t)v[i];
          acc += (uint64_t)(mul ? xa * xb : xa - xb);
        }
      }
    }
    return true;
  }
  __device__ void end(const Params&, const StageCtx&, const Lane&) {
    if (A->proj == TP_PROJ_COUNT) acc += __popc(alive);
  }
  __device__ void finish(const Params&, const Lane& g, uint32_t*) {
    const uint64_t s = warp_sum_u64(acc);
    if (g.lane == 0) atomicAdd(out, (unsigned long long)s);
  }
};

// ------------------------------------------------------------------ star-join queries
// SSB as one tile kernel: FK columns probe dimension lookup tables
// (Crystal's perfect hash, key - key_min), payloads build a dense group index,
// measures are aggregated per group.  Columns come in the host's order (most selective
// first); the last column is the aggregating measure, a first measure (MUL / SUB) is read
// back when it aggregates.
//
// GPU-FOR / GPU-DFOR / None columns: per column a warp picks one of two evaluation modes
// (warp-uniform):
//  * dense  -- while many of its 1024 rows are alive: decode all 32 rows per thread
//    (tile decode) and apply the column's role to each;
//  * sparse -- once few rows survive: visit only the alive rows and read each one's value
//    straight out of the staged tile (random access into a FOR miniblock, Alg. 1 for one
//    entry) -- no work for dead rows.
// GPU-RFOR columns are evaluated in RUN space (rfor_col): a range or a probe once per run
// (the rows of a run share its value) -- the run's passing bit reaches its rows
// through one 64-bit add per thread -- and measures / group payloads per alive row through
// the row's run number; the run expansion of the decode is never materialised.
// The group index lives in per-warp shared memory laid out [row i][lane] (conflict-free for
// any mix of rows).  The first of two measures stays in its ring item (held until the
// round's last column aggregates) and is re-read per alive row; only a DFOR / RFOR first
// measure is staged in a per-warp array.  Grouped queries pre-aggregate in a per-CTA
// shared-memory hash table (open addressing) and flush it once, so hot groups (q4.1 has 35)
// do not serialise on global atomics.
struct StarArgs {
  int32_t role[TP_MAX_COLS], lo[TP_MAX_COLS], hi[TP_MAX_COLS];
  const int32_t* table[TP_MAX_COLS];
  int32_t key_min[TP_MAX_COLS];
  uint32_t table_len[TP_MAX_COLS], stride[TP_MAX_COLS];
  uint32_t gmode[TP_MAX_COLS];   // probe: 0 filter only, 1 group = p * stride (first), 2 group += p * stride
  uint32_t mstage[TP_MAX_COLS];  // measure: 1 = the first of two, 0 = the aggregating one
  int agg;
  uint32_t ngroups;
  uint32_t gzero;                // grouped without payload probes: every row is group 0
  uint32_t gs_off, ws_off;       // per-warp scratch (words): group index, staged first measure
  uint32_t ra_off, sb_off;       // per-warp scratch: RFOR run array (1024), start / pass / alive words (3 x 33)
  uint32_t ht_slots, ht_shift;   // shared-memory aggregation table (grouped queries)
  uint32_t sparse_max;           // warp alive-row count at or below which a column is evaluated sparsely
  uint32_t sparse_lane_max;      // ... and the busiest lane's alive rows: the sparse loop runs for the
                                 // warp's maximum (alive rows cluster: runs of an order's lines)
  uint32_t hint_mask;            // bit c: column c's dense probes load with L1::no_allocate + L2 evict_last
  uint32_t rfor_sparse_max;      // a GPU-RFOR column with at most this many alive rows (<= 64) in the
                                 // warp goes sparse (run lengths only + a binary search per row)
  long long* sums;
  unsigned long long* counts;
};

#ifndef TP_HT_MAX_SLOTS
#define TP_HT_MAX_SLOTS 1024
#endif
constexpr uint32_t HT_MAX_SLOTS = TP_HT_MAX_SLOTS, HT_EMPTY = 0xffffffffu, HT_PROBES = 64;
// slots: a power of two >= 2 x the dense group count (at most HT_MAX_SLOTS); 4 words per slot:
// key, sum lo, sum hi, count
static inline uint32_t ht_slots(uint32_t ngroups) {
  uint32_t s = 256;
  while (s < HT_MAX_SLOTS && s < 2u * ngroups) s <<= 1;
  return s;
}
#ifndef TP_STAR_PAIR
#define TP_STAR_PAIR 1  // ungrouped queries: the run-space RFOR pass over both blocks of a round at once
                        // (q1.2 / q1.3 -8 %; in the grouped kernel q4.x -3 % but q3.2 +14 %: off there)
#endif
#ifndef TP_DENSE_PROBE_HINT
#define TP_DENSE_PROBE_HINT 1
#endif
#ifndef TP_PROBE_HINT_MIN
#define TP_PROBE_HINT_MIN 800000u  // table entries from which dense probes take the hint (SF20: the part table;
                                  // the 600K-entry customer table loses with it, None q3.x +20-30 %, measured)
#endif
__device__ __forceinline__ int32_t probe_ld(const int32_t* p) { return __ldg(p); }
// the dense probe of grouped queries (every alive row of a FOR / None column, the bulk of the
// lookups of q2.x): L1::no_allocate + L2 evict_last (q2.x -9 %, q3.2 -2 %, measured; either hint
// alone: no gain / +20 %; in the ungrouped kernel the changed code cost q1.1 4 %)
__device__ __forceinline__ int32_t dense_probe_ld(const int32_t* p) {
#if TP_DENSE_PROBE_HINT
  int32_t v;
  uint64_t pol;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
  return v;
#else
  return probe_ld(p);
#endif
}
constexpr uint32_t STAR_RA_WORDS = 1024, STAR_SB_WORDS = 3 * 33 + 1;
#ifndef TP_RFOR_CC8
#define TP_RFOR_CC8 0  // RFOR run decode: 4 entries per lane and pass only (one body: instruction cache)
#endif
#ifndef TP_HT_NOINLINE
#define TP_HT_NOINLINE 0
#endif
#ifndef TP_STAR_RING_WORDS
#define TP_STAR_RING_WORDS 8192u           // 32 KB
#endif
#ifndef TP_RING_SLACK_WORDS
#define TP_RING_SLACK_WORDS 2048u          // the ring holds the largest item + 8 KB
#endif
#ifndef TP_STAR_RING_WORDS_GROUPED
#define TP_STAR_RING_WORDS_GROUPED 6144u   // 24 KB
#endif

template <uint32_t MASK, bool GROUPED>
struct StarOp : OpBase {
  static constexpr uint32_t kMask = MASK;
  const StarArgs* A;
  uint64_t acc, cnt;  // ungrouped (q1.x): reduce in registers
  uint32_t alive;
  uint32_t* keys;
  uint32_t* hlo;   // 64-bit sums as lo/hi words: native 32-bit shared atomics with a carry
  uint32_t* hhi;   // (a 64-bit shared atomicAdd is a CAS loop on sm_100)
  uint32_t* hcnt;
  uint32_t hmask, hshift;

  __device__ void cta_init(const Params& P, uint32_t* smem) {
    if (GROUPED) {
      keys = smem + P.agg_off;
      hlo = keys + A->ht_slots;
      hhi = keys + 2 * A->ht_slots;
      hcnt = keys + 3 * A->ht_slots;
      hmask = A->ht_slots - 1u;
      hshift = A->ht_shift;
      for (uint32_t i = threadIdx.x; i < A->ht_slots; i += blockDim.x) {
        keys[i] = HT_EMPTY;
        hlo[i] = 0u;
        hhi[i] = 0u;
        hcnt[i] = 0u;
      }
    }
  }
#if TP_HT_NOINLINE
  __device__ __noinline__ void ht_add(uint32_t key, int64_t v) {
#else
  __device__ __forceinline__ void ht_add(uint32_t key, int64_t v) {
#endif
    uint32_t slot = (key * 0x9E3779B1u) >> hshift;  // multiplicative hash
#pragma unroll 1
    for (uint32_t p = 0; p < HT_PROBES; ++p) {
      uint32_t cur = keys[slot];
      if (cur == HT_EMPTY) {
        cur = atomicCAS(&keys[slot], HT_EMPTY, key);
        if (cur == HT_EMPTY) cur = key;
      }
      if (cur == key) {
        const uint32_t lo = (uint32_t)(uint64_t)v, hi = (uint32_t)((uint64_t)v >> 32);
        const uint32_t old = atomicAdd(&hlo[slot], lo);
        const uint32_t carry = old + lo < old ? 1u : 0u;
        if (hi + carry) atomicAdd(&hhi[slot], hi + carry);
        atomicAdd(&hcnt[slot], 1u);
        return;
      }
      slot = (slot + 1u) & hmask;
    }
    atomicAdd(reinterpret_cast<unsigned long long*>(A->sums) + key, (unsigned long long)v);  // table crowded
    atomicAdd(A->counts + key, 1ull);
  }
  __device__ void begin(const Params& P, const StageCtx& C, const Lane& g) { alive = valid_rows(P, C, g); }

  // the role of column c applied to row i (value x) -- shared by every mode
  __device__ __forceinline__ void apply_range(uint32_t c, uint32_t i, uint32_t x) {
    if ((uint32_t)((int32_t)x - A->lo[c]) > (uint32_t)(A->hi[c] - A->lo[c])) alive &= ~(1u << i);
  }
  __device__ __forceinline__ void apply_payload(uint32_t c, uint32_t i, int32_t p, uint32_t* G, uint32_t lane) {
    if (p < 0) {
      alive &= ~(1u << i);
    } else if (GROUPED && A->gmode[c]) {
      uint32_t* gp = G + 32u * i + lane;
      *gp = (A->gmode[c] == 1 ? 0u : *gp) + (uint32_t)p * A->stride[c];
    }
  }
  // payloads p[i] (-1 = miss) of the alive rows: one lean pass, warp-uniform values hoisted
  __device__ __forceinline__ void dense_payload(uint32_t c, const uint32_t (&p)[32], uint32_t* G, uint32_t lane) {
    uint32_t miss = 0u;
#pragma unroll
    for (int i = 0; i < 32; ++i) miss |= (p[i] >> 31) << i;
    alive &= ~miss;
    // dead rows' group entries are never read again: write all 32 (no per-row branch)
    if (GROUPED && A->gmode[c] == 1) {
      const uint32_t stride = A->stride[c];
#pragma unroll
      for (int i = 0; i < 32; ++i) G[32u * i + lane] = p[i] * stride;
    } else if (GROUPED && A->gmode[c] == 2) {
      const uint32_t stride = A->stride[c];
#pragma unroll
      for (int i = 0; i < 32; ++i) G[32u * i + lane] += p[i] * stride;
    }
  }
  // measure role of row i: its own filter; the first measure is staged, the aggregating one
  // combines with it and aggregates
  __device__ __forceinline__ void apply_measure(uint32_t c, uint32_t i, uint32_t x, const uint32_t* G, uint32_t* W,
                                                uint32_t lane) {
    if ((uint32_t)((int32_t)x - A->lo[c]) > (uint32_t)(A->hi[c] - A->lo[c])) {
      alive &= ~(1u << i);
      return;
    }
    if (A->mstage[c]) {
      W[32u * i + lane] = x;
      return;
    }
    int64_t y = (int32_t)x;
    if (A->agg == TP_AGG_MUL) y *= (int64_t)(int32_t)W[32u * i + lane];
    else if (A->agg == TP_AGG_SUB) y = (int64_t)(int32_t)W[32u * i + lane] - y;
    if (GROUPED) ht_add(A->gzero ? 0u : G[32u * i + lane], y);
    else acc += (uint64_t)y;
  }

  // ---------------- GPU-RFOR in run space
  // rows R .. R + L - 1 of the warp round hold an alive row (runs longer than 32 rows: assumed)
  __device__ __forceinline__ static bool run_alive(const uint32_t* AW, uint32_t R, uint32_t L) {
    if (L > 32u) return true;
    const uint32_t w = R >> 5;
    const uint64_t win = ((uint64_t)AW[w + 1] << 32) | AW[w];
    return ((win >> (R & 31u)) & ((1ull << L) - 1ull)) != 0ull;
  }
  // one stream block pair (rows 512 h .. 512 h + 511 of the round), CC entries per lane and pass
  // PAIR: both blocks at once, lanes 16 h .. 16 h + 15 on block h (bV / bL / r per lane, rm = the
  // larger r): one header decode and one 16-lane scan per pass serve both blocks
  template <int CC, bool PAIR = false>
  __device__ __forceinline__ void rfor_runs(const uint32_t* bV, const uint32_t* bL, uint32_t r, uint32_t h,
                                            uint32_t c, bool range, bool per_run, bool need_ra, bool all_alive,
                                            uint32_t* RA, uint32_t* SB, uint32_t* PB, const uint32_t* AW,
                                            uint32_t lane, uint32_t rm = 0u) {
    if (PAIR) h = lane >> 4;
    const uint32_t refV = bV[1], refL = bL[1];  // references (FOR on both arrays)
    const uint4 wv = make_uint4(bV[2], bV[3], bV[4], bV[5]), wl = make_uint4(bL[2], bL[3], bL[4], bL[5]);
    const int32_t* __restrict__ T = A->table[c];
    const uint32_t kmin = (uint32_t)A->key_min[c], tlen = A->table_len[c];
    const int32_t lo = A->lo[c];
    const uint32_t span = (uint32_t)(A->hi[c] - lo);
    uint32_t rowbase = 0u;  // rows of the block covered by earlier passes
#pragma unroll 1
    for (uint32_t e00 = 0; e00 < (PAIR ? rm : r); e00 += (PAIR ? 16u : 32u) * CC) {
      const uint32_t e0 = e00 + CC * (PAIR ? lane & 15u : lane), m = (e0 >> 5) & 15u, pos = e0 & 31u;
      const uint32_t bv = checked_bw(byte_of(wv, m)), bl = checked_bw(byte_of(wl, m));  // R2, R17
      const uint32_t* mV = bV + 6 + bytes_before(wv, m);  // miniblocks before m are full (R17)
      const uint32_t* mL = bL + 6 + bytes_before(wl, m);
      const uint32_t mv = __funnelshift_lc(0xffffffffu, 0u, bv), ml = __funnelshift_lc(0xffffffffu, 0u, bl);
      uint32_t len[CC], val[CC];
      uint32_t run = 0u;
      extract_c<CC>(mL, pos, bl, ml, len);
#pragma unroll
      for (int k = 0; k < CC; ++k) {  // run lengths (scan step 1)
        len[k] = e0 + k < r ? refL + len[k] : 0u;
        run += len[k];
      }
      const uint32_t incl = PAIR ? seg16_inclusive_scan(run) : warp_inclusive_scan(run, lane);
      uint32_t S = 512u * h + rowbase + incl - run;  // round row of entry e0's run start
      rowbase += __shfl_sync(FULL, incl, PAIR ? lane | 15u : 31u);
      extract_c<CC>(mV, pos, bv, mv, val);
#pragma unroll
      for (int k = 0; k < CC; ++k) val[k] += refV;
      uint32_t pass = 0u;  // bit k: run k passes the column's role
      if (per_run) {
        if (range) {
#pragma unroll
          for (int k = 0; k < CC; ++k) pass |= ((uint32_t)((int32_t)val[k] - lo) <= span ? 1u : 0u) << k;
        } else {
          // probes: every live run's lookup in flight before any result is used
          uint32_t Sk = S;
#pragma unroll
          for (int k = 0; k < CC; ++k) {
            const uint32_t key = val[k] - kmin;
            const bool live = e0 + k < r && key < tlen && (all_alive || run_alive(AW, Sk, len[k]));
            val[k] = live ? (uint32_t)probe_ld(T + key) : 0xffffffffu;  // payload, -1 = miss
            Sk += len[k];
          }
#pragma unroll
          for (int k = 0; k < CC; ++k) pass |= ((int32_t)val[k] >= 0 ? 1u : 0u) << k;
        }
      }
#pragma unroll
      for (int k = 0; k < CC; ++k) {
        if (e0 + k < r) {
          const uint32_t bit = 1u << (S & 31u);
          atomicOr(&SB[S >> 5], bit);
          if ((pass >> k) & 1u) atomicOr(&PB[S >> 5], bit);
          if (need_ra) RA[512u * h + e0 + k] = val[k];  // run number e0 + k of block h
        }
        S += len[k];
      }
    }
  }
  // sparse GPU-RFOR (few alive rows): only the run-length stream is unpacked -- its scan gives
  // every run's start row (Sarr[e], e < r) -- and each alive row finds its run by binary search
  // and unpacks that one run value (random access into the value stream block, Alg. 1 for one
  // entry); the alive rows are spread one per lane (compaction), so the warp runs one pass for
  // up to 32 rows whatever their owner lanes
  __device__ __forceinline__ void rfor_starts(const uint32_t* bL, uint32_t r, uint32_t lane, uint32_t* Sarr) {
    const uint32_t refL = bL[1];
    const uint4 wl = make_uint4(bL[2], bL[3], bL[4], bL[5]);
    uint32_t rows = 0u;
#pragma unroll 1
    for (uint32_t e00 = 0; e00 < r; e00 += 128u) {
      const uint32_t e0 = e00 + 4u * lane, m = (e0 >> 5) & 15u, pos = e0 & 31u;
      const uint32_t bl = checked_bw(byte_of(wl, m));
      const uint32_t* mL = bL + 6 + bytes_before(wl, m);
      const uint32_t ml = __funnelshift_lc(0xffffffffu, 0u, bl);
      uint32_t len[4], run = 0u;
      extract_c<4>(mL, pos, bl, ml, len);
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        len[k] = e0 + k < r ? refL + len[k] : 0u;
        run += len[k];
      }
      const uint32_t incl = warp_inclusive_scan(run, lane);
      uint32_t S = rows + incl - run;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        if (e0 + k < r) Sarr[e0 + k] = S;
        S += len[k];
      }
      rows += __shfl_sync(FULL, incl, 31);
    }
  }
  __device__ void rfor_col_sparse(const Params& P, const StageCtx& C, const Lane& g, uint32_t* scratch, uint32_t c,
                                  int role, uint32_t nal) {
    const Col& col = P.col[c];
    const StreamView vv = stream_view<true>(P, col.s0, C, 0), vl = stream_view<true>(P, col.s1, C, 1);
    uint32_t* RA = scratch + A->ra_off;  // run starts of both blocks (block h at 512 h)
    uint32_t* LS = scratch + A->sb_off;  // the warp's alive rows, compacted (<= 64)
    uint32_t* AW = LS + 66;              // alive words
    uint32_t* G = scratch + A->gs_off;
    uint32_t* W = scratch + A->ws_off;
    const uint32_t lane = g.lane;
    __syncwarp();  // the previous RFOR column's readers are done
    {
      const uint32_t cnt = __popc(alive);
      uint32_t off = warp_inclusive_scan(cnt, lane) - cnt, m = alive;
      while (m) {
        const uint32_t i = __ffs(m) - 1u;
        m &= m - 1u;
        LS[off++] = (lane << 5) | i;
      }
      AW[lane] = alive;
    }
    const uint32_t live_lanes = __ballot_sync(FULL, alive != 0u);
    const uint32_t* bV0 = nullptr;
    const uint32_t* bV1 = nullptr;
    uint32_t r0 = 0u, r1 = 0u;
#pragma unroll
    for (uint32_t h = 0; h < 2; ++h) {
      const uint32_t tl = C.round_base + 2u * g.cw + h;
      if (C.t0s + tl >= C.tile_end) break;                          // warp-uniform
      if (((live_lanes >> (16u * h)) & 0xffffu) == 0u) continue;  // no alive row in this block
      const uint32_t* bV = vv.sd + (vv.ss[vv.sshift + tl] - vv.lo + vv.dshift);
      const uint32_t* bL = vl.sd + (vl.ss[vl.sshift + tl] - vl.lo + vl.dshift);
      uint32_t r = bL[0];
      if (r > 512u) {
        tp_flag_error(4u);  // TP_DEVERR_RUNS
        r = 512u;
      }
      if (h == 0) { bV0 = bV; r0 = r; } else { bV1 = bV; r1 = r; }
      rfor_starts(bL, r, lane, RA + 512u * h);
    }
    __syncwarp();
#pragma unroll 1
    for (uint32_t t = lane; t < nal; t += 32u) {  // (up to 2 alive rows per lane)
      const uint32_t id = LS[t], j = id >> 5, i = id & 31u, h = j >> 4;
      const uint32_t q = 32u * (j & 15u) + i;  // the row within its block
      const uint32_t* Sa = RA + 512u * h;
      uint32_t lo = 0u, hi = h ? r1 : r0;  // the last run starting at or before q (row 0 starts run 0)
      while (hi - lo > 1u) {
        const uint32_t mid = (lo + hi) >> 1;
        if (Sa[mid] <= q) lo = mid; else hi = mid;
      }
      const uint32_t* bV = h ? bV1 : bV0;
      const uint4 wv = make_uint4(bV[2], bV[3], bV[4], bV[5]);
      const uint32_t mb = lo >> 5, bv = checked_bw(byte_of(wv, mb));
      const uint32_t x = bV[1] + extract_at(bV + 6 + bytes_before(wv, mb), (lo & 31u) * bv,
                                            __funnelshift_lc(0xffffffffu, 0u, bv));  // the run's value
      bool kill = false;
      if (role == TP_ROLE_RANGE) {
        kill = (uint32_t)((int32_t)x - A->lo[c]) > (uint32_t)(A->hi[c] - A->lo[c]);
      } else if (role == TP_ROLE_PROBE) {
        const uint32_t kk = x - (uint32_t)A->key_min[c];
        const int32_t p = kk < A->table_len[c] ? probe_ld(A->table[c] + kk) : -1;
        kill = p < 0;
        if (!kill && GROUPED && A->gmode[c]) {
          uint32_t* gp = G + 32u * i + j;
          *gp = (A->gmode[c] == 1 ? 0u : *gp) + (uint32_t)p * A->stride[c];
        }
      } else if ((uint32_t)((int32_t)x - A->lo[c]) > (uint32_t)(A->hi[c] - A->lo[c])) {
        kill = true;  // the measure's own filter
      } else if (A->mstage[c]) {
        W[32u * i + j] = x;
      } else {
        int64_t y = (int32_t)x;
        if (A->agg == TP_AGG_MUL) y *= (int64_t)(int32_t)W[32u * i + j];
        else if (A->agg == TP_AGG_SUB) y = (int64_t)(int32_t)W[32u * i + j] - y;
        if (GROUPED) ht_add(A->gzero ? 0u : G[32u * i + j], y);
        else acc += (uint64_t)y;
      }
      if (kill) atomicAnd(&AW[j], ~(1u << i));
    }
    __syncwarp();
    alive = AW[lane];
  }

  __device__ void rfor_col(const Params& P, const StageCtx& C, const Lane& g, uint32_t* scratch, uint32_t c,
                           int role) {
    const Col& col = P.col[c];
    const StreamView vv = stream_view<true>(P, col.s0, C, 0), vl = stream_view<true>(P, col.s1, C, 1);
    uint32_t* RA = scratch + A->ra_off;
    uint32_t* SB = scratch + A->sb_off;  // run-start bits per lane word
    uint32_t* PB = SB + 33;              // passing-run-start bits
    uint32_t* AW = PB + 33;              // alive words (+ a zero word)
    uint32_t* G = scratch + A->gs_off;
    uint32_t* W = scratch + A->ws_off;
    const uint32_t lane = g.lane;
    const bool range = role == TP_ROLE_RANGE;
    const bool per_run = role != TP_ROLE_MEASURE;
    const bool payload = GROUPED && role == TP_ROLE_PROBE && A->gmode[c];
    const bool need_ra = !per_run || payload;
    const bool all_alive = __all_sync(FULL, alive == FULL);
    __syncwarp();  // the previous RFOR column's readers are done
    SB[lane] = 0u;
    PB[lane] = 0u;
    AW[lane] = alive;
    if (lane == 0) AW[32] = 0u;
    __syncwarp();
    const uint32_t live_lanes = __ballot_sync(FULL, alive != 0u);
#if TP_STAR_PAIR
    if (!GROUPED) {
      const uint32_t tl0 = C.round_base + 2u * g.cw, hb = lane >> 4;
      const bool v1 = C.t0s + tl0 + 1u < C.tile_end;  // (block 0 is inside the range: alive rows)
      const bool go = (hb == 0u || v1) && ((live_lanes >> (16u * hb)) & 0xffffu) != 0u;
      const uint32_t tl = tl0 + (hb && v1 ? 1u : 0u);
      const uint32_t* bV = vv.sd + (vv.ss[vv.sshift + tl] - vv.lo + vv.dshift);
      const uint32_t* bL = vl.sd + (vl.ss[vl.sshift + tl] - vl.lo + vl.dshift);
      uint32_t r = go ? bV[0] : 0u;  // run / value count; 0: the half's block is skipped
      if (r > 512u) {
        tp_flag_error(4u);  // TP_DEVERR_RUNS
        r = 512u;
      }
      rfor_runs<8, true>(bV, bL, r, hb, c, range, per_run, need_ra, all_alive, RA, SB, PB, AW, lane,
                         __reduce_max_sync(FULL, r));
    } else
#endif
#pragma unroll 1
    for (uint32_t h = 0; h < 2; ++h) {
      const uint32_t tl = C.round_base + 2u * g.cw + h;
      if (C.t0s + tl >= C.tile_end) break;                    // warp-uniform
      if (((live_lanes >> (16u * h)) & 0xffffu) == 0u) continue;  // no alive row in this block
      const uint32_t* bV = vv.sd + (vv.ss[vv.sshift + tl] - vv.lo + vv.dshift);
      const uint32_t* bL = vl.sd + (vl.ss[vl.sshift + tl] - vl.lo + vl.dshift);
      uint32_t r = bV[0];  // run / value count
      if (r > 512u) {
        tp_flag_error(4u);  // TP_DEVERR_RUNS
        r = 512u;
      }
#if TP_RFOR_CC8
      if (r > 128u) rfor_runs<8>(bV, bL, r, h, c, range, per_run, need_ra, all_alive, RA, SB, PB, AW, lane);
      else
#endif
      rfor_runs<4>(bV, bL, r, h, c, range, per_run, need_ra, all_alive, RA, SB, PB, AW, lane);
    }
    __syncwarp();
    const uint32_t sb = SB[lane];
    if (per_run) {
      // the passing bit of the run covering the row before this lane's first row: the status of
      // the last run start at or before it, a 16-lane segmented scan (row 0 of a block starts a run)
      const uint32_t pb = PB[lane];
      uint32_t has = sb != 0u, st = has ? (pb >> (31u - __clz(sb))) & 1u : 0u;
#if TP_RFOR_BALLOT_CARRY
      // the nearest earlier lane of the block with a run start (lane 0 of a block has one): its
      // last start's passing bit, by two ballots
      const uint32_t hm = __ballot_sync(FULL, has) & ((1u << lane) - 1u) & (lane >= 16u ? 0xffff0000u : 0xffffu);
      const uint32_t stm = __ballot_sync(FULL, st);
      const uint32_t cin = hm ? (stm >> (31u - __clz(hm))) & 1u : 0u;
#else
      const uint32_t jj = lane & 15u;
#pragma unroll
      for (int d = 1; d < 16; d <<= 1) {
        const uint32_t yh = __shfl_up_sync(FULL, has, d, 16), ys = __shfl_up_sync(FULL, st, d, 16);
        if (jj >= (uint32_t)d && !has) { has = yh; st = ys; }
      }
      const uint32_t up = __shfl_up_sync(FULL, st, 1, 16);
      const uint32_t cin = jj ? up : 0u;
#endif
      // rows of passing runs: adding 1 right above each passing start (and above a virtual start
      // at row -1 carrying cin) into the continuation mask carries through the run's rows
      const uint64_t cont = (uint64_t)(~sb) << 1;
      const uint64_t add = ((uint64_t)pb << 2) | ((uint64_t)cin << 1);
      alive &= (uint32_t)(((cont + add) ^ cont) >> 2);
    }
    if (need_ra && __any_sync(FULL, alive != 0u)) {
      // run number of row i = run starts in the block up to row i - 1 (popc prefix over 16 lanes)
      const uint32_t cl = __popc(sb);
      const uint32_t base = seg16_inclusive_scan(cl) - cl + 512u * (lane >> 4) - 1u;
      uint32_t m = alive;
      while (m) {
        const uint32_t i = __ffs(m) - 1u;
        m &= m - 1u;
        const uint32_t x = RA[base + __popc(sb & (0xffffffffu >> (31u - i)))];
        if (payload) apply_payload(c, i, (int32_t)x, G, lane);
        else apply_measure(c, i, x, G, W, lane);
      }
    }
  }

  __device__ bool col(const Params& P, const StageCtx& C, const Lane& g, uint32_t* scratch, uint32_t c, uint32_t) {
    if (!__any_sync(FULL, alive != 0u)) return true;  // nothing survives in this warp's rows: skip the decode
    const int role = A->role[c];
    const Col& col = P.col[c];
    if ((MASK & M_RFOR) && col.scheme == S_RFOR) {
      const uint32_t nal = __reduce_add_sync(FULL, __popc(alive));
      if (nal <= A->rfor_sparse_max) rfor_col_sparse(P, C, g, scratch, c, role, nal);
      else rfor_col(P, C, g, scratch, c, role);
      return true;
    }
    const bool dfor = (MASK & M_DFOR) && col.scheme == S_DFOR;  // prefix sums: no random access
    const bool none = (MASK & M_NONE) && col.scheme == S_NONE;
    uint32_t* G = scratch + A->gs_off;
    uint32_t* W = scratch + A->ws_off;
    const uint32_t lane = g.lane;
    const uint32_t nal = __reduce_add_sync(FULL, __popc(alive));
    const bool sparse =
        !dfor && ((nal <= A->sparse_max &&
                   // a FOR filter / measure decodes densely for a few instructions a row: it goes
                   // sparse only if the busiest lane's rows are few too (probes save far more per
                   // skipped row: L2 lookups)
                   (role == TP_ROLE_PROBE || __reduce_max_sync(FULL, __popc(alive)) <= A->sparse_lane_max)) ||
                  (GROUPED && role == TP_ROLE_MEASURE && !A->mstage[c]));
    if (!sparse) {
      // ---------------- dense: every row of the warp's round
      uint32_t v[32];
      decode_col<MASK & ~M_RFOR, TP_QUERY_COMPACT, true>(P, c, C, g, scratch, v);
      if (role == TP_ROLE_RANGE) {
#pragma unroll
        for (int i = 0; i < 32; ++i) apply_range(c, i, v[i]);
      } else if (role == TP_ROLE_PROBE) {
        // all 32 probes are issued before any result is used (32 L2 requests in flight)
        const int32_t* __restrict__ T = A->table[c];
        const uint32_t kmin = (uint32_t)A->key_min[c], len = A->table_len[c];
        const uint32_t m = alive;
        if (GROUPED && ((A->hint_mask >> c) & 1u)) {  // a table larger than L1 (host's choice)
#pragma unroll
          for (int i = 0; i < 32; ++i) {
            const uint32_t kk = v[i] - kmin;
            v[i] = ((m >> i) & 1u) && kk < len ? (uint32_t)dense_probe_ld(T + kk) : 0xffffffffu;
          }
        } else {
#pragma unroll
          for (int i = 0; i < 32; ++i) {
            const uint32_t kk = v[i] - kmin;
            v[i] = ((m >> i) & 1u) && kk < len ? (uint32_t)probe_ld(T + kk) : 0xffffffffu;
          }
        }
        dense_payload(c, v, G, lane);
      } else {
        const int32_t lo = A->lo[c];
        const uint32_t span = (uint32_t)(A->hi[c] - lo);
#pragma unroll
        for (int i = 0; i < 32; ++i)
          if ((uint32_t)((int32_t)v[i] - lo) > span) alive &= ~(1u << i);
        if (A->mstage[c]) {
#pragma unroll
          for (int i = 0; i < 32; ++i) W[32u * i + lane] = v[i];
        } else {
          // (grouped: only a DFOR aggregating measure gets here, the others go sparse) -- static
          // row indices throughout: v[] stays in registers
          const uint32_t m = alive;
#pragma unroll
          for (int i = 0; i < 32; ++i) {
            if (m & (1u << i)) {
              int64_t y = (int32_t)v[i];
              if (A->agg == TP_AGG_MUL) y *= (int64_t)(int32_t)W[32u * i + lane];
              else if (A->agg == TP_AGG_SUB) y = (int64_t)(int32_t)W[32u * i + lane] - y;
              if (GROUPED) ht_add(A->gzero ? 0u : G[32u * i + lane], y);
              else acc += (uint64_t)y;
            }
          }
        }
      }
      return true;
    }
    // ---------------- sparse: alive rows only, values read out of the staged tile
    MbView mv;
    uint32_t bmask = 0u, nsw = 0u;
    const uint32_t* nw = nullptr;
    if (none) {
      nw = none_row<true>(P, col, C, g, nsw);
    } else {
      const StreamView sv = stream_view<true>(P, col.s0, C, 0);
      uint32_t tl;
      bool tv;
      mv = for_mb(P, col, C, g, sv, tl, tv);
      bmask = __funnelshift_lc(0xffffffffu, 0u, mv.b);
    }
    uint32_t m = alive;
    if (role == TP_ROLE_MEASURE) {
      // one row at a time (the aggregation's code once: instruction cache); few rows get here
      while (m) {
        const uint32_t i = __ffs(m) - 1u;
        m &= m - 1u;
        const uint32_t x = none ? none_at(nw, nsw, i) : mv.ref + extract_at(mv.w, i * mv.b, bmask);  // Alg. 1
        apply_measure(c, i, x, G, W, lane);
      }
      return true;
    }
    while (m) {
      uint32_t ii[4], xx[4];
      bool ok[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        ok[q] = m != 0u;
        ii[q] = ok[q] ? __ffs(m) - 1u : 0u;
        m &= m - 1u;
        xx[q] = none ? none_at(nw, nsw, ii[q]) : mv.ref + extract_at(mv.w, ii[q] * mv.b, bmask);  // Alg. 1, one entry
      }
      if (role == TP_ROLE_RANGE) {
#pragma unroll
        for (int q = 0; q < 4; ++q)
          if (ok[q]) apply_range(c, ii[q], xx[q]);
      } else {
        const int32_t* __restrict__ T = A->table[c];
        const uint32_t kmin = (uint32_t)A->key_min[c], len = A->table_len[c];
        int32_t pl[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const uint32_t kk = xx[q] - kmin;
          pl[q] = ok[q] && kk < len ? probe_ld(T + kk) : -1;
        }
#pragma unroll
        for (int q = 0; q < 4; ++q)
          if (ok[q]) apply_payload(c, ii[q], pl[q], G, lane);
      }
    }
    return true;
  }
  __device__ void end(const Params&, const StageCtx&, const Lane&) {
    if (!GROUPED) cnt += __popc(alive);
  }
  __device__ void finish(const Params&, const Lane& g, uint32_t*) {
    if (GROUPED) {
      consumers_sync();
      for (uint32_t i = threadIdx.x - 32u; i < A->ht_slots; i += CONSUMER_WARPS * 32u) {
        const uint32_t k = keys[i];
        if (k != HT_EMPTY) {
          atomicAdd(reinterpret_cast<unsigned long long*>(A->sums) + k,
                    ((unsigned long long)hhi[i] << 32) | hlo[i]);
          atomicAdd(A->counts + k, (unsigned long long)hcnt[i]);
        }
      }
    } else {
      const uint64_t s = warp_sum_u64(acc), k = warp_sum_u64(cnt);
      if (g.lane == 0) {
        atomicAdd(reinterpret_cast<unsigned long long*>(A->sums), (unsigned long long)s);
        atomicAdd(A->counts, (unsigned long long)k);
      }
    }
  }
};

// ------------------------------------------------------------------ kernels
#ifndef TP_DFOR_LEAN
#define TP_DFOR_LEAN 1
#endif
#ifndef TP_SUM_MINB
#define TP_SUM_MINB 4
#endif
template <uint32_t MASK, bool LEAN = false>
__global__ void __launch_bounds__(THREADS, TP_SUM_MINB) k_decode_sum(const __grid_constant__ Params P, unsigned long long* out) {
  SumOp<MASK, LEAN> op;
  op.out = out;
  op.acc = 0;
  run_pipeline(P, op);
}

template <uint32_t MASK>
__global__ void __launch_bounds__(THREADS, 4)
    k_decode_global(const __grid_constant__ Params P, const __grid_constant__ CUtensorMap tmap, int32_t* out) {
  GlobalOp<MASK> op;
  op.tmap = &tmap;
  op.out = out;
  op.full_rows32 = P.n >> 5;
  run_pipeline(P, op);
}

template <uint32_t MASK>
__global__ void __launch_bounds__(THREADS, 3)
    k_select_sum(const __grid_constant__ Params P, const __grid_constant__ SelectArgs A, unsigned long long* out) {
  SelectOp<MASK> op;
  op.A = &A;
  op.out = out;
  op.acc = 0;
  op.alive = 0;
  run_query_pipeline(P, op);
}

// grouped queries: 3 CTAs / SM (the hash table and the group array); q1.x: 3 (at 4 the RFOR
// run decode spills, measured in the ptxas report)
#ifndef TP_STAR_MINB_UNGROUPED
#define TP_STAR_MINB_UNGROUPED 3
#endif
template <uint32_t MASK, bool GROUPED>
__global__ void __launch_bounds__(THREADS, GROUPED ? 3 : TP_STAR_MINB_UNGROUPED)
    k_star_query(const __grid_constant__ Params P, const __grid_constant__ StarArgs A) {
  StarOp<MASK, GROUPED> op;
  op.A = &A;
  op.acc = 0;
  op.cnt = 0;
  op.alive = 0;
  run_query_pipeline(P, op);
}


// ------------------------------------------------------------------ random access (bitvector)
// a predicate bitvector selects rows; a compressed tile whose 512 bits are all
// zero is skipped entirely (no block_starts, header or data read), otherwise it is decoded
// and the bitvector applied.  Here the skip goes further for GPU-FOR and None: a 32-row
// miniblock whose bitvector word is zero is not read either (FOR reads the block header and
// the miniblock's b words, None its one 128-byte line); GPU-DFOR / GPU-RFOR
// decode the whole tile (the prefix sum / run expansion needs every earlier entry).
// One warp per pair of tiles, lane = miniblock (the pipeline's mapping), straight from
// global memory (L1-cached loads; no staging: the access pattern is data-dependent).
template <uint32_t MASK>
__global__ void __launch_bounds__(256) k_bitmap_sum(const __grid_constant__ Params P, const uint32_t* __restrict__ bm,
                                                    unsigned long long* out) {
  extern __shared__ __align__(16) uint32_t rsm[];
  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  const uint32_t seg = lane >> 4, j = lane & 15u;
  const Col& c = P.col[0];
  const Stream& st = P.st[c.s0];
  uint32_t* scratch = rsm + warp * RFOR_SCRATCH_WORDS;
  const uint32_t npairs = (P.ntiles + 1u) >> 1;
  const uint32_t nmb = (P.n + 31u) >> 5;
  uint64_t acc = 0;
  for (uint32_t pair = blockIdx.x * (blockDim.x >> 5) + warp; pair < npairs; pair += gridDim.x * (blockDim.x >> 5)) {
    const uint32_t t = 2u * pair + seg;
    const uint32_t mb = 16u * t + j;
    uint32_t w = 0u;
    if (mb < nmb) {
      w = __ldg(bm + mb);
      const uint32_t rows = P.n - 32u * mb;
      if (rows < 32u) w &= (1u << rows) - 1u;  // bits past the column's end
    }
    const uint32_t any = __ballot_sync(FULL, w != 0u);
    if (any == 0u) continue;  // both tiles unselected: skipped without a read
    const bool tile_any = ((any >> (16u * seg)) & 0xffffu) != 0u;
    if ((MASK & M_NONE) && c.scheme == S_NONE) {
      if (w) {  // one 128-byte line per selected miniblock
        const uint4* line = reinterpret_cast<const uint4*>(st.data + 32u * mb);
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          const uint4 a = __ldg(line + q);
          const uint32_t v4[4] = {a.x, a.y, a.z, a.w};
#pragma unroll
          for (int k = 0; k < 4; ++k)
            if ((w >> (4 * q + k)) & 1u) acc += (uint64_t)(int64_t)(int32_t)v4[k];
        }
      }
    } else if ((MASK & M_FOR) && c.scheme == S_FOR) {
      // Alg. 1 for the selected miniblocks only: block_starts -> header -> the b words (the
      // bitwidth-specialised unpack, warp-collective: unselected lanes take b = 0)
      uint32_t ref = 0u, b = 0u;
      const uint32_t* mw = st.data;
      if (w) {
        const uint32_t s = __ldg(st.starts + (mb >> 2));
        ref = __ldg(st.data + s);
        const uint32_t bw = __ldg(st.data + s + 1);
        b = checked_bw((bw >> (8u * (mb & 3u))) & 255u);
        mw = st.data + s + 2 + bw_prefix(bw, mb & 3u);
      }
      uint32_t e[32];
      unpack_mb(mw, b, e);
#pragma unroll
      for (int i = 0; i < 32; ++i)
        if ((w >> i) & 1u) acc += (uint64_t)(int64_t)(int32_t)(ref + e[i]);
    } else if ((MASK & M_DFOR) && c.scheme == S_DFOR) {
      // the whole tile: deltas of every miniblock, exclusive prefix inside the tile (R13)
      uint32_t run = 0u, first = 0u, ref = 0u, b = 0u;
      const uint32_t* mw = st.data;
      const bool live = tile_any && (mb >> 2) < c.nblocks;
      if (live) {
        const uint32_t s = __ldg(st.starts + (mb >> 2));
        first = __ldg(st.data + __ldg(st.starts + 4u * t) - 1u);
        ref = __ldg(st.data + s);
        const uint32_t bw = __ldg(st.data + s + 1);
        b = checked_bw((bw >> (8u * (mb & 3u))) & 255u);
        mw = st.data + s + 2 + bw_prefix(bw, mb & 3u);
      }
      uint32_t e[32];
      unpack_mb(mw, b, e);  // b = 0 (all zero) for lanes outside a selected tile
      uint32_t val[32];
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        val[i] = run;
        run += ref + e[i];
      }
      const uint32_t incl = seg16_inclusive_scan(run);
      const uint32_t base = first + (incl - run);
#pragma unroll
      for (int i = 0; i < 32; ++i)
        if ((w >> i) & 1u) acc += (uint64_t)(int64_t)(int32_t)(val[i] + base);
    } else if (MASK & M_RFOR) {
      // the whole tile: value / run-length streams scattered and expanded (steps 1-4 of
      // decode_rfor, reading the stream blocks from global memory)
      const Stream& sl = P.st[c.s1];
      __syncwarp();
#pragma unroll 1
      for (uint32_t h = 0; h < 2; ++h) {
        uint32_t* A = rfor_A(scratch, h);
        uint8_t* F = rfor_F(scratch, h);
        rfor_clear_flags(F, lane);
        __syncwarp();
        const uint32_t th = 2u * pair + h;
        if (th >= P.ntiles || !((any >> (16u * h)) & 0xffffu)) continue;  // warp-uniform
        const uint32_t* bV = st.data + __ldg(st.starts + th);
        const uint32_t* bL = sl.data + __ldg(sl.starts + th);
        uint32_t r = __ldg(bV);
        if (r > 512u) {
          tp_flag_error(4u);  // TP_DEVERR_RUNS
          r = 512u;
        }
        rfor_block_scatter<true>(bV, bL, r, lane, A, F);
      }
      __syncwarp();
      const RforChunk k = rfor_chunk(scratch, lane);
      uint32_t val[32];
      rfor_fill(k, rfor_carry(k), val);
#pragma unroll
      for (int i = 0; i < 32; ++i)
        if ((w >> i) & 1u) acc += (uint64_t)(int64_t)(int32_t)val[i];
    }
  }
  acc = warp_sum_u64(acc);
  if (lane == 0 && acc) atomicAdd(out, (unsigned long long)acc);
}

// dimension lookup tables (the hash-table build of Crystal's star joins)
__global__ void k_fill(int32_t* __restrict__ t, uint32_t len, int32_t v) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < len; i += gridDim.x * blockDim.x) t[i] = v;
}
struct DimArgs {
  tp_dim_pred pred[4];
  int npreds;
};
__global__ void k_lookup_build(const int32_t* __restrict__ keys, uint32_t nrows, int32_t key_min, uint32_t len,
                               const __grid_constant__ DimArgs D, const int32_t* __restrict__ payload,
                               int32_t* __restrict__ table) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < nrows; i += gridDim.x * blockDim.x) {
    bool ok = true;
    for (int p = 0; p < D.npreds; ++p) {
      const int32_t a = D.pred[p].attr[i];
      ok &= (a >= D.pred[p].lo1 && a <= D.pred[p].hi1) || (a >= D.pred[p].lo2 && a <= D.pred[p].hi2);
    }
    const uint32_t k = (uint32_t)(keys[i] - key_min);
    if (ok && k < len) table[k] = payload ? payload[i] : 0;
  }
}

// uncompressed int32 scan -> sum ("None"): the HBM read roof of the same consumer
__global__ void __launch_bounds__(256) k_plain_sum(const int4* __restrict__ x4, const int32_t* __restrict__ x,
                                                   uint64_t n, unsigned long long* out) {
  uint64_t acc = 0;
  const uint64_t n4 = n >> 2;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride) {
    int4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                 : "l"(x4 + i));
    acc += (uint64_t)((int64_t)v.x + (int64_t)v.y + (int64_t)v.z + (int64_t)v.w);
  }
  if (blockIdx.x == 0 && threadIdx.x < (n & 3)) acc += (uint64_t)(int64_t)x[(n & ~uint64_t(3)) + threadIdx.x];
  acc = warp_sum_u64(acc);
  if ((threadIdx.x & 31) == 0) atomicAdd(out, (unsigned long long)acc);
}

// ================================================================== host side
static int g_sms = 0;
static int sm_count() {
  if (g_sms == 0) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_sms, cudaDevAttrMultiProcessorCount, dev);
    if (g_sms <= 0) g_sms = 148;
  }
  return g_sms;
}

#ifndef TP_MAX_STAGES
#define TP_MAX_STAGES 8
#endif
#ifndef TP_RING_KB
#define TP_RING_KB 40
#endif
#ifndef TP_QUERY_RING_KB
#define TP_QUERY_RING_KB 24
#endif
static PFN_cuTensorMapEncodeTiled_v12000 tensor_map_encoder() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  }
  return fn;
}

static uint32_t worst_tile_words(uint32_t scheme) {
  if (scheme == TP_NONE) return TILE_ROWS;
  return scheme == TP_FOR || scheme == TP_FORNM ? 4u * (2u + 128u) : scheme == TP_DFOR ? 1u + 4u * (2u + 128u) : 6u + 512u;
}
static uint32_t align4(uint32_t w) { return (w + 3u) & ~3u; }

// Validate the columns and lay out one ring item: per stream of the item's column a
// data region (TPR * rounds tiles of at most max_tile_words + alignment slop) and a
// block_starts region; item size = the largest column's.  extra_scratch: words per
// consumer warp (after the view table); agg_words: per-CTA aggregation table.
// query pipeline: the largest ring item column k can produce (a range of TPR tiles: data words
// + alignment + the unpack's over-read, block_starts words + alignment; None: one tensor box)
static uint32_t query_item_words(const tp_column& k) {
  if (k.scheme == TP_NONE) return TPR * TILE_ROWS + 256u;  // + the box's 1024-byte alignment
  uint32_t w = 0;
  for (int s = 0; s < (k.scheme == TP_RFOR ? 2 : 1); ++s) {
    uint32_t mtw = s == 0 ? k.max_tile_words0 : k.max_tile_words1;
    if (mtw == 0 || mtw > worst_tile_words(k.scheme)) mtw = worst_tile_words(k.scheme);
    const uint32_t starts = k.scheme == TP_RFOR ? TPR + 1u : 4u * TPR + 1u;
    w += align4(TPR * mtw + 6u) + 4u + align4(starts + 6u);
  }
  return w;
}

static tp_status build_params(const tp_column* cols, int ncols, uint32_t extra_scratch, uint32_t agg_words,
                              Params& P, size_t& smem_bytes, bool query = false, bool rfor_scratch = true,
                              uint32_t ring_min_words = 0) {
  memset(&P, 0, sizeof(P));
  if (!cols || ncols < 1 || ncols > TP_MAX_COLS) return TP_EINVAL;
  const uint64_t n = cols[0].n;
  if (n >= (1ull << 32)) return TP_EUNSUPPORTED;
  bool any_rfor = false, any_none = false;
  uint32_t mtws[MAX_STREAMS];
  uint32_t max_round_words = 0;  // data words of one round (TPR tiles) of the widest column
  for (int c = 0; c < ncols; ++c) {
    const tp_column& k = cols[c];
    if (k.n != n) return TP_EINVAL;
    if (k.words0 >= (1ull << 32) || k.words1 >= (1ull << 32)) return TP_EUNSUPPORTED;
    const bool rf = k.scheme == TP_RFOR;
    if (k.scheme == TP_NONE) {
      if (k.block_size != 512 || k.num_blocks != (n + 511) / 512 || k.words0 < n) return TP_EFORMAT;
      if (reinterpret_cast<uintptr_t>(k.data0) & 15u) return TP_EINVAL;
    } else if (k.scheme == TP_FOR || k.scheme == TP_DFOR) {
      if (k.block_size != 128 || k.miniblock_count != 4 || k.num_blocks != (n + 127) / 128) return TP_EFORMAT;
    } else if (k.scheme == TP_FORNM) {
      if (ncols != 1) return TP_EINVAL;  // decode / decode_sum only
      if (k.block_size != 128 || k.miniblock_count != 1 || k.num_blocks != (n + 127) / 128) return TP_EFORMAT;
    } else if (rf) {
      if (k.block_size != 512 || k.miniblock_count != 16 || k.num_blocks != (n + 511) / 512) return TP_EFORMAT;
      if (!k.starts1 || !k.data1) return TP_EINVAL;
    } else {
      return TP_EINVAL;
    }
    if (n > 0 && (!k.starts0 || !k.data0)) return TP_EINVAL;
    any_rfor |= rf;
    Col& cc = P.col[c];
    cc.scheme = k.scheme == TP_FOR ? S_FOR : k.scheme == TP_DFOR ? S_DFOR : k.scheme == TP_RFOR ? S_RFOR
              : k.scheme == TP_FORNM ? S_FORNM : S_NONE;
    cc.nblocks = (uint32_t)k.num_blocks;
    uint32_t rw = 0;
    for (int s = 0; s < (rf ? 2 : 1); ++s) {
      Stream& st = P.st[P.nstreams];
      st.data = s == 0 ? k.data0 : k.data1;
      st.starts = s == 0 ? k.starts0 : k.starts1;
      st.kind = rf ? K_RFOR : k.scheme == TP_DFOR ? K_DFOR : k.scheme == TP_NONE ? K_NONE : K_FOR;
      st.nblocks = (uint32_t)k.num_blocks;
      uint32_t mtw = s == 0 ? k.max_tile_words0 : k.max_tile_words1;
      if (mtw == 0 || mtw > worst_tile_words(k.scheme)) mtw = worst_tile_words(k.scheme);
      if (k.scheme == TP_NONE) {
        mtw = TILE_ROWS;
        any_none = true;
        // [words0 / 32][32] int32 tensor, boxes of 16 rows per tile, 128-byte swizzle (the
        // consumers' 16-byte reads of a 32-row miniblock are then bank-conflict free)
        if (n > 0) {
          auto enc = tensor_map_encoder();
          if (!enc) return TP_ECUDA;
          cuuint64_t dims[2] = {32, (cuuint64_t)(k.words0 / 32)};
          cuuint64_t strides[1] = {128};
          cuuint32_t box[2] = {32, (cuuint32_t)(TPR * (TILE_ROWS / 32))};
          cuuint32_t estr[2] = {1, 1};
          if (enc(&P.tmap[c], CU_TENSOR_MAP_DATA_TYPE_INT32, 2, const_cast<uint32_t*>(k.data0), dims, strides, box,
                  estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
            return TP_ECUDA;
        }
      }
      mtws[P.nstreams] = mtw;
      rw += TPR * mtw;
      if (s == 0) cc.s0 = P.nstreams; else cc.s1 = P.nstreams;
      ++P.nstreams;
    }
    max_round_words = std::max(max_round_words, rw);
  }
  if (query) {
    // the byte ring of the query pipeline (run_query_pipeline): at least twice the largest item
    uint32_t max_item = 0;
    for (int c = 0; c < ncols; ++c) max_item = std::max(max_item, query_item_words(cols[c]));
    P.rounds = 1;
    P.ncols = (uint32_t)ncols;
    P.n = (uint32_t)n;
    P.ntiles = (uint32_t)((n + TILE_ROWS - 1) / TILE_ROWS);
    P.ring_words = (std::max(ring_min_words, max_item + TP_RING_SLACK_WORDS) + 255u) & ~255u;
    P.nstages = 0;
    P.stage_words = 0;
    P.staging_off = (any_rfor && rfor_scratch) ? RFOR_SCRATCH_WORDS : 0u;
    P.scratch_words_per_warp = align4(P.staging_off + extra_scratch);
    P.scratch_off = P.ring_words;
    P.agg_off = P.scratch_off + CONSUMER_WARPS * P.scratch_words_per_warp;
    P.bar_off = align4(P.agg_off + agg_words);
    if (P.bar_off & 1u) ++P.bar_off;
    smem_bytes = (size_t)P.bar_off * 4 + 2 * QNS * 8 + QNS * 16 + 16;
    return TP_OK;
  }
  // rounds per item: single-column kernels carry ~16 KB of compressed words per item
  // (bytes in flight at low bitwidths, where one round is a few hundred bytes); queries
  // keep per-round row state across columns, so they use one round per item
#ifndef TP_TARGET_WORDS
#define TP_TARGET_WORDS 8192u  // ~32 KB of compressed words per GPU-FOR item (NEXT-4 sweep: b = 16
                               // 0.169 -> 0.159 ms vs 16 KB items, profiles/r02_tile_sweep*.json)
#endif
#ifndef TP_TARGET_WORDS_OTHER
#define TP_TARGET_WORDS_OTHER 4096u  // ~16 KB for the instruction-bound DFOR / RFOR decodes: their
                                     // 24 KB ring keeps 4 CTAs / SM (32 KB items: RFOR runs of 4
                                     // 0.72 -> 1.15 ms at 2 CTAs / SM, same-box A/B)
#endif
  const bool for_item = ncols == 1 && (cols[0].scheme == TP_FOR || cols[0].scheme == TP_FORNM);
  const uint32_t target_words = for_item ? TP_TARGET_WORDS : TP_TARGET_WORDS_OTHER;
  P.rounds = ncols > 1 ? 1u
                       : std::max<uint32_t>(1u, std::min<uint32_t>(8u, target_words / std::max(max_round_words, 1u)));
#ifdef TP_FIXED_ROUNDS  // the tiles-per-item sweep (NEXT-4, Fig. 5): items of 8 x TP_FIXED_ROUNDS tiles
  if (ncols == 1) P.rounds = TP_FIXED_ROUNDS;
#endif
  const uint32_t TPS = TPR * P.rounds;
  uint32_t item = 0;
  for (int c = 0; c < ncols; ++c) {
    uint32_t off = 0;
    const uint32_t q0 = P.col[c].s0, q1 = P.col[c].scheme == S_RFOR ? P.col[c].s1 : q0;
    for (uint32_t q = q0; q <= q1; ++q) {
      Stream& st = P.st[q];
      if (st.kind == K_NONE) {  // a 1024-byte aligned swizzled box, no block_starts region
        off = (off + 255u) & ~255u;
        st.data_off = off;
        off += TPS * TILE_ROWS;
        st.starts_off = off;
        continue;
      }
      st.data_off = off;
      const uint32_t region = align4(std::max<uint32_t>(TPS * mtws[q] + 12u, 48u));  // + alignment slop + unpack over-read
      // bytes the producer may copy: the region minus the unpack over-read words (16-byte multiple)
      st.data_cap = (region - 8u) * 4u & ~15u;
      off += region;
      st.starts_off = off;
      off += align4((st.kind == K_RFOR ? TPS + 1u : 4u * TPS + 1u) + 8u);
    }
    item = std::max(item, off);
  }
  P.ncols = (uint32_t)ncols;
  P.n = (uint32_t)n;
  P.ntiles = (uint32_t)((n + TILE_ROWS - 1) / TILE_ROWS);
  P.stage_words = any_none ? (item + 255u) & ~255u : align4(item);  // NONE boxes: 1024-byte aligned
  P.staging_off = any_rfor ? RFOR_SCRATCH_WORDS : 0u;
  P.scratch_words_per_warp = align4(P.staging_off + extra_scratch);
  // ring depth: 2..8 items within ~40 KB, so that several CTAs (16+ consumer warps) share
  // an SM while ~100+ KB of TMA traffic stays in flight per SM
  uint32_t nstg = TP_MAX_STAGES;
  // queries hold more per-warp state (3 CTAs/SM at most): a smaller ring keeps them at 3
  // (FOR-only single columns are HBM-bound and get the big ring; DFOR / RFOR decodes are
  // instruction-bound and trade ring space for one more resident CTA)
  const bool for_only = ncols == 1 && (P.col[0].scheme == S_FOR || P.col[0].scheme == S_FORNM);
  const uint32_t ring_kb = ncols > 1 ? TP_QUERY_RING_KB : (for_only ? TP_RING_KB : TP_QUERY_RING_KB);
  while (nstg > 2 && (size_t)nstg * P.stage_words * 4 > ring_kb * 1024) --nstg;
  P.nstages = nstg;
  P.scratch_off = (nstg * P.stage_words + 255u) & ~255u;  // 1024-byte aligned (RFOR staging in scratch)
  P.agg_off = P.scratch_off + CONSUMER_WARPS * P.scratch_words_per_warp;
  P.bar_off = align4(P.agg_off + agg_words);
  if (P.bar_off & 1u) ++P.bar_off;  // 8-byte aligned barriers
  smem_bytes = (size_t)P.bar_off * 4 + 2 * nstg * 8 + 16;
  return TP_OK;
}

template <class K>
static int grid_for(K kernel, size_t smem) {
  // the attribute + occupancy queries are host round trips into the driver in front of every
  // launch: cached per (kernel, device) -- the largest dynamic shared-memory size set so far (a
  // launch above it raises it) -- and per (kernel, size, device) for the occupancy
  struct Attr { const void* k; int dev; size_t smem; };
  struct Occ { const void* k; int dev; size_t smem; int occ; };
  static Attr attrs[64];
  static Occ occs[128];
  static int nattr = 0, nocc = 0;
  static std::mutex mu;
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lock(mu);
  int ai = -1;
  for (int i = 0; i < nattr; ++i)
    if (attrs[i].k == (const void*)kernel && attrs[i].dev == dev) ai = i;
  if (ai < 0 || attrs[ai].smem < smem) {
    cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (ai >= 0) attrs[ai].smem = smem;
    else if (nattr < 64) attrs[nattr++] = Attr{(const void*)kernel, dev, smem};
  }
  for (int i = 0; i < nocc; ++i)
    if (occs[i].k == (const void*)kernel && occs[i].dev == dev && occs[i].smem == smem) return sm_count() * occs[i].occ;
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, THREADS, smem);
  if (occ < 1) occ = 1;
  if (occ > 8) occ = 8;
  if (nocc < 128) occs[nocc++] = Occ{(const void*)kernel, dev, smem, occ};
  return sm_count() * occ;
}

static uint32_t scheme_mask(const Params& P) {
  uint32_t m = 0;
  for (uint32_t c = 0; c < P.ncols; ++c) m |= 1u << P.col[c].scheme;
  return m;
}

template <class K, class... Args>
static void launch(K kernel, size_t smem, int cap, void* stream, Args... args) {
  const int grid = std::max(1, std::min<int>(grid_for(kernel, smem), cap));
  static const bool dbg = getenv("TILEPACK_DEBUG_LAUNCH") != nullptr;  // tuning: grid / smem per launch
  if (dbg) fprintf(stderr, "TPLAUNCH grid=%d ctas_per_sm=%d smem=%zu\n", grid, grid / sm_count(), smem);
  kernel<<<grid, THREADS, smem, (cudaStream_t)stream>>>(args...);
}

static tp_status launched() {
  g_launches.fetch_add(1, std::memory_order_relaxed);
  return cudaGetLastError() == cudaSuccess ? TP_OK : TP_ECUDA;
}


#define TP_DISPATCH_MASK(MASKV, CALL)                               \
  switch (MASKV) {                                                  \
    case M_FOR: { constexpr uint32_t MK = M_FOR; CALL; } break;     \
    case M_DFOR: { constexpr uint32_t MK = M_DFOR; CALL; } break;   \
    case M_RFOR: { constexpr uint32_t MK = M_RFOR; CALL; } break;   \
    case M_FOR | M_DFOR: { constexpr uint32_t MK = M_FOR | M_DFOR; CALL; } break; \
    case M_FOR | M_RFOR: { constexpr uint32_t MK = M_FOR | M_RFOR; CALL; } break; \
    case M_DFOR | M_RFOR: { constexpr uint32_t MK = M_DFOR | M_RFOR; CALL; } break; \
    case M_NONE: { constexpr uint32_t MK = M_NONE; CALL; } break;   \
    default: { constexpr uint32_t MK = M_FOR | M_DFOR | M_RFOR | M_NONE; CALL; } break; \
  }

}  // namespace tp

using namespace tp;

extern "C" {

tp_status tp_decode_sum(const tp_column* dcol, int64_t* d_sum, void* stream) {
  if (!dcol || !d_sum) return TP_EINVAL;
  if (dcol->n == 0) return TP_OK;
  Params P;
  size_t smem = 0;
  tp_status st = build_params(dcol, 1, 0, 0, P, smem);
  if (st != TP_OK) return st;
  auto out = reinterpret_cast<unsigned long long*>(d_sum);
  const int cap = (int)((P.ntiles + 1) / 2);
  switch (scheme_mask(P)) {
    case M_FOR:
      // tiles of <= 12-bit miniblocks (4 x (2 + 4 x 12) words): the instruction-bound variant
      // (measured: lean -2.5 % at b = 12, +2.7 % at b = 16)
      if (dcol->max_tile_words0 != 0 && dcol->max_tile_words0 <= 200u)
        launch(k_decode_sum<M_FOR, true>, smem, cap, stream, P, out);
      else
        launch(k_decode_sum<M_FOR>, smem, cap, stream, P, out);
      break;
    case M_DFOR:
#if TP_DFOR_LEAN
      launch(k_decode_sum<M_DFOR, true>, smem, cap, stream, P, out);
#else
      launch(k_decode_sum<M_DFOR>, smem, cap, stream, P, out);
#endif
      break;
    case M_NONE: launch(k_decode_sum<M_NONE>, smem, cap, stream, P, out); break;
    case M_FORNM: launch(k_decode_sum<M_FORNM>, smem, cap, stream, P, out); break;
    default: launch(k_decode_sum<M_RFOR>, smem, cap, stream, P, out); break;
  }
  return launched();
}

}  // extern "C"

namespace tp {
// decode -> global through the tile pipeline; raw = packed offsets only (FOR / DFOR blocks)
tp_status decode_global_impl(const tp_column* dcol, int32_t* d_out, bool raw, void* stream) {
  if (!dcol || !d_out) return TP_EINVAL;
  if (dcol->n == 0) return TP_OK;
  if (reinterpret_cast<uintptr_t>(d_out) & 15u) return TP_EINVAL;
  if (raw && dcol->scheme == TP_RFOR) return TP_EINVAL;
  Params P;
  size_t smem = 0;
  // per warp: 2 x 4 KB swizzled staging + 1 KB alignment slop (RFOR: staged in its expansion
  // scratch).  GPU-DFOR at >= TP_DFOR_SINGLE_BITS bits / int takes one buffer -- 4 CTAs / SM
  // instead of 3; measured on 500M rows: sorted-uniform (3.6 bits) -12 %, near-sorted (5.9) -6 %,
  // but D1 (1.8, closer to the HBM roof) +5 %.  (A slop-free double buffer costs FOR b = 4 7 %.)
  const bool single = TP_GLOBAL_SINGLE_DFOR && dcol->scheme == TP_DFOR && !raw &&
                      (double)dcol->words0 * 32.0 >= TP_DFOR_SINGLE_BITS * (double)dcol->n;
  const uint32_t staging = dcol->scheme == TP_RFOR ? 0u : (single ? 1024u : 2048u) + 256u;
  tp_status st = build_params(dcol, 1, staging, 0, P, smem);
  if (st != TP_OK) return st;
  P.single_staging = single ? 1u : 0u;
  CUtensorMap tmap;
  memset(&tmap, 0, sizeof(tmap));
  const uint32_t rows32 = (uint32_t)(dcol->n / 32);
  if (rows32 > 0) {
    auto enc = tensor_map_encoder();
    if (!enc) return TP_ECUDA;
    cuuint64_t dims[2] = {32, rows32};
    cuuint64_t strides[1] = {128};
    cuuint32_t box[2] = {32, 32};
    cuuint32_t estr[2] = {1, 1};
    if (enc(&tmap, CU_TENSOR_MAP_DATA_TYPE_INT32, 2, d_out, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return TP_ECUDA;
  }
  const int cap = (int)((P.ntiles + 1) / 2);
  if (raw) {
    launch(k_decode_global<M_RAW>, smem, cap, stream, P, tmap, d_out);
    return launched();
  }
  switch (scheme_mask(P)) {
    case M_FOR: launch(k_decode_global<M_FOR>, smem, cap, stream, P, tmap, d_out); break;
    case M_FORNM: launch(k_decode_global<M_FORNM>, smem, cap, stream, P, tmap, d_out); break;
    case M_DFOR: launch(k_decode_global<M_DFOR>, smem, cap, stream, P, tmap, d_out); break;
    case M_NONE: launch(k_decode_global<M_NONE>, smem, cap, stream, P, tmap, d_out); break;
    default: launch(k_decode_global<M_RFOR>, smem, cap, stream, P, tmap, d_out); break;
  }
  return launched();
}
}  // namespace tp

extern "C" {

tp_status tp_decode(const tp_column* dcol, int32_t* d_out, void* stream) {
  return decode_global_impl(dcol, d_out, false, stream);
}

tp_status tp_select_project_sum(const tp_column* dcols, int ncols, const int32_t* lo, const int32_t* hi, int proj_op,
                                int a, int b, int64_t* d_result, void* stream) {
  if (!dcols || !lo || !hi || !d_result || ncols < 1 || ncols > TP_MAX_COLS) return TP_EINVAL;
  if (proj_op < TP_PROJ_COL || proj_op > TP_PROJ_COUNT) return TP_EINVAL;
  for (int c = 0; c < ncols; ++c)
    if (dcols[c].scheme == TP_FORNM) return TP_EINVAL;  // the ablation format: decode / decode_sum only
  if (proj_op != TP_PROJ_COUNT && (a < 0 || a >= ncols)) return TP_EINVAL;
  if ((proj_op == TP_PROJ_MUL || proj_op == TP_PROJ_SUB) && (b < 0 || b >= ncols)) return TP_EINVAL;
  if (dcols[0].n == 0) return TP_OK;
  // evaluation order: predicate-only columns first, then a, then b (a == b decodes twice;
  // predicates are idempotent)
  const bool use_a = proj_op != TP_PROJ_COUNT, use_b = proj_op == TP_PROJ_MUL || proj_op == TP_PROJ_SUB;
  tp_column ord[TP_MAX_COLS + 1];
  SelectArgs A;
  memset(&A, 0, sizeof(A));
  A.proj = proj_op;
  int k = 0;
  for (int c = 0; c < ncols; ++c) {
    if ((use_a && c == a) || (use_b && c == b)) continue;
    ord[k] = dcols[c]; A.lo[k] = lo[c]; A.hi[k] = hi[c]; ++k;
  }
  A.npred = (uint32_t)k;
  if (use_a) { ord[k] = dcols[a]; A.lo[k] = lo[a]; A.hi[k] = hi[a]; ++k; A.has_a = 1; }
  if (use_b) {
    if (k >= TP_MAX_COLS) return TP_EINVAL;
    ord[k] = dcols[b]; A.lo[k] = lo[b]; A.hi[k] = hi[b]; ++k; A.has_b = 1;
  }
  Params P;
  size_t smem = 0;
  uint32_t ring_min = TP_STAR_RING_WORDS;
  if (const char* e = getenv("TILEPACK_QUERY_RING_WORDS")) ring_min = (uint32_t)atoi(e);  // tests: a tight ring
  tp_status st = build_params(ord, k, 0, 0, P, smem, true, true, ring_min);
  if (st != TP_OK) return st;
  auto out = reinterpret_cast<unsigned long long*>(d_result);
  const int cap = (int)((P.ntiles + 1) / 2);
  TP_DISPATCH_MASK(scheme_mask(P), launch(k_select_sum<MK>, smem, cap, stream, P, A, out));
  return launched();
}

tp_status tp_lookup_build(const int32_t* d_keys, uint64_t nrows, int32_t key_min, uint32_t table_len,
                          const tp_dim_pred* preds, int npreds, const int32_t* d_payload, int32_t* d_table,
                          void* stream) {
  if (!d_table || (nrows && !d_keys) || npreds < 0 || npreds > 4 || (npreds && !preds)) return TP_EINVAL;
  if (nrows >= (1ull << 32)) return TP_EUNSUPPORTED;
  DimArgs D;
  memset(&D, 0, sizeof(D));
  for (int p = 0; p < npreds; ++p) {
    if (!preds[p].attr) return TP_EINVAL;
    D.pred[p] = preds[p];
  }
  D.npreds = npreds;
  const int grid = sm_count() * 4;
  k_fill<<<grid, 256, 0, (cudaStream_t)stream>>>(d_table, table_len, -1);
  tp_status st = launched();
  if (st != TP_OK || nrows == 0) return st;
  k_lookup_build<<<grid, 256, 0, (cudaStream_t)stream>>>(d_keys, (uint32_t)nrows, key_min, table_len, D, d_payload,
                                                         d_table);
  return launched();
}

tp_status tp_star_query(const tp_column* dcols, const tp_star_col* roles, int ncols, int agg, int64_t* d_sums,
                        uint64_t* d_counts, uint32_t ngroups, void* stream) {
  if (!dcols || !roles || !d_sums || !d_counts || ncols < 1 || ncols > TP_MAX_COLS || ngroups < 1) return TP_EINVAL;
  if (agg < TP_AGG_SUM || agg > TP_AGG_SUB) return TP_EINVAL;
  for (int c = 0; c < ncols; ++c)
    if (dcols[c].scheme == TP_FORNM) return TP_EINVAL;  // the ablation format: decode / decode_sum only
  int nmeas = 0;
  for (int c = 0; c < ncols; ++c) {
    const tp_star_col& r = roles[c];
    if (r.role < TP_ROLE_RANGE || r.role > TP_ROLE_MEASURE) return TP_EINVAL;
    if (r.role == TP_ROLE_PROBE && (!r.table || r.table_len == 0)) return TP_EINVAL;
    if (r.role == TP_ROLE_MEASURE) ++nmeas;
  }
  // the last column aggregates; with MUL / SUB one earlier measure is staged
  if (roles[ncols - 1].role != TP_ROLE_MEASURE || nmeas != (agg == TP_AGG_SUM ? 1 : 2)) return TP_EINVAL;
  if (dcols[0].n == 0) return TP_OK;
  const bool grouped = ngroups > 1;
  StarArgs A;
  memset(&A, 0, sizeof(A));
  bool gseen = false;
  for (int c = 0; c < ncols; ++c) {
    A.role[c] = roles[c].role; A.lo[c] = roles[c].lo; A.hi[c] = roles[c].hi;
    A.table[c] = roles[c].table; A.key_min[c] = roles[c].key_min;
    A.table_len[c] = roles[c].table_len; A.stride[c] = roles[c].stride;
    if (roles[c].role == TP_ROLE_PROBE && grouped && roles[c].stride) {
      A.gmode[c] = gseen ? 2u : 1u;
      gseen = true;
    }
    A.mstage[c] = roles[c].role == TP_ROLE_MEASURE && c != ncols - 1;
  }
  A.gzero = grouped && !gseen;
  // dense probes into a table too large for L1 bypass it and stay in L2 (evict_last); smaller
  // tables (supplier, date) keep their L1 hits
  uint32_t hint_min = TP_PROBE_HINT_MIN;
  if (const char* e = getenv("TILEPACK_PROBE_HINT_MIN")) hint_min = (uint32_t)atoi(e);  // tuning
  for (int c = 0; c < ncols; ++c)
    if (roles[c].role == TP_ROLE_PROBE && roles[c].table_len >= hint_min) A.hint_mask |= 1u << c;
  A.agg = agg;
  A.ngroups = ngroups;
  A.sparse_max = TP_SPARSE_MAX;
  A.sparse_lane_max = TP_SPARSE_LANE_MAX;
  A.rfor_sparse_max = TP_RFOR_SPARSE_MAX;
  if (const char* e = getenv("TILEPACK_RFOR_SPARSE_MAX")) A.rfor_sparse_max = std::min(64, atoi(e));  // tests
  if (const char* e = getenv("TILEPACK_SPARSE_LANE_MAX")) A.sparse_lane_max = (uint32_t)atoi(e);  // tuning
  if (const char* e = getenv("TILEPACK_SPARSE_MAX")) A.sparse_max = (uint32_t)atoi(e);  // tests: force a mode
  const uint32_t hts = grouped ? ht_slots(ngroups) : 0u;
  // byte ring: 24 KB next to the grouped queries' hash table and group arrays (3 CTAs / SM),
  // 32 KB for q1.x (4 CTAs / SM); at least twice the largest item either way
  uint32_t ring_min = grouped ? TP_STAR_RING_WORDS_GROUPED : TP_STAR_RING_WORDS;
  if (const char* e = getenv("TILEPACK_QUERY_RING_WORDS")) ring_min = (uint32_t)atoi(e);  // tests: a tight ring
  bool any_rfor = false;
  for (int c = 0; c < ncols; ++c) any_rfor |= dcols[c].scheme == TP_RFOR;
  const uint32_t gwords = grouped ? 32u * 32u : 0u, wwords = nmeas == 2 ? 32u * 32u : 0u;
  const uint32_t rwords = any_rfor ? STAR_RA_WORDS + STAR_SB_WORDS : 0u;
  Params P;
  size_t smem = 0;
  tp_status st = build_params(dcols, ncols, gwords + wwords + rwords, 4u * hts, P, smem, true, false, ring_min);
  if (st != TP_OK) return st;
  A.gs_off = 0;
  A.ws_off = gwords;
  A.ra_off = gwords + wwords;
  A.sb_off = A.ra_off + STAR_RA_WORDS;
  A.ht_slots = hts;
  A.ht_shift = 32u - (uint32_t)__builtin_ctz(hts ? hts : 1u);
  A.sums = reinterpret_cast<long long*>(d_sums);
  A.counts = reinterpret_cast<unsigned long long*>(d_counts);
  const int cap = (int)((P.ntiles + 1) / 2);
  if (grouped) {
    TP_DISPATCH_MASK(scheme_mask(P), (launch(k_star_query<MK, true>, smem, cap, stream, P, A)));
  } else {
    TP_DISPATCH_MASK(scheme_mask(P), (launch(k_star_query<MK, false>, smem, cap, stream, P, A)));
  }
  return launched();
}

tp_status tp_plain_sum(const int32_t* d_x, uint64_t n, int64_t* d_sum, void* stream) {
  if (!d_x || !d_sum) return TP_EINVAL;
  if (n == 0) return TP_OK;
  if (reinterpret_cast<uintptr_t>(d_x) & 15u) return TP_EINVAL;
  const int grid = sm_count() * 8;
  k_plain_sum<<<grid, 256, 0, (cudaStream_t)stream>>>(reinterpret_cast<const int4*>(d_x), d_x, n,
                                                      reinterpret_cast<unsigned long long*>(d_sum));
  return launched();
}

tp_status tp_bitmap_sum(const tp_column* dcol, const uint32_t* d_bitmap, int64_t* d_sum, void* stream) {
  if (!dcol || !d_bitmap || !d_sum || dcol->scheme == TP_FORNM) return TP_EINVAL;
  if (dcol->n == 0) return TP_OK;
  Params P;
  size_t smem_unused = 0;
  tp_status st = build_params(dcol, 1, 0, 0, P, smem_unused);
  if (st != TP_OK) return st;
  auto out = reinterpret_cast<unsigned long long*>(d_sum);
  const bool rf = dcol->scheme == TP_RFOR;
  const size_t smem = rf ? 8u * RFOR_SCRATCH_WORDS * 4u : 0u;
  const uint32_t npairs = (P.ntiles + 1) / 2;
  auto go = [&](auto kernel) {
    cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, 256, smem);
    const int grid = std::max(1, std::min<int>(sm_count() * std::max(1, occ), (int)((npairs + 7) / 8)));
    kernel<<<grid, 256, smem, (cudaStream_t)stream>>>(P, d_bitmap, out);
  };
  switch (scheme_mask(P)) {
    case M_FOR: go(k_bitmap_sum<M_FOR>); break;
    case M_DFOR: go(k_bitmap_sum<M_DFOR>); break;
    case M_NONE: go(k_bitmap_sum<M_NONE>); break;
    default: go(k_bitmap_sum<M_RFOR>); break;
  }
  return launched();
}

uint64_t tp_launch_count(void) { return g_launches.load(); }

tp_status tp_device_errors(uint32_t* flags, void* stream) {
  if (!flags) return TP_EINVAL;
  if (cudaStreamSynchronize((cudaStream_t)stream) != cudaSuccess) return TP_ECUDA;
  uint32_t v = 0;
  if (cudaMemcpyFromSymbol(&v, g_tp_err, sizeof(v)) != cudaSuccess) return TP_ECUDA;
  static const uint32_t zero = 0;
  if (cudaMemcpyToSymbol(g_tp_err, &zero, sizeof(zero)) != cudaSuccess) return TP_ECUDA;
  *flags = v;
  return TP_OK;
}

/* profiling builds (-DTP_PROFILE_WAITS): copy out and reset the cycle counters */
tp_status tp_debug_counters(uint64_t* out16) {
  if (cudaMemcpyFromSymbol(out16, g_prof, sizeof(unsigned long long) * 16) != cudaSuccess) return TP_ECUDA;
  static const unsigned long long zero[16] = {0};
  if (cudaMemcpyToSymbol(g_prof, zero, sizeof(zero)) != cudaSuccess) return TP_ECUDA;
  return TP_OK;
}

tp_status tp_device_info(int* sms, int* ctas_per_sm) {
  if (sms) *sms = sm_count();
  if (ctas_per_sm) {
    tp_column c;
    memset(&c, 0, sizeof(c));
    c.scheme = TP_FOR; c.block_size = 128; c.miniblock_count = 4; c.n = 1 << 20; c.num_blocks = (1 << 20) / 128;
    c.starts0 = reinterpret_cast<const uint32_t*>(16); c.data0 = c.starts0;
    c.max_tile_words0 = 4 * (2 + 4 * 16);  // the bench column (b = 16)
    Params P;
    size_t smem = 0;
    build_params(&c, 1, 0, 0, P, smem);
    *ctas_per_sm = grid_for(k_decode_sum<M_FOR>, smem) / sm_count();
  }
  return TP_OK;
}

}  // extern "C"
