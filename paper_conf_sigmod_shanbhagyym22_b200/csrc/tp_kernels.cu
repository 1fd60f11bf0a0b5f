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
#include <cstring>

#include "tilepack.h"
#include "tp_device.cuh"

namespace tp {

std::atomic<uint64_t> g_launches{0};

// ------------------------------------------------------------------ stage context
struct StageCtx {
  const uint32_t* stage;  // this stage's shared words
  uint32_t tile_base;     // first tile of the stage
  uint32_t tile_end;      // one past the last tile of the stage (CTA range)
};

struct StreamView {
  const uint32_t* sd;  // data region
  const uint32_t* ss;  // block_starts region
  uint32_t lo;         // first copied data word (global index)
  uint32_t dshift, sshift;
};

__device__ __forceinline__ StreamView stream_view(const Params& P, uint32_t s, const StageCtx& C) {
  const Stream& st = P.st[s];
  StreamView v;
  const uint32_t sidx = st.kind == K_RFOR ? C.tile_base : 4u * C.tile_base;
  v.ss = C.stage + st.starts_off;
  v.sshift = align_shift(st.starts, sidx);
  v.lo = v.ss[v.sshift] - (st.kind == K_DFOR ? 1u : 0u);
  v.sd = C.stage + st.data_off;
  v.dshift = align_shift(st.data, v.lo);
  return v;
}

// lane geometry inside a consumer warp: 2 tiles x 16 miniblocks
struct Lane {
  uint32_t lane, cw;          // lane id, consumer warp id
  uint32_t tile_local;        // tile inside the stage
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

// ---------------------------------------------------------------- GPU-FOR decode
// LoadBitPack analogue: the thread's 32 rows of the tile.
__device__ __forceinline__ void decode_for(const Params& P, const Col& c, const StageCtx& C, const Lane& g,
                                           uint32_t (&val)[32]) {
  const StreamView v = stream_view(P, c.s0, C);
  const uint32_t lb = 4u * g.tile_local + (g.mb >> 2);
  const bool tv = C.tile_base + g.tile_local < C.tile_end;
  const MbView m = for_view(v.sd, v.ss, v.lo, v.dshift, v.sshift, tv ? 4u * C.tile_base + lb : UINT_MAX,
                            c.nblocks, lb, g.mb & 3u);
  uint32_t e[32];
  unpack_mb(m.w, m.b, e);
#pragma unroll
  for (int i = 0; i < 32; ++i) val[i] = m.ref + e[i];  // Alg. 1 line 18
}

// ---------------------------------------------------------------- GPU-DFOR decode
// LoadDBitPack analogue: unpack the deltas of the thread's 32
// slots, then the tile-wide exclusive prefix sum (R13) -- a
// register scan inside the thread plus a 16-lane shuffle scan across the
// tile's miniblocks -- plus the tile's first value (Fig. 6).
__device__ __forceinline__ void decode_dfor(const Params& P, const Col& c, const StageCtx& C, const Lane& g,
                                            uint32_t (&val)[32]) {
  const StreamView v = stream_view(P, c.s0, C);
  const uint32_t lb = 4u * g.tile_local + (g.mb >> 2);
  const bool tv = C.tile_base + g.tile_local < C.tile_end;
  const MbView m = for_view(v.sd, v.ss, v.lo, v.dshift, v.sshift, tv ? 4u * C.tile_base + lb : UINT_MAX,
                            c.nblocks, lb, g.mb & 3u);
  uint32_t first = 0u;
  if (tv) first = v.sd[v.ss[v.sshift + 4u * g.tile_local] - 1u - v.lo + v.dshift];
  uint32_t e[32];
  unpack_mb(m.w, m.b, e);
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
// LoadRBitPack analogue: unpack the value and run-length stream
// blocks of the row block (lane j of a 16-lane half takes entries 32j..32j+31
// of both streams), exclusive scan of the run lengths -> run starts S, then
// each thread expands its 32 rows by a search + forward walk over S in the
// warp's scratch (result == repeat(V, L), R19).
__device__ __forceinline__ uint32_t pad33(uint32_t e) { return e + (e >> 5); }
constexpr uint32_t RFOR_HALF_WORDS = 1072;  // S (529) + V (528), padded so the halves' banks differ by 16
constexpr uint32_t RFOR_SCRATCH_WORDS = 2 * RFOR_HALF_WORDS;

struct RforHdr {
  const uint32_t* w;
  uint32_t ref, b, r, cnt;
};
__device__ __forceinline__ RforHdr rfor_hdr(const StreamView& v, uint32_t tile_local, uint32_t j, bool tv) {
  RforHdr h;
  h.r = 0u; h.cnt = 0u; h.ref = 0u; h.b = 0u; h.w = v.sd;
  if (!tv) return h;
  const uint32_t* blk = v.sd + (v.ss[v.sshift + tile_local] - v.lo + v.dshift);
  h.r = blk[0];       // run / value count
  h.ref = blk[1];
  uint32_t off = 0u;
#pragma unroll
  for (uint32_t q = 0; q < 4; ++q) {
    const uint32_t bw = blk[2 + q];
    if (q < (j >> 2)) off += (bw * 0x01010101u) >> 24;
    else if (q == (j >> 2)) { off += bw_prefix(bw, j & 3u); h.b = min((bw >> (8u * (j & 3u))) & 255u, 32u); }
  }
  h.w = blk + 6u + off;  // [r][ref][4 bitwidth words] then tight miniblocks (R17)
  const int rem = (int)h.r - 32 * (int)j;
  h.cnt = rem <= 0 ? 0u : (rem >= 32 ? 32u : (uint32_t)rem);
  return h;
}

__device__ __forceinline__ void decode_rfor(const Params& P, const Col& c, const StageCtx& C, const Lane& g,
                                            uint32_t* scratch, uint32_t (&val)[32]) {
  const StreamView vv = stream_view(P, c.s0, C), vl = stream_view(P, c.s1, C);
  const bool tv = C.tile_base + g.tile_local < C.tile_end;
  const uint32_t j = g.mb;
  const RforHdr hv = rfor_hdr(vv, g.tile_local, j, tv), hl = rfor_hdr(vl, g.tile_local, j, tv);  // hv.r == hl.r
  uint32_t* S = scratch + (g.lane >> 4) * RFOR_HALF_WORDS;
  uint32_t* V = S + 529;
  uint32_t ev[32], el[32];
  unpack_mb(hv.w, hv.b, ev);
  unpack_mb(hl.w, hl.b, el);
  // local exclusive scan of the run lengths of entries 32j..32j+cnt-1
  uint32_t run = 0u;
#pragma unroll
  for (int i = 0; i < 32; ++i) {
    const uint32_t len = (uint32_t)i < hl.cnt ? hl.ref + el[i] : 0u;
    el[i] = run;
    run += len;
  }
  const uint32_t incl = seg16_inclusive_scan(run);
  const uint32_t sbase = incl - run;
#pragma unroll
  for (int i = 0; i < 32; ++i) {
    if ((uint32_t)i < hl.cnt) {
      S[33u * j + i] = sbase + el[i];
      V[33u * j + i] = hv.ref + ev[i];
    }
  }
  if (j == 0 && hl.r > 0u) S[pad33(hl.r)] = 0x7fffffffu;  // sentinel
  __syncwarp();
  // expand: rows 32j .. 32j+31 of the row block
  const uint32_t row0 = 32u * j, r = hl.r;
  if (r > 0u) {
    uint32_t a = 0u, bnd = r;
    while (bnd - a > 1u) {
      const uint32_t mid = (a + bnd) >> 1;
      if (S[pad33(mid)] <= row0) a = mid; else bnd = mid;
    }
    uint32_t cur = a, nxt = S[pad33(a + 1u)], x = V[pad33(a)];
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      if (row0 + i >= nxt) {
        ++cur;
        x = V[pad33(cur)];
        nxt = S[pad33(cur + 1u)];
      }
      val[i] = x;
    }
  } else {
#pragma unroll
    for (int i = 0; i < 32; ++i) val[i] = 0u;
  }
  __syncwarp();
}

__device__ __forceinline__ void decode_col(const Params& P, uint32_t ci, const StageCtx& C, const Lane& g,
                                           uint32_t* scratch, uint32_t (&val)[32]) {
  const Col& c = P.col[ci];
  if (c.scheme == S_FOR) decode_for(P, c, C, g, val);
  else if (c.scheme == S_DFOR) decode_dfor(P, c, C, g, val);
  else decode_rfor(P, c, C, g, scratch, val);
}

// ------------------------------------------------------------------ the pipeline
// warp 0: TMA producer; warps 1..CONSUMER_WARPS: consumers (Op::stage).
template <class Op>
__device__ __forceinline__ void run_pipeline(const Params& P, Op& op) {
  extern __shared__ __align__(1024) uint32_t smem[];
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31u;
  // CTA tile range, in pairs of tiles so that a consumer warp's 1024 rows
  // never straddle two CTAs (decode->global stores whole warp boxes)
  const uint32_t npairs = (P.ntiles + 1u) >> 1;
  const uint32_t p0 = (uint32_t)((uint64_t)blockIdx.x * npairs / gridDim.x);
  const uint32_t p1 = (uint32_t)((uint64_t)(blockIdx.x + 1) * npairs / gridDim.x);
  const uint32_t t0 = 2u * p0, t1 = min(2u * p1, P.ntiles);
  if (t0 >= t1) return;
  const uint32_t nst = (t1 - t0 + TPS - 1) / TPS;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + P.scratch_off + CONSUMER_WARPS * P.scratch_words_per_warp);
  uint64_t* empty = full + P.nstages;
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
    for (uint32_t sb = 0; sb < nst; sb += 31) {
      // lane i prefetches every stream's block_starts entry at the start of stage sb+i
      const uint32_t tb = min(t0 + (sb + lane) * TPS, t1);
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
      const uint32_t se = min(sb + 31, nst);
      for (uint32_t s = sb; s < se; ++s) {
        const uint32_t slot = s % P.nstages;
        if (s >= P.nstages) mbar_wait(&empty[slot], ((s / P.nstages) + 1u) & 1u);
        const uint32_t tile_base = t0 + s * TPS, tile_end = min(tile_base + TPS, t1);
        uint32_t mylo = 0u, myhi = 0u;
#pragma unroll
        for (int q = 0; q < MAX_STREAMS; ++q) {
          if ((uint32_t)q < P.nstreams) {
            const uint32_t a = __shfl_sync(FULL, bnd[q], s - sb);
            const uint32_t b = __shfl_sync(FULL, bnd[q], s - sb + 1);
            if (lane == (uint32_t)q) { mylo = a; myhi = b; }
          }
        }
        uint32_t bytes = 0u;
        const char *dsrc = nullptr, *ssrc = nullptr;
        uint32_t dbytes = 0u, sbytes = 0u;
        uint32_t* dst_d = nullptr;
        uint32_t* dst_s = nullptr;
        if (lane < P.nstreams) {
          const Stream& st = P.st[lane];
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
          uint32_t* sbase = smem + slot * P.stage_words;
          dst_d = sbase + st.data_off;
          dst_s = sbase + st.starts_off;
          bytes = dbytes + sbytes;
        }
        const uint32_t total = __reduce_add_sync(FULL, bytes);
        if (lane == 0) mbar_arrive_expect_tx(&full[slot], total);
        __syncwarp();
        if (lane < P.nstreams) {
          bulk_g2s(dst_d, dsrc, dbytes, &full[slot], pol);
          bulk_g2s(dst_s, ssrc, sbytes, &full[slot], pol);
        }
      }
    }
  } else {
    // ---------------- consumers
    const Lane g = lane_geom();
    uint32_t* scratch = smem + P.scratch_off + g.cw * P.scratch_words_per_warp;
    for (uint32_t s = 0; s < nst; ++s) {
      const uint32_t slot = s % P.nstages;
      mbar_wait(&full[slot], (s / P.nstages) & 1u);
      StageCtx C;
      C.stage = smem + slot * P.stage_words;
      C.tile_base = t0 + s * TPS;
      C.tile_end = min(C.tile_base + TPS, t1);
      op.stage(P, C, g, scratch, s);
      __syncwarp();
      if (g.lane == 0) mbar_arrive(&empty[slot]);
    }
    op.finish(P, g);
  }
}

// ------------------------------------------------------------------ consumers
__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t x) {
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) x += __shfl_xor_sync(FULL, x, d);
  return x;
}

// decode -> sum (decode-only microbenchmark)
struct SumOp {
  unsigned long long* out;
  uint64_t acc;
  __device__ void stage(const Params& P, const StageCtx& C, const Lane& g, uint32_t* scratch, uint32_t) {
    const Col& c = P.col[0];
    const uint32_t tile = C.tile_base + g.tile_local;
    const uint32_t row0 = tile * TILE_ROWS + g.mb * MB_ROWS;
    const bool tv = tile < C.tile_end;
    if (c.scheme == S_FOR) {
      const StreamView v = stream_view(P, c.s0, C);
      const uint32_t lb = 4u * g.tile_local + (g.mb >> 2);
      const MbView m = for_view(v.sd, v.ss, v.lo, v.dshift, v.sshift, tv ? 4u * C.tile_base + lb : UINT_MAX,
                                c.nblocks, lb, g.mb & 3u);
      if (tv && row0 + MB_ROWS <= P.n) {
        const uint64_t se = sum_mb(m.w, m.b);
        acc += se + (uint64_t)((int64_t)(int32_t)m.ref * 32);
      } else {
        uint32_t e[32];
        unpack_mb(m.w, m.b, e);
#pragma unroll
        for (int i = 0; i < 32; ++i)
          if (tv && row0 + i < P.n) acc += (uint64_t)(int64_t)(int32_t)(m.ref + e[i]);
      }
    } else {
      uint32_t val[32];
      decode_col(P, 0, C, g, scratch, val);
      if (tv && row0 + MB_ROWS <= P.n) {
#pragma unroll
        for (int i = 0; i < 32; ++i) acc += (uint64_t)(int64_t)(int32_t)val[i];
      } else {
#pragma unroll
        for (int i = 0; i < 32; ++i)
          if (tv && row0 + i < P.n) acc += (uint64_t)(int64_t)(int32_t)val[i];
      }
    }
  }
  __device__ void finish(const Params&, const Lane& g) {
    const uint64_t s = warp_sum_u64(acc);
    if (g.lane == 0) atomicAdd(out, (unsigned long long)s);
  }
};

// decode -> global (Fig. 7a mode): the warp's 1024 rows go to a
// 128B-swizzled 4 KB shared buffer (conflict-free 16-byte stores) and leave by
// one TMA tensor store; the partial last miniblock (n % 32 rows) is stored directly.
struct GlobalOp {
  const CUtensorMap* tmap;
  int32_t* out;
  uint32_t full_rows32;  // n / 32: rows of the [n/32][32] tensor
  __device__ void stage(const Params& P, const StageCtx& C, const Lane& g, uint32_t* scratch, uint32_t s) {
    uint32_t val[32];
    decode_col(P, 0, C, g, scratch, val);
    const uint32_t pair_tile = C.tile_base + 2u * g.cw;
    if (pair_tile >= C.tile_end) return;  // warp-uniform
    // staging buffers: 2 x 4 KB per warp, 1024-aligned, after the RFOR scratch
    uint32_t* buf = scratch + P.staging_off;
    buf = reinterpret_cast<uint32_t*>((reinterpret_cast<uintptr_t>(buf) + 1023) & ~uintptr_t(1023));
    buf += (s & 1u) * 1024u;
    if (g.lane == 0) bulk_wait_read<1>();  // the store issued from this buffer two stages ago is done reading
    __syncwarp();
    const uint32_t l = g.lane;
#pragma unroll
    for (uint32_t q = 0; q < 8; ++q) {
      uint4 v4 = make_uint4(val[4 * q], val[4 * q + 1], val[4 * q + 2], val[4 * q + 3]);
      *reinterpret_cast<uint4*>(buf + l * 32u + ((q ^ (l & 7u)) << 2)) = v4;
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
  __device__ void finish(const Params&, const Lane& g) {
    if (g.lane == 0) bulk_wait_all();
    __syncwarp();
  }
};

// select / project / aggregate over up to 6 columns
struct SelectOp {
  int32_t lo[TP_MAX_COLS], hi[TP_MAX_COLS];
  int proj, a, b;
  unsigned long long* out;
  uint64_t acc;
  __device__ void stage(const Params& P, const StageCtx& C, const Lane& g, uint32_t* scratch, uint32_t) {
    const uint32_t tile = C.tile_base + g.tile_local;
    const uint32_t row0 = tile * TILE_ROWS + g.mb * MB_ROWS;
    uint32_t alive = 0u;
    if (tile < C.tile_end && row0 < P.n) {
      const uint32_t nrows = P.n - row0;
      alive = nrows >= 32u ? 0xffffffffu : ((1u << nrows) - 1u);
    }
    uint32_t va[32], vb[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) { va[i] = 0u; vb[i] = 0u; }
    for (uint32_t c = 0; c < P.ncols; ++c) {
      uint32_t v[32];
      decode_col(P, c, C, g, scratch, v);
      const int32_t l = lo[c], h = hi[c];
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        const int32_t x = (int32_t)v[i];
        if (x < l || x > h) alive &= ~(1u << i);
      }
      if ((int)c == a) {
#pragma unroll
        for (int i = 0; i < 32; ++i) va[i] = v[i];
      }
      if ((int)c == b) {
#pragma unroll
        for (int i = 0; i < 32; ++i) vb[i] = v[i];
      }
    }
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      if (alive & (1u << i)) {
        int64_t t;
        const int64_t xa = (int32_t)va[i], xb = (int32_t)vb[i];
        if (proj == TP_PROJ_COL) t = xa;
        else if (proj == TP_PROJ_MUL) t = xa * xb;
        else if (proj == TP_PROJ_SUB) t = xa - xb;
        else t = 1;
        acc += (uint64_t)t;
      }
    }
  }
  __device__ void finish(const Params&, const Lane& g) {
    const uint64_t s = warp_sum_u64(acc);
    if (g.lane == 0) atomicAdd(out, (unsigned long long)s);
  }
};

__global__ void __launch_bounds__(THREADS) k_decode_sum(const __grid_constant__ Params P, unsigned long long* out) {
  SumOp op;
  op.out = out;
  op.acc = 0;
  run_pipeline(P, op);
}

__global__ void __launch_bounds__(THREADS)
    k_decode_global(const __grid_constant__ Params P, const __grid_constant__ CUtensorMap tmap, int32_t* out) {
  GlobalOp op;
  op.tmap = &tmap;
  op.out = out;
  op.full_rows32 = P.n >> 5;
  run_pipeline(P, op);
}

struct SelectArgs {
  int32_t lo[TP_MAX_COLS], hi[TP_MAX_COLS];
  int proj, a, b;
};
__global__ void __launch_bounds__(THREADS)
    k_select_sum(const __grid_constant__ Params P, const __grid_constant__ SelectArgs A, unsigned long long* out) {
  SelectOp op;
  for (int c = 0; c < TP_MAX_COLS; ++c) { op.lo[c] = A.lo[c]; op.hi[c] = A.hi[c]; }
  op.proj = A.proj; op.a = A.a; op.b = A.b;
  op.out = out;
  op.acc = 0;
  run_pipeline(P, op);
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

static uint32_t worst_tile_words(uint32_t scheme) {
  return scheme == TP_FOR ? 4u * (2u + 128u) : scheme == TP_DFOR ? 1u + 4u * (2u + 128u) : 6u + 512u;
}
static uint32_t align4(uint32_t w) { return (w + 3u) & ~3u; }

// Validate columns and lay the stage out: per stream a data region
// (TPS tiles of at most max_tile_words + alignment slop) and a block_starts region.
static tp_status build_params(const tp_column* cols, int ncols, uint32_t extra_scratch,
                              Params& P, size_t& smem_bytes) {
  memset(&P, 0, sizeof(P));
  if (!cols || ncols < 1 || ncols > TP_MAX_COLS) return TP_EINVAL;
  const uint64_t n = cols[0].n;
  if (n >= (1ull << 32)) return TP_EUNSUPPORTED;
  uint32_t off = 0;
  bool any_rfor = false;
  for (int c = 0; c < ncols; ++c) {
    const tp_column& k = cols[c];
    if (k.n != n) return TP_EINVAL;
    if (k.words0 >= (1ull << 32) || k.words1 >= (1ull << 32)) return TP_EUNSUPPORTED;
    const bool rf = k.scheme == TP_RFOR;
    if (k.scheme == TP_FOR || k.scheme == TP_DFOR) {
      if (k.block_size != 128 || k.miniblock_count != 4 || k.num_blocks != (n + 127) / 128) return TP_EFORMAT;
    } else if (rf) {
      if (k.block_size != 512 || k.miniblock_count != 16 || k.num_blocks != (n + 511) / 512) return TP_EFORMAT;
      if (!k.starts1 || !k.data1) return TP_EINVAL;
    } else {
      return TP_EINVAL;
    }
    if (n > 0 && (!k.starts0 || !k.data0)) return TP_EINVAL;
    any_rfor |= rf;
    Col& cc = P.col[c];
    cc.scheme = k.scheme == TP_FOR ? S_FOR : k.scheme == TP_DFOR ? S_DFOR : S_RFOR;
    cc.nblocks = (uint32_t)k.num_blocks;
    for (int s = 0; s < (rf ? 2 : 1); ++s) {
      Stream& st = P.st[P.nstreams];
      st.data = s == 0 ? k.data0 : k.data1;
      st.starts = s == 0 ? k.starts0 : k.starts1;
      st.kind = rf ? K_RFOR : (k.scheme == TP_DFOR ? K_DFOR : K_FOR);
      st.nblocks = (uint32_t)k.num_blocks;
      uint32_t mtw = s == 0 ? k.max_tile_words0 : k.max_tile_words1;
      if (mtw == 0 || mtw > worst_tile_words(k.scheme)) mtw = worst_tile_words(k.scheme);
      st.data_off = off;
      off += align4(std::max<uint32_t>(TPS * mtw + 12u, 48u));
      st.starts_off = off;
      off += align4((rf ? TPS + 1u : 4u * TPS + 1u) + 8u);
      if (s == 0) cc.s0 = P.nstreams; else cc.s1 = P.nstreams;
      ++P.nstreams;
    }
  }
  P.ncols = (uint32_t)ncols;
  P.n = (uint32_t)n;
  P.ntiles = (uint32_t)((n + TILE_ROWS - 1) / TILE_ROWS);
  P.stage_words = align4(off);
  P.staging_off = any_rfor ? RFOR_SCRATCH_WORDS : 0u;
  const uint32_t scratch = P.staging_off + extra_scratch;
  P.scratch_words_per_warp = align4(scratch);
  // ring depth: up to 4 stages, keep the CTA under ~100 KB so >= 2 CTAs fit an SM
  uint32_t nstg = 4;
  while (nstg > 2 && (size_t)(nstg * P.stage_words + CONSUMER_WARPS * P.scratch_words_per_warp) * 4 > 100 * 1024)
    --nstg;
  P.nstages = nstg;
  P.scratch_off = nstg * P.stage_words;
  smem_bytes = (size_t)(P.scratch_off + CONSUMER_WARPS * P.scratch_words_per_warp) * 4 + 2 * nstg * 8 + 16;
  return TP_OK;
}

template <class K>
static int grid_for(K kernel, size_t smem) {
  cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, THREADS, smem);
  if (occ < 1) occ = 1;
  if (occ > 8) occ = 8;
  return sm_count() * occ;
}

static tp_status launched() {
  g_launches.fetch_add(1, std::memory_order_relaxed);
  return cudaGetLastError() == cudaSuccess ? TP_OK : TP_ECUDA;
}

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

}  // namespace tp

using namespace tp;

extern "C" {

tp_status tp_decode_sum(const tp_column* dcol, int64_t* d_sum, void* stream) {
  if (!dcol || !d_sum) return TP_EINVAL;
  if (dcol->n == 0) return TP_OK;
  Params P;
  size_t smem = 0;
  tp_status st = build_params(dcol, 1, 0, P, smem);
  if (st != TP_OK) return st;
  const int grid = std::min<int>(grid_for(k_decode_sum, smem), (int)((P.ntiles + 1) / 2));
  k_decode_sum<<<grid, THREADS, smem, (cudaStream_t)stream>>>(P, reinterpret_cast<unsigned long long*>(d_sum));
  return launched();
}

tp_status tp_decode(const tp_column* dcol, int32_t* d_out, void* stream) {
  if (!dcol || !d_out) return TP_EINVAL;
  if (dcol->n == 0) return TP_OK;
  if (reinterpret_cast<uintptr_t>(d_out) & 15u) return TP_EINVAL;
  Params P;
  size_t smem = 0;
  // per warp: RFOR scratch + 2 x 4 KB swizzled staging + 1 KB alignment slop
  tp_status st = build_params(dcol, 1, 2048u + 256u, P, smem);
  if (st != TP_OK) return st;
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
  const int grid = std::min<int>(grid_for(k_decode_global, smem), (int)((P.ntiles + 1) / 2));
  k_decode_global<<<grid, THREADS, smem, (cudaStream_t)stream>>>(P, tmap, d_out);
  return launched();
}

tp_status tp_select_project_sum(const tp_column* dcols, int ncols, const int32_t* lo, const int32_t* hi, int proj_op,
                                int a, int b, int64_t* d_result, void* stream) {
  if (!dcols || !lo || !hi || !d_result || ncols < 1 || ncols > TP_MAX_COLS) return TP_EINVAL;
  if (proj_op < TP_PROJ_COL || proj_op > TP_PROJ_COUNT) return TP_EINVAL;
  if (proj_op != TP_PROJ_COUNT && (a < 0 || a >= ncols)) return TP_EINVAL;
  if ((proj_op == TP_PROJ_MUL || proj_op == TP_PROJ_SUB) && (b < 0 || b >= ncols)) return TP_EINVAL;
  if (dcols[0].n == 0) return TP_OK;
  Params P;
  size_t smem = 0;
  tp_status st = build_params(dcols, ncols, 0, P, smem);
  if (st != TP_OK) return st;
  SelectArgs A;
  memset(&A, 0, sizeof(A));
  for (int c = 0; c < TP_MAX_COLS; ++c) {
    A.lo[c] = c < ncols ? lo[c] : INT_MIN;
    A.hi[c] = c < ncols ? hi[c] : INT_MAX;
  }
  A.proj = proj_op; A.a = a; A.b = b;
  const int grid = std::min<int>(grid_for(k_select_sum, smem), (int)((P.ntiles + 1) / 2));
  k_select_sum<<<grid, THREADS, smem, (cudaStream_t)stream>>>(P, A, reinterpret_cast<unsigned long long*>(d_result));
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

uint64_t tp_launch_count(void) { return g_launches.load(); }

tp_status tp_device_info(int* sms, int* ctas_per_sm) {
  if (sms) *sms = sm_count();
  if (ctas_per_sm) {
    tp_column c;
    memset(&c, 0, sizeof(c));
    c.scheme = TP_FOR; c.block_size = 128; c.miniblock_count = 4; c.n = 1 << 20; c.num_blocks = (1 << 20) / 128;
    c.starts0 = reinterpret_cast<const uint32_t*>(16); c.data0 = c.starts0;
    Params P;
    size_t smem = 0;
    build_params(&c, 1, 0, P, smem);
    *ctas_per_sm = grid_for(k_decode_sum, smem) / sm_count();
  }
  return TP_OK;
}

}  // extern "C"
