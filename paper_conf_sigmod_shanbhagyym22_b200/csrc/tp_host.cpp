// tp_host.cpp -- host half of the C ABI (include/tilepack.h): the one-time
// column encoder, the GPU-* scheme chooser and the
// tile-range sharder.  Multi-threaded over independent blocks.
//
// Byte layout: DESIGN.md "Formats" (readings R1-R18).  Written independently of
// oracle/oracle.c; tests/test_host_encoder.py checks the two byte for byte.
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <thread>
#include <vector>

#include "tilepack.h"

namespace {

constexpr uint32_t kBlock = 128;    // FOR / DFOR block
constexpr uint32_t kTile = 512;     // D = 4 blocks / RFOR block
constexpr uint32_t kGuard = TP_GUARD_WORDS;

inline uint32_t bit_length(uint32_t u) { return u ? 32u - (uint32_t)__builtin_clz(u) : 0u; }

// run fn(lo, hi) over [0, count) split across hardware threads
template <class F>
void parallel_for(uint64_t count, F fn, uint64_t min_grain = 4096) {
  unsigned hw = std::max(1u, std::thread::hardware_concurrency());
  uint64_t nthreads = std::min<uint64_t>(hw, (count + min_grain - 1) / min_grain);
  if (nthreads <= 1) {
    if (count) fn(0, count);
    return;
  }
  std::vector<std::thread> th;
  th.reserve(nthreads);
  for (uint64_t t = 0; t < nthreads; ++t) {
    uint64_t lo = count * t / nthreads, hi = count * (t + 1) / nthreads;
    th.emplace_back([=] { fn(lo, hi); });
  }
  for (auto& x : th) x.join();
}

// Bit writer: appends b-bit fields LSB-first into consecutive words (R1).
struct BitWriter {
  uint32_t* out;
  uint64_t acc = 0;
  uint32_t fill = 0;
  explicit BitWriter(uint32_t* o) : out(o) {}
  inline void put(uint32_t v, uint32_t b) {
    if (b == 0) return;
    acc |= (uint64_t)v << fill;
    fill += b;
    if (fill >= 32) {
      *out++ = (uint32_t)acc;
      acc >>= 32;
      fill -= 32;
    }
  }
  inline uint32_t* flush() {
    if (fill) { *out++ = (uint32_t)acc; acc = 0; fill = 0; }
    return out;
  }
};

// ---- one FOR-packed block of up to 128 entries: ref, 4 widths, sizes
struct ForBlockPlan {
  int32_t ref;
  uint32_t bw;     // packed bitwidth word
  uint32_t words;  // 2 + sum of widths
};

// values v[0..cnt) (cnt <= 128); slots cnt..127 are neutral pads (R8, R13)
inline ForBlockPlan plan_for_block(const int32_t* v, uint32_t cnt) {
  ForBlockPlan p{0, 0, 2};
  if (cnt == 0) return p;
  int32_t mn = v[0];
  for (uint32_t i = 1; i < cnt; ++i) mn = std::min(mn, v[i]);
  p.ref = mn;
  for (uint32_t j = 0; j < 4; ++j) {
    uint32_t mx = 0;
    for (uint32_t i = 32 * j; i < std::min(cnt, 32 * j + 32); ++i) mx = std::max(mx, (uint32_t)v[i] - (uint32_t)mn);
    const uint32_t b = bit_length(mx);
    p.bw |= b << (8 * j);
    p.words += b;
  }
  return p;
}

inline uint32_t* write_for_block(const int32_t* v, uint32_t cnt, const ForBlockPlan& p, uint32_t* out) {
  *out++ = (uint32_t)p.ref;
  *out++ = p.bw;
  for (uint32_t j = 0; j < 4; ++j) {
    const uint32_t b = (p.bw >> (8 * j)) & 255u;
    BitWriter w(out);
    for (uint32_t i = 32 * j; i < 32 * j + 32; ++i) w.put(i < cnt ? (uint32_t)v[i] - (uint32_t)p.ref : 0u, b);
    out = w.flush();
  }
  return out;
}

// ---- GPU-FOR without miniblocks: one bitwidth per 128-value block
inline ForBlockPlan plan_fornm_block(const int32_t* v, uint32_t cnt) {
  ForBlockPlan p{0, 0, 2};
  if (cnt == 0) return p;
  int32_t mn = v[0];
  for (uint32_t i = 1; i < cnt; ++i) mn = std::min(mn, v[i]);
  uint32_t mx = 0;
  for (uint32_t i = 0; i < cnt; ++i) mx = std::max(mx, (uint32_t)v[i] - (uint32_t)mn);
  p.ref = mn;
  p.bw = bit_length(mx);  // byte 0 (R2 with one miniblock)
  p.words = 2 + 4 * p.bw;
  return p;
}
inline uint32_t* write_fornm_block(const int32_t* v, uint32_t cnt, const ForBlockPlan& p, uint32_t* out) {
  *out++ = (uint32_t)p.ref;
  *out++ = p.bw;
  BitWriter w(out);
  for (uint32_t i = 0; i < kBlock; ++i) w.put(i < cnt ? (uint32_t)v[i] - (uint32_t)p.ref : 0u, p.bw);
  return w.flush();
}

// ---- GPU-FOR
struct ForEnc {
  static uint64_t nblocks(uint64_t n) { return (n + kBlock - 1) / kBlock; }
  static uint32_t block_words(const int32_t* x, uint64_t n, uint64_t i) {
    const uint32_t cnt = (uint32_t)std::min<uint64_t>(kBlock, n - i * kBlock);
    return plan_for_block(x + i * kBlock, cnt).words;
  }
};

// ---- GPU-DFOR tile: m values -> first + up to 4 FOR blocks of deltas
inline uint32_t dfor_tile_deltas(const int32_t* x, uint32_t m, int32_t* d) {
  for (uint32_t s = 0; s + 1 < m; ++s) d[s] = (int32_t)((uint32_t)x[s + 1] - (uint32_t)x[s]);
  return m - 1;  // real deltas
}

// ---- GPU-RFOR stream block: [r][ref][4 bw words][16 tight miniblocks]
struct RforPlan {
  int32_t ref;
  uint32_t bw[4];
  uint32_t words;
};
inline RforPlan plan_rfor_stream(const int32_t* s, uint32_t r) {
  RforPlan p{};
  int32_t mn = s[0];
  for (uint32_t i = 1; i < r; ++i) mn = std::min(mn, s[i]);
  p.ref = mn;
  p.words = 6;
  for (uint32_t j = 0; j < 16; ++j) {
    uint32_t mx = 0;
    const uint32_t lo = 32 * j, hi = std::min(r, lo + 32);
    for (uint32_t i = lo; i < hi; ++i) mx = std::max(mx, (uint32_t)s[i] - (uint32_t)mn);
    const uint32_t b = lo < r ? bit_length(mx) : 0u;
    p.bw[j / 4] |= b << (8 * (j % 4));
    const uint32_t cnt = hi > lo ? hi - lo : 0;
    p.words += (uint32_t)(((uint64_t)cnt * b + 31) / 32);
  }
  return p;
}
inline uint32_t* write_rfor_stream(const int32_t* s, uint32_t r, const RforPlan& p, uint32_t* out) {
  *out++ = r;
  *out++ = (uint32_t)p.ref;
  for (int q = 0; q < 4; ++q) *out++ = p.bw[q];
  for (uint32_t j = 0; j < 16; ++j) {
    const uint32_t b = (p.bw[j / 4] >> (8 * (j % 4))) & 255u;
    const uint32_t lo = 32 * j, hi = std::min(r, lo + 32);
    BitWriter w(out);
    for (uint32_t i = lo; i < hi; ++i) w.put((uint32_t)s[i] - (uint32_t)p.ref, b);
    out = w.flush();
  }
  return out;
}
inline uint32_t rle_block(const int32_t* x, uint32_t m, int32_t* V, int32_t* L) {
  uint32_t r = 0;
  for (uint32_t i = 0; i < m;) {
    uint32_t k = i + 1;
    while (k < m && x[k] == x[i]) ++k;
    V[r] = x[i];
    L[r] = (int32_t)(k - i);
    ++r;
    i = k;
  }
  return r;
}

// exclusive prefix sum of per-unit word counts (sequential; units are few per value)
uint64_t exclusive_scan(std::vector<uint32_t>& w, std::vector<uint64_t>& off) {
  off.resize(w.size() + 1);
  uint64_t acc = 0;
  for (size_t i = 0; i < w.size(); ++i) { off[i] = acc; acc += w[i]; }
  off[w.size()] = acc;
  return acc;
}

struct Sizes {
  uint64_t nb = 0, w0 = 0, w1 = 0;
  std::vector<uint32_t> u0, u1;  // per-unit words (blocks for FOR, tiles for DFOR, row blocks for RFOR)
};

Sizes compute_sizes(int scheme, const int32_t* x, uint64_t n) {
  Sizes s;
  if (scheme == TP_NONE) {  // plain values, 512-row tiles, padded to whole 32-row miniblocks
    s.nb = (n + kTile - 1) / kTile;
    s.w0 = (n + 31) / 32 * 32;
  } else if (scheme == TP_FOR || scheme == TP_FORNM) {
    s.nb = (n + kBlock - 1) / kBlock;
    s.u0.resize(s.nb);
    const bool nm = scheme == TP_FORNM;
    parallel_for(s.nb, [&](uint64_t lo, uint64_t hi) {
      for (uint64_t i = lo; i < hi; ++i)
        s.u0[i] = nm ? plan_fornm_block(x + i * kBlock, (uint32_t)std::min<uint64_t>(kBlock, n - i * kBlock)).words
                     : ForEnc::block_words(x, n, i);
    });
    for (uint32_t w : s.u0) s.w0 += w;
  } else if (scheme == TP_DFOR) {
    s.nb = (n + kBlock - 1) / kBlock;
    const uint64_t nt = (n + kTile - 1) / kTile;
    s.u0.resize(nt);
    parallel_for(nt, [&](uint64_t lo, uint64_t hi) {
      int32_t d[kTile];
      for (uint64_t t = lo; t < hi; ++t) {
        const uint32_t m = (uint32_t)std::min<uint64_t>(kTile, n - t * kTile);
        const uint32_t real = dfor_tile_deltas(x + t * kTile, m, d);
        uint32_t w = 1;  // first value
        for (uint32_t k = 0; k < (m + kBlock - 1) / kBlock; ++k) {
          const uint32_t lo2 = k * kBlock;
          const uint32_t cnt = real > lo2 ? std::min(kBlock, real - lo2) : 0u;
          w += plan_for_block(d + lo2, cnt).words;
        }
        s.u0[t] = w;
      }
    }, 512);
    for (uint32_t w : s.u0) s.w0 += w;
  } else {
    s.nb = (n + kTile - 1) / kTile;
    s.u0.resize(s.nb);
    s.u1.resize(s.nb);
    parallel_for(s.nb, [&](uint64_t lo, uint64_t hi) {
      int32_t V[kTile], L[kTile];
      for (uint64_t k = lo; k < hi; ++k) {
        const uint32_t m = (uint32_t)std::min<uint64_t>(kTile, n - k * kTile);
        const uint32_t r = rle_block(x + k * kTile, m, V, L);
        s.u0[k] = plan_rfor_stream(V, r).words;
        s.u1[k] = plan_rfor_stream(L, r).words;
      }
    }, 512);
    for (uint32_t w : s.u0) s.w0 += w;
    for (uint32_t w : s.u1) s.w1 += w;
  }
  return s;
}

}  // namespace

extern "C" {

tp_status tp_encode_size(int scheme, const int32_t* x, uint64_t n, uint64_t* num_blocks, uint64_t* words0,
                         uint64_t* words1) {
  if (scheme < TP_FOR || scheme > TP_FORNM || (n && !x)) return TP_EINVAL;
  if (n >= (1ull << 32)) return TP_EUNSUPPORTED;
  Sizes s = compute_sizes(scheme, x, n);
  if (s.w0 >= (1ull << 32) || s.w1 >= (1ull << 32)) return TP_EUNSUPPORTED;
  if (num_blocks) *num_blocks = s.nb;
  if (words0) *words0 = s.w0;
  if (words1) *words1 = s.w1;
  return TP_OK;
}

tp_status tp_encode(int scheme, const int32_t* x, uint64_t n, uint32_t* starts0, uint32_t* data0, uint32_t* starts1,
                    uint32_t* data1, tp_column* out) {
  if (scheme < TP_FOR || scheme > TP_FORNM || (n && !x) || !starts0 || !data0 || !out) return TP_EINVAL;
  if (scheme == TP_RFOR && (!starts1 || !data1)) return TP_EINVAL;
  if (n >= (1ull << 32)) return TP_EUNSUPPORTED;
  Sizes s = compute_sizes(scheme, x, n);
  if (s.w0 >= (1ull << 32) || s.w1 >= (1ull << 32)) return TP_EUNSUPPORTED;
  std::vector<uint64_t> off0, off1;
  exclusive_scan(s.u0, off0);
  memset(out, 0, sizeof(*out));
  out->scheme = (uint32_t)scheme;
  out->n = n;
  out->num_blocks = s.nb;
  uint32_t mtw0 = 0, mtw1 = 0;
  if (scheme == TP_NONE) {
    parallel_for(s.nb, [&](uint64_t lo, uint64_t hi) {
      for (uint64_t k = lo; k < hi; ++k) {
        const uint64_t r0 = k * kTile, r1 = std::min<uint64_t>(n, r0 + kTile);
        starts0[k] = (uint32_t)r0;
        memcpy(data0 + r0, x + r0, (r1 - r0) * 4);
      }
    });
    memset(data0 + n, 0, (s.w0 - n) * 4);
    starts0[s.nb] = (uint32_t)s.w0;
    mtw0 = kTile;
    out->block_size = kTile; out->miniblock_count = 1; out->tile_blocks = 1;
  } else if (scheme == TP_FOR || scheme == TP_FORNM) {
    const bool nm = scheme == TP_FORNM;
    parallel_for(s.nb, [&](uint64_t lo, uint64_t hi) {
      for (uint64_t i = lo; i < hi; ++i) {
        const uint32_t cnt = (uint32_t)std::min<uint64_t>(kBlock, n - i * kBlock);
        const int32_t* v = x + i * kBlock;
        starts0[i] = (uint32_t)off0[i];
        if (nm) write_fornm_block(v, cnt, plan_fornm_block(v, cnt), data0 + off0[i]);
        else write_for_block(v, cnt, plan_for_block(v, cnt), data0 + off0[i]);
      }
    });
    starts0[s.nb] = (uint32_t)s.w0;
    for (uint64_t t = 0; t * 4 < s.nb; ++t)
      mtw0 = std::max<uint32_t>(mtw0, starts0[std::min<uint64_t>(4 * t + 4, s.nb)] - starts0[4 * t]);
    out->block_size = kBlock; out->miniblock_count = nm ? 1 : 4; out->tile_blocks = 4;
  } else if (scheme == TP_DFOR) {
    const uint64_t nt = (n + kTile - 1) / kTile;
    parallel_for(nt, [&](uint64_t lo, uint64_t hi) {
      int32_t d[kTile];
      for (uint64_t t = lo; t < hi; ++t) {
        const uint32_t m = (uint32_t)std::min<uint64_t>(kTile, n - t * kTile);
        const uint32_t real = dfor_tile_deltas(x + t * kTile, m, d);
        uint32_t* o = data0 + off0[t];
        *o++ = (uint32_t)x[t * kTile];  // first value
        for (uint32_t k = 0; k < (m + kBlock - 1) / kBlock; ++k) {
          const uint32_t lo2 = k * kBlock;
          const uint32_t cnt = real > lo2 ? std::min(kBlock, real - lo2) : 0u;
          starts0[4 * t + k] = (uint32_t)(o - data0);
          o = write_for_block(d + lo2, cnt, plan_for_block(d + lo2, cnt), o);
        }
      }
    }, 512);
    starts0[s.nb] = (uint32_t)s.w0;
    for (uint32_t w : s.u0) mtw0 = std::max(mtw0, w);
    out->block_size = kBlock; out->miniblock_count = 4; out->tile_blocks = 4;
  } else {
    exclusive_scan(s.u1, off1);
    parallel_for(s.nb, [&](uint64_t lo, uint64_t hi) {
      int32_t V[kTile], L[kTile];
      for (uint64_t k = lo; k < hi; ++k) {
        const uint32_t m = (uint32_t)std::min<uint64_t>(kTile, n - k * kTile);
        const uint32_t r = rle_block(x + k * kTile, m, V, L);
        starts0[k] = (uint32_t)off0[k];
        starts1[k] = (uint32_t)off1[k];
        write_rfor_stream(V, r, plan_rfor_stream(V, r), data0 + off0[k]);
        write_rfor_stream(L, r, plan_rfor_stream(L, r), data1 + off1[k]);
      }
    }, 512);
    starts0[s.nb] = (uint32_t)s.w0;
    starts1[s.nb] = (uint32_t)s.w1;
    for (uint32_t w : s.u0) mtw0 = std::max(mtw0, w);
    for (uint32_t w : s.u1) mtw1 = std::max(mtw1, w);
    out->block_size = kTile; out->miniblock_count = 16; out->tile_blocks = 1;
    memset(starts1 + s.nb + 1, 0, kGuard * 4);
    memset(data1 + s.w1, 0, kGuard * 4);
    out->starts1 = starts1; out->data1 = data1; out->words1 = s.w1;
  }
  memset(starts0 + s.nb + 1, 0, kGuard * 4);
  memset(data0 + s.w0, 0, kGuard * 4);
  out->starts0 = starts0; out->data0 = data0; out->words0 = s.w0;
  out->max_tile_words0 = mtw0;
  out->max_tile_words1 = mtw1;
  return TP_OK;
}

tp_status tp_choose_scheme(const int32_t* x, uint64_t n, int* scheme, uint64_t* bytes) {
  if ((n && !x) || !scheme) return TP_EINVAL;
  if (n >= (1ull << 32)) return TP_EUNSUPPORTED;
  int best = 0;
  uint64_t best_bytes = 0;
  for (int s = TP_FOR; s <= TP_RFOR; ++s) {  // ties -> FOR < DFOR < RFOR (R20)
    Sizes z = compute_sizes(s, x, n);
    const uint64_t b = 4 * (3 + (z.nb + 1) * (s == TP_RFOR ? 2 : 1) + z.w0 + z.w1);
    if (best == 0 || b < best_bytes) { best = s; best_bytes = b; }
  }
  *scheme = best;
  if (bytes) *bytes = best_bytes;
  return TP_OK;
}

uint64_t tp_compressed_bytes(const tp_column* c) {
  if (!c) return 0;
  const uint64_t streams = c->scheme == TP_RFOR ? 2 : 1;
  if (c->scheme == TP_NONE) return 4 * c->n;  // the plain column (header / starts: pipeline artefacts)
  return 4 * (3 + streams * (c->num_blocks + 1) + c->words0 + c->words1);
}

tp_status tp_shard(const tp_column* c, uint64_t row_lo, uint64_t row_hi, uint32_t* r0, uint32_t* r1,
                   tp_column* view) {
  if (!c || !view || !r0 || row_lo > row_hi || row_hi > c->n || (row_lo % kTile)) return TP_EINVAL;
  if (row_hi != c->n && (row_hi % kTile)) return TP_EINVAL;
  const bool rf = c->scheme == TP_RFOR;
  if (rf && !r1) return TP_EINVAL;
  const uint64_t per = (rf || c->scheme == TP_NONE) ? kTile : kBlock;
  const uint64_t b0 = row_lo / per, b1 = (row_hi + per - 1) / per;
  *view = *c;
  if (row_lo == row_hi) {  // an empty range (also of an empty column): no blocks, no words
    view->n = 0;
    view->num_blocks = 0;
    r0[0] = 0;
    memset(r0 + 1, 0, kGuard * 4);
    view->starts0 = r0;
    view->words0 = 0;
    view->max_tile_words0 = 0;
    if (rf) {
      r1[0] = 0;
      memset(r1 + 1, 0, kGuard * 4);
      view->starts1 = r1;
      view->words1 = 0;
      view->max_tile_words1 = 0;
    }
    return TP_OK;
  }
  view->n = row_hi - row_lo;
  view->num_blocks = b1 - b0;
  const bool dfor = c->scheme == TP_DFOR;
  // stream 0 (and 1): rebase block_starts to the view's first word
  const uint32_t base0 = c->starts0[b0] - (dfor ? 1u : 0u);
  for (uint64_t b = b0; b <= b1; ++b) r0[b - b0] = c->starts0[b] - base0;
  memset(r0 + (b1 - b0) + 1, 0, kGuard * 4);
  view->starts0 = r0;
  view->data0 = c->data0 + base0;
  const uint64_t end0 = (dfor && b1 < c->num_blocks) ? (uint64_t)c->starts0[b1] - 1 : c->starts0[b1];
  view->words0 = end0 - base0;
  // a DFOR view ending before the next tile stops at that tile's first value: last entry = total words
  if (dfor && b1 < c->num_blocks) r0[b1 - b0] = (uint32_t)view->words0;
  if (rf) {
    const uint32_t base1 = c->starts1[b0];
    for (uint64_t b = b0; b <= b1; ++b) r1[b - b0] = c->starts1[b] - base1;
    memset(r1 + (b1 - b0) + 1, 0, kGuard * 4);
    view->starts1 = r1;
    view->data1 = c->data1 + base1;
    view->words1 = c->starts1[b1] - base1;
  }
  return TP_OK;
}

// Format check of a HOST column (include/tilepack.h tp_validate): header fields, block_starts
// monotone and inside the data, every bitwidth byte <= 32 (R3, R5) and unused bytes zero,
// every block exactly as long as its header says (Alg. 1 lines 13-14: 2 + sum of b words;
// RFOR layout B, R17: 6 + tight miniblocks), RFOR run counts <= the block's rows; the exact
// max_tile_words of each stream (what the decoders size their shared-memory ring with).
tp_status tp_validate(const tp_column* c, uint32_t* mtw0_out, uint32_t* mtw1_out) {
  if (!c) return TP_EINVAL;
  const uint64_t n = c->n;
  if (n >= (1ull << 32) || c->words0 >= (1ull << 32) || c->words1 >= (1ull << 32)) return TP_EUNSUPPORTED;
  const uint32_t sch = c->scheme;
  const bool rf = sch == TP_RFOR;
  uint64_t per;
  uint32_t mbc;
  if (sch == TP_FOR || sch == TP_DFOR) { per = kBlock; mbc = 4; }
  else if (sch == TP_FORNM) { per = kBlock; mbc = 1; }
  else if (rf) { per = kTile; mbc = 16; }
  else if (sch == TP_NONE) { per = kTile; mbc = 1; }
  else return TP_EINVAL;
  if (c->block_size != per || c->miniblock_count != mbc || c->num_blocks != (n + per - 1) / per) return TP_EFORMAT;
  if (!c->starts0 || (c->words0 && !c->data0) || (rf && (!c->starts1 || (c->words1 && !c->data1))))
    return TP_EINVAL;
  const uint64_t nb = c->num_blocks;
  const uint32_t* s0 = c->starts0;
  uint32_t mtw0 = 0, mtw1 = 0;
  for (uint64_t b = 0; b < nb; ++b)
    if (s0[b] > s0[b + 1]) return TP_EFORMAT;
  if (s0[nb] != c->words0) return TP_EFORMAT;
  if (sch == TP_NONE) {
    for (uint64_t b = 0; b < nb; ++b)
      if (s0[b] != b * kTile) return TP_EFORMAT;
    if (c->words0 < n) return TP_EFORMAT;
    mtw0 = kTile;
  } else if (!rf) {
    const bool dfor = sch == TP_DFOR;
    for (uint64_t b = 0; b < nb; ++b) {
      // DFOR: the tile's first value precedes its first block (Fig. 6)
      const uint64_t start = s0[b];
      if (dfor && (b % 4) == 0 && start < 1) return TP_EFORMAT;
      const uint64_t next = (dfor && (b + 1) % 4 == 0 && b + 1 < nb) ? (uint64_t)s0[b + 1] - 1 : s0[b + 1];
      if (next < start + 2 || next > c->words0) return TP_EFORMAT;
      const uint32_t bw = c->data0[start + 1];
      uint32_t words = 2;
      for (uint32_t j = 0; j < 4; ++j) {
        const uint32_t bj = (bw >> (8 * j)) & 255u;
        if (j >= mbc ? bj != 0 : bj > 32) return TP_EFORMAT;
        words += mbc == 1 ? 4 * bj : bj;
      }
      if (next - start != words) return TP_EFORMAT;
    }
    for (uint64_t t = 0; 4 * t < nb; ++t) {
      const uint64_t lo = dfor ? (uint64_t)s0[4 * t] - 1 : s0[4 * t];
      const uint64_t hi = std::min<uint64_t>(4 * t + 4, nb) == nb ? c->words0
                          : (dfor ? (uint64_t)s0[4 * t + 4] - 1 : s0[4 * t + 4]);
      mtw0 = std::max<uint32_t>(mtw0, (uint32_t)(hi - lo));
    }
  } else {
    const uint32_t* s1 = c->starts1;
    for (uint64_t b = 0; b < nb; ++b)
      if (s1[b] > s1[b + 1]) return TP_EFORMAT;
    if (s1[nb] != c->words1) return TP_EFORMAT;
    for (int q = 0; q < 2; ++q) {
      const uint32_t* st = q ? s1 : s0;
      const uint32_t* d = q ? c->data1 : c->data0;
      uint32_t& mtw = q ? mtw1 : mtw0;
      for (uint64_t b = 0; b < nb; ++b) {
        const uint64_t start = st[b], span = (uint64_t)st[b + 1] - start;
        if (span < 6) return TP_EFORMAT;
        const uint32_t rows = (uint32_t)std::min<uint64_t>(kTile, n - b * kTile);
        const uint32_t r = d[start];
        if (r > rows || (rows > 0 && r == 0)) return TP_EFORMAT;
        uint64_t words = 6;
        for (uint32_t j = 0; j < 16; ++j) {
          const uint32_t bj = (d[start + 2 + j / 4] >> (8 * (j % 4))) & 255u;
          const uint32_t cnt = r > 32 * j ? std::min(32u, r - 32 * j) : 0u;
          if (bj > 32 || (cnt == 0 && bj != 0)) return TP_EFORMAT;
          words += (cnt * bj + 31) / 32;
        }
        if (span != words) return TP_EFORMAT;
        if (q == 0 && d[start] != c->data1[s1[b]]) return TP_EFORMAT;  // both streams count the same runs
        mtw = std::max<uint32_t>(mtw, (uint32_t)span);
      }
    }
  }
  if (mtw0_out) *mtw0_out = mtw0;
  if (mtw1_out) *mtw1_out = mtw1;
  return TP_OK;
}

const char* tp_status_string(tp_status s) {
  switch (s) {
    case TP_OK: return "ok";
    case TP_EINVAL: return "invalid argument";
    case TP_ESIZE: return "buffer too small";
    case TP_EFORMAT: return "malformed column";
    case TP_ECUDA: return "CUDA error";
    case TP_EUNSUPPORTED: return "unsupported size (n or word offsets >= 2^32)";
  }
  return "unknown status";
}

}  // extern "C"
