/*
 * tilepack.h -- C ABI of the B200-native (sm_100a) implementation of
 *   A. Shanbhag, B. Yogatama, X. Yu, S. Madden,
 *   "Tile-based Lightweight Integer Compression in GPU", SIGMOD '22.
 * Citations "P:<lines>" refer to /root/reference/PAPER.md; "R<n>" to the
 * readings listed in DESIGN.md (section "Readings of the paper").
 *
 * The boundary follows the paper's problem statement:
 *   - encode a column into blocks / miniblocks / tiles
 *   - decode a column
 *   - decode fused into a select / project / aggregate
 *   - shard a column by 512-row tile ranges            (multi-GPU)
 *
 * Conventions (all functions):
 *   - Plain pointers and sizes only.  "host" pointers are ordinary CPU memory,
 *     "device" pointers are CUDA global memory of the current device.
 *   - Ownership: the CALLER owns every buffer.  The library never frees caller
 *     memory and never allocates on the decode path.
 *   - Errors: a tp_status is returned; nothing is thrown across the ABI.  Device
 *     calls check cudaGetLastError() after each launch and return TP_ECUDA.
 *   - Device calls are asynchronous on `stream` (a cudaStream_t passed as
 *     void*; NULL = legacy default stream).  Results land in device memory.
 *   - Data arrays (data0/data1) and block_starts arrays (starts0/starts1)
 *     must be allocated with TP_GUARD_WORDS extra zero words after their last
 *     used word (R9: Alg. 1 line 15 reads data[s+1]; the tile stager reads
 *     16-byte aligned supersets).  Device arrays must be 16-byte aligned.
 *   - Counts: n < 2^32 (the header's total count is a 32-bit word)
 *     and every word offset < 2^32 (block_starts are u32, R6); larger inputs
 *     return TP_EUNSUPPORTED.  Shard larger columns with tp_shard.
 *   - All values are int32; decode arithmetic is mod 2^32 (R4); aggregates
 *     are int64 mod 2^64 (R24).
 */
#ifndef TILEPACK_H
#define TILEPACK_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define TP_GUARD_WORDS 4u

typedef enum {
  TP_OK = 0,
  TP_EINVAL = 1,        /* bad argument (NULL pointer, unknown scheme, bad op)  */
  TP_ESIZE = 2,         /* a caller-provided buffer is too small                */
  TP_EFORMAT = 3,       /* header / bitwidth inconsistent with the scheme       */
  TP_ECUDA = 4,         /* a CUDA launch or API call failed                     */
  TP_EUNSUPPORTED = 5   /* n >= 2^32 or word offsets >= 2^32                    */
} tp_status;

typedef enum {
  TP_FOR = 1,   /* GPU-FOR   header [128, 4, n]                          */
  TP_DFOR = 2,  /* GPU-DFOR header [128, 4, n], tiles of D = 4 blocks   */
  TP_RFOR = 3,  /* GPU-RFOR header [512, 16, n], value + run streams     */
  TP_NONE = 4,  /* "None" (Fig. 11): the plain int32 column, header [512, 1, n];
                 * block_starts[k] = 512 k (one 512-row tile per block), data = the
                 * values padded with zeros to a multiple of 32 words (words0 = that
                 * padded count).  The uncompressed baseline the paper compares GPU-*
                 * against, run through the same tile pipeline.  Never chosen by GPU-*. */
  TP_FORNM = 5  /* GPU-FOR WITHOUT miniblocks (the paper's ablation): header
                 * [128, 1, n]; block = [ref][bitwidth word: byte 0 = b of the whole 128-value
                 * block][128 entries x b bits, LSB-first] = 2 + 4 b words.  Host encoder and
                 * decode / decode_sum only (measurement of the miniblock trade-off); never
                 * chosen by GPU-*, not accepted by the GPU encoder or the query operators. */
} tp_scheme;

/*
 * A NON-OWNING view of one encoded column.  The pointers are either all host
 * or all device (tp_encode fills host pointers; the caller copies the arrays
 * to the device and repoints them).
 *   header (Fig. 3, R7) = {block_size, miniblock_count, n}
 *   FOR/DFOR: starts0 = block_starts (num_blocks+1 u32 word offsets into
 *             data0, R6), data0 = blocks; starts1/data1 unused.
 *             DFOR: the first value of tile t is data0[starts0[4t]-1] (Fig. 6).
 *   RFOR:     starts0/data0 = value stream, starts1/data1 = run-length stream,
 *             one stream block per 512-row block (R17).
 *   max_tile_words0/1: largest word span of one 512-row tile in stream 0/1
 *             (filled by tp_encode / tp_gpu_encode / tp_shard / tp_validate;
 *             0 = unknown, the decoder then assumes the format's worst case).
 *             Sizes the shared-memory ring; a value below the column's real
 *             span is detected on the device (TP_DEVERR_TILE_WORDS).
 */
typedef struct {
  uint32_t scheme;            /* tp_scheme                                      */
  uint32_t block_size;        /* 128 (FOR, DFOR) or 512 (RFOR)                  */
  uint32_t miniblock_count;   /* 4 (FOR, DFOR) or 16 (RFOR)                     */
  uint32_t tile_blocks;       /* blocks per 512-row tile: 4 (FOR, DFOR), 1 (RFOR) */
  uint64_t n;                 /* total count                                    */
  uint64_t num_blocks;        /* ceil(n/128) (FOR, DFOR) or ceil(n/512) (RFOR)  */
  const uint32_t* starts0;
  const uint32_t* data0;
  uint64_t words0;            /* used words of data0 (excluding guard words)   */
  const uint32_t* starts1;
  const uint32_t* data1;
  uint64_t words1;
  uint32_t max_tile_words0;
  uint32_t max_tile_words1;
} tp_column;

/* ------------------------------------------------------------------ host */

/* Sizes tp_encode will produce for `scheme` on host column x[0..n).
 * Outputs (host): *num_blocks, *words0, *words1 (0 unless RFOR).
 * Allocate starts0/starts1 with num_blocks+1+TP_GUARD_WORDS words and
 * data0/data1 with words+TP_GUARD_WORDS words.  Multi-threaded. */
tp_status tp_encode_size(int scheme, const int32_t* x, uint64_t n,
                         uint64_t* num_blocks, uint64_t* words0, uint64_t* words1);

/* Encode host column x[0..n) (compression is a one-time host
 * step).  Writes starts/data (host, caller-allocated as above, guard words
 * zeroed by the library) and fills *out with host pointers.  starts1/data1
 * may be NULL unless scheme == TP_RFOR.  Byte layout: DESIGN.md "Formats". */
tp_status tp_encode(int scheme, const int32_t* x, uint64_t n,
                    uint32_t* starts0, uint32_t* data0,
                    uint32_t* starts1, uint32_t* data1, tp_column* out);

/* GPU-* (P:1206-1217): the scheme with the smallest footprint; ties resolve
 * FOR < DFOR < RFOR (R20).  Outputs (host): *scheme, *bytes. */
tp_status tp_choose_scheme(const int32_t* x, uint64_t n, int* scheme, uint64_t* bytes);

/* Compressed footprint in bytes: 3-word header + block_starts + data
 * (P:1459-1471).  0 for a NULL column. */
uint64_t tp_compressed_bytes(const tp_column* col);

/* A view of rows [row_lo, row_hi) of a HOST column; row_lo must be a multiple
 * of 512 (one tile), row_hi a multiple of 512 or n.
 * Writes rebased block_starts into rebased0 (and rebased1 for RFOR), each
 * with (blocks in range)+1+TP_GUARD_WORDS words; the view's data pointers
 * alias the parent's data (DFOR views start at the tile's first value). */
tp_status tp_shard(const tp_column* host_col, uint64_t row_lo, uint64_t row_hi,
                   uint32_t* rebased0, uint32_t* rebased1, tp_column* view);

/* Format check of a HOST column (R1-R19): header fields
 * (block_size / miniblock_count / num_blocks of the scheme), block_starts
 * non-decreasing and ending at words0 (words1), every bitwidth byte <= 32
 * (R3, R5) with the unused bytes zero, every block exactly 2 + sum of its
 * miniblock widths words (Alg. 1 lines 13-14; FORNM 2 + 4 b;
 * RFOR 6 + its tight miniblocks, R17), RFOR run counts in [1, rows of the
 * block] and equal in both streams.  Returns TP_EFORMAT at the first
 * violation, TP_OK otherwise, and writes the column's exact largest tile
 * span per stream (the value max_tile_words0/1 must not be below) to
 * *max_tile_words0 / *max_tile_words1 (either may be NULL).  O(num_blocks)
 * reads, single-threaded; the device calls do NOT run it (they trust the
 * bytes -- see tp_device_errors for what they do check). */
tp_status tp_validate(const tp_column* host_col, uint32_t* max_tile_words0, uint32_t* max_tile_words1);

/* ---------------------------------------------------------------- device */

/* Format violations the DEVICE calls detect while they run (bit flags; the kernel
 * stays inside its buffers -- a tile range longer than the ring region sized from
 * max_tile_words is copied only up to the region, a run count above 512 is used as
 * 512 -- and the affected results are undefined):
 *   TP_DEVERR_TILE_WORDS a tile range spans more words than max_tile_words0/1 says
 *   TP_DEVERR_RUNS       an RFOR stream block counts more than 512 runs (R17)
 * A miniblock bitwidth byte > 32 (R3, R5) is used as 32 on the device (memory-safe, the
 * values undefined) and NOT flagged there -- checking it per miniblock cost 2-4 % of the
 * decode kernels; tp_validate reports it (TP_EFORMAT) for a host column.
 * tp_device_errors synchronizes `stream`, writes the flags accumulated by this
 * library's kernels on the current device since the last call to *flags (host), and
 * clears them.  Returns TP_ECUDA if the synchronisation or the read fails. */
enum { TP_DEVERR_TILE_WORDS = 2, TP_DEVERR_RUNS = 4 };
tp_status tp_device_errors(uint32_t* flags, void* stream);

/* Decode the whole DEVICE column into d_out[0..n) (int32, device).
 * One pass over HBM: each 512-row tile is staged once into shared memory by
 * TMA bulk copies and unpacked there (tile-based decompression);
 * decoded rows are written back by TMA tensor stores (decode-to-global mode
 * of Fig. 7a). */
tp_status tp_decode(const tp_column* dcol, int32_t* d_out, void* stream);

/* Decode fused into an int64 sum (the paper's decode-only microbenchmark,
 * P:720-724, with a consumer that keeps every value live).  ADDS the sum of
 * all n values into *d_sum (device int64; the caller zeroes it). */
tp_status tp_decode_sum(const tp_column* dcol, int64_t* d_sum, void* stream);

/* Fused select / project / aggregate over ncols DEVICE columns of equal n
 * (the decoders replace the tile load inside the query kernel):
 *   *d_result += sum over rows i with lo[c] <= col_c[i] <= hi[c] for all c
 *                of proj(i)
 * proj_op: TP_PROJ_COL -> col_a[i];  TP_PROJ_MUL -> col_a[i]*col_b[i];
 *          TP_PROJ_SUB -> col_a[i]-col_b[i];  TP_PROJ_COUNT -> 1.
 * lo/hi: host arrays of ncols int32 (inclusive); [INT32_MIN, INT32_MAX]
 * means "no predicate".  ncols <= TP_MAX_COLS. */
#define TP_MAX_COLS 6
enum { TP_PROJ_COL = 0, TP_PROJ_MUL = 1, TP_PROJ_SUB = 2, TP_PROJ_COUNT = 3 };
tp_status tp_select_project_sum(const tp_column* dcols, int ncols,
                                const int32_t* lo, const int32_t* hi,
                                int proj_op, int a, int b,
                                int64_t* d_result, void* stream);

/* ---------------------------------------------------- star-join queries
 * The SSB workload of P:1874-1888 (13 queries, dictionary-encoded):
 * decoded fact-table foreign keys probe dimension lookup tables (Crystal-style
 * perfect hashing: table[key - key_min]), payloads form a dense group index,
 * and the measures are aggregated per group -- all inside one tile kernel
 * (SURVEY 8(a) rows a7-a8).
 *
 * tp_lookup_build: DEVICE table[0..table_len) := -1, then for every dimension
 * row i whose attributes pass all preds:
 *     table[keys[i] - key_min] = payload ? payload[i] : 0
 * pred p passes when lo1 <= attr[i] <= hi1 OR lo2 <= attr[i] <= hi2
 * (set lo2 > hi2 for a single range).  keys/attr/payload are DEVICE int32
 * arrays of nrows; keys must lie in [key_min, key_min + table_len); payloads
 * must be >= 0.  npreds <= 4.  Two kernels, asynchronous on `stream`. */
typedef struct {
  const int32_t* attr;
  int32_t lo1, hi1, lo2, hi2;
} tp_dim_pred;
tp_status tp_lookup_build(const int32_t* d_keys, uint64_t nrows, int32_t key_min, uint32_t table_len,
                          const tp_dim_pred* preds, int npreds, const int32_t* d_payload,
                          int32_t* d_table, void* stream);

/* tp_star_query: one fused pass over ncols (<= TP_MAX_COLS) DEVICE columns
 * of equal n.  roles[c] says what column c does, applied in the order given:
 *   TP_ROLE_RANGE   : row survives iff lo <= v <= hi
 *   TP_ROLE_PROBE   : p = table[v - key_min] (v outside the table -> -1);
 *                     row survives iff p >= 0; group += p * stride
 *   TP_ROLE_MEASURE : the row's measure (lo/hi also filter it: use
 *                     [INT32_MIN, INT32_MAX] for none); agg (below) combines
 *                     the measures: TP_AGG_SUM: sum(m0); TP_AGG_MUL:
 *                     sum(m0 * m1); TP_AGG_SUB: sum(m0 - m1)  (int64, R24)
 * The LAST column is the aggregating measure (m1 for MUL / SUB, m0 for SUM);
 * with MUL / SUB exactly one earlier column is a MEASURE (m0), which may sit
 * anywhere before it (its value is staged per row; filters after it still
 * apply).  Columns are evaluated in the order given: put the most selective
 * first -- once few rows of a warp survive, later columns are read row by row
 * (random access into the staged tile) instead of decoded whole.
 * Errors: TP_EINVAL for a bad role / missing table / measure layout.
 * For every surviving row:
 *   d_sums[group] += aggregate, d_counts[group] += 1
 * (DEVICE int64 / uint64 arrays of ngroups, caller-zeroed).  Rows whose group
 * is >= ngroups are a caller error (not checked per row). */
enum { TP_ROLE_RANGE = 0, TP_ROLE_PROBE = 1, TP_ROLE_MEASURE = 2 };
enum { TP_AGG_SUM = 0, TP_AGG_MUL = 1, TP_AGG_SUB = 2 };
typedef struct {
  int32_t role;
  int32_t lo, hi;            /* RANGE */
  const int32_t* table;      /* PROBE (DEVICE) */
  int32_t key_min;
  uint32_t table_len;
  uint32_t stride;
} tp_star_col;
tp_status tp_star_query(const tp_column* dcols, const tp_star_col* roles, int ncols, int agg,
                        int64_t* d_sums, uint64_t* d_counts, uint32_t ngroups, void* stream);

/* Random access under a predicate bitvector:
 *   *d_sum += sum of x[i] over the rows i whose bit is set,
 * bit i of the bitvector = bit (i mod 32) of DEVICE word d_bitmap[i / 32] (LSB-first; at least
 * ceil(n / 32) words; bits past n are ignored).  A 512-row tile whose bits are all zero is
 * skipped without reading any of its compressed words; GPU-FOR and None also skip every
 * 32-row miniblock whose bitvector word is zero (a FOR miniblock is read through its block
 * header, Alg. 1), GPU-DFOR / GPU-RFOR decode each selected tile whole.  Any scheme, one
 * kernel, asynchronous on `stream`. */
tp_status tp_bitmap_sum(const tp_column* dcol, const uint32_t* d_bitmap, int64_t* d_sum, void* stream);

/* The uncompressed baseline "None": *d_sum += sum of the n int32
 * values of DEVICE array d_x (16-byte aligned), 128-bit streaming loads.
 * Used as the measured HBM read roof of the same consumer. */
tp_status tp_plain_sum(const int32_t* d_x, uint64_t n, int64_t* d_sum, void* stream);

/* ------------------------------------------------ cascading baseline (ablation)
 * The paper's CASCADING decompression model, the baseline of
 * Fig. 7a: the same encoded DEVICE column decoded one layer per kernel, every layer
 * reading and writing global memory -- FOR+BitPack 2 passes, Delta+FOR+BitPack 3,
 * RLE+FOR+BitPack 8.  d_out receives the n decoded values (as tp_decode); d_work is a
 * DEVICE scratch of tp_cascaded_workspace_words(col) u32 words.  For measurement only
 * (SURVEY.md NEXT-1). */
uint64_t tp_cascaded_workspace_words(const tp_column* col);
tp_status tp_decode_cascaded(const tp_column* dcol, int32_t* d_out, uint32_t* d_work, void* stream);

/* ------------------------------------------------------ GPU encoder (tile-parallel)
 * The paper compresses once on the host; every 512-row tile is encoded
 * independently, so the encoder also runs on the GPU
 * in one pass over a DEVICE column: warps plan and pack tiles, a decoupled look-back over
 * chunks (16384 rows for FOR / DFOR, 8192 for RFOR) gives each tile its word offset
 * (SURVEY.md NEXT-3).  The bytes are
 * identical to tp_encode's.  d_x must be 16-byte aligned.
 *
 * d_work: DEVICE scratch of tp_gpu_encode_workspace_bytes(n) bytes (8-byte aligned), owned
 * by the caller; the calls zero it themselves (stream-ordered). */
uint64_t tp_gpu_encode_workspace_bytes(uint64_t n);

/* Capacity that always suffices for scheme on n rows (host arithmetic, no device work):
 * *num_blocks as tp_encode_size; *words0 / *words1 = worst-case data words (every miniblock
 * 32 bits wide: FOR 130 words per 128 rows, DFOR + 1 per tile, RFOR 518 per 512 rows and
 * stream, None n rounded up to 32).  Allocate starts with num_blocks+1+TP_GUARD_WORDS words and
 * data with words+TP_GUARD_WORDS words. */
tp_status tp_gpu_encode_bound(int scheme, uint64_t n, uint64_t* num_blocks, uint64_t* words0, uint64_t* words1);

/* Exact data words of all three formats for DEVICE d_x[0..n), one pass (GPU-* analysis,
 * P:1206-1217): words4 (host) = {FOR, DFOR, RFOR values, RFOR run lengths}.  Blocks until
 * the counts are on the host. */
tp_status tp_gpu_encode_sizes(const int32_t* d_x, uint64_t n, void* d_work, uint64_t* words4, void* stream);

/* GPU-* on a DEVICE column (same rule as tp_choose_scheme: smallest footprint, ties
 * FOR < DFOR < RFOR, R20).  Blocks. */
tp_status tp_gpu_choose_scheme(const int32_t* d_x, uint64_t n, void* d_work, int* scheme, uint64_t* bytes,
                               void* stream);

/* Encode DEVICE d_x[0..n) into DEVICE arrays: starts0/data0 (+ starts1/data1 for RFOR) as
 * for tp_encode; cap0 / cap1 = usable data words (guards excluded; tp_gpu_encode_bound or
 * tp_gpu_encode_sizes give a sufficient value).  Writes every used word, the last
 * block_starts entry and the zero guard words.  tp_gpu_encode_launch is asynchronous on
 * `stream`; tp_gpu_encode_result waits for it and fills *out with the device pointers, word
 * counts and max_tile_words (TP_ESIZE if a capacity was too small -- the arrays are then
 * incomplete).  tp_gpu_encode = launch + result. */
tp_status tp_gpu_encode_launch(int scheme, const int32_t* d_x, uint64_t n, uint32_t* d_starts0, uint32_t* d_data0,
                               uint64_t cap0, uint32_t* d_starts1, uint32_t* d_data1, uint64_t cap1, void* d_work,
                               void* stream);
tp_status tp_gpu_encode_result(int scheme, uint64_t n, const uint32_t* d_starts0, const uint32_t* d_data0,
                               const uint32_t* d_starts1, const uint32_t* d_data1, const void* d_work,
                               tp_column* out, void* stream);
tp_status tp_gpu_encode(int scheme, const int32_t* d_x, uint64_t n, uint32_t* d_starts0, uint32_t* d_data0,
                        uint64_t cap0, uint32_t* d_starts1, uint32_t* d_data1, uint64_t cap1, void* d_work,
                        tp_column* out, void* stream);

/* ---------------------------------------------- measurement (not the method)
 * The INT32 issue roof of SURVEY.md 8(d): the low-bitwidth decoders are bound by
 * integer instruction issue, not HBM (P:1705-1707 for DFOR on the paper's GPU).
 * Launches one microbenchmark kernel on every SM (8 CTAs x 256 threads, 8 independent
 * dependency chains per thread) asynchronously on `stream`; *warp_insts (host) = the
 * warp instructions of the measured kind it executes (the caller times the launch).
 * kind (three register operands): 0 SHF, 1 LOP3, 2 IADD3, 3 IMAD, 4 SHF / LOP3 / IADD3
 * mix (ALU pipe), 5 LOP3 / IMAD alternating (ALU + FMA pipes); (two registers + an
 * immediate): 6 SHF, 7 LOP3, 8 IMAD, 9 LOP3 / SHF / IMAD over both pipes (the per-SMSP
 * issue limit).  d_sink: one DEVICE u32 (practically never written). */
tp_status tp_bench_int_roof(int kind, uint32_t iters, uint32_t* d_sink, uint64_t* warp_insts, void* stream);

/* --------------------------------------------------------------- utility */

const char* tp_status_string(tp_status s);

/* Number of CUDA kernels this library has launched in this process
 * (bench.py reports it as gpu_launches). */
uint64_t tp_launch_count(void);
/* Profiling builds only (-DTP_PROFILE_WAITS): copy 16 cycle counters of the query pipeline
 * (consumer data waits, per-column work, producer slot waits) to out16 (host) and reset
 * them.  Other builds report zeros. */
tp_status tp_debug_counters(uint64_t* out16);

/* Number of SMs of the current device and the decoder's CTAs per SM
 * (persistent grid = SMs x CTAs/SM). */
tp_status tp_device_info(int* sm_count, int* ctas_per_sm);

#ifdef __cplusplus
}
#endif
#endif /* TILEPACK_H */
