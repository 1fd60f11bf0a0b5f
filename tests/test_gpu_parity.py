"""GPU parity: the sm_100a decoders and fused operators vs the CPU oracle, through the C ABI.
Integer work: every comparison is bit-exact."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import datagen  # noqa: E402
import oracle  # noqa: E402
from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp  # noqa: E402

SCHEMES = ("for", "dfor", "rfor")


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.set_device(0)


def _check_column(x, scheme):
    h = tp.encode(x, scheme)
    e = oracle.encode(scheme, x)
    want = oracle.decode(e)
    d = h.to_device()
    got = tp.decode(d).cpu().numpy()
    assert np.array_equal(got, want), f"{scheme} n={len(x)} first bad row {np.flatnonzero(got != want)[:5]}"
    s = int(tp.decode_sum(d).item())
    assert s == oracle.column_sum(want)


@pytest.mark.parametrize("scheme", SCHEMES)
def test_mixed_ragged_columns(scheme):
    for name, x in datagen.mixed_columns(seed=11):
        if len(x) == 0:
            continue
        _check_column(x, scheme)


@pytest.mark.parametrize("scheme", SCHEMES)
def test_tiny_columns(scheme):
    for x in list(datagen.small_alphabet_columns(2))[1:]:
        _check_column(x, scheme)


def test_every_bitwidth_for():
    for b in range(0, 33):
        _check_column(datagen.uniform_bits(b, 512 * 37 + 13, seed=100 + b), "for")


def test_mixed_bitwidths_within_warp():
    """lanes of one warp disagree on b: the runtime-bitwidth fallback path."""
    rng = np.random.default_rng(4)
    parts = [rng.integers(0, 2 ** int(rng.integers(0, 32)), 32, dtype=np.int64) for _ in range(2000)]
    x = np.concatenate(parts).astype(np.int32)
    for s in SCHEMES:
        _check_column(x, s)


@pytest.mark.parametrize("scheme,gen", [
    ("for", lambda n: datagen.uniform_bits(16, n, seed=5)),
    ("dfor", lambda n: datagen.sorted_uniform(n, seed=6)),
    ("dfor", lambda n: datagen.d1_sorted(n, 2**28)),
    ("rfor", lambda n: datagen.runs(n, 4, seed=7)),
    ("rfor", lambda n: datagen.runs(n, 64, seed=8)),
])
def test_many_ctas(scheme, gen):
    """several stages per CTA, every CTA busy, ragged tail"""
    n = 5_000_000 + 321
    _check_column(gen(n), scheme)


def test_empty_column():
    h = tp.encode(np.zeros(0, np.int32), "for")
    d = h.to_device()
    assert int(tp.decode_sum(d).item()) == 0


def test_select_project_sum_parity():
    rng = np.random.default_rng(3)
    n = 1_000_000 + 77
    qty = rng.integers(1, 51, n, dtype=np.int32)
    disc = rng.integers(0, 11, n, dtype=np.int32)
    price = rng.integers(90000, 10_000_000, n, dtype=np.int32)
    date = np.repeat(rng.integers(19920101, 19981231, n // 4 + 1, dtype=np.int32), 4)[:n]
    cols = [date, qty, disc, price]
    schemes = ["rfor", "for", "for", "dfor"]
    dc = [tp.encode(c, s).to_device() for c, s in zip(cols, schemes)]
    lo = [19930101, 1, 1, -(2**31)]
    hi = [19931231, 24, 3, 2**31 - 1]
    for proj, a, b in (("mul", 3, 2), ("col", 3, 0), ("sub", 3, 1), ("count", 0, 0)):
        got = int(tp.select_project_sum(dc, lo, hi, proj, a, b).item())
        assert got == oracle.select_project_sum(cols, lo, hi, proj, a, b), proj


def test_plain_sum():
    x = datagen.uniform_bits(32, 1_000_003, seed=2)
    t = torch.from_numpy(x).cuda()
    out = torch.zeros(1, dtype=torch.int64, device="cuda")
    tp.tp_plain_sum(t, len(x), out)
    assert int(out.item()) == oracle.column_sum(x)


@pytest.mark.slow
def test_bench_size_for_b16_sampled():
    """BASELINE config 2 at the bench's launch configuration: 500M U[0,2^16) rows.
    Fused sum == the plain int64 sum; decoded rows at 20k sampled positions == Alg. 1."""
    n = 500_000_000
    x = datagen.uniform_bits(16, n)
    h = tp.encode(x, "for")
    assert h.nbytes() == 4 * (3 + (n // 128) + 1 + (n // 128) * (2 + 4 * 16))
    d = h.to_device()
    assert int(tp.decode_sum(d).item()) == int(x.astype(np.int64).sum())
    out = tp.decode(d)
    rng = np.random.default_rng(0)
    idx = np.sort(rng.integers(0, n, 20_000))
    got = out[torch.from_numpy(idx).cuda()].cpu().numpy()
    e = oracle.Encoded(scheme="for", header=h.header(), starts=h.starts0[: h.col.num_blocks + 1],
                       data=h.data0[: h.col.words0])
    dg = h.data0  # already has guard words
    want = np.array([oracle.for_decode_range(e, int(i), int(i) + 1, dg)[0] for i in idx[:2000]], np.int32)
    assert np.array_equal(got[:2000], want)
    assert np.array_equal(got, x[idx])
    tail = out[n - 1000:].cpu().numpy()
    assert np.array_equal(tail, oracle.for_decode_range(e, n - 1000, n, dg))
    # the whole decoded column == x (decode(encode(x)) == x, the oracle-pinned definition)
    assert torch.equal(out, torch.from_numpy(x).cuda())
    assert tp.tp_device_errors() == 0


@pytest.mark.parametrize("b", [0, 1, 4, 8, 12])
def test_lean_for_sum_full_rounds(b):
    """The low-bitwidth decode->sum variant (k_decode_sum<FOR, LEAN>, max_tile_words <= 200) on a
    column long enough that every CTA runs many full rounds of 8 tiles per item (24M rows = 46,875
    tiles over <= 740 CTAs), plus a ragged tail: the fused sum == the int64 sum of x, the decoded
    column == x element by element (Alg. 1; bitwidth sweep P:1419-1423)."""
    n = 24_000_000 + 333
    x = datagen.uniform_bits(b, n, seed=7000 + b)
    h = tp.encode(x, "for")
    assert h.col.max_tile_words0 <= 200  # the lean kernel is the one dispatched
    d = h.to_device()
    assert int(tp.decode_sum(d).item()) == oracle.column_sum(x)
    xd = torch.from_numpy(x).cuda()
    assert torch.equal(tp.decode(d), xd)
    # every 512-row tile-range shard boundary inside a CTA's range: a sub-range starting mid-column
    from paper_conf_sigmod_shanbhagyym22_b200 import dist as tpd
    lo, hi = tpd.tile_range(n, 1, 3)
    ds = tpd.ShardColumn(h, lo, hi).to_device()
    assert int(tp.decode_sum(ds).item()) == oracle.column_sum(x[lo:hi])
    assert tp.tp_device_errors() == 0


def test_device_format_errors_flagged():
    """Format violations the kernels meet are flagged (tp_device_errors), not silent: a
    max_tile_words below the column's real tile span (the ring stays in bounds, the flag says the
    result is undefined) and an RFOR run count > 512; a bitwidth byte > 32 (R3, R5) is used as 32
    on the device (memory-safe) and reported by tp_validate on the host."""
    assert tp.tp_device_errors() == 0
    x = datagen.uniform_bits(10, 5_000_000 + 5, seed=3)  # many tiles per CTA: items of many tiles
    h = tp.encode(x, "for")
    d = h.to_device()
    tp.decode_sum(d)
    assert tp.tp_device_errors() == 0
    bw = int(h.starts0[9]) + 1
    bad = h.data0.copy()
    bad[bw] = (bad[bw] & ~np.uint32(0xff0000)) | np.uint32(45 << 16)
    d.data0.copy_(torch.from_numpy(bad.view(np.int32)))
    tp.decode_sum(d)
    torch.cuda.synchronize()  # completes without a fault (the byte is used as 32)
    old_word = h.data0[bw]
    h.data0[bw] = bad[bw]
    with pytest.raises(tp.TilepackError, match="malformed"):
        tp.tp_validate(h.col)
    h.data0[bw] = old_word
    d = h.to_device()
    d.col.max_tile_words0 = 8  # far below the 4 x (2 + 4 x 10) words of a tile
    tp.decode_sum(d)
    assert tp.tp_device_errors() & tp.TP_DEVERR_TILE_WORDS
    r = tp.encode(datagen.runs(512 * 8, 4, seed=2), "rfor")
    dr = r.to_device()
    bad = r.data0.copy()
    bad[int(r.starts0[3])] = 900  # run count > 512
    dr.data0.copy_(torch.from_numpy(bad.view(np.int32)))
    tp.decode_sum(dr)
    assert tp.tp_device_errors() & tp.TP_DEVERR_RUNS
    assert tp.tp_device_errors() == 0  # read-and-clear


@pytest.mark.parametrize("scheme", SCHEMES)
def test_fake_multi_gpu_shards(scheme):
    """shard into k tile ranges, decode each shard on GPU 0, the pieces
    concatenate to the column and the shard sums add up to the whole-column sum."""
    from paper_conf_sigmod_shanbhagyym22_b200 import dist as tpd
    n = 512 * 301 + 77
    x = {"for": datagen.uniform_bits(20, n, seed=1), "dfor": datagen.sorted_uniform(n, seed=2),
         "rfor": datagen.runs(n, 5, seed=3)}[scheme]
    h = tp.encode(x, scheme)
    for world in (2, 3, 8):
        acc = torch.zeros(1, dtype=torch.int64, device="cuda")
        pieces = []
        for r in range(world):
            d = tpd.shard(h, r, world).to_device()
            pieces.append(tp.decode(d).cpu().numpy())
            tp.decode_sum(d, out=acc)
        assert np.array_equal(np.concatenate(pieces), x)
        assert int(acc.item()) == oracle.column_sum(x)


@pytest.mark.parametrize("scheme", SCHEMES)
def test_cascaded_baseline_parity(scheme):
    """NEXT-1: the cascading-decompression baseline decodes the same bytes to the same values."""
    for name, x in list(datagen.mixed_columns(seed=21))[::3]:
        if len(x) == 0:
            continue
        d = tp.encode(x, scheme).to_device()
        assert np.array_equal(tp.decode_cascaded(d).cpu().numpy(), x), (scheme, name)
    x = {"for": datagen.uniform_bits(12, 3_000_001, seed=4), "dfor": datagen.near_sorted(3_000_001, seed=4),
         "rfor": datagen.runs(3_000_001, 6, seed=4)}[scheme]
    d = tp.encode(x, scheme).to_device()
    assert np.array_equal(tp.decode_cascaded(d).cpu().numpy(), x)


@pytest.mark.parametrize("n", [1, 31, 512, 512 * 8 + 5, 512 * 37 + 77, 3_000_001])
def test_none_plain_column(n):
    """TP_NONE (the uncompressed baseline): decode == the column itself, through the
    TMA tensor-box path (ragged tails zero-filled by the box, masked by the consumer)."""
    x = np.random.default_rng(n).integers(-(2**31), 2**31, n, dtype=np.int64).astype(np.int32)
    d = tp.encode(x, "none").to_device()
    assert np.array_equal(tp.decode(d).cpu().numpy(), x)
    assert int(tp.decode_sum(d).item()) == oracle.column_sum(x)
    got = int(tp.select_project_sum([d, d], [-(2**30), 0], [2**30, 2**31 - 1], "col", 1, 0).item())
    want = oracle.select_project_sum([x, x], [-(2**30), 0], [2**30, 2**31 - 1], "col", 1, 0)
    assert got == want


@pytest.mark.parametrize("scheme", ("for", "dfor", "rfor", "none"))
def test_bitmap_random_access(scheme):
    """NEXT-4 random access: the sum of the rows a predicate bitvector selects,
    across selectivities from 0 (every tile skipped) to 1, ragged tail, == the oracle."""
    for n in (512 * 301 + 77, 2_000_003):
        x = {"for": datagen.uniform_bits(17, n, seed=1), "dfor": datagen.near_sorted(n, seed=2),
             "rfor": datagen.runs(n, 9, seed=3), "none": datagen.uniform_bits(31, n, seed=4)}[scheme]
        d = tp.encode(x, scheme).to_device()
        for k, sigma in enumerate((0.0, 1e-5, 1 / 512, 0.01, 0.3, 1.0)):
            bm = datagen.bernoulli_bitmap(n, sigma, seed=10 + k)
            got = int(tp.bitmap_sum(d, torch.from_numpy(bm.view(np.int32)).cuda()).item())
            assert got == oracle.bitmap_sum(x, bm), (scheme, n, sigma)
    # one selected row in the last, partial miniblock; bits past n set (ignored)
    bm = np.zeros((n + 31) // 32, np.uint32)
    bm[-1] = np.uint32(0xffffffff)
    got = int(tp.bitmap_sum(d, torch.from_numpy(bm.view(np.int32)).cuda()).item())
    assert got == int(x[(n // 32) * 32:].astype(np.int64).sum())


@pytest.mark.slow
@pytest.mark.parametrize("scheme,gen", [
    ("dfor", lambda n: datagen.d1_sorted(n, 2**28)),        # BASELINE config 3
    ("rfor", lambda n: datagen.runs(n, 4)),                 # BASELINE config 4, shortest runs
])
def test_full_size_dfor_rfor(scheme, gen):
    """configs 3 / 4 at the suite's full size (500M rows), in the launch configuration
    scripts/bench_suite.py times: the GPU decode of the encoded bytes == the oracle's decode of
    the same bytes (whole column), and the fused sum == the oracle's int64 sum."""
    n = 500_000_000
    x = gen(n)
    h = tp.encode(x, scheme)
    a = h.arrays()
    if scheme == "dfor":
        e = oracle.Encoded(scheme="dfor", header=a["header"], starts=a["starts0"], data=a["data0"])
    else:
        e = oracle.Encoded(scheme="rfor", header=a["header"], startsV=a["starts0"], dataV=a["data0"],
                           startsL=a["starts1"], dataL=a["data1"])
    want = oracle.decode(e)
    d = h.to_device()
    got = tp.decode(d)
    assert torch.equal(got, torch.from_numpy(want).cuda())
    assert int(tp.decode_sum(d).item()) == oracle.column_sum(want)


def test_no_miniblock_variant():
    """the miniblock ablation: GPU decode / decode_sum of GPU-FOR without miniblocks
    == the oracle's decode, every bitwidth and ragged lengths; query operators refuse it."""
    for b in (0, 1, 7, 16, 31, 32):
        _check_column(datagen.uniform_bits(b, 512 * 23 + 45, seed=b), "fornm")
    for name, x in list(datagen.mixed_columns(seed=31))[::4]:
        if len(x):
            _check_column(x, "fornm")
    rng = np.random.default_rng(5)  # skewed: a few outliers widen a whole block (vs one miniblock)
    x = rng.integers(0, 2**6, 3_000_017, dtype=np.int64)
    x[rng.integers(0, len(x), 3000)] = 2**20
    _check_column(x.astype(np.int32), "fornm")
    d = tp.encode(x.astype(np.int32), "fornm").to_device()
    with pytest.raises(tp.TilepackError):
        tp.select_project_sum([d], [0], [5], "col", 0)
