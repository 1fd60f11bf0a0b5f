"""Host encoder of the product library (C++, multi-threaded) vs the oracle, byte for byte.
No GPU needed: encoding is the paper's one-time host step."""
import numpy as np
import pytest

import datagen
import oracle
from paper_conf_sigmod_shanbhagyym22_b200 import tilepack as tp

SCHEMES = ("for", "dfor", "rfor")


def _same(h, e):
    a = h.arrays()
    assert np.array_equal(a["header"], e["header"])
    if e["scheme"] == "rfor":
        assert np.array_equal(a["starts0"], e["startsV"]) and np.array_equal(a["data0"], e["dataV"])
        assert np.array_equal(a["starts1"], e["startsL"]) and np.array_equal(a["data1"], e["dataL"])
    else:
        assert np.array_equal(a["starts0"], e["starts"]) and np.array_equal(a["data0"], e["data"])
    assert h.nbytes() == e.nbytes()


def test_bruteforce_tiny_columns_byte_identical():
    for x in datagen.small_alphabet_columns(3):
        for s in SCHEMES:
            _same(tp.encode(x, s), oracle.encode(s, x))


@pytest.mark.parametrize("scheme", SCHEMES)
def test_mixed_columns_byte_identical(scheme):
    for name, x in datagen.mixed_columns(seed=5):
        _same(tp.encode(x, scheme), oracle.encode(scheme, x))


def test_c1_columns_byte_identical():
    for b in (1, 7, 16):
        x = datagen.c1_column(b)
        _same(tp.encode(x, "for"), oracle.for_encode(x))


def test_large_multithreaded_byte_identical():
    n = 3_000_000 + 123
    for s, x in (("for", datagen.uniform_bits(11, n, seed=9)), ("dfor", datagen.near_sorted(n, seed=8)),
                 ("rfor", datagen.runs(n, 5, seed=7))):
        _same(tp.encode(x, s), oracle.encode(s, x))


def test_choose_scheme_matches_oracle():
    for x in (datagen.d1_prefix(200_000, 2**28, 250_000_000), datagen.runs(200_000, 16, seed=2),
              datagen.uniform_bits(9, 200_000, seed=3), np.zeros(1000, np.int32)):
        s, b = tp.tp_choose_scheme(x)
        os_, oe = oracle.choose_scheme(x)
        assert tp.SCHEME_NAMES[s] == os_ and b == oe.nbytes()


def test_max_tile_words():
    x = datagen.uniform_bits(16, 512 * 10 + 5, seed=1)
    h = tp.encode(x, "for")
    s = h.starts0[: h.col.num_blocks + 1].astype(np.int64)
    spans = [s[min(4 * t + 4, len(s) - 1)] - s[4 * t] for t in range((len(s) - 1 + 3) // 4)]
    assert h.col.max_tile_words0 == max(spans)


@pytest.mark.parametrize("scheme", SCHEMES)
def test_shard_views_decode_to_slices(scheme):
    """tp_shard: a 512-row-aligned range view decodes (by the oracle) to the slice."""
    n = 512 * 13 + 200
    x = {"for": datagen.uniform_bits(9, n, seed=1), "dfor": datagen.near_sorted(n, seed=1),
         "rfor": datagen.runs(n, 7, seed=1)}[scheme]
    h = tp.encode(x, scheme)
    for lo, hi in ((0, 512 * 5), (512 * 5, 512 * 9), (512 * 9, n), (0, n), (512 * 13, n)):
        nbv = -(-(hi - lo) // (512 if scheme == "rfor" else 128))
        r0 = np.zeros(nbv + 1 + tp.GUARD_WORDS, np.uint32)
        r1 = np.zeros(nbv + 1 + tp.GUARD_WORDS, np.uint32) if scheme == "rfor" else None
        v = tp.tp_shard(h.col, lo, hi, r0, r1)
        assert v.n == hi - lo and v.num_blocks == nbv
        import ctypes

        def words(ptr, k):
            return np.ctypeslib.as_array((ctypes.c_uint32 * k).from_address(ptr)).copy()
        if scheme == "rfor":
            e = oracle.Encoded(scheme="rfor", header=np.array([512, 16, hi - lo], np.uint32),
                               startsV=r0[:nbv + 1], dataV=words(v.data0, v.words0),
                               startsL=r1[:nbv + 1], dataL=words(v.data1, v.words1))
        else:
            e = oracle.Encoded(scheme=scheme, header=np.array([128, 4, hi - lo], np.uint32),
                               starts=r0[:nbv + 1], data=words(v.data0, v.words0))
        assert np.array_equal(oracle.decode(e), x[lo:hi])


def test_errors():
    x = np.arange(1000, dtype=np.int32)
    with pytest.raises(tp.TilepackError):
        tp.tp_encode_size(7, x)
    h = tp.encode(x, "for")
    r0 = np.zeros(64, np.uint32)
    with pytest.raises(tp.TilepackError):
        tp.tp_shard(h.col, 100, 600, r0)   # not tile aligned


def test_none_layout():
    """TP_NONE: block_starts = 512 k, data = the values zero-padded to 32 words, bytes = 4 n."""
    for n in (0, 1, 511, 512, 513, 5000):
        x = np.arange(n, dtype=np.int32) * 3 - 7
        h = tp.encode(x, "none")
        nb = (n + 511) // 512
        assert int(h.col.num_blocks) == nb and int(h.col.words0) == (n + 31) // 32 * 32
        assert list(h.starts0[:nb]) == [512 * k for k in range(nb)] and h.starts0[nb] == h.col.words0
        assert np.array_equal(h.data0[:n].view(np.int32), x) and not h.data0[n:].any()
        assert h.nbytes() == 4 * n


def test_no_miniblock_variant_byte_identical():
    """GPU-FOR without miniblocks: the product's host encoder == the oracle's FOR
    with one 128-entry miniblock per block, byte for byte; size = 4 (3 + nb + 1 + sum(2 + 4 b))."""
    for name, x in datagen.mixed_columns(seed=9):
        h = tp.encode(x, "fornm")
        e = oracle.encode("fornm", x)
        _same(h, e)
        assert int(h.col.miniblock_count) == 1
    for x in datagen.small_alphabet_columns(3):
        _same(tp.encode(x, "fornm"), oracle.encode("fornm", x))
    # uniform b bits: every block has width b -> exactly the miniblock format's size
    x = datagen.uniform_bits(13, 128 * 1000, seed=2)
    assert tp.encode(x, "fornm").nbytes() == tp.encode(x, "for").nbytes()


def test_gpu_encode_bound_covers_every_encoding():
    """tp_gpu_encode_bound (host arithmetic): a capacity that always suffices -- never below the
    words the encoder actually produces (worst case: every miniblock 32 bits wide / every row its
    own run), equal to it for full-range data; the workspace grows with the chunk count."""
    cols = [datagen.uniform_bits(32, 5000 + 77, seed=1), datagen.runs(9000, 1, seed=2),
            np.zeros(1, np.int32), datagen.uniform_bits(7, 512 * 9, seed=3)]
    for x in cols:
        for s in ("for", "dfor", "rfor", "none"):
            sc = tp.SCHEMES[s]
            nb, w0, w1 = tp.tp_gpu_encode_bound(sc, len(x))
            h = tp.encode(x, s)
            assert nb == h.col.num_blocks and w0 >= h.col.words0 and w1 >= h.col.words1, (s, len(x))
    x = datagen.uniform_bits(32, 128 * 40, seed=4)
    assert tp.tp_gpu_encode_bound(tp.TP_FOR, len(x))[1] == tp.encode(x, "for").col.words0
    assert tp.tp_gpu_encode_workspace_bytes(10**8) > tp.tp_gpu_encode_workspace_bytes(10**6) > 0


@pytest.mark.parametrize("scheme", ("for", "dfor", "rfor", "none", "fornm"))
def test_validate_accepts_encoder_output(scheme):
    """tp_validate accepts every encoded column and reports the encoder's max_tile_words."""
    for name, x in list(datagen.mixed_columns(seed=8)) + [("c16", datagen.uniform_bits(16, 100_003, seed=1))]:
        h = tp.encode(x, scheme)
        m0, m1 = tp.tp_validate(h.col)
        assert (m0, m1) == (h.col.max_tile_words0, h.col.max_tile_words1), (scheme, name)


def _expect_eformat(col):
    with pytest.raises(tp.TilepackError, match="malformed"):
        tp.tp_validate(col)


def test_validate_rejects_corruptions():
    """Each corruption a decoder could not survive is TP_EFORMAT (include/tilepack.h tp_validate)."""
    x = datagen.uniform_bits(9, 512 * 6 + 40, seed=2)
    h = tp.encode(x, "for")
    bw_word = int(h.starts0[3]) + 1
    old = h.data0[bw_word]
    h.data0[bw_word] = (old & ~np.uint32(0xff00)) | np.uint32(40 << 8)   # bitwidth byte 40 > 32
    _expect_eformat(h.col)
    h.data0[bw_word] = old
    tp.tp_validate(h.col)
    h.starts0[5], h.starts0[6] = h.starts0[6], h.starts0[5]              # block_starts not monotone
    _expect_eformat(h.col)
    h = tp.encode(x, "for")
    h.col.num_blocks = h.col.num_blocks - 1                               # header inconsistent with n
    _expect_eformat(h.col)
    h = tp.encode(x, "fornm")
    h.data0[int(h.starts0[2]) + 1] |= np.uint32(1 << 8)                   # FORNM: bytes 1..3 must be 0
    _expect_eformat(h.col)
    r = tp.encode(datagen.runs(512 * 4, 5, seed=1), "rfor")
    r.data0[int(r.starts0[1])] = 600                                      # run count > 512
    _expect_eformat(r.col)
    r = tp.encode(datagen.runs(512 * 4, 5, seed=1), "rfor")
    r.data1[int(r.starts1[2])] += 1                                       # streams disagree on the run count
    _expect_eformat(r.col)
    d = tp.encode(datagen.near_sorted(512 * 3 + 9, seed=3), "dfor")
    d.col.words0 = d.col.words0 - 1                                       # data shorter than block_starts says
    _expect_eformat(d.col)


@pytest.mark.parametrize("scheme", ("for", "dfor", "rfor", "none"))
def test_shard_empty_range(scheme):
    """An empty tile range (and a shard of an empty column) is an empty view, no underflow."""
    from paper_conf_sigmod_shanbhagyym22_b200 import dist as tpd
    x = datagen.uniform_bits(5, 512 * 3, seed=1)
    for col in (x, np.zeros(0, np.int32)):
        h = tp.encode(col, scheme)
        s = tpd.ShardColumn(h, 0, 0)
        assert s.n == 0 and int(s.col.num_blocks) == 0 and int(s.col.words0) == 0 and int(s.col.words1) == 0
    h = tp.encode(np.zeros(0, np.int32), scheme)
    s = tpd.shard(h, 1, 4)
    assert s.n == 0 and int(s.col.words0) == 0
