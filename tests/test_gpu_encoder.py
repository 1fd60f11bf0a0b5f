"""GPU parity of the tile-parallel encoder (tp_gpu_encode) against the oracle:
the bytes the GPU writes (header, block_starts, data) are compared word for word with
oracle.encode of the same seeded column; GPU-* sizes / choice against oracle.choose_scheme.
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


def _dev(x):
    return torch.from_numpy(np.ascontiguousarray(x, np.int32)).cuda()


def _same(g, e):
    a = g.arrays()
    assert np.array_equal(a["header"], e["header"])
    if e["scheme"] == "rfor":
        assert np.array_equal(a["starts0"], e["startsV"]), "startsV"
        assert np.array_equal(a["data0"], e["dataV"]), f"dataV first bad {np.flatnonzero(a['data0'] != e['dataV'])[:4]}"
        assert np.array_equal(a["starts1"], e["startsL"]), "startsL"
        assert np.array_equal(a["data1"], e["dataL"]), "dataL"
    else:
        assert np.array_equal(a["starts0"], e["starts"]), "starts"
        assert np.array_equal(a["data0"], e["data"]), f"data first bad {np.flatnonzero(a['data0'] != e['data'])[:4]}"
    assert g.nbytes() == e.nbytes()


def _guards_zero(g):
    nb = int(g.col.num_blocks)
    assert not g.starts0[nb + 1: nb + 1 + tp.GUARD_WORDS].any()
    assert not g.data0[g.col.words0: g.col.words0 + tp.GUARD_WORDS].any()
    if g.data1 is not None:
        assert not g.starts1[nb + 1: nb + 1 + tp.GUARD_WORDS].any()
        assert not g.data1[g.col.words1: g.col.words1 + tp.GUARD_WORDS].any()


def _check(x, scheme, exact=False):
    g = tp.gpu_encode(_dev(x), scheme, exact=exact)
    _same(g, oracle.encode(scheme, x))
    _guards_zero(g)
    return g


def test_bruteforce_tiny_columns_byte_identical():
    """every column of length <= 3 over {INT32_MIN, -1, 0, 1, 2, 3, INT32_MAX}"""
    for x in datagen.small_alphabet_columns(3):
        if len(x) == 0:
            continue
        for s in SCHEMES:
            _check(x, s)


@pytest.mark.parametrize("scheme", SCHEMES)
def test_mixed_ragged_columns(scheme):
    for name, x in datagen.mixed_columns(seed=13):
        if len(x) == 0:
            continue
        _check(x, scheme)


def test_every_bitwidth_for():
    for b in range(0, 33):
        _check(datagen.uniform_bits(b, 512 * 21 + 13 * b, seed=300 + b), "for", exact=(b % 2 == 0))


@pytest.mark.parametrize("scheme,gen", [
    ("for", lambda n: datagen.uniform_bits(16, n, seed=5)),
    ("for", lambda n: datagen.uniform_bits(32, n, seed=6)),
    ("dfor", lambda n: datagen.sorted_uniform(n, seed=6)),
    ("dfor", lambda n: datagen.near_sorted(n, seed=9)),
    ("dfor", lambda n: datagen.d1_sorted(n, 2**28)),
    ("rfor", lambda n: datagen.runs(n, 4, seed=7)),
    ("rfor", lambda n: datagen.runs(n, 64, seed=8)),
    ("rfor", lambda n: datagen.uniform_bits(16, n, seed=10)),  # r = 512 almost everywhere
])
def test_many_chunks_lookback(scheme, gen):
    """thousands of 4096-row chunks: every tile offset comes out of the decoupled look-back"""
    n = 5_000_000 + 321
    x = gen(n)
    g = _check(x, scheme, exact=True)
    # and the GPU-encoded column decodes through the product decoder
    assert np.array_equal(tp.decode(g).cpu().numpy(), x)


def test_sizes_and_choice_match_oracle():
    for x in (datagen.d1_prefix(200_000, 2**28, 250_000_000), datagen.runs(200_000, 16, seed=2),
              datagen.uniform_bits(9, 200_000, seed=3), np.zeros(1000, np.int32), datagen.consecutive(77_777),
              datagen.uniform_bits(32, 5000, seed=1)):
        d = _dev(x)
        work = torch.empty((tp.tp_gpu_encode_workspace_bytes(len(x)) + 7) // 8, dtype=torch.int64, device="cuda")
        w = tp.tp_gpu_encode_sizes(d, len(x), work)
        ef, ed, er = (oracle.encode(s, x) for s in SCHEMES)
        assert w == [len(ef["data"]), len(ed["data"]), len(er["dataV"]), len(er["dataL"])]
        s, b = tp.tp_gpu_choose_scheme(d, len(x), work)
        os_, oe = oracle.choose_scheme(x)
        assert tp.SCHEME_NAMES[s] == os_ and b == oe.nbytes()
        assert tp.gpu_encode(d, "auto").scheme == os_


def test_max_tile_words_match_host_encoder_rule():
    for s, x in (("for", datagen.uniform_bits(16, 512 * 10 + 5, seed=1)), ("dfor", datagen.near_sorted(40_000)),
                 ("rfor", datagen.runs(40_000, 3, seed=2))):
        g = tp.gpu_encode(_dev(x), s)
        h = tp.encode(x, s)
        assert (g.col.max_tile_words0, g.col.max_tile_words1) == (h.col.max_tile_words0, h.col.max_tile_words1)


def test_capacity_too_small_is_an_error():
    x = _dev(datagen.uniform_bits(20, 100_000, seed=1))
    n = x.numel()
    work = torch.empty((tp.tp_gpu_encode_workspace_bytes(n) + 7) // 8, dtype=torch.int64, device="cuda")
    nb, w0, _ = tp.tp_gpu_encode_bound(tp.TP_FOR, n)
    starts = torch.empty(nb + 1 + 4, dtype=torch.int32, device="cuda")
    data = torch.empty(1000 + 4, dtype=torch.int32, device="cuda")
    with pytest.raises(tp.TilepackError, match="too small"):
        tp.tp_gpu_encode(tp.TP_FOR, x, n, starts, data, 1000, None, None, 0, work)


def test_empty_and_none_columns():
    for s in SCHEMES:
        g = tp.gpu_encode(torch.zeros(0, dtype=torch.int32, device="cuda"), s)
        assert g.col.words0 == 0 and g.nbytes() == tp.encode(np.zeros(0, np.int32), s).nbytes()
        assert g.arrays()["starts0"].tolist() == [0]
    for n in (1, 33, 512 * 9 + 7):
        x = np.random.default_rng(n).integers(-(2**31), 2**31, n, dtype=np.int64).astype(np.int32)
        g = tp.gpu_encode(_dev(x), "none")
        h = tp.encode(x, "none")
        a, b = g.arrays(), h.arrays()
        for k in ("header", "starts0", "data0"):
            assert np.array_equal(a[k], b[k]), k
        assert np.array_equal(a["data0"][:n].view(np.int32), x)


@pytest.mark.slow
def test_bench_size_gpu_encode_for_b16():
    """the bench column (500M rows U[0,2^16), BASELINE config 2) encoded on the GPU: the
    closed-form size (b + 0.75 bits/int), a 4M-row tile-aligned slice byte-identical
    to the oracle's encoding of that slice, sampled rows decoded by the oracle's Alg. 1 from the
    GPU's bytes, and the fused sum."""
    n = 500_000_000
    x = datagen.uniform_bits(16, n)
    g = tp.gpu_encode(_dev(x), "for")
    assert g.nbytes() == 4 * (3 + (n // 128) + 1 + (n // 128) * (2 + 4 * 16))
    lo = 512 * 300_000
    k = 4_000_000
    e = oracle.encode("for", x[lo:lo + k])
    ds = g.data0[int(g.starts0[lo // 128].item()): int(g.starts0[(lo + k) // 128].item())].cpu().numpy().view(np.uint32)
    assert np.array_equal(ds, e["data"])
    a = g.arrays()
    enc = oracle.Encoded(scheme="for", header=a["header"], starts=a["starts0"], data=a["data0"])
    dg = enc.guarded("data")
    rng = np.random.default_rng(1)
    for i in rng.integers(0, n, 2000):
        assert oracle.for_decode_range(enc, int(i), int(i) + 1, dg)[0] == x[i]
    assert np.array_equal(oracle.for_decode_range(enc, n - 1000, n, dg), x[n - 1000:])
    assert int(tp.decode_sum(g).item()) == int(x.astype(np.int64).sum())
