"""GPU parity of the sort offload (include/blu_sort.h; §3)
against the CPU oracle (oracle/sort_oracle.cpp) on the same seeded inputs: partial keys, the sorted
partial key buffer and its payload order (stability), duplicate ranges and the completed sort are
all compared exactly (integer work: bit-exact)."""
import numpy as np
import pytest

import blugen
import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def bg():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sigmod_merajispcksygnk16_b200 import blugby
    return blugby


def u32(t):
    return t.cpu().numpy().view(np.uint32)


def dev_u32(a):
    return torch.from_numpy(np.ascontiguousarray(a, np.uint32).view(np.int32)).cuda()


@pytest.mark.parametrize("W", [4, 12, 16])
def test_partial_keys(bg, W):
    rows = blugen.sort_rows(100_003, W, seed=W)
    d = torch.from_numpy(rows).cuda()
    for w in range(W // 4):
        assert np.array_equal(u32(bg.blu_sort_partial_keys(d, w)), oracle.partial_keys(rows, w))


@pytest.mark.parametrize("n,card", [(1, 5), (31, 5), (4095, 7), (4097, 2**32), (100_003, 300),
                                    (1_000_003, 2**32), (1_000_003, 1), (3_000_001, 1 << 20)])
def test_sort_pairs_stable(bg, n, card):
    """Keys sorted, and payloads in the oracle's stable order (ties by buffer order) — across tiles,
    CTAs and ragged tails; card=1 (all keys equal) must return the payload unchanged."""
    rng = np.random.default_rng(n)
    keys = rng.integers(0, card, n, dtype=np.uint64).astype(np.uint32)
    pay = rng.permutation(n).astype(np.uint32)
    ko, po = bg.blu_sort_pairs(dev_u32(keys), dev_u32(pay))
    eko, epo = oracle.sort_pairs(keys, pay)
    assert np.array_equal(u32(ko), eko)
    assert np.array_equal(u32(po), epo)


@pytest.mark.parametrize("n,card", [(1, 3), (2, 1), (9999, 3), (500_000, 200_000), (2_000_001, 1000)])
def test_dup_ranges(bg, n, card):
    rng = np.random.default_rng(card)
    keys = np.sort(rng.integers(0, card, n)).astype(np.uint32)
    st, ln = bg.blu_sort_dup_ranges(dev_u32(keys))
    est, eln = oracle.dup_ranges(keys)
    assert np.array_equal(st.cpu().numpy(), est) and np.array_equal(ln.cpu().numpy(), eln)


@pytest.mark.parametrize("seg", ["1", "0"])
@pytest.mark.parametrize("n,W", [(0, 8), (1, 8), (2, 4), (4097, 8), (300_007, 16), (1_000_003, 12), (2_000_000, 16)])
def test_sort_rows(bg, monkeypatch, n, W, seg):
    """The completed sort: identical permutation (stable lexicographic order), with short
    ranges sorted by the shared-memory window sort (default) or by the batched radix sort."""
    if seg == "0":
        monkeypatch.setenv("BLU_SORT_NO_SEG", "1")
    rows = blugen.sort_rows(n, W, seed=n + W)
    perm, stats = bg.blu_sort_rows(torch.from_numpy(rows).cuda())
    assert np.array_equal(u32(perm), oracle.sort_rows(rows))
    if n > 1000:
        assert stats["levels"] >= 2 and stats["ranges"][0] > 0  # the date word alone leaves duplicates


def test_sort_rows_small_alphabet_all_levels(bg):
    """Bytes from {0,1,2}: duplicate ranges survive every level and fully equal rows remain at the
    end (they must stay in row order)."""
    rng = np.random.default_rng(4)
    rows = rng.integers(0, 3, (200_000, 12), dtype=np.uint8)
    perm, stats = bg.blu_sort_rows(torch.from_numpy(rows).cuda())
    assert np.array_equal(u32(perm), oracle.sort_rows(rows))
    assert stats["levels"] == 3 and stats["active"][2] > 0


def test_sort_rows_special_cases(bg):
    n, W = 50_000, 8
    same = np.zeros((n, W), np.uint8)
    perm, _ = bg.blu_sort_rows(torch.from_numpy(same).cuda())
    assert np.array_equal(u32(perm), np.arange(n, dtype=np.uint32))
    rev = np.stack([np.frombuffer(int(x).to_bytes(W, "big"), np.uint8) for x in range(n)])[::-1].copy()
    perm, stats = bg.blu_sort_rows(torch.from_numpy(rev).cuda())
    assert np.array_equal(u32(perm), np.arange(n, dtype=np.uint32)[::-1])


@pytest.mark.parametrize("sw", ["2048", "4096", "2048-nowarp"])
@pytest.mark.parametrize("run", [1, 2, 7, 33, 100, 256, 257, 300, 1024, 1025, 2048, 2049, 5000])
def test_sort_rows_window_boundaries(bg, monkeypatch, run, sw):
    """Level-1 ranges of a fixed length (word 0 = row // run) whose level-1 keys are random with many
    ties (word 1 from {0..3}): ranges of up to 256 rows take the warp sort (every network size), up to
    sw/2 rows the window sort (straddling the sw-row windows at every offset), longer ones the batched
    radix sort. Word 2 = row id reversed keeps
    a third level for the tied rows."""
    monkeypatch.setenv("BLU_SORT_SEG_W", sw[:4])
    if sw.endswith("nowarp"):  # ranges <= 256 rows take the window sort instead of the warp sort
        monkeypatch.setenv("BLU_SORT_NO_WARP", "1")
    n = 60_001
    rng = np.random.default_rng(run)
    i = np.arange(n, dtype=np.uint64)
    w0 = (i // run).astype(np.uint32)
    w1 = rng.integers(0, 4, n).astype(np.uint32)
    w2 = (n - i).astype(np.uint32)
    rows = np.stack([w0, w1, w2], 1).astype(">u4").view(np.uint8).reshape(n, 12).copy()
    perm, stats = bg.blu_sort_rows(torch.from_numpy(rows).cuda())
    assert np.array_equal(u32(perm), oracle.sort_rows(rows))
    if run > 1:
        assert stats["levels"] >= 2
