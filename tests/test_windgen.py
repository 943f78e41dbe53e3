"""Pins for the shared input generator (windgen): splitmix64 against its published
first outputs, the content layout, and the workload statistics it is fitted to."""
import math

import numpy as np

import windgen as W


def test_splitmix64_published_values():
    # SplitMix64 seeded with 0 (Steele, Lea, Flood 2014; Vigna's splitmix64.c):
    # first outputs e220a8397b1dcdaf, 6e789e6aa1b965f4, 06c45d188009454f.
    assert W.splitmix64_scalar(0) == 0xE220A8397B1DCDAF
    assert W.splitmix64_scalar(W.GOLDEN) == 0x6E789E6AA1B965F4
    assert W.splitmix64_scalar(2 * W.GOLDEN & W.MASK64) == 0x06C45D188009454F


def test_content_words_match_scalar():
    key = W.content_key(3001, 7)
    idx = np.array([0, 1, 2, 12345, 2**40 + 3], dtype=np.uint64)
    got = W.content_words(3001, 7, idx)
    for i, w in zip(idx.tolist(), got.tolist()):
        assert w == W.splitmix64_scalar(key ^ i)


def test_content_bytes_little_endian():
    b = W.content_bytes(1, 2, 16, 16)
    w = W.content_words(1, 2, np.array([2, 3], np.uint64))
    assert b.tobytes() == int(w[0]).to_bytes(8, "little") + int(w[1]).to_bytes(8, "little")


def test_tags_distinguish_pools():
    a = W.content_bytes(9, 1, 0, 4096)
    b = W.content_bytes(9, 2, 0, 4096)
    assert (a != b).mean() > 0.95


def test_sharegpt_fit():
    """C2 lengths: log-normal fitted to Table 2's ShareGPT median 695 / P90 1556,
    then clipped to 256..2048: the unclipped fit reproduces the median and P90."""
    rng_l = W.lengths_sharegpt(200000, 1, lo=1, hi=10**9)
    assert abs(np.median(rng_l) - 695) / 695 < 0.02
    assert abs(np.percentile(rng_l, 90) - 1556) / 1556 < 0.03
    c2 = W.request_lengths("C2")
    assert c2.size == 64 and c2.min() >= 256 and c2.max() <= 2048


def test_longbench_fit():
    x = W.lengths_longbench(200000, 1, lo=-10**9, hi=10**9)
    assert abs(x.mean() - 2890.4) < 10
    assert abs(np.percentile(x, 90) - 3792) < 25


def test_blocks_and_cases():
    assert W.blocks_for_tokens(0) == 0 and W.blocks_for_tokens(1) == 1
    assert W.blocks_for_tokens(16) == 1 and W.blocks_for_tokens(17) == 2
    c = W.migration_case("C1")
    assert c.n == 256 and c.nb_src == math.ceil(1.1 * 256)
    assert len(set(c.dst_bt.tolist())) == c.n and len(set(c.src_bt.tolist())) == c.n
    assert c.shape.chunk_bytes == 24576
    s = W.migration_case("C2", variant="sequential")
    assert (s.src_bt == np.arange(s.n)).all()
    # C2 is ~40 GiB of payload
    c2 = W.migration_case("C2")
    payload = 2 * c2.shape.n_layers * c2.n * c2.shape.chunk_bytes
    assert 30 * 2**30 < payload < 50 * 2**30


def test_hash_shuffle_uniformish():
    d = W.hash_shuffle_dest(8000, 8, 5)
    cnt = np.bincount(d, minlength=8)
    assert cnt.min() > 850 and cnt.max() < 1150


def test_seed_offset_zero_is_the_survey_seeds_and_nonzero_changes_the_case():
    """bench --seed: offset 0 reproduces S§8(d)'s seeds exactly; another offset draws a new
    case from the same distributions (same request count, different lengths / slots /
    content seed)."""
    from windgen import migration_case
    a, b = migration_case("C2"), migration_case("C2", seed_offset=0)
    assert np.array_equal(a.src_bt, b.src_bt) and np.array_equal(a.dst_bt, b.dst_bt)
    assert a.content_seed == b.content_seed == 3002
    c = migration_case("C2", seed_offset=5)
    assert c.lengths.size == a.lengths.size and c.content_seed == 3007
    assert not np.array_equal(c.lengths, a.lengths)
    assert c.lengths.min() >= 256 and c.lengths.max() <= 2048
