"""windgen — seeded synthetic INPUT generators shared by the oracle side and the CUDA side.

This module holds none of the method's arithmetic (no block addressing, no table
validation, no copy).  It only synthesises what SURVEY.md §8(d) calls the common
generator:

* request-length mixes fitted to the paper's workloads
  (ShareGPT / LongBench statistics, Table 2; the Fig. 8
  decode set; OPT's 2048-token maximum context);
* block-table slot choices (a seeded permutation for the "shuffled" source,
  lowest-free-first destination slots in a pool with a seeded 30 % of slots
  pre-occupied);
* pool *content*: the counter-based splitmix64 byte pattern of SURVEY §8(c) O9.
  The same generator is implemented a second time, in CUDA, in
  ``windgen/csrc/windgen_fill.cu`` (``libwindgen_cuda.so``) so 40-110 GiB device pools
  can be filled and checked without a host copy; ``tests/test_windgen.py`` pins the two
  implementations against each other and against published splitmix64 values.

Everything is deterministic in its seeds: ``len_seed = 1000+k``, ``slot_seed = 2000+k``,
``content_seed = 3000+k`` for config Ck.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

MASK64 = (1 << 64) - 1
GOLDEN = 0x9E3779B97F4A7C15          # splitmix64 increment (Steele et al. 2014)
TAG_MUL = 0xD1B54A32D192ED03         # tag multiplier of SURVEY §8(c) O9
SM_M1 = 0xBF58476D1CE4E5B9
SM_M2 = 0x94D049BB133111EB

BLOCK_SIZE = 16  # tokens per block (BJ:configs)


# --------------------------------------------------------------------------- content

def splitmix64_scalar(x: int) -> int:
    """Reference scalar splitmix64 finaliser on a 64-bit counter x (returns the output
    for state x, i.e. z = x + GOLDEN then the two xor-shift-multiply rounds)."""
    z = (x + GOLDEN) & MASK64
    z = ((z ^ (z >> 30)) * SM_M1) & MASK64
    z = ((z ^ (z >> 27)) * SM_M2) & MASK64
    return z ^ (z >> 31)


def content_key(seed: int, tag: int) -> int:
    """The per-pool 64-bit key: seed*GOLDEN xor tag*TAG_MUL (mod 2^64)."""
    return ((seed * GOLDEN) & MASK64) ^ ((tag * TAG_MUL) & MASK64)


def content_words(seed: int, tag: int, word_index: np.ndarray) -> np.ndarray:
    """Vectorised O9 content: word w (the 8-byte word at pool byte offset 8*w) is
    splitmix64(key xor w).  Returns uint64 of the same shape as ``word_index``."""
    key = np.uint64(content_key(seed, tag))
    x = np.bitwise_xor(np.asarray(word_index, dtype=np.uint64), key)
    with np.errstate(over="ignore"):
        z = x + np.uint64(GOLDEN)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(SM_M1)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(SM_M2)
        z = z ^ (z >> np.uint64(31))
    return z


def content_bytes(seed: int, tag: int, byte_offset: int, nbytes: int) -> np.ndarray:
    """Bytes [byte_offset, byte_offset+nbytes) of the O9 pattern for pool (seed, tag),
    as uint8.  Offsets and sizes must be multiples of 8 (every pool chunk is)."""
    if byte_offset % 8 or nbytes % 8:
        raise ValueError("content_bytes needs 8-byte aligned offset and size")
    w0 = byte_offset // 8
    words = content_words(seed, tag, np.arange(w0, w0 + nbytes // 8, dtype=np.uint64))
    return words.view(np.uint8)  # little-endian word -> bytes, same as the device


# ------------------------------------------------------------------- request lengths

def blocks_for_tokens(tokens: np.ndarray | int, block_size: int = BLOCK_SIZE):
    """ceil(tokens / block_size): the number of paged blocks a request holds (A3: whole
    blocks are stored, the last possibly partial; A19: 0 tokens -> 0 blocks)."""
    t = np.asarray(tokens, dtype=np.int64)
    return (t + block_size - 1) // block_size


def lengths_sharegpt(n: int, seed: int, lo: int = 256, hi: int = 2048) -> np.ndarray:
    """Prompt lengths ~ clip(round(lognormal(mu=ln 695, sigma=ln(1556/695)/1.2816)), lo, hi):
    a log-normal matched to ShareGPT's median 695 and P90 1556 (Table 2),
    clipped to the C2 range 256-2048 (BJ:configs[1]; OPT max context 2048)."""
    rng = np.random.default_rng(seed)
    sigma = math.log(1556 / 695) / 1.2815515655446004
    x = rng.lognormal(mean=math.log(695), sigma=sigma, size=n)
    return np.clip(np.rint(x), lo, hi).astype(np.int64)


def lengths_longbench(n: int, seed: int, lo: int = 16, hi: int = 4096) -> np.ndarray:
    """Prompt lengths ~ clip(round(N(2890.4, 706.2)), 16, 4096): a normal matched to
    LongBench's mean 2890.4 and P90 3792 (sigma = (3792-2887)/1.2816 = 706.2), PAPER.md
    P:281 Table 2, within LLaMA-2's 4K context."""
    rng = np.random.default_rng(seed)
    x = rng.normal(loc=2890.4, scale=706.2, size=n)
    return np.clip(np.rint(x), lo, hi).astype(np.int64)


def lengths_longtail(n: int, seed: int, lo: int = 16, hi: int = 8192) -> np.ndarray:
    """C5's long-tail mix: clip(round(lognormal(ln 695, 1.0)), 16, 8192)."""
    rng = np.random.default_rng(seed)
    x = rng.lognormal(mean=math.log(695), sigma=1.0, size=n)
    return np.clip(np.rint(x), lo, hi).astype(np.int64)


# ---------------------------------------------------------------------- model shapes

@dataclass(frozen=True)
class KVShape:
    """The KV geometry a BJ:configs entry names (SURVEY §8 geometry table)."""
    name: str
    n_layers: int
    n_kv_heads: int
    head_dim: int
    elem_bytes: int
    block_size: int = BLOCK_SIZE

    @property
    def chunk_bytes(self) -> int:  # C = H*bs*d*e_b (bytes of one (layer, K|V, block))
        return self.n_kv_heads * self.block_size * self.head_dim * self.elem_bytes


SHAPES = {
    "C1": KVShape("OPT-125M", 12, 12, 64, 2),
    "C2": KVShape("OPT-13B", 40, 40, 128, 2),
    "C3": KVShape("OPT-66B", 64, 72, 128, 2),
    "C4": KVShape("Llama-2-70B-GQA-bf16", 80, 8, 128, 2),
    "C5": KVShape("Llama-3-8B-GQA-fp8", 32, 8, 128, 1),
}


def request_lengths(cfg: str, scale: float = 1.0, seed_offset: int = 0) -> np.ndarray:
    """Token lengths of the requests each config migrates.  ``scale`` < 1
    shrinks the request COUNT (not the distribution) for small parity cases;
    ``seed_offset`` shifts the config's seed (bench --seed)."""
    k = int(cfg[1])
    seed = 1000 + k + seed_offset
    if cfg == "C1":
        n = max(1, round(8 * scale))
        return np.full(n, 512, dtype=np.int64)
    if cfg == "C2":
        return lengths_sharegpt(max(1, round(64 * scale)), seed)
    if cfg == "C3":
        return np.full(max(1, round(4 * scale)), 2048, dtype=np.int64)
    if cfg == "C4":
        return lengths_longbench(max(1, round(32 * scale)), seed)
    if cfg == "C5":
        return lengths_longtail(max(1, round(1024 * scale)), seed)
    raise KeyError(cfg)


# ----------------------------------------------------------------------- slot choice

def shuffled_slots(n: int, n_slots: int, seed: int) -> np.ndarray:
    """The first n entries of a seeded permutation of [0, n_slots): fragmented sources."""
    if n > n_slots:
        raise ValueError("n > n_slots")
    rng = np.random.default_rng(seed)
    return rng.permutation(n_slots)[:n].astype(np.int32)


def occupied_mask(n_slots: int, frac: float, seed: int) -> np.ndarray:
    """A seeded random `frac` of [0, n_slots) marked occupied (bool array)."""
    rng = np.random.default_rng(seed)
    occ = np.zeros(n_slots, dtype=bool)
    k = int(round(frac * n_slots))
    occ[rng.permutation(n_slots)[:k]] = True
    return occ


def lowest_free(occupied: np.ndarray, n: int) -> np.ndarray:
    """Host KV-manager allocation, lowest free slot first."""
    free = np.flatnonzero(~occupied)
    if free.size < n:
        raise ValueError("not enough free slots")
    return free[:n].astype(np.int32)


@dataclass
class MigrationCase:
    """One synthetic migration: pool sizes, block tables, content seeds and tags."""
    cfg: str
    shape: KVShape
    lengths: np.ndarray
    req_blocks: np.ndarray          # blocks per request
    nb_src: int
    nb_dst: int
    src_bt: np.ndarray              # int32 [n]
    dst_bt: np.ndarray              # int32 [n]
    content_seed: int
    src_tag: int = 1
    dst_tag: int = 2
    variant: str = "shuffled"
    extra: dict = field(default_factory=dict)

    @property
    def n(self) -> int:
        return int(self.src_bt.size)


def migration_case(cfg: str, variant: str = "shuffled", scale: float = 1.0,
                   lengths: np.ndarray | None = None, shape: KVShape | None = None,
                   occupied_frac: float = 0.30, seed_offset: int = 0) -> MigrationCase:
    """The common generator of SURVEY §8(d): NB_src = ceil(1.1*n); sources = first n of
    a seeded permutation (shuffled) or 0..n-1 (sequential); the destination pool has a
    seeded 30 % of slots pre-occupied and takes the lowest free slots (A10).
    ``seed_offset`` shifts every seed of the config (len / slot / content; bench --seed)."""
    k = int(cfg[1]) + seed_offset
    shape = shape or SHAPES[cfg]
    lens = (request_lengths(cfg, scale, seed_offset) if lengths is None
            else np.asarray(lengths, np.int64))
    req_blocks = blocks_for_tokens(lens, shape.block_size)
    n = int(req_blocks.sum())
    nb_src = max(1, math.ceil(1.1 * n))
    if variant == "sequential":
        nb_dst = max(1, n)
        src_bt = np.arange(n, dtype=np.int32)
        dst_bt = np.arange(n, dtype=np.int32)
    elif variant == "shuffled":
        nb_dst = max(1, math.ceil(1.1 * n / (1.0 - occupied_frac)))
        src_bt = shuffled_slots(n, nb_src, 2000 + k)
        occ = occupied_mask(nb_dst, occupied_frac, 2000 + k + 100)
        dst_bt = lowest_free(occ, n)
    else:
        raise KeyError(variant)
    return MigrationCase(cfg, shape, lens, req_blocks, nb_src, nb_dst, src_bt, dst_bt,
                         content_seed=3000 + k, variant=variant)


def live_mask_after_free(n_slots: int, req_blocks: np.ndarray, free_frac: float,
                         seed: int):
    """C5 compaction input: requests laid out in a pool slot by slot (seeded shuffled
    placement), then a seeded `free_frac` of requests freed.  Returns (live mask,
    per-request slot lists of the surviving requests)."""
    rng = np.random.default_rng(seed)
    total = int(req_blocks.sum())
    if total > n_slots:
        raise ValueError("pool too small")
    slots = rng.permutation(n_slots)[:total].astype(np.int32)
    tables, pos = [], 0
    for b in req_blocks:
        tables.append(slots[pos:pos + int(b)])
        pos += int(b)
    keep = rng.random(len(req_blocks)) >= free_frac
    live = np.zeros(n_slots, dtype=np.uint8)
    kept = []
    for t, kp in zip(tables, keep):
        if kp:
            live[t] = 1
            kept.append(t)
    return live, kept


def skewed_placement(n_req: int, n_gpus: int, seed: int,
                     weights=(.25, .20, .15, .12, .10, .08, .06, .04)) -> np.ndarray:
    """C5's skewed request placement over GPUs; weights renormalised to
    the first n_gpus entries."""
    w = np.asarray(weights[:n_gpus], dtype=np.float64)
    w = w / w.sum()
    rng = np.random.default_rng(seed)
    return rng.choice(n_gpus, size=n_req, p=w).astype(np.int32)


def hash_shuffle_dest(n_req: int, n_gpus: int, seed: int) -> np.ndarray:
    """The uniform all-to-all shuffle: request r moves to GPU splitmix64(seed ^ r) mod G."""
    return np.array([splitmix64_scalar((seed ^ r) & MASK64) % n_gpus
                     for r in range(n_req)], dtype=np.int32)
