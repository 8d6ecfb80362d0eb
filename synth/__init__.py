"""synth — seeded synthetic inputs shared by the oracle tests, the GPU parity
tests and bench.py.

This module holds NONE of the method's arithmetic: it only draws cube cells,
query boxes, op codes, dictionary strings and fact rows.  Both sides (oracle/
and the CUDA path) consume what it produces; neither is imported here.

Recipes follow SURVEY.md §8(d) (the paper prints no workload; DESIGN.md
"Input recipe" states them):
  C1  4-D int32 32^4, 1,000 random boxes, per-dim (f,t) a sorted uniform pair.
  C2  6-D float32 2^28 cells (C2a (16,16,16,16,16,256), C2b (16,16,32,32,32,32)),
      target fraction phi log-uniform in [1e-4,1], l_d = max(1, round(n_d*phi^(1/6))).
  C3  3-D (2048,2048,2048), phi log-uniform in [1e-5, 1].
  C4  TPC-DS store_sales-shaped fact table with four text dimensions.
  C5  (1024*G, 4096, 8192) float32, small boxes of 4 KiB .. 4 MiB.

Cells use a counter-based generator (splitmix64 of seed and linear index) so
any cell can be recomputed anywhere; oracle/ and the CUDA fill kernel each
implement the same formula independently.
"""
from __future__ import annotations

import numpy as np

SEED_BASE = 0x5EED0000

SUM, COUNT, MIN, MAX, AVG = 0, 1, 2, 3, 4
GEN_UNIFORM, GEN_AFFINE = 1, 2

CONFIGS = {
    "C1": dict(extents=(32, 32, 32, 32), dtype=np.int32, nq=1000, seed=SEED_BASE + 0),
    "C2a": dict(extents=(16, 16, 16, 16, 16, 256), dtype=np.float32, nq=4096, seed=SEED_BASE + 1),
    "C2b": dict(extents=(16, 16, 32, 32, 32, 32), dtype=np.float32, nq=4096, seed=SEED_BASE + 1),
    "C3": dict(extents=(2048, 2048, 2048), dtype=np.float32, nq=4096, seed=SEED_BASE + 2),
    "C5": dict(extents=(1024, 4096, 8192), dtype=np.float32, nq=65536, seed=SEED_BASE + 4),
}

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def splitmix64(seed: int, idx) -> np.ndarray:
    """splitmix64(seed + (idx+1)*golden) for an array of indices (uint64 wraparound)."""
    idx = np.asarray(idx, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + (idx + np.uint64(1)) * np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def uniform_cells(ncells: int, dtype, seed: int, first: int = 0, chunk: int = 1 << 24) -> np.ndarray:
    """Counter-hash cells: int32 uniform in [-2^20, 2^20), float32 k*2^-24 in [0,1)."""
    dtype = np.dtype(dtype)
    out = np.empty(ncells, dtype=dtype)
    for a in range(0, ncells, chunk):
        b = min(ncells, a + chunk)
        z = splitmix64(seed, np.arange(first + a, first + b, dtype=np.uint64))
        if dtype == np.int32:
            out[a:b] = (z >> np.uint64(43)).astype(np.int64) - (1 << 20)
        else:
            out[a:b] = (z >> np.uint64(40)).astype(np.float32) * np.float32(1.0 / 16777216.0)
    return out


def affine_cells(extents, dtype, params) -> np.ndarray:
    """v(x) = c0 + sum_d c_d x_d on the full (small) grid, row-major."""
    grids = np.indices(extents, dtype=np.float64)
    v = np.full(tuple(extents), float(params[0]))
    for d in range(len(extents)):
        v = v + float(params[1 + d]) * grids[d]
    return v.astype(dtype).reshape(-1)


def cube(extents, dtype, gen=GEN_UNIFORM, seed=0, params=None) -> np.ndarray:
    n = int(np.prod(extents))
    if gen == GEN_UNIFORM:
        return uniform_cells(n, dtype, seed)
    return affine_cells(extents, dtype, params)


# ---------------------------------------------------------------- queries

def random_boxes(extents, nq: int, rng: np.random.Generator) -> np.ndarray:
    """C1 recipe: per dimension a sorted pair of uniform draws (inclusive)."""
    nd = len(extents)
    r = np.empty((nq, nd, 2), dtype=np.int64)
    for d, n in enumerate(extents):
        a = rng.integers(0, n, size=nq)
        b = rng.integers(0, n, size=nq)
        r[:, d, 0] = np.minimum(a, b)
        r[:, d, 1] = np.maximum(a, b)
    return r


def fraction_boxes(extents, nq: int, rng: np.random.Generator, phi_lo: float, phi_hi: float = 1.0,
                   size_extents=None):
    """C2/C3 recipe: phi log-uniform, l_d = max(1, round(n_d * phi^(1/N))), offsets uniform.
    `size_extents` (weak scaling over GPUs): box lengths from these (the one-GPU cube), offsets
    uniform over `extents` (the grown global cube), so every query reads what it would at N = 1."""
    nd = len(extents)
    sizes = extents if size_extents is None else size_extents
    phi = np.exp(rng.uniform(np.log(phi_lo), np.log(phi_hi), size=nq))
    r = np.empty((nq, nd, 2), dtype=np.int64)
    for d, n in enumerate(extents):
        ell = np.clip(np.rint(sizes[d] * phi ** (1.0 / nd)).astype(np.int64), 1, n)
        off = (rng.random(nq) * (n - ell + 1)).astype(np.int64)
        r[:, d, 0] = off
        r[:, d, 1] = off + ell - 1
    return r


def small_boxes(extents, nq: int, rng: np.random.Generator, cell_bytes: int = 4,
                bytes_lo: int = 4096, bytes_hi: int = 4 << 20):
    """C5 recipe: box bytes log-uniform in [4 KiB, 4 MiB], aspect = random simplex split of log2(cells)."""
    nd = len(extents)
    cells = np.exp(rng.uniform(np.log(bytes_lo / cell_bytes), np.log(bytes_hi / cell_bytes), size=nq))
    w = rng.dirichlet(np.ones(nd), size=nq)
    r = np.empty((nq, nd, 2), dtype=np.int64)
    for d, n in enumerate(extents):
        ell = np.clip(np.rint(cells ** w[:, d]).astype(np.int64), 1, n)
        off = (rng.random(nq) * (n - ell + 1)).astype(np.int64)
        r[:, d, 0] = off
        r[:, d, 1] = off + ell - 1
    return r


def ops_uniform(nq: int, rng: np.random.Generator) -> np.ndarray:
    return rng.integers(0, 5, size=nq).astype(np.int32)


def ops_mix(nq: int, rng: np.random.Generator) -> np.ndarray:
    """C2 mix: SUM 40%, MIN 20%, MAX 20%, AVG 10%, COUNT 10%."""
    return rng.choice(np.array([SUM, MIN, MAX, AVG, COUNT], dtype=np.int32), size=nq,
                      p=[0.4, 0.2, 0.2, 0.1, 0.1]).astype(np.int32)


def config_queries(name: str, nq: int | None = None, seed: int | None = None, extents=None, size_extents=None):
    """Boxes and ops of a config.  `size_extents`: weak scaling (see fraction_boxes); C5's boxes
    have absolute sizes already, C1's are uniform pairs."""
    cfg = CONFIGS[name]
    ext = tuple(extents) if extents is not None else cfg["extents"]
    nq = cfg["nq"] if nq is None else nq
    rng = np.random.default_rng(cfg["seed"] if seed is None else seed)
    if name == "C1":
        return random_boxes(ext, nq, rng), ops_uniform(nq, rng)
    if name in ("C2a", "C2b"):
        return fraction_boxes(ext, nq, rng, 1e-4, size_extents=size_extents), ops_mix(nq, rng)
    if name == "C3":
        return fraction_boxes(ext, nq, rng, 1e-5, size_extents=size_extents), ops_mix(nq, rng)
    if name == "C5":
        return small_boxes(ext, nq, rng), ops_mix(nq, rng)
    raise KeyError(name)


# ---------------------------------------------------------------- C4 (TPC-DS store_sales-shaped)

def tpcds_dates() -> list[str]:
    """d_date members: every day 1998-01-01 .. 2002-12-31 (1,826 values), ISO format."""
    import datetime as _dt
    d0 = _dt.date(1998, 1, 1)
    return [(d0 + _dt.timedelta(days=i)).isoformat() for i in range(1826)]


def tpcds_members(seed: int = SEED_BASE + 3) -> dict[str, list[str]]:
    """Member strings of the four text columns (cardinalities approximate TPC-DS; parameters)."""
    rng = np.random.default_rng(seed)
    alpha = np.frombuffer(b"ABCDEFGHIJKLMNOPQRSTUVWXYZ", dtype=np.uint8)
    stores = []
    for i in range(128):
        tail = bytes(rng.choice(alpha, size=8)).decode()
        stores.append(f"AAAAAAAA{tail}")               # 16-char s_store_id
    words = ["accessories", "athletic", "baseball", "bedding", "blinds/shades", "bracelets",
             "camcorders", "classical", "computers", "country", "decor", "dresses", "earings",
             "fiction", "fishing", "fragrances", "furniture", "glassware", "guns", "history",
             "infants", "jewelry boxes", "kids", "lighting", "maternity", "mens watches",
             "mystery", "newborn", "outdoor", "pants", "personal", "pop", "portable", "reference",
             "rock", "romance", "scanners", "school-uniforms", "self-help", "shirts", "sports",
             "stereo", "swimwear", "televisions", "tennis", "toddlers", "travel", "wallpaper",
             "womens watches", "audio"]
    classes = []
    for i in range(100):
        w = words[i % len(words)] + ("" if i < len(words) else f" {i // len(words)}")
        classes.append(w[:50])
    states = ["AK", "AL", "AR", "AZ", "CA", "CO", "CT", "DC", "DE", "FL", "GA", "HI", "IA", "ID", "IL",
              "IN", "KS", "KY", "LA", "MA", "MD", "ME", "MI", "MN", "MO", "MS", "MT", "NC", "ND", "NE",
              "NH", "NJ", "NM", "NV", "NY", "OH", "OK", "OR", "PA", "RI", "SC", "SD", "TN", "TX", "UT",
              "VA", "VT", "WA", "WI", "WV", "WY", "PR"]
    return {"d_date": tpcds_dates(), "s_store_id": stores, "i_class": classes, "ca_state": states}


def tpcds_facts(nrows: int, members: dict[str, list[str]], seed: int = SEED_BASE + 3):
    """store_sales-shaped rows: per text column a member index (strings are members[col][idx]),
    ss_quantity int32 in [1,100] and ss_net_paid float32 (whole cents / 100 -> stored as cents
    to stay exactly representable)."""
    rng = np.random.default_rng(seed + 1)
    cols = {c: rng.integers(0, len(m), size=nrows).astype(np.int64) for c, m in members.items()}
    qty = rng.integers(1, 101, size=nrows).astype(np.int32)
    cents = rng.integers(0, 1 << 14, size=nrows).astype(np.float32)
    return cols, qty, cents


def text_column(members: list[str], idx, chunk: int = 1 << 22):
    """A fact table's raw text column: row r holds the string members[idx[r]] (length-delimited
    bytes, the C-ABI key layout).  Returns (bytes uint8[...], offsets int64[n+1])."""
    idx = np.asarray(idx)
    enc = [m.encode() for m in members]
    lens = np.array([len(e) for e in enc], np.int64)
    width = max(int(lens.max()), 1)
    table = np.zeros((len(enc), width), np.uint8)
    for i, e in enumerate(enc):
        table[i, :len(e)] = np.frombuffer(e, np.uint8)
    rl = lens[idx]
    offs = np.zeros(len(idx) + 1, np.int64)
    np.cumsum(rl, out=offs[1:])
    out = np.empty(max(int(offs[-1]), 1), np.uint8)
    col = np.arange(width)
    for a in range(0, len(idx), chunk):
        b = min(len(idx), a + chunk)
        rows = table[idx[a:b]]
        out[offs[a]:offs[b]] = rows[col[None, :] < rl[a:b, None]]
    return out, offs


def tpcds_queries(nq: int, members: dict[str, list[str]], seed: int = SEED_BASE + 3):
    """Query strings: a d_date range (two dates), 0-3 equality predicates on store/class/state, op."""
    rng = np.random.default_rng(seed + 2)
    dates = members["d_date"]
    out = []
    for _ in range(nq):
        a, b = sorted(rng.integers(0, len(dates), size=2))
        q = {"d_date": (dates[a], dates[b])}
        for col in ("s_store_id", "i_class", "ca_state"):
            if rng.random() < 0.5:
                m = members[col]
                if rng.random() < 0.05:
                    q[col] = m[rng.integers(0, len(m))] + "?"       # a miss: not a member
                else:
                    q[col] = m[rng.integers(0, len(m))]
        q["op"] = int(rng.choice([SUM, COUNT, MIN, MAX, AVG]))
        out.append(q)
    return out


def random_keys(n: int, seed: int, min_len: int = 1, max_len: int = 24, alphabet: bytes | None = None):
    """n random byte-string keys (duplicates possible), for dictionary stress tests."""
    rng = np.random.default_rng(seed)
    lens = rng.integers(min_len, max_len + 1, size=n)
    if alphabet is None:
        raw = rng.integers(0, 256, size=int(lens.sum()), dtype=np.uint8)
    else:
        a = np.frombuffer(alphabet, dtype=np.uint8)
        raw = a[rng.integers(0, len(a), size=int(lens.sum()))]
    blob = raw.tobytes()
    offs = np.zeros(n + 1, dtype=np.int64)
    offs[1:] = np.cumsum(lens)
    return [blob[offs[i]:offs[i + 1]] for i in range(n)]


# ---------------------------------------------------------------- multi-resolution hierarchies (NEXT #3)

def date_hierarchy():
    """d_date members 1998-01-01 .. 2002-12-31 at levels year (0), month (1), day (2):
    finest-member -> level-id arrays (ids are ranks in time order)."""
    import datetime as _dt
    d0 = _dt.date(1998, 1, 1)
    days = [d0 + _dt.timedelta(days=i) for i in range(1826)]
    year = np.array([d.year - 1998 for d in days], dtype=np.int32)
    month = np.array([(d.year - 1998) * 12 + d.month - 1 for d in days], dtype=np.int32)
    return [year, month, np.arange(1826, dtype=np.int32)]


def random_hierarchy(n_finest: int, levels: int, rng: np.random.Generator):
    """A monotone hierarchy: level L-1 is the identity; each coarser level groups
    consecutive members of the next finer level into random-size blocks."""
    ids = [np.arange(n_finest, dtype=np.int32)]
    for _ in range(levels - 1):
        prev = ids[0]
        n_prev = int(prev.max()) + 1
        cuts = np.sort(rng.choice(np.arange(1, n_prev), size=max(0, min(n_prev - 1, n_prev // 3)), replace=False)) \
            if n_prev > 1 else np.zeros(0, dtype=np.int64)
        group = np.searchsorted(cuts, np.arange(n_prev), side="right").astype(np.int32)
        ids.insert(0, group[prev])
    return ids
