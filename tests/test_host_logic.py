"""Host-side logic of the product library, CPU only: block-cyclic shard geometry
(brute force against the definition), the fast division used by the kernels'
address generation, and the dictionary hash's host implementation."""
import os
import ctypes

import numpy as np
import pytest

import paper_conf_ipps_malikrse12_b200 as olap

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _owned(r, G, g, b):
    return (r // b) % G == g


def _local(r, G, b):
    return (r // (b * G)) * b + r % b


@pytest.mark.parametrize("n0", [1, 7, 64, 100, 2048])
@pytest.mark.parametrize("G,b", [(1, 1), (2, 1), (3, 2), (4, 4), (8, 1), (8, 16), (5, 3)])
def test_shard_local_rows_brute_force(n0, G, b):
    rng = np.random.default_rng(n0 * 131 + G * 7 + b)
    pairs = [(lo, hi) for lo in range(min(n0, 24)) for hi in range(lo, min(n0, 24))]
    pairs += [tuple(sorted(rng.integers(0, n0, size=2))) for _ in range(300)]
    for g in range(G):
        for lo, hi in pairs:
            lo, hi = int(lo), int(hi)
            owned = [r for r in range(lo, hi + 1) if _owned(r, G, g, b)]
            llo, lhi = olap.shard_local_rows(n0, (G, g, b), lo, hi)
            if not owned:
                assert llo > lhi
            else:
                loc = [_local(r, G, b) for r in owned]
                assert loc == list(range(loc[0], loc[-1] + 1))     # one contiguous local range
                assert (llo, lhi) == (loc[0], loc[-1])
    # every row owned by exactly one shard; local indices dense per shard
    for g in range(G):
        rows = [r for r in range(n0) if _owned(r, G, g, b)]
        assert [_local(r, G, b) for r in rows] == list(range(len(rows)))


def test_shard_local_rows_errors():
    with pytest.raises(olap.OlapError):
        olap.shard_local_rows(10, (2, 0, 1), 0, 10)
    with pytest.raises(olap.OlapError):
        olap.shard_local_rows(10, (2, 2, 1), 0, 3)
    assert olap.shard_local_rows(10, (2, 1, 1), 4, 3)[0] > olap.shard_local_rows(10, (2, 1, 1), 4, 3)[1]


def _fastdiv(d, n):
    n = np.ascontiguousarray(n, dtype=np.uint32)
    q = np.empty_like(n)
    assert olap.lib.olap_selftest_fastdiv(d, n.ctypes.data, n.size, q.ctypes.data) == 0
    return q


def test_fastdiv_exact():
    rng = np.random.default_rng(0)
    small = np.arange(0, 1 << 16, dtype=np.uint32)
    for d in list(range(1, 300)) + [1023, 1024, 1025, 4095, 65535, 65536]:
        assert np.array_equal(_fastdiv(d, small), small // d)
    big = np.concatenate([rng.integers(0, 1 << 31, size=20000, dtype=np.int64),
                          [(1 << 31) - 1, (1 << 31) - 2, 0, 1]]).astype(np.uint32)
    for d in list(rng.integers(1, 1 << 31, size=200)) + [(1 << 30) + 1, (1 << 31) - 1, 3, 7, 1 << 20]:
        d = int(d)
        assert np.array_equal(_fastdiv(d, big), big // d), d
        edge = np.array([k * d - 1 for k in range(1, 40) if k * d - 1 < (1 << 31)] +
                        [k * d for k in range(1, 40) if k * d < (1 << 31)], dtype=np.uint32)
        assert np.array_equal(_fastdiv(d, edge), edge // d), d


def _ref_hash(key: bytes) -> int:
    """The documented hash (common.cuh): fmix64(sum_j fmix64((j<<32|w_j)+K1) + len*K2) mod 2^64."""
    M = (1 << 64) - 1

    def fmix(k):
        k ^= k >> 33
        k = (k * 0xff51afd7ed558ccd) & M
        k ^= k >> 33
        k = (k * 0xc4ceb9fe1a85ec53) & M
        k ^= k >> 33
        return k

    s = 0
    for j in range(0, (len(key) + 3) // 4):
        w = int.from_bytes(key[4 * j:4 * j + 4].ljust(4, b"\0"), "little")
        s = (s + fmix((((j << 32) | w) + 0x9E3779B97F4A7C15) & M)) & M
    return fmix((s + len(key) * 0xD6E8FEB86659FD93) & M)


def test_dict_hash_host_matches_definition():
    for key in [b"", b"a", b"abcd", b"abcde", b"2001-01-01", bytes(range(256)), b"\0\0\0", b"\0\0\0\0"]:
        assert olap.lib.olap_selftest_hash(key, len(key)) == _ref_hash(key)
    # zero padding must not collide keys of different lengths
    assert olap.lib.olap_selftest_hash(b"ab", 2) != olap.lib.olap_selftest_hash(b"ab\0", 3)


def test_hier_convert_matches_oracle():
    """olap_hier_convert (host code in the product library) vs oracle.convert_range."""
    import oracle
    import synth
    rng = np.random.default_rng(21)
    hier_ids = [synth.date_hierarchy(), synth.random_hierarchy(50, 3, rng), [np.zeros(7, np.int32),
                                                                             np.zeros(7, np.int32),
                                                                             np.arange(7, dtype=np.int32)]]
    h = olap.Hierarchy(hier_ids)
    assert h.extents(2) == (1826, 50, 7) and h.extents(0)[0] == 5
    for target in (1, 2):
        ranges, levels = [], []
        for _ in range(200):
            q, lq = [], []
            for d in range(3):
                r = int(rng.integers(0, target + 1))
                n = int(hier_ids[d][r].max()) + 1
                a, b = sorted(rng.integers(0, n, size=2))
                if rng.random() < 0.05:
                    a, b = b + 1, a
                q.append((int(a), int(b)))
                lq.append(r)
            ranges.append(q)
            levels.append(lq)
        got = h.convert(ranges, levels, target)
        for qi in range(200):
            for d in range(3):
                want = oracle.convert_range(hier_ids[d], levels[qi][d], target, *ranges[qi][d])
                g = tuple(got[qi, d])
                if want[0] > want[1]:
                    assert g[0] > g[1]
                else:
                    assert g == want
    with pytest.raises(olap.OlapError):
        olap.Hierarchy([[np.array([0, 2, 2], np.int32), np.arange(3, dtype=np.int32)]])   # gap in ids
    with pytest.raises(olap.OlapError):
        h.convert([[(0, 9), (0, 1), (0, 1)]], [[0, 0, 0]], 2)                              # year 9 does not exist


def test_bench_scaling_modes():
    """bench.py's N>1 workloads (host logic): weak scaling grows the global cube and the global
    batch with N; C3 defaults to strong scaling (the fixed 32 GiB cube split N ways)."""
    import bench
    assert bench.scaled_workload("C2a", 4, "weak") == ((64, 16, 16, 16, 16, 256), 4096 * 4)
    assert bench.scaled_workload("C3", 8, "strong") == ((2048, 2048, 2048), 4096)
    assert bench.scaled_workload("C5", 2, "weak") == ((2048, 4096, 8192), 65536 * 2)
    assert bench.default_scaling("C3") == "strong" and bench.default_scaling("C2a") == "weak"


def test_bench_weak_scaling_keeps_per_query_work():
    """Weak scaling over N GPUs: the batch of N x 4,096 queries on the N-fold cube keeps the box
    sizes of the one-GPU recipe (the same phi draws give the same lengths), offsets span the global
    cube, so the bytes per GPU per step stay those of N = 1 and queries/s can grow N-fold."""
    import bench
    import synth
    base = synth.CONFIGS["C2a"]["extents"]
    ext, nq = bench.scaled_workload("C2a", 4, "weak")
    one = synth.config_queries("C2a", nq=nq, seed=99, extents=base)[0]
    weak = bench.batches("C2a", ext, nq, 1, 99 - 1000, size_extents=base)[0][0]
    assert np.array_equal(weak[:, :, 1] - weak[:, :, 0], one[:, :, 1] - one[:, :, 0])
    assert (weak[:, :, 0] >= 0).all() and (weak[:, :, 1] < np.array(ext)).all()
    assert weak[:, 0, 1].max() >= base[0]  # offsets reach beyond the one-GPU rows
    # block-cyclic shards (b = 1) own rows r = g mod N: each GPU's owned rows sum to ~1/N of them
    owned = [sum(len(range(lo + ((g - lo) % 4), hi + 1, 4)) for lo, hi in weak[:, 0]) for g in range(4)]
    total = int((weak[:, 0, 1] - weak[:, 0, 0] + 1).sum())
    assert sum(owned) == total and max(owned) <= 1.05 * total / 4


def test_bench_refuses_mismatched_world():
    """--gpus N under a launcher that started a different number of ranks is an error, never a
    silent 1-GPU run."""
    import subprocess
    import sys
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "1"],
                       capture_output=True, text=True, env=env, timeout=120)
    assert r.returncode != 0 and "WORLD_SIZE=1" in (r.stderr + r.stdout)


def test_column_mode_reciprocal_table():
    """cube.cu's kInv32 (column mode's division-free n / d, d <= 32) holds ceil(2^32 / d), and the
    multiply-high quotient is exact for every n < 2^27 it is used on (brute force at the edges)."""
    import os
    import re
    src = open(os.path.join(ROOT, "paper_conf_ipps_malikrse12_b200", "csrc", "cube.cu")).read()
    body = re.search(r"kInv32\[33\] = \{([^}]*)\}", src).group(1)
    tab = [int(x.strip().rstrip("ul")) for x in body.replace("\n", " ").split(",") if x.strip()]
    assert tab == [0] + [-(-(1 << 32) // d) for d in range(1, 33)]
    for d in range(1, 33):
        for n in list(range(0, 4096)) + [(1 << 27) - k for k in range(1, 4096)]:
            assert (n * tab[d]) >> 32 == n // d
