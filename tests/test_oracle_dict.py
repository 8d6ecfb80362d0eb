"""Pins of the oracle's text-to-integer dictionaries (§III-F;
reading R11: id = rank in byte-lexicographic order) and of the fact-scan oracle
 against invariants, Python's own bytes ordering and an
independent cube-building path.  CPU only."""
import bisect

import numpy as np

import oracle
import synth


def test_dict_bijection_order_roundtrip():
    keys = synth.random_keys(3000, seed=5, min_len=0, max_len=12, alphabet=b"ab\x00\xffz ")
    d = oracle.Dict(keys)
    distinct = sorted(set(keys))                      # Python bytes order == memcmp, shorter prefix first
    assert len(d) == len(distinct)
    ids = d.translate(keys)
    for k, i in zip(keys, ids):
        assert distinct[i] == k                        # id = rank
    for i, k in enumerate(distinct):
        assert d.lookup(i) == k                        # lookup(translate(s)) = s
        assert d.translate([k])[0] == i                # translate(lookup(i)) = i
    assert sorted(set(ids.tolist())) == list(range(len(distinct)))


def test_dict_near_misses_and_empty_key():
    members = ["CA", "CAL", "NY", "", "a b", "2001-01-01"]
    d = oracle.Dict(members)
    assert d.translate([""])[0] == 0                   # empty string is a valid key, sorts first
    probes = ["C", "ca", "CA ", " CA", "CAL\x00", "NY\x00", "2001-01-1", "2001-01-01 ", "a  b", "b"]
    assert (d.translate(probes) == -1).all()
    assert d.translate(["CA", "CAL"]).tolist() == [2, 3]   # "" < "2001-01-01" < "CA" < "CAL"


def test_dict_permutation_and_duplicate_invariance():
    keys = synth.random_keys(500, seed=9, max_len=6, alphabet=b"xyz")
    d1 = oracle.Dict(keys)
    rng = np.random.default_rng(0)
    shuffled = [keys[i] for i in rng.permutation(len(keys))] + keys[:100]
    d2 = oracle.Dict(shuffled)
    assert len(d1) == len(d2)
    for i in range(len(d1)):
        assert d1.lookup(i) == d2.lookup(i)


def test_dict_bounds_match_bisect():
    members = synth.tpcds_dates()
    d = oracle.Dict(members)
    s = sorted(members)
    for probe in ["1997-12-31", "1998-01-01", "1999-06-15", "1999-06-15x", "2002-12-31", "2003-01-01",
                  "2000-02-30", ""]:
        assert d.bound(probe) == bisect.bisect_left(s, probe)
        assert d.bound(probe, upper=True) == bisect.bisect_right(s, probe)
    # ISO dates sort chronologically: id order is date order
    assert [d.lookup(i).decode() for i in range(len(members))] == members


def test_factscan_equals_cube_sum():
    """Independent path: fact scan over translated rows == SUM query on the cube built from them."""
    members = synth.tpcds_members()
    small = {k: v[:n] for (k, v), n in zip(members.items(), (40, 6, 5, 4))}
    cols, qty, cents = synth.tpcds_facts(20000, small)
    dicts = {c: oracle.Dict(m) for c, m in small.items()}
    order = list(small)                                 # d_date, s_store_id, i_class, ca_state
    ids = np.stack([dicts[c].translate([small[c][i] for i in cols[c]]) for c in order]).astype(np.int32)
    ext = tuple(len(small[c]) for c in order)
    cube_q = np.zeros(ext, dtype=np.int64)
    np.add.at(cube_q, tuple(ids), qty)
    cube_n = np.zeros(ext, dtype=np.int64)
    np.add.at(cube_n, tuple(ids), 1)
    rng = np.random.default_rng(1)
    boxes = synth.random_boxes(ext, 300, rng)
    s, c = oracle.factscan(ids, qty, boxes)
    rq = oracle.query(ext, boxes, np.full(300, oracle.SUM, np.int32), cube_q.astype(np.int32).ravel())
    rn = oracle.query(ext, boxes, np.full(300, oracle.SUM, np.int32), cube_n.astype(np.int32).ravel())
    assert np.array_equal(s, rq["i"])
    assert np.array_equal(c, rn["i"])
    # float data column
    cube_f = np.zeros(ext, dtype=np.float64)
    np.add.at(cube_f, tuple(ids), cents.astype(np.float64))
    sf, _ = oracle.factscan(ids, cents, boxes)
    rf = oracle.query(ext, boxes, np.full(300, oracle.SUM, np.int32), cube_f.astype(np.float32).ravel())
    assert np.array_equal(sf, rf["d"])                 # integer-valued cents: exact
