"""Pins of the prior-art simulation (oracle/prior_art.py: the paper's X-shuffle flush, Alg. 3 +
GPU_Collect) against what the paper prints and against brute force (-m "not gpu").

These pin the CPU side of §8(f) N3; tests/test_gpu_prior_art.py checks the CUDA comparison
kernels against it."""
import json
import random

from oracle import prior_art as pa

import synth


def test_mu_eq1_reading_s21():
    # P@31646: "2^eta = 16, 32, 64, 128 -> mu(eta) = 2, 4, 8, 16"; mu(8) = 80
    assert [pa.mu(e) for e in range(4, 9)] == [2, 4, 8, 16, 80]
    # the lambda values App. A.1 lists
    assert [pa.lam(4, i) for i in range(1, 5)] == [11, 16, 16, 12]
    assert pa.lam(5, 4) == 32 and pa.lam(6, 8) == 64 and pa.lam(7, 8) == 120 and pa.lam(8, 8) == 184


def _w5():
    d = json.load(open(synth.golden_path("w5_xshuffle.json")))
    return [tuple(x) for x in d["lanes"]], d["eta"]


def test_w5_fig3_printed_facts():
    """Fig. 3 (P@28428-30196): after the first shuffle (mask 1000) lane 0010's cache [a1]
    becomes [a5]; lane 1010 receives a1, keeps [a5] and sends a5 on; lane 0000 with [b0]
    receives a4 and caches [a4, b0]; at the end only a4 and a5 of object a remain and no
    object has more than mu(4) = 2 messages."""
    row, eta = _w5()
    assert row[0b0010] == ("a", 1) and row[0b1010] == ("a", 5)
    assert row[0b0000] == ("b", 0) and row[0b1000] == ("a", 4)
    trace = []
    fin = pa.x_shuffle_bundle(row, eta, trace)
    assert trace[0][0b0010] == [("a", 5)]
    assert trace[0][0b1010] == [("a", 5)]
    assert sorted(trace[0][0b0000]) == [("a", 4), ("b", 0)]
    assert sorted({m for m in fin if m[0] == "a"}) == [("a", 4), ("a", 5)]
    for o in {m[0] for m in row}:
        assert len({m for m in fin if m[0] == o}) <= pa.mu(eta)
        newest = max(m for m in row if m[0] == o)
        assert newest in fin  # the newest message of every object survives


def test_w5_listing_order_contradicts_the_figure():
    """As the listing prints it (compare, then shuffle; the last message not compared), a4
    travels 1000 -> 0000 -> 0100 -> 0110 and meets the a5 lane 0110 cached one round earlier,
    so a4 can never survive — the figure's outcome needs the text's order (reading R23)."""
    row, eta = _w5()
    fin = pa.x_shuffle_bundle(row, eta, order="listing")
    assert ("a", 4) not in fin and ("a", 5) in fin
    rng = random.Random(0)
    for _ in range(300):  # whatever the other lanes hold
        r = list(row)
        for lane in range(16):
            if lane not in (0b0000, 0b0010, 0b1000, 0b1010):
                r[lane] = (rng.choice("bcde"), rng.randrange(20))
        assert ("a", 4) not in pa.x_shuffle_bundle(r, eta, order="listing")


def test_app_a2_counterexample_listing_order():
    """under the listing's order this two-object eta=4 bundle leaves object 1
    with 3 distinct messages (14, 13, 11) > mu(4) = 2."""
    row = [(1, 14), (0, 15), (1, 2), (0, 5), (1, 1), (0, 0), (1, 13), (0, 7), (0, 3), (1, 9), (1, 12),
           (0, 8), (0, 6), (1, 11), (1, 4), (0, 10)]
    fin = pa.x_shuffle_bundle(row, 4, order="listing")
    assert sorted({m[1] for m in fin if m[0] == 1}) == [11, 13, 14]
    assert sorted({m[1] for m in pa.x_shuffle_bundle(row, 4) if m[0] == 1}) == [13, 14]


def test_single_object_bundles_keep_only_the_newest():
    rng = random.Random(1)
    for eta in (4, 5):
        for _ in range(400):
            ts = rng.sample(range(10_000), 2 ** eta)
            fin = pa.x_shuffle_bundle([(0, t) for t in ts], eta)
            assert set(fin) == {(0, max(ts))}


def test_mixed_bundles_break_the_mu_bound_and_the_write_loop():
    """Theorem 1's bound does not hold for bundles mixing objects (App. A.2, here under R23):
    object 0 keeps 3 > mu(4) messages, and mu(4) rounds of 'write if newer' with highest-lane
    arbitration install 854 instead of the newest 912 — the prior-art hazard the comparison
    kernel counts (objects_wrong)."""
    row = [(0, 433), (1, 162), (1, 601), (1, 943), (0, 836), (1, 782), (1, 909), (0, 802), (0, 44), (1, 296),
           (0, 854), (1, 145), (1, 832), (0, 912), (1, 889), (0, 586)]
    fin = pa.x_shuffle_bundle(row, 4)
    assert len({m for m in fin if m[0] == 0}) == 3 > pa.mu(4)
    table = pa.t_table_write({}, 0, fin, 4)
    assert table[(0, 0)] == (0, 854) and table[(1, 0)] == (1, 943)
    # and such bundles are common: three objects in 16 lanes exceed the bound readily
    worst = 0
    rng = random.Random(2)
    for _ in range(2000):
        ts = rng.sample(range(1, 1000), 16)
        r = list(zip([rng.randrange(3) for _ in range(16)], ts))
        f = pa.x_shuffle_bundle(r, 4)
        worst = max(worst, max(len({m for m in f if m[0] == o}) for o in range(3)))
    assert worst > pa.mu(4)


def test_clean_equals_brute_force_when_bundles_hold_one_object():
    """Alg. 2 steps 3-4 over buckets whose bundles are object-pure: the per-object newest."""
    rng = random.Random(3)
    buckets = []
    for b in range(64):
        o = b // 16  # bundles of 16 buckets share one object
        buckets.append([(o, rng.randrange(100_000)) for _ in range(rng.randrange(1, 9))])
    got = pa.clean(buckets, 4)
    want = {}
    for bk in buckets:
        for o, t in bk:
            want[o] = max(want.get(o, -1), t)
    assert {o: m[1] for o, m in got.items()} == want
