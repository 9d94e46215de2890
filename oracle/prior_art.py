"""The paper's own flush design (prior art), simulated on the CPU as printed.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py): pins the comparison kernels of §8(f) N3
(csrc/prior_art.cu) to the paper's text.  Pure Python loops over small bundles; no code is
shared with the CUDA path.

* mu(eta) — Eq. (1), P@31247-31646, under reading S21: the smallest
  i <= 8 with lambda(eta, i) >= 2^eta, else 2^eta - lambda(eta, 8) + 8, where
  lambda(eta, i) = i*C(eta+1, 2) - sum_{j=1..i} (14-j)(j-1)/2 + i.
* x_shuffle_bundle — Alg. 3 lines 1-10 (P@24850-26135, Fig. 3 P@28428-30196) for one bundle
  of 2^eta lanes, in the order the text and Fig. 3 describe (reading R23: own message into the
  cache Gamma, then eta rounds of shuffle_xor(2^(eta-j)) + compare) or as the listing prints
  it (compare, then shuffle; the last received message is not compared).
  Messages are (obj, t); "newer" compares t (the paper's rule; the CUDA comparison kernel
  compares the (t, seq) key of reading R7, which is the same order for distinct t).
* t_table_write — lines 11-13: repeat mu(eta) times, every lane whose message is newer than
  T[o][bundle] writes it.  Same-address writes of one round resolve to the highest lane
  (what a warp store does on NVIDIA GPUs); the round structure is what the paper relies on.
* collect — GPU_Collect (P@23216-23566): per object the newest message over the bundles.
"""
from __future__ import annotations

from math import comb


def lam(eta: int, i: int) -> float:
    return i * comb(eta + 1, 2) - sum((14 - j) * (j - 1) / 2 for j in range(1, i + 1)) + i


def mu(eta: int) -> int:
    for i in range(1, 9):
        if lam(eta, i) >= 2 ** eta:
            return i
    return int(2 ** eta - lam(eta, 8) + 8)


def _cache_step(cache, cur):
    """Every lane looks its current message's object up in its cache: absent -> add; cached
    one older -> replace; otherwise continue with the cached (newer) message."""
    nxt = list(cur)
    for lane, m in enumerate(cur):
        if m is None:
            continue
        hit = next((c for c in cache[lane] if c[0] == m[0]), None)
        if hit is None:
            cache[lane].append(m)
        elif hit[1] < m[1]:
            cache[lane][cache[lane].index(hit)] = m
        else:
            nxt[lane] = hit
    return nxt


def x_shuffle_bundle(msgs, eta: int, trace=None, order: str = "text"):
    """msgs: list of 2^eta (obj, t) tuples (None = no message).  Returns the message each lane
    holds after the cache-and-shuffle step.  trace (optional list) receives the lanes' caches
    (lists of (obj, t)) after every compare step.

    order="text" (reading R23; P@28428-30196 and Fig. 3): each lane adds its own
      message, then eta times: shuffle_xor(2^(eta-j)), compare with the cache.
    order="listing" (Alg. 3 lines 4-10 as printed): eta times: compare, then shuffle; the
      message received by the last shuffle is not compared.
    Only "text" reproduces the figure's outcome (a4 and a5 both survive); under "listing" a4
    always meets the cached a5 (see tests/test_prior_art.py)."""
    n = 2 ** eta
    assert len(msgs) == n
    cache = [[] for _ in range(n)]  # Gamma per lane
    cur = list(msgs)
    if order == "text":
        cur = _cache_step(cache, cur)  # "each thread first adds its message to its cache"
        for j in range(1, eta + 1):
            mask = 2 ** (eta - j)
            cur = [cur[lane ^ mask] for lane in range(n)]  # butterfly shuffle
            cur = _cache_step(cache, cur)
            if trace is not None:
                trace.append([list(c) for c in cache])
        return cur
    for j in range(1, eta + 1):
        cur = _cache_step(cache, cur)
        if trace is not None:
            trace.append([list(c) for c in cache])
        mask = 2 ** (eta - j)
        cur = [cur[lane ^ mask] for lane in range(n)]
    return cur


def t_table_write(table: dict, bundle: int, final_msgs, eta: int):
    """Lines 11-13: mu(eta) rounds of 'if T[o][bundle].t < m.t then write'; in each round the
    writers of one address resolve to the highest lane."""
    for _ in range(mu(eta)):
        writes = {}
        for lane, m in enumerate(final_msgs):
            if m is None:
                continue
            cur = table.get((m[0], bundle))
            if cur is None or cur[1] < m[1]:
                writes[(m[0], bundle)] = m  # later lanes overwrite earlier ones
        table.update(writes)
    return table


def collect(table: dict):
    """GPU_Collect: per object, the newest message over all bundles."""
    best = {}
    for (o, _b), m in table.items():
        if o not in best or best[o][1] < m[1]:
            best[o] = m
    return best


def clean(buckets, eta: int):
    """Alg. 2 steps 3-4 over a list of buckets (each a list of (obj, t), processed from its
    last message to its first, one thread per bucket): the per-object newest message found."""
    n = 2 ** eta
    table = {}
    depth = max((len(b) for b in buckets), default=0)
    for b0 in range(0, len(buckets), n):
        bundle = b0 // n
        lanes = buckets[b0:b0 + n] + [[]] * (n - len(buckets[b0:b0 + n]))
        for i in range(depth - 1, -1, -1):
            msgs = [lane[i] if i < len(lane) else None for lane in lanes]
            t_table_write(table, bundle, x_shuffle_bundle(msgs, eta), eta)
    return collect(table)
