"""Pins for the CPU oracle (oracle/ac_oracle.c) against what the paper and the
mathematics fix -- never against the oracle itself or the CUDA path.

* the worked example printed in PAPER.md Section II (tests/golden/ushers.txt)
* the definitions: trie states <-> pattern prefixes, f(s) = longest proper
  suffix that is a prefix, delta(s,a) = longest suffix of str(s)+a that is a
  prefix, output(s) = patterns that are suffixes of str(s)
* brute-force substring search on tiny random inputs (tests/brute.py)
* closed forms: a^n with {a^1..a^K}; all |A|^k strings; no pattern byte;
  a single pattern's overlapping occurrences
* invariants: count = sum of per-pattern occurrence counts, chunking
  invariance, permutation equivariance, shift under prefixing, concatenation
  with a separator byte
"""
from __future__ import annotations

import itertools
import random
from pathlib import Path

import numpy as np
import pytest

from brute import brute_matches
from oracle import Oracle

GOLDEN = Path(__file__).resolve().parent / "golden"


def _pairs(ends, pids):
    return list(zip(ends.tolist(), pids.tolist()))


def _parse_golden(path):
    rec = {"goto": [], "delta": [], "output": {}, "match": []}
    for line in path.read_text().splitlines():
        if not line or line.startswith("#"):
            continue
        k, *v = line.split()
        if k == "patterns":
            rec["patterns"] = [x.encode() for x in v]
        elif k == "text":
            rec["text"] = v[0].encode()
        elif k in ("goto", "delta"):
            rec[k].append((int(v[0]), ord(v[1]), None if v[2] == "fail" else int(v[2])))
        elif k == "fail":
            rec["fail"] = [int(x) for x in v]
        elif k == "output":
            rec["output"][int(v[0])] = v[1:]
        elif k == "match":
            rec["match"].append((int(v[0]), v[1].encode()))
    return rec


# ---------------------------------------------------------------------------
# P1: the printed worked example
# ---------------------------------------------------------------------------
def test_worked_example_goto_fail_output():
    g = _parse_golden(GOLDEN / "ushers.txt")
    o = Oracle(g["patterns"])
    assert o.num_states == 10
    for s, a, t in g["goto"]:
        assert o.goto(s, a) == t, (s, chr(a))
    assert [o.fail(s) for s in range(10)] == g["fail"]
    names = {p: i for i, p in enumerate(g["patterns"])}
    for s in range(10):
        want = sorted(names[w.encode()] for w in g["output"].get(s, []))
        assert o.output(s) == want, s
    for s, a, t in g["delta"]:
        assert o.delta(s, a) == t


def test_worked_example_matches():
    g = _parse_golden(GOLDEN / "ushers.txt")
    o = Oracle(g["patterns"])
    ends, pids = o.match(g["text"])
    names = {p: i for i, p in enumerate(g["patterns"])}
    assert _pairs(ends, pids) == [(e, names[w]) for e, w in g["match"]]
    # north_star's start form: she@1, he@2, hers@2
    starts = [e - len(g["patterns"][p]) + 1 for e, p in _pairs(ends, pids)]
    assert list(zip(starts, [g["patterns"][p] for p in pids.tolist()])) == [(1, b"she"), (2, b"he"), (2, b"hers")]


def test_root_is_total():
    o = Oracle([b"he", b"she", b"his", b"hers", b"\x00\xff"])
    for a in range(256):
        assert o.goto(0, a) is not None  # P:51 g(0,sigma) != fail


def test_empty_pattern_rejected():
    with pytest.raises(ValueError):
        Oracle([b"ab", b""])


# ---------------------------------------------------------------------------
# the definitions of g, f, delta and output, checked from pattern prefixes
# ---------------------------------------------------------------------------
def _state_strings(o: Oracle, alphabet):
    strs = {0: b""}
    frontier = [0]
    while frontier:
        nxt = []
        for s in frontier:
            for a in alphabet:
                t = o.goto(s, a)
                if t is None or (s == 0 and t == 0):
                    continue
                assert t not in strs
                strs[t] = strs[s] + bytes([a])
                nxt.append(t)
        frontier = nxt
    return strs


@pytest.mark.parametrize("seed", range(60))
def test_functions_match_their_definitions(seed):
    rng = random.Random(seed)
    A = rng.randint(1, 4)
    alphabet = list(range(97, 97 + A))
    pats = [bytes(rng.choice(alphabet) for _ in range(rng.randint(1, 6))) for _ in range(rng.randint(1, 8))]
    o = Oracle(pats)
    strs = _state_strings(o, alphabet)
    prefixes = {p[:i] for p in pats for i in range(len(p) + 1)}
    assert set(strs.values()) == prefixes and len(strs) == o.num_states
    by_str = {v: k for k, v in strs.items()}
    for s, w in strs.items():
        assert o.depth(s) == len(w)  # depth = length of the state's string (trie level)
        if s:
            suf = next(w[i:] for i in range(1, len(w) + 1) if w[i:] in prefixes)
            assert o.fail(s) == by_str[suf]
        assert o.output(s) == sorted(i for i, p in enumerate(pats) if w.endswith(p))
        for a in alphabet + [0x7A + 1]:
            wa = w + bytes([a])
            suf = next(wa[i:] for i in range(len(wa) + 1) if wa[i:] in prefixes)
            assert o.delta(s, a) == by_str[suf]


# ---------------------------------------------------------------------------
# P3: brute force on tiny random inputs
# ---------------------------------------------------------------------------
def _tiny_case(rng):
    A = rng.randint(1, 4)
    alphabet = list(range(97, 97 + A)) if rng.random() < 0.8 else [0, 255, 1, 128][:A]
    pats = [bytes(rng.choice(alphabet) for _ in range(rng.randint(1, 6))) for _ in range(rng.randint(1, 8))]
    text = bytes(rng.choice(alphabet + [ord("z")]) for _ in range(rng.randint(0, 256)))
    return pats, text


def test_brute_force_random():
    rng = random.Random(1234)
    for _ in range(3000):
        pats, text = _tiny_case(rng)
        o = Oracle(pats)
        assert _pairs(*o.match(text)) == brute_matches(text, pats)


def test_brute_force_chunked_and_windows():
    rng = random.Random(99)
    for _ in range(800):
        pats, text = _tiny_case(rng)
        o = Oracle(pats)
        want = brute_matches(text, pats)
        chunk = rng.randint(1, 40)
        assert _pairs(*o.match_chunked(text, chunk)) == want
        lo = rng.randint(0, len(text))
        hi = rng.randint(lo, len(text))
        base = rng.randint(0, 1 << 40)
        got = _pairs(*o.match_window(text, lo, hi, base=base))
        exp = [(e + base, p) for e, p in want if lo <= e - len(pats[p]) + 1 < hi]
        assert got == exp


# ---------------------------------------------------------------------------
# P4: closed forms
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("n,K", [(0, 3), (1, 5), (7, 7), (100, 1), (1000, 32), (4096, 17)])
def test_closed_form_runs(n, K):
    pats = [b"a" * k for k in range(1, K + 1)]
    o = Oracle(pats)
    ends, pids = o.match(b"a" * n)
    m = min(n, K)
    assert ends.size == (K * n - K * (K - 1) // 2 if n >= K else n * (n + 1) // 2)
    want = [(s + p, p) for s in range(n) for p in range(K) if s + p < n]
    assert _pairs(ends, pids) == want
    assert m == 0 or ends.size > 0


@pytest.mark.parametrize("A,k", [(2, 3), (3, 4), (4, 5), (4, 1)])
def test_closed_form_all_kmers(A, k):
    alphabet = bytes(range(65, 65 + A))
    pats = [bytes(t) for t in itertools.product(alphabet, repeat=k)]  # lexicographic ids
    rng = np.random.default_rng(A * 100 + k)
    digits = rng.integers(0, A, size=3000)
    text = bytes(alphabet[d] for d in digits)
    ends, pids = o_match = Oracle(pats).match(text)
    assert ends.size == len(text) - k + 1
    for i, (e, p) in enumerate(zip(ends.tolist(), pids.tolist())):
        assert e == i + k - 1
        val = 0
        for d in digits[i:i + k]:
            val = val * A + int(d)
        assert p == val
    del o_match


def test_closed_form_no_pattern_bytes():
    o = Oracle([b"xyz", b"q", b"\x00\x01"])
    assert o.count(bytes(range(32, 100)).replace(b"q", b"").replace(b"x", b"") * 50) == 0


@pytest.mark.parametrize("p,t,c", [(b"aa", b"aaaa", 3), (b"aba", b"ababa", 2), (b"abc", b"abcabcab", 2),
                                   (b"\x00", b"\x00\x01\x00", 2), (b"zz", b"z", 0)])
def test_closed_form_single_pattern(p, t, c):
    assert Oracle([p]).count(t) == c


# ---------------------------------------------------------------------------
# P5: invariants
# ---------------------------------------------------------------------------
def _occ(text: bytes, p: bytes) -> int:
    c, i = 0, text.find(p)
    while i >= 0:
        c += 1
        i = text.find(p, i + 1)
    return c


def test_count_is_sum_of_occurrences():
    import synth
    w = synth.make("c1", n=1 << 16)
    o = Oracle(w.patterns)
    text = w.text.tobytes()
    assert o.count(text) == sum(_occ(text, p) for p in w.patterns)


@pytest.mark.parametrize("chunk", [1, 2, 15, 16, 17, 333, 4096])
def test_chunking_invariance(chunk):
    import synth
    w = synth.make("c2", n=1 << 15, n_patterns=200)
    o = Oracle(w.patterns)
    e0, p0 = o.match(w.text)
    e1, p1 = o.match_chunked(w.text, chunk)
    assert np.array_equal(e0, e1) and np.array_equal(p0, p1)


def test_permutation_equivariance():
    rng = random.Random(5)
    for _ in range(200):
        pats, text = _tiny_case(rng)
        perm = list(range(len(pats)))
        rng.shuffle(perm)  # new id j holds old pattern perm[j]
        a = set(_pairs(*Oracle(pats).match(text)))
        b = set((e, perm[p]) for e, p in _pairs(*Oracle([pats[j] for j in perm]).match(text)))
        assert a == b


def test_prefix_shift_and_concatenation():
    rng = random.Random(6)
    for _ in range(200):
        pats, t1 = _tiny_case(rng)
        _, t2 = _tiny_case(rng)
        o = Oracle(pats)
        sep = b"#"  # not in any pattern alphabet
        k = rng.randint(0, 9)
        a = _pairs(*o.match(t1))
        assert _pairs(*o.match(sep * k + t1)) == [(e + k, p) for e, p in a]
        b = _pairs(*o.match(t2))
        joined = _pairs(*o.match(t1 + sep + t2))
        assert joined == a + [(e + len(t1) + 1, p) for e, p in b]


def test_duplicate_and_nested_patterns():
    pats = [b"ab", b"ab", b"b", b"abab", b"bab"]
    text = b"xababab"
    o = Oracle(pats)
    assert _pairs(*o.match(text)) == brute_matches(text, pats)
    assert o.count(text) == 3 * 2 + 3 + 2 + 2


def test_all_byte_values():
    rng = np.random.default_rng(7)
    text = rng.integers(0, 256, size=5000, dtype=np.uint8).tobytes()
    pats = [bytes([b]) for b in range(256)] + [text[100:104], text[4000:4010], b"\x00\x00"]
    o = Oracle(pats)
    assert _pairs(*o.match(text)) == brute_matches(text, pats)


# ---------------------------------------------------------------------------
# Whole-text runners used by the full-size GPU parity tests: the parallel
# window runner and the multiset digest, pinned to brute force
# ---------------------------------------------------------------------------
_M64 = (1 << 64) - 1


def _mix64(x: int) -> int:
    """splitmix64 (Steele, Lea, Flood 2014), written out independently."""
    z = (x + 0x9E3779B97F4A7C15) & _M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _M64
    return z ^ (z >> 31)


def test_mix64_known_values():
    # splitmix64 stream seeded with 0: the published first outputs
    assert _mix64(0) == 0xE220A8397B1DCDAF
    assert _mix64(0x9E3779B97F4A7C15) == 0x6E789E6AA1B965F4


@pytest.mark.parametrize("seed", range(200))
def test_digest_window_against_brute_force(seed):
    rng = random.Random(7000 + seed)
    A = rng.randint(1, 4)
    alphabet = list(range(97, 97 + A))
    pats = [bytes(rng.choice(alphabet) for _ in range(rng.randint(1, 6))) for _ in range(rng.randint(1, 8))]
    text = bytes(rng.choice(alphabet) for _ in range(rng.randint(0, 200)))
    lo = rng.randint(0, len(text))
    hi = rng.randint(lo, len(text) + 3)
    base = rng.choice([0, 1, 12345, 1 << 33])
    o = Oracle(pats)
    want = [(e - len(pats[p]) + 1, p) for e, p in brute_matches(text, pats)]
    want = [(st, p) for st, p in want if lo <= st < min(hi, len(text))]
    hs = [_mix64(((base + st) << 24) | p) for st, p in want]
    sm, x = 0, 0
    for h in hs:
        sm = (sm + h) & _M64
        x ^= h
    assert o.digest_window(text, lo, hi, base=base) == (len(want), sm, x)


@pytest.mark.parametrize("seed", range(40))
def test_parallel_runners_against_brute_force(seed):
    rng = random.Random(9100 + seed)
    A = rng.randint(1, 3)
    alphabet = list(range(97, 97 + A))
    pats = [bytes(rng.choice(alphabet) for _ in range(rng.randint(1, 7))) for _ in range(rng.randint(1, 10))]
    text = bytes(rng.choice(alphabet) for _ in range(rng.randint(0, 3000)))
    o = Oracle(pats)
    # tiny windows so the 3000-byte text is split many times across threads
    o._windows = lambda n, threads, min_window=37: Oracle._windows(o, n, 5, min_window)
    want = brute_matches(text, pats)
    ends, pids = o.match_parallel(text)
    assert _pairs(ends, pids) == want
    hs = [_mix64(((e - len(pats[p]) + 1) << 24) | p) for e, p in want]
    sm, x = 0, 0
    for h in hs:
        sm = (sm + h) & _M64
        x ^= h
    assert o.digest_parallel(text) == (len(want), sm, x)


def test_canonical_sort_is_reentrant():
    # many threads sorting different dictionaries' lists at once must each
    # get their own canonical order (the comparator keeps no shared state)
    from concurrent.futures import ThreadPoolExecutor
    cases = []
    for seed in range(16):
        rng = random.Random(seed)
        pats = [bytes(rng.choice(b"ab") for _ in range(rng.randint(1, 9))) for _ in range(6)]
        text = bytes(rng.choice(b"ab") for _ in range(20000))
        cases.append((Oracle(pats), text, brute_matches(text, pats)))

    def run(c):
        o, text, want = c
        ends, pids = o.match(text)
        return _pairs(ends, pids) == want

    with ThreadPoolExecutor(8) as ex:
        assert all(ex.map(run, cases * 2))


# ---------------------------------------------------------------------------
# P6: the walk is O(n): one goto transition per symbol, and at most as
# many failure transitions (AC'75: each failure move lowers the depth, each
# goto move raises it by at most one)
# ---------------------------------------------------------------------------
def test_transitions_worked_example():
    # "ushers": g(5,'r') = fail -> f(5) = 2 is the only failure move
    o = Oracle([b"he", b"she", b"his", b"hers"])
    assert o.transitions(b"ushers") == (6, 1)


@pytest.mark.parametrize("seed", range(80))
def test_transitions_linear(seed):
    rng = random.Random(31000 + seed)
    A = rng.randint(1, 4)
    alphabet = list(range(97, 97 + A))
    pats = [bytes(rng.choice(alphabet) for _ in range(rng.randint(1, 7))) for _ in range(rng.randint(1, 9))]
    text = bytes(rng.choice(alphabet) for _ in range(rng.randint(0, 500)))
    o = Oracle(pats)
    gotos, fails = o.transitions(text)
    assert gotos == len(text) and fails <= gotos


def test_transitions_closed_forms():
    # a^n with {a^1..a^K}: the walk climbs to depth K, then every further 'a'
    # is one failure move (a^K -> a^(K-1)) and one goto move: n - K failures
    K, n = 5, 1000
    o = Oracle([b"a" * k for k in range(1, K + 1)])
    assert o.transitions(b"a" * n) == (n, n - K)
    # no pattern byte in the text: the root loops, no failure move
    assert Oracle([b"xyz"]).transitions(b"abc" * 50) == (150, 0)
