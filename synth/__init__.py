"""Seeded synthetic inputs for the Aho-Corasick scan (texts and dictionaries).

This module is shared by the oracle side (tests, cpu_baseline) and the CUDA
side (tests, bench) and therefore holds NONE of the method's arithmetic: no
automaton, no matching, no counting -- only random bytes with the shapes of
the paper's workloads ("input data sizes in the range of 50KB -
200MB and the numbers of patterns in the range of 100 - 20,000", patterns
"extracted" from the corpus) and of BASELINE.json's five configs.  The
recipes are stated in DESIGN.md section "Inputs".

Determinism: text is produced in 1 MiB blocks; block j draws from
PCG64(splitmix64(seed * 2^32 + j)), so any block can be regenerated on its
own, every consumer sees identical bytes, and no block shares a stream with
another seed's generator.  Seeds are 1000*cfg + 0 (text),
1000*cfg + 1 (patterns), 1000*cfg + 2 (vocabulary).
"""
from __future__ import annotations

import os
from concurrent.futures import ThreadPoolExecutor
from dataclasses import dataclass, field

import numpy as np

BLOCK = 1 << 20
MASK64 = (1 << 64) - 1


def splitmix64(x: int) -> int:
    """One splitmix64 output for a 64-bit input (seed derivation only)."""
    x = (x + 0x9E3779B97F4A7C15) & MASK64
    z = x
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def rng_for(seed: int, j: int = 0) -> np.random.Generator:
    """Stream j of seed: PCG64 seeded with splitmix64(seed * 2^32 + j).  (Round 1
    used seed ^ j, which made text block 1 of seed 1000c replay the pattern
    stream 1000c + 1 -- C3's second MiB then held its dictionary's own bytes,
    3x the planted matches and 200+ per chain, a hot spot the recipe does not
    call for.)"""
    return np.random.Generator(np.random.PCG64(splitmix64(((seed << 32) + j) & MASK64)))


def _blocks(n: int, seed: int, fill, block0: int = 0) -> np.ndarray:
    """Allocate n bytes and fill them block by block with fill(rng, view, j);
    the text starts at block ``block0`` of the (endless) seeded stream."""
    out = np.empty(n, dtype=np.uint8)

    def one(j):
        lo = j * BLOCK
        fill(rng_for(seed, block0 + j), out[lo:min(n, lo + BLOCK)], block0 + j)

    nb = (n + BLOCK - 1) // BLOCK
    if nb >= 8:  # blocks are independent: fill them on every host core
        with ThreadPoolExecutor(min(nb, os.cpu_count() or 1)) as ex:
            list(ex.map(one, range(nb)))
    else:
        for j in range(nb):
            one(j)
    return out


# ---------------------------------------------------------------------------
# C1: iid lowercase text, iid lowercase patterns
# ---------------------------------------------------------------------------
def text_lowercase(n: int, seed: int, block0: int = 0) -> np.ndarray:
    def fill(rng, v, j):
        v[:] = rng.integers(ord("a"), ord("z") + 1, size=v.size, dtype=np.uint8)
    return _blocks(n, seed, fill, block0)


def patterns_random(count: int, lmin: int, lmax: int, seed: int, alphabet: bytes) -> list[bytes]:
    rng = rng_for(seed)
    al = np.frombuffer(alphabet, dtype=np.uint8)
    lens = rng.integers(lmin, lmax + 1, size=count)
    return [al[rng.integers(0, al.size, size=int(L))].tobytes() for L in lens]


# ---------------------------------------------------------------------------
# C2: English-like text (Zipf over a seeded vocabulary), substring patterns
# ---------------------------------------------------------------------------
# relative English letter frequencies a..z (percent), for vocabulary letters
_EN_FREQ = np.array([8.2, 1.5, 2.8, 4.3, 12.7, 2.2, 2.0, 6.1, 7.0, 0.15, 0.77, 4.0, 2.4,
                     6.7, 7.5, 1.9, 0.095, 6.0, 6.3, 9.1, 2.8, 0.98, 2.4, 0.15, 2.0, 0.074])


@dataclass
class Vocabulary:
    flat: np.ndarray   # concatenated word bytes
    off: np.ndarray    # word w = flat[off[w]:off[w] + lens[w]]
    lens: np.ndarray
    cdf: np.ndarray    # Zipf(s=1) cumulative distribution over ranks


def english_vocabulary(seed: int, words: int = 20000, mean_len: float = 5.0, max_len: int = 20) -> Vocabulary:
    rng = rng_for(seed)
    lens = np.minimum(1 + np.floor(rng.exponential(mean_len, size=words)).astype(np.int64), max_len)
    p = _EN_FREQ / _EN_FREQ.sum()
    flat = (ord("a") + rng.choice(26, size=int(lens.sum()), p=p)).astype(np.uint8)
    off = np.concatenate([[0], np.cumsum(lens)[:-1]])
    w = 1.0 / np.arange(1, words + 1)
    cdf = np.cumsum(w / w.sum())
    cdf[-1] = 1.0
    return Vocabulary(flat, off, lens, cdf)


def text_english(n: int, seed: int, vocab: Vocabulary, punct: float = 0.05, words_per_line: int = 12,
                 block0: int = 0) -> np.ndarray:
    def fill(rng, v, j):
        pos = 0
        while pos < v.size:
            m = max(64, (v.size - pos) // 3)
            ids = np.searchsorted(vocab.cdf, rng.random(m), side="right")
            ids = np.minimum(ids, vocab.lens.size - 1)
            wl = vocab.lens[ids]
            has_p = rng.random(m) < punct
            pch = np.where(rng.random(m) < 0.5, ord(","), ord(".")).astype(np.uint8)
            sep = np.where(rng.random(m) < 1.0 / words_per_line, ord("\n"), ord(" ")).astype(np.uint8)
            tok = wl + has_p + 1
            starts = np.concatenate([[0], np.cumsum(tok)[:-1]])
            total = int(tok.sum())
            buf = np.empty(total, dtype=np.uint8)
            within = np.arange(int(wl.sum())) - np.repeat(np.cumsum(wl) - wl, wl)
            buf[np.repeat(starts, wl) + within] = vocab.flat[np.repeat(vocab.off[ids], wl) + within]
            buf[(starts + wl)[has_p]] = pch[has_p]
            buf[starts + wl + has_p] = sep
            take = min(total, v.size - pos)
            v[pos:pos + take] = buf[:take]
            pos += take
    return _blocks(n, seed, fill, block0)


def patterns_substrings(text: np.ndarray, count: int, lmin: int, lmax: int, seed: int) -> list[bytes]:
    """Patterns "extracted" from the text: substrings at seeded starts."""
    rng = rng_for(seed)
    lens = rng.integers(lmin, lmax + 1, size=count)
    starts = rng.integers(0, max(1, text.size - lmax), size=count)
    return [text[int(s):int(s) + int(L)].tobytes() for s, L in zip(starts, lens)]


# ---------------------------------------------------------------------------
# C3: Snort-like byte patterns over packet-payload text
# ---------------------------------------------------------------------------
def patterns_snort(count: int, seed: int, mean_extra: float = 11.0, lmin: int = 4, lmax: int = 64) -> list[bytes]:
    rng = rng_for(seed)
    lens = np.minimum(lmin + np.floor(rng.exponential(mean_extra, size=count)).astype(np.int64), lmax)
    printable = rng.random(count) < 0.7
    out = []
    for L, pr in zip(lens, printable):
        if pr:
            out.append(rng.integers(0x20, 0x7F, size=int(L), dtype=np.uint8).tobytes())
        else:
            out.append(rng.integers(0, 256, size=int(L), dtype=np.uint8).tobytes())
    return out


def text_payload(n: int, seed: int, patterns: list[bytes], chunk: int = 64,
                 p_printable: float = 0.60, p_planted: float = 0.02, block0: int = 0) -> np.ndarray:
    pat_flat = np.frombuffer(b"".join(patterns), dtype=np.uint8)
    pat_len = np.array([len(p) for p in patterns], dtype=np.int64)
    pat_off = np.concatenate([[0], np.cumsum(pat_len)[:-1]])

    def fill(rng, v, j):
        m = (v.size + chunk - 1) // chunk
        kind = rng.random(m)
        pr = rng.integers(0x20, 0x7F, size=m * chunk, dtype=np.uint8)
        un = rng.integers(0, 256, size=m * chunk, dtype=np.uint8)
        is_un = np.repeat((kind >= p_printable) & (kind < 1.0 - p_planted), chunk)
        buf = np.where(is_un, un, pr)
        planted = np.nonzero(kind >= 1.0 - p_planted)[0]
        if planted.size and len(patterns):
            pid = rng.integers(0, len(patterns), size=planted.size)
            L = np.minimum(pat_len[pid], chunk)
            off = (rng.random(planted.size) * (chunk - L + 1)).astype(np.int64)
            within = np.arange(int(L.sum())) - np.repeat(np.cumsum(L) - L, L)
            dst = np.repeat(planted * chunk + off, L) + within
            buf[dst] = pat_flat[np.repeat(pat_off[pid], L) + within]
        v[:] = buf[:v.size]
    return _blocks(n, seed, fill, block0)


# ---------------------------------------------------------------------------
# C4: DNA text with 'N' runs, k-mer patterns
# ---------------------------------------------------------------------------
_ACGT = np.frombuffer(b"ACGT", dtype=np.uint8)


def text_dna(n: int, seed: int, p_n_run: float = 1e-4, max_run: int = 100, block0: int = 0) -> np.ndarray:
    def fill(rng, v, j):
        v[:] = _ACGT[rng.integers(0, 4, size=v.size, dtype=np.uint8)]
        k = rng.binomial(v.size, p_n_run)
        if k:
            st = rng.integers(0, v.size, size=k)
            L = rng.integers(1, max_run + 1, size=k)
            within = np.arange(int(L.sum())) - np.repeat(np.cumsum(L) - L, L)
            idx = np.repeat(st, L) + within
            v[idx[idx < v.size]] = ord("N")
    return _blocks(n, seed, fill, block0)


def patterns_kmers(text: np.ndarray, count: int, seed: int, lmin: int = 20, lmax: int = 32,
                   frac_from_text: float = 0.5) -> list[bytes]:
    rng = rng_for(seed)
    lens = rng.integers(lmin, lmax + 1, size=count)
    from_text = rng.random(count) < frac_from_text
    starts = rng.integers(0, max(1, text.size - lmax), size=count)
    out = []
    for L, ft, s in zip(lens, from_text, starts):
        if ft:
            # sample a window free of 'N' (reads with N are not k-mer queries)
            s = int(s)
            for _ in range(64):
                w = text[s:s + int(L)]
                if not (w == ord("N")).any():
                    break
                s = int(rng.integers(0, max(1, text.size - lmax)))
            out.append(w.tobytes())
        else:
            out.append(_ACGT[rng.integers(0, 4, size=int(L))].tobytes())
    return out


# ---------------------------------------------------------------------------
# C5 adversarial families
# ---------------------------------------------------------------------------
def text_repeat(n: int, unit: bytes) -> np.ndarray:
    # one n-byte allocation filled by doubling copies (C5 texts reach 16 GiB;
    # np.resize of a short unit concatenates n / len(unit) views)
    u = np.frombuffer(unit, dtype=np.uint8)
    out = np.empty(n, dtype=np.uint8)
    k = min(n, u.size)
    out[:k] = u[:k]
    while k < n:
        m = min(k, n - k)
        out[k:k + m] = out[:m]
        k += m
    return out


def patterns_runs(byte: int, kmax: int) -> list[bytes]:
    """{a^1, ..., a^kmax}: every position is the end of min(i+1, kmax) matches."""
    return [bytes([byte]) * k for k in range(1, kmax + 1)]


# ---------------------------------------------------------------------------
# Workloads (BASELINE.json configs)
# ---------------------------------------------------------------------------
@dataclass
class Workload:
    name: str
    text: np.ndarray
    patterns: list[bytes]
    meta: dict = field(default_factory=dict)


C_SIZES = {"c1": 1 << 20, "c2": 1 << 28, "c3": 1 << 30, "c4": 1 << 32}


def stream(w: Workload, name: str, block0: int, nbytes: int) -> np.ndarray:
    """nbytes of config `name`'s endless text stream starting at block0."""
    m = (nbytes + BLOCK - 1) // BLOCK * BLOCK
    b0 = block0
    if name == "c1":
        t = text_lowercase(m, 1000, b0)
    elif name == "c2":
        t = text_english(m, 2000, english_vocabulary(2002), block0=b0)
    elif name == "c3":
        t = text_payload(m, 3000, w.patterns, block0=b0)
    elif name == "c4":
        t = text_dna(m, 4000, block0=b0)
    else:
        raise ValueError(name)
    return t[:nbytes]


def segment(w: Workload, name: str, index: int, n: int, extra: int) -> np.ndarray:
    """Bytes [index*n, (index+1)*n + extra) of config `name`'s text stream
    (n a multiple of BLOCK): rank `index`'s shard plus its halo, for the
    weak-scaled multi-GPU bench.  Segment 0 without extra is w.text."""
    assert n % BLOCK == 0
    return stream(w, name, index * (n // BLOCK), n + extra)


def make(name: str, n: int | None = None, n_patterns: int | None = None) -> Workload:
    """Build a config's text and dictionary.  ``n`` scales the text down for
    oracle-sized tests (dictionary recipe unchanged unless n_patterns given)."""
    if name == "c1":
        n = C_SIZES["c1"] if n is None else n
        P = 100 if n_patterns is None else n_patterns
        pats = patterns_random(P, 2, 16, 1001, b"abcdefghijklmnopqrstuvwxyz")
        return Workload("c1", text_lowercase(n, 1000), pats,
                        {"text": "iid a-z", "patterns": f"{P} iid a-z, len U{{2..16}}"})
    if name == "c2":
        n = C_SIZES["c2"] if n is None else n
        P = 1000 if n_patterns is None else n_patterns
        voc = english_vocabulary(2002)
        text = text_english(n, 2000, voc)
        pats = patterns_substrings(text, P, 4, 32, 2001)
        return Workload("c2", text, pats, {"text": "English-like Zipf(1) over 20k words",
                                           "patterns": f"{P} substrings, len U{{4..32}}"})
    if name == "c3":
        n = C_SIZES["c3"] if n is None else n
        P = 10000 if n_patterns is None else n_patterns
        pats = patterns_snort(P, 3001)
        return Workload("c3", text_payload(n, 3000, pats), pats,
                        {"text": "64B payload chunks 60/38/2", "patterns": f"{P} Snort-like bytes"})
    if name == "c4":
        n = C_SIZES["c4"] if n is None else n
        P = 20000 if n_patterns is None else n_patterns
        text = text_dna(n, 4000)
        pats = patterns_kmers(text, P, 4001)
        return Workload("c4", text, pats, {"text": "ACGT + 0.01% N runs", "patterns": f"{P} k-mers U{{20..32}}"})
    if name.startswith("c5-"):
        # c5-<family>-<P>-<log2 n>, family in {english, snort}; or c5-adv-<kind>-<log2 n>
        parts = name.split("-")
        fam = parts[1]
        if fam == "adv":
            kind = parts[2]
            n = (1 << int(parts[3])) if n is None else n
            runs = patterns_runs(ord("a"), 32)
            if kind == "a":
                return Workload(name, text_repeat(n, b"a"), runs, {"text": "a^n", "patterns": "{a^1..a^32}"})
            unit = patterns_random(1, 7, 7, 5003, b"abcdefghijklmnopqrstuvwxyz")[0]
            voc = english_vocabulary(5002)
            pats = patterns_substrings(text_english(1 << 20, 5000, voc), 1000, 4, 32, 5001) + runs + [unit]
            return Workload(name, text_repeat(n, unit + b"aaaaaaaa"), pats,
                            {"text": "period-15 repeat", "patterns": "1000 english + runs + unit"})
        P = int(parts[2]) if n_patterns is None else n_patterns
        n = (1 << int(parts[3])) if n is None else n
        if fam == "english":
            voc = english_vocabulary(5002)
            text = text_english(n, 5000, voc)
            return Workload(name, text, patterns_substrings(text, P, 4, 32, 5001), {})
        if fam == "snort":
            pats = patterns_snort(P, 5011)
            return Workload(name, text_payload(n, 5010, pats), pats, {})
    raise ValueError(f"unknown workload {name!r}")
