"""Brute-force substring search: the plain definition of the result.

Independent of oracle/ and of the product: every (end, pid) with
text[end-len+1 .. end] == pattern[pid], in canonical (start, pid) order.
"""
from __future__ import annotations


def brute_matches(text: bytes, patterns: list[bytes]) -> list[tuple[int, int]]:
    occ = []
    for pid, p in enumerate(patterns):
        L = len(p)
        for s in range(0, len(text) - L + 1):
            if text[s:s + L] == p:
                occ.append((s, pid, s + L - 1))
    occ.sort()
    return [(end, pid) for (_s, pid, end) in occ]
