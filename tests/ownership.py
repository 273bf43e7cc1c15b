"""Chunk ownership for tests (reading A10: a token belongs to the chunk holding its first byte):
the oracle's counts of the tokens whose first byte lies in [s, e).  Pinned in test_oracle.py
(the owned counts of any partition sum to the whole-text counts)."""
import numpy as np

import oracle


def is_word(c: int) -> bool:
    return (48 <= c <= 57) or (65 <= c <= 90) or (97 <= c <= 122) or c == 95


def owned_counts(data: bytes, s: int, e: int, words) -> np.ndarray:
    """Counts of the sub-buffer that starts at the first token start >= s and ends where the
    token open at e ends (its boundaries are then genuine token boundaries of `data`)."""
    a = s
    if s > 0:
        while a < e and is_word(data[a - 1]) and is_word(data[a]):
            a += 1
    if a >= e:
        return np.zeros(len(words), dtype=np.uint64)
    b = e
    while b < len(data) and is_word(data[b - 1]) and is_word(data[b]):
        b += 1
    return oracle.count_tokens(data[a:b], words)
