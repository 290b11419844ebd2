"""classes — TEST INFRASTRUCTURE ONLY (task rule ③). Plain definition of the equivalence classes
that partial simulation produces.

PAPER.md:41 (§II-B): nodes are simulated on random patterns and "nodes with identical partial truth
tables are put into the same equivalence class"; the representative is the node with the minimum
id and a class of n nodes yields n-1 candidate pairs (representative, member). :61 / :183 / :187:
the partial simulator also simulates counter-example patterns to split the classes of disproved
pairs. Pairs are literals, so a node and the complement of another are in one
class too (relative phase = 1).

Patterns (the same counter-based generator the product uses, written out again here, Q19):
pattern p = 32 w + b takes PI id i to bit b of word w, where for w < num_words the word is the low
32 bits of splitmix64(seed ^ (i << 32) ^ w) and for w >= num_words it is the caller's word
pi_words[i - 1][w - num_words] (e.g. counter-examples).

Definition, one assignment at a time: evaluate every node on every pattern (oracle.eval_all), take
each node's vector of values v(n); n and m are in one class iff v(n) = v(m) or v(n) = !v(m). For
every AND node m that is not the minimum id of its class, emit (repr, m, phase) with phase = 1 iff
v(m) = !v(repr); pairs ordered by m. PIs and the constant only ever appear as representatives.
Pins: tests/test_classes_oracle.py (published splitmix64 outputs; with the full input cube as
patterns the classes equal the exact functional classes of the brute-force evaluator; hand cases).
"""
from __future__ import annotations

from typing import List, Optional, Sequence, Tuple

import numpy as np

M64 = (1 << 64) - 1


def splitmix64(x: int) -> int:
    """splitmix64 output for state x (Steele, Lea, Flood 2014; the state is incremented first)."""
    z = (x + 0x9E3779B97F4A7C15) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def pattern_words(num_pis: int, num_words: int, seed: int,
                  pi_words: Optional[np.ndarray] = None) -> List[List[int]]:
    """words[i-1] = the u32 words of PI id i: num_words random ones, then the caller's."""
    words = []
    for i in range(1, num_pis + 1):
        row = [splitmix64((seed ^ (i << 32) ^ w) & M64) & 0xFFFFFFFF for w in range(num_words)]
        if pi_words is not None:
            row += [int(x) for x in pi_words[i - 1]]
        words.append(row)
    return words


def classes(orc, num_words: int, seed: int, pi_words: Optional[np.ndarray] = None
            ) -> List[Tuple[int, int, int]]:
    """(repr, member, phase) for every AND member, ordered by member (see module docstring)."""
    I = orc.num_pis
    N = 1 + I + orc.num_ands
    words = pattern_words(I, num_words, seed, pi_words)
    total = len(words[0]) if I else num_words + (0 if pi_words is None else pi_words.shape[1])
    vals = np.zeros((N, 32 * total), dtype=np.uint8)
    for p in range(32 * total):
        w, b = divmod(p, 32)
        pis = np.array([(words[i][w] >> b) & 1 for i in range(I)], dtype=np.uint8)
        vals[:, p] = orc.eval_all(pis)
    first = {}
    phase = np.zeros(N, dtype=np.uint8)
    pairs = []
    for n in range(N):
        v = vals[n]
        inv = int(v[0])
        key = (v ^ inv).tobytes()
        phase[n] = inv
        if key in first:
            r = first[key]
            if n > I:
                pairs.append((r, n, inv ^ int(phase[r])))
        else:
            first[key] = n
    return pairs
