"""Oracle of the row grouping step — TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

PAPER.md:84-88 (§III-A) and Table I: rows are divided into groups by
their number of intermediate products (step 2) or of output non-zeros (step 6); a group
is a contiguous key range.  Given the inclusive upper bounds of the groups (ascending;
the bin table is a *parameter* of the implementation, read from the library under test),
the group of a row is the first group whose upper bound is >= its key.  Rows with key 0
belong to no group (reading R13: nothing to compute), reported as -1; keys above the
last bound get len(upper) (the overflow / global-memory group).
"""
from __future__ import annotations

import numpy as np


def bin_of(keys, upper) -> np.ndarray:
    keys = np.asarray(keys, dtype=np.int64)
    upper = np.asarray(upper, dtype=np.int64)
    out = np.empty(len(keys), dtype=np.int64)
    for i, kv in enumerate(keys.tolist()) if len(keys) < 4096 else []:
        if kv <= 0:
            out[i] = -1
            continue
        g = 0
        while g < len(upper) and kv > upper[g]:
            g += 1
        out[i] = g
    if len(keys) >= 4096:  # same rule, vectorised for large inputs
        out[:] = np.searchsorted(upper, keys, side="left")
        out[keys <= 0] = -1
    return out


def group_histogram(keys, upper) -> np.ndarray:
    """Number of rows per group (index len(upper) = overflow group)."""
    b = bin_of(keys, upper)
    return np.bincount(b[b >= 0], minlength=len(upper) + 1)
