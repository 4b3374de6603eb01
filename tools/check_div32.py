#!/usr/bin/env python
"""Checks Div32 (common.cuh): floor(x / d) = mulhi32(x, m) >> k for every d in [2, 16] on the top
2^21 values below 2^31 (where the multiplier's error is largest) and 2M random x < 2^31."""
import numpy as np


def params(d):
    c = (d - 1).bit_length()
    return -(-(1 << (31 + c)) // d), c - 1


def main():
    for d in range(2, 17):
        m, k = params(d)
        assert m < (1 << 32)
        xs = np.concatenate([np.arange((1 << 31) - (1 << 21), 1 << 31, dtype=np.uint64),
                             np.random.default_rng(d).integers(0, 1 << 31, 2_000_000, dtype=np.uint64)])
        q = ((xs * np.uint64(m)) >> np.uint64(32)) >> np.uint64(k)
        assert np.array_equal(q, xs // np.uint64(d)), d
    print("Div32 exact for d in [2, 16], x < 2^31")


if __name__ == "__main__":
    main()
