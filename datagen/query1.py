"""Query-1-family inputs (PAPER.md P:41 Query 1, P:53 non-equality variant).

Tables R(col1, col2) and S(col1, col2), int32, as in Query 1.  The paper
prints no distributions (reading R12); the recipe below follows
SURVEY.md §8(d):

=======  =========  ==================================  ==============  ====
config   |R|=|S|    col1 (correlated key)               col2 (value)    seed
=======  =========  ==================================  ==============  ====
C1       1000       U[0,250); 10% of R.col1 U[250,275)   U[0,16)         1
C2       1M         U[0,2^18)  (or Zipf(1.0) variant)    U[0,16)         2
C5       16M        U[0,2^31-1)                          U[0,2^20)       7
=======  =========  ==================================  ==============  ====

C1's 10% out-of-range R keys produce empty subqueries (NULL aggregates,
COUNT = 0), which the paper is silent on (reading R1).
"""
import numpy as np

CONFIGS = {
    "C1": dict(n_r=1000, n_s=1000, key_hi=250, val_hi=16, seed=1,
               empty_frac=0.10, empty_hi=275),
    "C2": dict(n_r=1_000_000, n_s=1_000_000, key_hi=1 << 18, val_hi=16, seed=2),
    "C2z": dict(n_r=1_000_000, n_s=1_000_000, key_hi=1 << 18, val_hi=16, seed=2,
                zipf=1.0),
    "C5": dict(n_r=16_000_000, n_s=16_000_000, key_hi=(1 << 31) - 1,
               val_hi=1 << 20, seed=7),
}

# C2's op x agg sweep (BASELINE.json configs[1]); exists and count compare
# R.col2 as in Query 1 where an outer comparison applies.
C2_SWEEP = [(op, agg) for op in ("=", "<", ">", "!=")
            for agg in ("min", "count", "exists")]


def _zipf_keys(rng, n, key_hi, s):
    # Zipf(s) over ranks 1..key_hi, ranks mapped to keys by a random
    # permutation so hot keys are spread over the key domain.
    ranks = np.arange(1, key_hi + 1, dtype=np.float64)
    w = ranks ** (-s)
    w /= w.sum()
    idx = rng.choice(key_hi, size=n, p=w)
    perm = rng.permutation(key_hi)
    return perm[idx].astype(np.int32)


def tables(n_r, n_s, key_hi, val_hi, seed, empty_frac=0.0, empty_hi=None,
           zipf=None, null_frac=0.0):
    """Return {"R": {"col1", "col2"}, "S": {...}} int32 arrays and, when
    ``null_frac > 0``, validity masks under ``"R_valid"`` / ``"S_valid"``
    (uint8, 1 = not NULL) for every column."""
    rng = np.random.Generator(np.random.PCG64(seed))
    if zipf:
        r1 = _zipf_keys(rng, n_r, key_hi, zipf)
        s1 = _zipf_keys(rng, n_s, key_hi, zipf)
    else:
        r1 = rng.integers(0, key_hi, size=n_r, dtype=np.int64).astype(np.int32)
        s1 = rng.integers(0, key_hi, size=n_s, dtype=np.int64).astype(np.int32)
    if empty_frac:
        m = rng.random(n_r) < empty_frac
        r1[m] = rng.integers(key_hi, empty_hi, size=int(m.sum()))
    r2 = rng.integers(0, val_hi, size=n_r, dtype=np.int64).astype(np.int32)
    s2 = rng.integers(0, val_hi, size=n_s, dtype=np.int64).astype(np.int32)
    out = {"R": {"col1": r1, "col2": r2}, "S": {"col1": s1, "col2": s2}}
    if null_frac:
        out["R_valid"] = {c: (rng.random(n_r) >= null_frac).astype(np.uint8)
                          for c in ("col1", "col2")}
        out["S_valid"] = {c: (rng.random(n_s) >= null_frac).astype(np.uint8)
                          for c in ("col1", "col2")}
    return out


def config(name, **override):
    kw = dict(CONFIGS[name])
    kw.update(override)
    return tables(**kw)


def random_small(seed, n_r, n_s, key_hi=4, val_lo=-3, val_hi=4, null_frac=0.2,
                 extra_cols=True):
    """Tiny randomized tables with NULLs, negative values and extra columns
    (col3 in R and S) for local-predicate tests."""
    rng = np.random.Generator(np.random.PCG64(seed))

    def col(n, lo, hi):
        return rng.integers(lo, hi, size=n, dtype=np.int64).astype(np.int32)

    R = {"col1": col(n_r, 0, key_hi), "col2": col(n_r, val_lo, val_hi)}
    S = {"col1": col(n_s, 0, key_hi), "col2": col(n_s, val_lo, val_hi)}
    if extra_cols:
        R["col3"] = col(n_r, 0, 3)
        S["col3"] = col(n_s, 0, 3)
    out = {"R": R, "S": S}
    if null_frac:
        out["R_valid"] = {c: (rng.random(n_r) >= null_frac).astype(np.uint8) for c in R}
        out["S_valid"] = {c: (rng.random(n_s) >= null_frac).astype(np.uint8) for c in S}
    return out
