"""Shared test helpers (no method arithmetic beyond the Philox words of the oracle)."""
import numpy as np

TOL = 1e-9   # north_star: dS / H / MDL within 1e-9 relative (floor of 1 nat for dS)


def close(gpu, ref, tol=TOL, floor=1.0):
    gpu = np.asarray(gpu, np.float64)
    ref = np.asarray(ref, np.float64)
    return np.abs(gpu - ref) <= tol * np.maximum(np.abs(ref), floor)


def mh_u(oracle_mod, seed, outer, itr, vs):
    """u = (w3 + 1/2) 2^-32 of each vertex's Philox counter (v, 0, itr, outer<<1|1)."""
    key = [seed & 0xffffffff, seed >> 32]
    return np.array([(int(oracle_mod.philox([int(v), 0, itr, (outer << 1) | 1], key)[3]) + 0.5) / 2 ** 32
                     for v in vs])


def ties(oracle_mod, seed, outer, itr, vs, p):
    """MH decisions within 1e-9 of the threshold: counted and reported, not failed."""
    u = mh_u(oracle_mod, seed, outer, itr, vs)
    return np.abs(u - p) <= 1e-9 * np.maximum(p, 1e-300)
