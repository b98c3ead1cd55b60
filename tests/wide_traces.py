"""Seeded adversarial traces for the full-size arithmetic paths (VERDICT r1 missing #1): one
kernel with more than 2^24 invocations concentrated in three point masses, so that
  * n * S2 >= 2^128 (the 256-bit tier test and bandwidth conversion, A5, A8),
  * D_j >= 2^63 at a grid point that coincides with a mass (u128 densities, A10),
  * the valley scan runs on u128 densities (A11),
plus a Tier-2 kernel near 2^44 with n * S2 >= 2^128, mixed into C1's rows in a seeded order.
Input construction only: none of the method's arithmetic lives here."""
import numpy as np

import gen


def point_mass_trace(seed=0x51E7E0AD):
    base = gen.make_trace("C1")
    K0 = base["K"]
    rng = np.random.default_rng(seed)
    a = 1 << 30
    d = 1 << 42
    masses = [(a, (1 << 23) + 3), (a + d, (1 << 22) + 1), (a + 2 * d, 3 * (1 << 21) + 5)]
    x3 = np.concatenate([np.full(m, v, np.uint64) for v, m in masses])
    # Tier-2 kernel near 2^44: Irwin-Hall-like integer noise of CoV ~ 1e-3, 2^24 invocations
    n2 = 1 << 24
    x2 = ((1 << 44) - (1 << 36) + rng.integers(-(1 << 33), 1 << 33, n2)).astype(np.uint64)
    kid = np.concatenate([base["kid"], np.full(len(x3), K0, np.uint32), np.full(n2, K0 + 1, np.uint32)])
    x = np.concatenate([base["x"], x3, x2])
    cta = np.concatenate([base["cta"], rng.choice(np.array([128, 256, 512], np.uint32), len(x3) + n2)])
    y = np.concatenate([base["y"], (x3 >> np.uint64(6)) + rng.integers(0, 1000, len(x3)).astype(np.uint64),
                        (x2 >> np.uint64(8)) + np.uint64(17)])
    perm = rng.permutation(len(kid))
    return {"kid": kid[perm], "x": x[perm], "cta": cta[perm], "y": y[perm], "K": K0 + 2}
