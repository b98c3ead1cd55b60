"""Independent big-int / Fraction brute force of the Sieve back-end -- TEST INFRASTRUCTURE ONLY.

A second, deliberately naive implementation of SURVEY.md 8(c), written from
the paper's definitions without looking at oracle/sieve_oracle.c's structure:

* moments and every comparison with Python integers (no overflow possible);
* CoV < theta as the exact rational comparison sigma^2 < theta^2 mu^2 with Fractions;
* fma emulated exactly: float(Fraction(a) * Fraction(b) + Fraction(c)) is correctly rounded
  (Python's int/int true division rounds to nearest-even), since Python 3.12 has no math.fma;
* the prediction C_pred = sum_s W_s y_rep / x_rep evaluated exactly as a Fraction.

Only for tiny traces (a few hundred invocations, small G).
"""
import math
from fractions import Fraction

LOG2E_256 = 256.0 * 1.4426950408889634074
LN2_256 = float.fromhex("0x1.62e42fefa39efp-9")     # rn(ln 2) / 256
KMAX = 10526
TWO52 = 2.0 ** 52


def fma(a, b, c):
    return float(Fraction(a) * Fraction(b) + Fraction(c))


def _exp2_neg_table():
    """2^(-j/256), j = 1..255, correctly rounded (60-digit decimal, then float() rounds); entry 0
    is 1 - 2^-53 (A10: no term is an exact half-integer)."""
    from decimal import Decimal, getcontext
    getcontext().prec = 60
    return [1.0 - 2.0 ** -53] + [float(Decimal(2) ** (Decimal(-j) / Decimal(256))) for j in range(1, 256)]


EXP2_NEG = _exp2_neg_table()


def _k(t):
    # nearest integer to the EXACT product t * 256 log2 e (single rounding, ties to even)
    return round(Fraction(t) * Fraction(LOG2E_256))


def _reduce(t, k):
    r = fma(-float(k), LN2_256, t)
    p = -float(Fraction(1, 6))           # P(r) = 1 - r + r^2/2 - r^3/6 (Horner, signed coefs)
    for c in (Fraction(1, 2), Fraction(-1), Fraction(1)):
        p = fma(p, r, float(c))
    return p, k & 255, k >> 8


def det_exp(t):
    k = _k(t)
    if k > KMAX:
        return 0.0
    p, j, m = _reduce(t, k)
    return math.ldexp(p * EXP2_NEG[j], -m)


def q_of_t(t):
    """rint(P * 2^(-j/256) * 2^(40-m)) with a single rounding (exact rational, then round)."""
    k = _k(t)
    if k > KMAX:
        return 0
    p, j, m = _reduce(t, k)
    v = Fraction(p) * Fraction(EXP2_NEG[j]) * Fraction(2) ** (40 - m)
    return round(v)                      # Fraction round(): nearest, ties to even


def q_term(g, x, inv_h, lo):
    """A10: z = rn(rn(g - lo) / h') - rn(rn(x - lo) / h') with 1/h' = inv_h (Python floats are
    IEEE doubles; x - lo is an exact integer below 2^44, so float() of it is exact)"""
    gs = (g - float(lo)) * inv_h
    xs = float(x - lo) * inv_h
    z = gs - xs
    t = (z * z) * 0.5
    return q_of_t(t)


def cov_below(vals, theta):
    """population CoV < theta, exactly (sigma = sqrt of the mean squared deviation)"""
    n = len(vals)
    mu = Fraction(sum(vals), n)
    var = sum((Fraction(v) - mu) ** 2 for v in vals) / n
    return var < theta * theta * mu * mu


def bandwidth(vals, bw_scale):
    n = len(vals)
    return bandwidth_from_moments(n, sum(vals), sum(v * v for v in vals), bw_scale)


def bandwidth_from_moments(n, s1, s2, bw_scale):
    num = n * s2 - s1 * s1                # exact integer
    var = float(num) / (float(n) * float(n))   # float(int) is correctly rounded
    h_raw = (bw_scale * math.sqrt(var)) * math.pow(float(n), -0.2)
    e = math.frexp(h_raw)[1] - 1 - 15    # ilogb(h_raw) - 15
    return math.ldexp(float(round(math.ldexp(h_raw, -e))), e)


def grid(lo, hi, G):
    return [float(lo) + float((hi - lo) * j) / float(G - 1) for j in range(G)]


def kde(vals, lo, hi, h, G):
    inv_h = 1.0 / h
    return [sum(q_term(g, x, inv_h, lo) for x in vals) for g in grid(lo, hi, G)]


def valley_cuts(D, shift):
    """indices m of the valleys: hysteresis delta = max(1, max D >> shift), run midpoints"""
    delta = max(1, max(D) >> shift)
    cuts = []
    mode = "up"
    top = D[0]
    for j in range(1, len(D)):
        d = D[j]
        if mode == "up":
            top = max(top, d)
            if d + delta <= top:
                mode, low, a, b = "down", d, j, j
        else:
            if d < low:
                low, a, b = d, j, j
            elif d == low and b == j - 1:
                b = j
            elif d >= low + delta:
                cuts.append((a + b) // 2)
                mode, top = "up", d
    return cuts


def stratify(kid, x, K, cta=None, cycles=None, theta=Fraction(2, 5), G=64, shift=10,
             bw_scale=1.06, max_rounds=64, split_kinds=None):
    """split_kinds: optional list that receives 1 (valley) or 2 (bisection) per KDE segment"""
    n = len(kid)
    kid = [int(k) for k in kid]
    x = [int(v) for v in x]
    cta = [0] * n if cta is None else [int(c) for c in cta]
    strata = []  # dicts
    for k in range(K):
        rows = [i for i in range(n) if kid[i] == k]
        if not rows:
            continue
        vals = [x[i] for i in rows]
        if min(vals) == max(vals):
            strata.append(dict(kid=k, tier=1, lo=min(vals), hi=max(vals), h=0.0, rnd=0))
            continue
        if cov_below(vals, theta):
            strata.append(dict(kid=k, tier=2, lo=min(vals), hi=max(vals), h=0.0, rnd=0))
            continue
        open_ = [vals]
        rnd = 0
        while open_:
            rnd += 1
            if rnd > max_rounds:
                raise RuntimeError("ELIMIT")
            nxt = []
            for seg in open_:
                lo, hi = min(seg), max(seg)
                h = bandwidth(seg, bw_scale)
                D = kde(seg, lo, hi, h, G)
                gs = grid(lo, hi, G)
                T = sorted({math.ceil(gs[m]) for m in valley_cuts(D, shift)})
                T = [t for t in T if lo < t <= hi]
                if split_kinds is not None:
                    split_kinds.append(1 if T else 2)
                if not T:
                    T = [(lo + hi + 1) // 2]
                bounds = [0] + T + [1 << 64]
                for a, b in zip(bounds[:-1], bounds[1:]):
                    part = [v for v in seg if a <= v < b]
                    if not part:
                        continue
                    if min(part) == max(part) or cov_below(part, theta):
                        strata.append(dict(kid=k, tier=3, lo=min(part), hi=max(part), h=h, rnd=rnd))
                    else:
                        nxt.append(part)
            open_ = nxt
    strata.sort(key=lambda s: (s["kid"], s["lo"]))
    sid = [None] * n
    for s_i, s in enumerate(strata):
        for i in range(n):
            if kid[i] == s["kid"] and s["lo"] <= x[i] <= s["hi"]:
                sid[i] = s_i
    for s_i, s in enumerate(strata):
        mem = [i for i in range(n) if sid[i] == s_i]
        s["count"] = len(mem)
        s["W"] = sum(x[i] for i in mem)
        if s["tier"] == 1:
            rep = min(mem)
        else:
            by_cta = {}
            for i in mem:
                by_cta.setdefault(cta[i], []).append(i)
            best = max(by_cta.values(), key=lambda l: (len(l), -min(l)))
            rep = min(best)
        s["rep"] = rep
        s["rep_instr"] = x[rep]
        s["rep_cycles"] = None if cycles is None else int(cycles[rep])
        s["rep_cta"] = cta[rep]
    return strata, sid


def predict(strata, cycles=None, rep_cycles=None):
    """C_pred exactly; IPC = 1 / sum_s w_s / IPC_s; error; speedup"""
    I = sum(s["W"] for s in strata)
    ys = rep_cycles if rep_cycles is not None else [s["rep_cycles"] for s in strata]
    c_pred = sum(Fraction(s["W"] * y, s["rep_instr"]) for s, y in zip(strata, ys))
    out = {"predicted_cycles_exact": c_pred, "predicted_cycles": float(c_pred),
           "predicted_ipc": float(Fraction(I) / c_pred) if c_pred else math.inf}
    if cycles is not None:
        cm = sum(int(c) for c in cycles)
        out["measured_cycles"] = float(cm)
        out["error"] = float(abs(c_pred - cm) / cm) if cm else math.nan
        out["speedup"] = float(Fraction(cm, sum(ys)))
    return out


def min_strata(vals, theta=Fraction(2, 5)):
    """NEXT-3 by exhaustion (reading A28): every way of cutting the sorted distinct values into
    runs; the minimum count whose runs all have CoV < theta (Fractions, population sigma), and
    the canonical optimum = the one whose cut positions, read from the last, are smallest."""
    from itertools import combinations
    d = sorted(set(int(v) for v in vals))
    m = len(d)
    groups = {v: [w for w in vals if int(w) == v] for v in d}
    for k in range(1, m + 1):
        found = []
        for cut in combinations(range(1, m), k - 1):
            bounds = (0,) + cut + (m,)
            if all(cov_below([w for v in d[bounds[t]:bounds[t + 1]] for w in groups[v]], theta)
                   for t in range(k)):
                found.append(cut)
        if found:
            best = min(found, key=lambda c: tuple(reversed(c)))
            return k, [d[i] for i in best]
    raise AssertionError("unreachable: single values are always valid")
