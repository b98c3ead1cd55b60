"""CPU oracle for the Sieve stratification back-end -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
import this package.  The product (paper_conf_ispass_naderantahanse23_b200/) never imports it;
the two share no code.  See oracle/sieve_oracle.c for the step-by-step implementation with
PAPER.md citations, and oracle/brute.py for an independent big-int brute force.
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

STRATUM_DTYPE = np.dtype([
    ("kernel_id", "<u4"), ("tier", "<u4"), ("index_in_kernel", "<u4"), ("rep_cta", "<u4"),
    ("lo", "<u8"), ("hi", "<u8"), ("count", "<u8"), ("instr_sum_lo", "<u8"), ("instr_sum_hi", "<u8"),
    ("rep_id", "<u8"), ("rep_instr", "<u8"), ("rep_cycles", "<u8"), ("bandwidth", "<f8"),
    ("split_round", "<u4"), ("pad", "<u4")])


class _Pred(ctypes.Structure):
    _fields_ = [("predicted_cycles", ctypes.c_double), ("predicted_ipc", ctypes.c_double),
                ("measured_cycles", ctypes.c_double), ("error", ctypes.c_double),
                ("speedup", ctypes.c_double), ("total_instr_lo", ctypes.c_uint64),
                ("total_instr_hi", ctypes.c_uint64)]


def _lib():
    global _LIB
    if _LIB is None:
        p = os.path.join(_HERE, "libsieve_oracle.so")
        if not os.path.exists(p):
            import sys
            sys.path.insert(0, os.path.dirname(_HERE))
            from tools.build_native import build_oracle
            build_oracle()
        L = ctypes.CDLL(p)
        u32, u64, dbl, vp = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_double, ctypes.c_void_p
        L.oracle_stratify.argtypes = [u64, u32, vp, vp, vp, vp, vp, u32, u32, u32, u32, u32, dbl,
                                      ctypes.c_int, ctypes.POINTER(vp)]
        L.oracle_stratify.restype = ctypes.c_int
        L.oracle_free.argtypes = [vp]
        L.oracle_predict.argtypes = [vp, vp, ctypes.POINTER(_Pred)]
        L.oracle_predict.restype = ctypes.c_int
        L.oracle_strata_count.argtypes = [vp]
        L.oracle_strata_count.restype = u64
        L.oracle_strata_copy.argtypes = [vp, vp]
        L.oracle_sid_copy.argtypes = [vp, vp]
        L.oracle_segment_count.argtypes = [vp]
        L.oracle_segment_count.restype = u64
        L.oracle_segment_get.argtypes = [vp, u64, vp, vp, ctypes.POINTER(dbl), vp, vp, vp]
        L.oracle_segment_get.restype = ctypes.c_int
        L.oracle_rounds.argtypes = [vp]
        L.oracle_rounds.restype = u32
        L.oracle_totals.argtypes = [vp, vp]
        L.oracle_det_exp.argtypes = [dbl]
        L.oracle_det_exp.restype = dbl
        L.oracle_q.argtypes = [dbl]
        L.oracle_q.restype = u64
        L.oracle_cycle_cov.argtypes = [vp, vp, vp, ctypes.POINTER(dbl)]
        L.oracle_cycle_cov.restype = ctypes.c_int
        L.oracle_min_strata.argtypes = [u64, u32, vp, vp, u32, u32, u64, vp, vp, u64, ctypes.POINTER(u64)]
        L.oracle_min_strata.restype = ctypes.c_int
        L.oracle_exp2_table.argtypes = [ctypes.c_int]
        L.oracle_exp2_table.restype = dbl
        L.oracle_tier.argtypes = [u64, u64, u64, u64, u64, u64, u64, u32, u32]
        L.oracle_tier.restype = ctypes.c_int
        L.oracle_bandwidth.argtypes = [u64, u64, u64, u64, u64, dbl]
        L.oracle_bandwidth.restype = dbl
        L.oracle_u256_to_double.argtypes = [vp]
        L.oracle_u256_to_double.restype = dbl
        L.oracle_grid_point.argtypes = [u64, u64, u32, u32]
        L.oracle_grid_point.restype = dbl
        L.oracle_kde.argtypes = [vp, u64, u64, u64, dbl, u32, vp, vp]
        L.oracle_valleys.argtypes = [vp, vp, u32, u32, vp]
        L.oracle_valleys.restype = u32
        L.oracle_sizeof_stratum.restype = ctypes.c_int
        assert L.oracle_sizeof_stratum() == STRATUM_DTYPE.itemsize
        _LIB = L
    return _LIB


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _u128(lo, hi):
    return (int(hi) << 64) | int(lo)


def _split(v):
    v = int(v)
    return v & ((1 << 64) - 1), v >> 64


class OracleError(RuntimeError):
    def __init__(self, code):
        super().__init__(f"oracle status {code}")
        self.code = code


class Result:
    """Oracle output: strata (structured array), per-row stratum ids, debug segments."""

    def __init__(self, handle, n, G):
        self._h = handle
        self.n = n
        self.G = G
        L = _lib()
        ns = L.oracle_strata_count(handle)
        self.strata = np.zeros(ns, STRATUM_DTYPE)
        if ns:
            L.oracle_strata_copy(handle, _p(self.strata))
        self.sid = np.zeros(n, np.uint32)
        if n:
            L.oracle_sid_copy(handle, _p(self.sid))
        self.rounds = L.oracle_rounds(handle)
        t = np.zeros(4, np.uint64)
        L.oracle_totals(handle, _p(t))
        self.total_instr = _u128(t[0], t[1])
        self.c_meas = _u128(t[2], t[3])

    def __del__(self):
        if getattr(self, "_h", None) and _LIB is not None:
            _LIB.oracle_free(self._h)
            self._h = None

    def segments(self, with_density=True):
        L = _lib()
        out = []
        for i in range(L.oracle_segment_count(self._h)):
            m4 = np.zeros(4, np.uint32)
            m3 = np.zeros(3, np.uint64)
            h = ctypes.c_double()
            dlo = np.zeros(self.G, np.uint64) if with_density else None
            dhi = np.zeros(self.G, np.uint64) if with_density else None
            L.oracle_segment_get(self._h, i, _p(m4), _p(m3), ctypes.byref(h), _p(dlo), _p(dhi), None)
            cuts = np.zeros(int(m4[3]), np.uint64)
            L.oracle_segment_get(self._h, i, _p(m4), _p(m3), ctypes.byref(h), None, None, _p(cuts))
            out.append({"kernel_id": int(m4[0]), "round": int(m4[1]), "split_kind": int(m4[2]),
                        "n_cuts": int(m4[3]), "lo": int(m3[0]), "hi": int(m3[1]),
                        "count": int(m3[2]), "bandwidth": h.value, "d_lo": dlo, "d_hi": dhi,
                        "cuts": cuts})
        return out

    def cycle_cov(self, cycles):
        """Per-stratum CoV of the members' cycles and its instruction-weighted mean (Fig. 4)."""
        cyc = np.ascontiguousarray(cycles, np.uint64)
        cov = np.zeros(len(self.strata), np.float64)
        w = ctypes.c_double()
        rc = _lib().oracle_cycle_cov(self._h, _p(cyc), _p(cov), ctypes.byref(w))
        if rc != 0:
            raise OracleError(rc)
        return cov, w.value

    def predict(self, rep_cycles=None):
        pr = _Pred()
        rc = _lib().oracle_predict(self._h, _p(None if rep_cycles is None else
                                                np.ascontiguousarray(rep_cycles, np.uint64)),
                                   ctypes.byref(pr))
        if rc != 0:
            raise OracleError(rc)
        return {"predicted_cycles": pr.predicted_cycles, "predicted_ipc": pr.predicted_ipc,
                "measured_cycles": pr.measured_cycles, "error": pr.error, "speedup": pr.speedup,
                "total_instr": _u128(pr.total_instr_lo, pr.total_instr_hi)}


def stratify(kid, x, K, cta=None, cycles=None, ids=None, theta=(2, 5), G=1024, valley_shift=10,
             max_rounds=64, bw_scale=1.06, keep_debug=False):
    """Run the oracle over a whole trace (or a kernel subset with explicit global ids)."""
    kid = np.ascontiguousarray(kid, np.uint32)
    x = np.ascontiguousarray(x, np.uint64)
    cta = None if cta is None else np.ascontiguousarray(cta, np.uint32)
    cycles = None if cycles is None else np.ascontiguousarray(cycles, np.uint64)
    ids = None if ids is None else np.ascontiguousarray(ids, np.uint64)
    h = ctypes.c_void_p()
    rc = _lib().oracle_stratify(len(kid), K, _p(kid), _p(x), _p(cta), _p(cycles), _p(ids),
                                theta[0], theta[1], G, valley_shift, max_rounds, bw_scale,
                                1 if keep_debug else 0, ctypes.byref(h))
    if rc != 0:
        raise OracleError(rc)
    return Result(h, len(kid), G)


def min_strata(kid, x, K, theta=(2, 5), max_distinct=1 << 62):
    """NEXT-3 (reading A28): exact minimum strata per kernel and the canonical optimal cuts.
    -> (counts[K] as uint32, list of per-kernel cut lists)."""
    kid = np.ascontiguousarray(kid, np.uint32)
    x = np.ascontiguousarray(x, np.uint64)
    counts = np.zeros(K, np.uint32)
    nc = ctypes.c_uint64()
    rc = _lib().oracle_min_strata(len(kid), K, _p(kid), _p(x), theta[0], theta[1], max_distinct,
                                  _p(counts), None, 0, ctypes.byref(nc))
    if rc != 0:
        raise OracleError(rc)
    cuts = np.zeros(max(1, nc.value), np.uint64)
    rc = _lib().oracle_min_strata(len(kid), K, _p(kid), _p(x), theta[0], theta[1], max_distinct,
                                  _p(counts), _p(cuts), nc.value, ctypes.byref(nc))
    if rc != 0:
        raise OracleError(rc)
    per, o = [], 0
    for c in counts.tolist():
        k = c - 1 if 2 <= c < 0xFFFFFFFF else 0
        per.append([int(v) for v in cuts[o:o + k]])
        o += k
    return counts, per


# ---- step functions exported for the pin tests ----
def det_exp(t):
    return _lib().oracle_det_exp(float(t))


def q_of_t(t):
    return int(_lib().oracle_q(float(t)))


def exp2_table():
    return [_lib().oracle_exp2_table(j) for j in range(256)]


def tier(values, theta=(2, 5)):
    n = len(values)
    s1 = sum(int(v) for v in values)
    s2 = sum(int(v) * int(v) for v in values)
    a, b = _split(s1)
    c, d = _split(s2)
    return _lib().oracle_tier(n, a, b, c, d, min(values), max(values), theta[0], theta[1])


def bandwidth(values, bw_scale=1.06):
    n = len(values)
    s1 = sum(int(v) for v in values)
    s2 = sum(int(v) * int(v) for v in values)
    a, b = _split(s1)
    c, d = _split(s2)
    return _lib().oracle_bandwidth(n, a, b, c, d, bw_scale)


def tier_moments(n, s1, s2, lo, hi, theta=(2, 5)):
    """O3 on explicit exact moments (n, S1, S2 as Python ints) -- the wide-regime pin hook."""
    a, b = _split(s1)
    c, d = _split(s2)
    return _lib().oracle_tier(n, a, b, c, d, lo, hi, theta[0], theta[1])


def bandwidth_moments(n, s1, s2, bw_scale=1.06):
    a, b = _split(s1)
    c, d = _split(s2)
    return _lib().oracle_bandwidth(n, a, b, c, d, bw_scale)


def u256_to_double(v):
    w = np.array([(int(v) >> (64 * i)) & ((1 << 64) - 1) for i in range(4)], np.uint64)
    return _lib().oracle_u256_to_double(_p(w))


def grid_point(lo, hi, j, G):
    return _lib().oracle_grid_point(lo, hi, j, G)


def kde(values, lo, hi, h, G):
    v = np.ascontiguousarray(values, np.uint64)
    dlo = np.zeros(G, np.uint64)
    dhi = np.zeros(G, np.uint64)
    _lib().oracle_kde(_p(v), len(v), lo, hi, h, G, _p(dlo), _p(dhi))
    return [_u128(a, b) for a, b in zip(dlo, dhi)]


def valleys(D, shift=10):
    G = len(D)
    dlo = np.array([int(d) & ((1 << 64) - 1) for d in D], np.uint64)
    dhi = np.array([int(d) >> 64 for d in D], np.uint64)
    out = np.zeros(G, np.uint32)
    nc = _lib().oracle_valleys(_p(dlo), _p(dhi), G, shift, _p(out))
    return [int(v) for v in out[:nc]]
