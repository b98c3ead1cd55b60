"""Seeded synthetic trace generator (shared test/bench input module).

Holds none of the method's arithmetic: it only produces the columns (kernel id, instruction
count, CTA size, cycles) that both the CPU oracle and the CUDA path consume.  The recipe is in
DESIGN.md section 4 and in gen/sieve_gen.h.

    from gen import make_trace, CONFIGS
    tr = make_trace("C1")            # dict of numpy arrays: kid u32, x u64, cta u32, y u64
    tr = make_trace("C4", first=0, n=1_000_000)   # a slice of a big config
"""
import ctypes
import os
from dataclasses import dataclass, replace

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


class _Params(ctypes.Structure):
    _fields_ = [("seed", ctypes.c_uint64), ("n_total", ctypes.c_uint64),
                ("K", ctypes.c_uint32), ("order", ctypes.c_uint32),
                ("homogeneous", ctypes.c_uint32), ("alt_cta_pct", ctypes.c_uint32),
                ("t1_pct", ctypes.c_uint32), ("t2_pct", ctypes.c_uint32), ("t3_pct", ctypes.c_uint32),
                ("t1_kernels", ctypes.c_uint32), ("t2_kernels", ctypes.c_uint32),
                ("t3_kernels", ctypes.c_uint32),
                ("m_min", ctypes.c_uint32), ("m_max", ctypes.c_uint32),
                ("phase_len_min", ctypes.c_uint32), ("phase_len_max", ctypes.c_uint32),
                ("n_phases", ctypes.c_uint32), ("rep_min", ctypes.c_uint32),
                ("rep_max", ctypes.c_uint32)]


@dataclass(frozen=True)
class GenConfig:
    name: str
    n: int
    K: int
    seed: int
    order: int = 1            # 0 = i.i.d. Zipf, 1 = training-loop phase schedule
    homogeneous: int = 0      # 1: cycles y = a_k * x exactly
    t_pct: tuple = (41, 40, 19)   # target invocation shares per intended tier shape
    t_kernels: tuple = (0, 0, 0)  # exact kernel counts per class (C1)
    modes: tuple = (2, 6)
    alt_cta_pct: int = 5
    phase_len: tuple = (200, 600)
    reps: tuple = (1, 16)


# BASELINE.json configs; seeds 0x51E7E000 + index
CONFIGS = {
    "C1": GenConfig("C1-tiny", 10_000, 20, 0x51E7E001, order=0, t_kernels=(8, 6, 6), modes=(2, 2)),
    "C2": GenConfig("C2-cactus", 500_000, 60, 0x51E7E002, modes=(2, 6)),
    "C3": GenConfig("C3-mlperf", 5_000_000, 300, 0x51E7E003, modes=(2, 8)),
    "C4": GenConfig("C4-scaled-mlperf", 100_000_000, 2000, 0x51E7E004, modes=(2, 8)),
    "C5": GenConfig("C5-kde-stress", 1_000_000_000, 2000, 0x51E7E005, t_pct=(30, 30, 40), modes=(5, 20)),
}


def lib_path():
    return os.path.join(_HERE, "libsievegen.so")


def _lib():
    global _LIB
    if _LIB is None:
        p = lib_path()
        if not os.path.exists(p):
            import sys
            sys.path.insert(0, os.path.dirname(_HERE))
            from tools.build_native import build_gen
            build_gen()
        L = ctypes.CDLL(p)
        L.sgen_build.argtypes = [ctypes.POINTER(_Params), ctypes.POINTER(ctypes.c_void_p)]
        L.sgen_build.restype = ctypes.c_int
        L.sgen_free.argtypes = [ctypes.c_void_p]
        L.sgen_fill.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64,
                                ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        L.sgen_kernel_class.argtypes = [ctypes.c_void_p, ctypes.c_uint32]
        L.sgen_kernel_class.restype = ctypes.c_uint32
        _LIB = L
    return _LIB


class Generator:
    """Tables for one config; fill any slice of the trace (counter-based, order-free)."""

    def __init__(self, cfg: GenConfig):
        self.cfg = cfg
        p = _Params(seed=cfg.seed, n_total=cfg.n, K=cfg.K, order=cfg.order,
                    homogeneous=cfg.homogeneous, alt_cta_pct=cfg.alt_cta_pct,
                    t1_pct=cfg.t_pct[0], t2_pct=cfg.t_pct[1], t3_pct=cfg.t_pct[2],
                    t1_kernels=cfg.t_kernels[0], t2_kernels=cfg.t_kernels[1],
                    t3_kernels=cfg.t_kernels[2], m_min=cfg.modes[0], m_max=cfg.modes[1],
                    phase_len_min=cfg.phase_len[0], phase_len_max=cfg.phase_len[1],
                    n_phases=8 + cfg.K // 64, rep_min=cfg.reps[0], rep_max=cfg.reps[1])
        h = ctypes.c_void_p()
        rc = _lib().sgen_build(ctypes.byref(p), ctypes.byref(h))
        if rc != 0:
            raise ValueError(f"sgen_build failed ({rc}) for {cfg}")
        self._h = h

    def __del__(self):
        if getattr(self, "_h", None) and _LIB is not None:
            _LIB.sgen_free(self._h)
            self._h = None

    def fill(self, first=0, n=None, out=None):
        n = self.cfg.n - first if n is None else n
        if out is None:
            out = {"kid": np.empty(n, np.uint32), "x": np.empty(n, np.uint64),
                   "cta": np.empty(n, np.uint32), "y": np.empty(n, np.uint64)}
        ptr = lambda a: None if a is None else a.ctypes.data_as(ctypes.c_void_p)
        _lib().sgen_fill(self._h, first, n, ptr(out["kid"]), ptr(out["x"]), ptr(out["cta"]),
                         ptr(out["y"]))
        return out

    def kernel_class(self, k):
        return _lib().sgen_kernel_class(self._h, k)


def get_config(name, **overrides):
    cfg = CONFIGS[name]
    return replace(cfg, **overrides) if overrides else cfg


def make_trace(name_or_cfg="C1", first=0, n=None, **overrides):
    cfg = name_or_cfg if isinstance(name_or_cfg, GenConfig) else get_config(name_or_cfg, **overrides)
    g = Generator(cfg)
    tr = g.fill(first, n)
    tr["K"] = cfg.K
    tr["first"] = first
    return tr
