"""Thin Python binding of libsieve.so (include/sieve.h): argument marshalling only.

Every step of the stratification path runs in the library's sm_100a kernels.  PyTorch is used
only for device memory (tensors), streams and process groups (the NCCL unique-id exchange).
There is no CPU fallback: if libsieve.so is missing or cannot load, importing this module raises.

    import paper_conf_ispass_naderantahanse23_b200 as sieve
    ctx = sieve.Ctx(device=0)
    tr = sieve.load_trace(ctx, kid, x, num_kernels=K, cta=cta, cycles=y)   # numpy or CUDA tensors
    st = sieve.stratify(tr)                 # -> Strata; st.table is a numpy structured array
    pred = sieve.predict(st, tr)            # dict: predicted_cycles, predicted_ipc, error, ...
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# SIEVE_LIB_PATH: an alternative build of the same library (A/B measurements of kernel variants)
LIB_PATH = os.environ.get("SIEVE_LIB_PATH") or os.path.join(_HERE, "libsieve.so")

SIEVE_OK, SIEVE_EINVAL, SIEVE_ERANGE, SIEVE_ENOMEM = 0, -1, -2, -3
SIEVE_ECUDA, SIEVE_ENCCL, SIEVE_EDOM, SIEVE_ELIMIT, SIEVE_ESTATE = -4, -5, -6, -7, -8
MEM_HOST, MEM_DEVICE, ADOPT, KID16, CTA16 = 0, 1, 2, 4, 8

STRATUM_DTYPE = np.dtype([
    ("kernel_id", "<u4"), ("tier", "<u4"), ("index_in_kernel", "<u4"), ("rep_cta", "<u4"),
    ("lo", "<u8"), ("hi", "<u8"), ("count", "<u8"), ("instr_sum_lo", "<u8"), ("instr_sum_hi", "<u8"),
    ("rep_id", "<u8"), ("rep_instr", "<u8"), ("rep_cycles", "<u8"), ("bandwidth", "<f8"),
    ("split_round", "<u4"), ("pad", "<u4")])

EXPORTED = [
    "sieve_get_unique_id", "sieve_ctx_create", "sieve_group_create", "sieve_group_destroy",
    "sieve_ctx_create_in_group", "sieve_ctx_set_allocator", "sieve_ctx_destroy",
    "sieve_load_trace", "sieve_trace_free", "sieve_params_default", "sieve_stratify",
    "sieve_strata_count", "sieve_strata_copy", "sieve_strata_stats", "sieve_strata_free",
    "sieve_segment_count", "sieve_segment_get", "sieve_predict", "sieve_last_error",
    "sieve_version", "sieve_u128_to_limbs", "sieve_limbs_to_u128", "sieve_ctx_set_timing",
    "sieve_ctx_set_term_count",
    "sieve_timing_get", "sieve_kernel_launches", "sieve_stratify_sweep", "sieve_tier_census",
    "sieve_predict_multi", "sieve_cycle_cov", "sieve_load_csv", "sieve_trace_copy",
    "sieve_trace_kernel_names", "sieve_min_strata",
]
PHASES = ["moments", "compact", "sort", "kde_plan", "kde", "refine", "assign", "reps", "predict"]


class Params(ctypes.Structure):
    _fields_ = [("theta_num", ctypes.c_uint32), ("theta_den", ctypes.c_uint32),
                ("grid_points", ctypes.c_uint32), ("valley_shift", ctypes.c_uint32),
                ("max_rounds", ctypes.c_uint32), ("keep_debug", ctypes.c_uint32),
                ("bw_scale", ctypes.c_double)]


class _Segment(ctypes.Structure):
    _fields_ = [("kernel_id", ctypes.c_uint32), ("round", ctypes.c_uint32),
                ("split_kind", ctypes.c_uint32), ("n_cuts", ctypes.c_uint32),
                ("lo", ctypes.c_uint64), ("hi", ctypes.c_uint64), ("count", ctypes.c_uint64),
                ("bandwidth", ctypes.c_double)]


class _Prediction(ctypes.Structure):
    _fields_ = [("predicted_cycles", ctypes.c_double), ("predicted_ipc", ctypes.c_double),
                ("measured_cycles", ctypes.c_double), ("error", ctypes.c_double),
                ("speedup", ctypes.c_double), ("total_instr_lo", ctypes.c_uint64),
                ("total_instr_hi", ctypes.c_uint64)]


class CsvSpec(ctypes.Structure):
    _fields_ = [("col_kernel", ctypes.c_int32), ("col_instr", ctypes.c_int32),
                ("col_cta", ctypes.c_int32), ("col_cycles", ctypes.c_int32),
                ("header_lines", ctypes.c_uint32), ("delimiter", ctypes.c_char)]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; "
                          "g.build()'` (no CPU fallback exists)")
    L = ctypes.CDLL(LIB_PATH, mode=ctypes.RTLD_GLOBAL)
    vp, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    P = ctypes.POINTER
    sig = {
        "sieve_get_unique_id": ([vp], i32),
        "sieve_ctx_create": ([i32, vp, i32, i32, vp, P(vp)], i32),
        "sieve_group_create": ([i32, P(vp)], i32),
        "sieve_group_destroy": ([vp], None),
        "sieve_ctx_create_in_group": ([i32, vp, vp, i32, P(vp)], i32),
        "sieve_ctx_set_allocator": ([vp, vp, vp, vp], i32),
        "sieve_ctx_destroy": ([vp], None),
        "sieve_load_trace": ([vp, u64, u64, u32, vp, vp, vp, vp, u32, P(vp)], i32),
        "sieve_trace_free": ([vp], None),
        "sieve_params_default": ([P(Params)], None),
        "sieve_stratify": ([vp, P(Params), vp, P(vp)], i32),
        "sieve_strata_count": ([vp, P(u64)], i32),
        "sieve_strata_copy": ([vp, vp, u64], i32),
        "sieve_strata_stats": ([vp, P(u32), P(u64), P(u64)], i32),
        "sieve_strata_free": ([vp], None),
        "sieve_segment_count": ([vp, P(u64)], i32),
        "sieve_segment_get": ([vp, u64, P(_Segment), vp, vp, vp], i32),
        "sieve_predict": ([vp, vp, vp, P(_Prediction)], i32),
        "sieve_last_error": ([], ctypes.c_char_p),
        "sieve_version": ([], ctypes.c_char_p),
        "sieve_u128_to_limbs": ([u64, u64, vp], None),
        "sieve_limbs_to_u128": ([vp, P(u64), P(u64)], None),
        "sieve_ctx_set_timing": ([vp, i32], i32),
        "sieve_ctx_set_term_count": ([vp, i32], i32),
        "sieve_timing_get": ([vp, u32, P(ctypes.c_double), P(u64), P(u64)], i32),
        "sieve_kernel_launches": ([], u64),
        "sieve_stratify_sweep": ([vp, P(Params), u32, vp, vp, vp], i32),
        "sieve_tier_census": ([vp, u32, vp, vp, vp, vp, vp], i32),
        "sieve_predict_multi": ([vp, vp, u32, vp, P(_Prediction)], i32),
        "sieve_cycle_cov": ([vp, vp, vp, vp, P(ctypes.c_double)], i32),
        "sieve_load_csv": ([vp, vp, u64, u32, P(CsvSpec), u64, P(vp), P(u32)], i32),
        "sieve_trace_copy": ([vp, vp, vp, vp, vp, P(u64), P(u32)], i32),
        "sieve_trace_kernel_names": ([vp, vp, u64, P(u64)], i32),
        "sieve_min_strata": ([vp, u32, u32, u32, vp, vp, u64, P(u64)], i32),
    }
    for name, (args, res) in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = res
    return L


_L = _load()


class SieveError(RuntimeError):
    def __init__(self, code, where):
        msg = _L.sieve_last_error().decode(errors="replace")
        super().__init__(f"{where} failed with status {code}: {msg}")
        self.code = code


def _check(code, where):
    if code != SIEVE_OK:
        raise SieveError(code, where)


def version():
    return _L.sieve_version().decode()


def u128_to_limbs(v):
    out = (ctypes.c_uint64 * 4)()
    _L.sieve_u128_to_limbs(v & ((1 << 64) - 1), v >> 64, out)
    return list(out)


def limbs_to_u128(limbs):
    arr = (ctypes.c_uint64 * 4)(*[int(l) for l in limbs])
    lo, hi = ctypes.c_uint64(), ctypes.c_uint64()
    _L.sieve_limbs_to_u128(arr, ctypes.byref(lo), ctypes.byref(hi))
    return (hi.value << 64) | lo.value


def get_unique_id():
    buf = (ctypes.c_uint8 * 128)()
    _check(_L.sieve_get_unique_id(buf), "sieve_get_unique_id")
    return bytes(buf)


def _stream_handle(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


class Group:
    """In-process rank group: `world` threads share one GPU (multi-rank parity tests)."""

    def __init__(self, world):
        h = ctypes.c_void_p()
        _check(_L.sieve_group_create(world, ctypes.byref(h)), "sieve_group_create")
        self._h = h
        self.world = world

    def __del__(self):
        if getattr(self, "_h", None):
            _L.sieve_group_destroy(self._h)
            self._h = None


class Ctx:
    """sieve_ctx: device, stream and (world > 1) an NCCL communicator."""

    def __init__(self, device=0, stream=None, rank=0, world=1, nccl_id=None, group=None):
        h = ctypes.c_void_p()
        sh = _stream_handle(stream)
        if group is not None:
            _check(_L.sieve_ctx_create_in_group(device, sh, group._h, rank, ctypes.byref(h)),
                   "sieve_ctx_create_in_group")
        else:
            idbuf = None if nccl_id is None else (ctypes.c_uint8 * 128)(*nccl_id)
            _check(_L.sieve_ctx_create(device, sh, rank, world, idbuf, ctypes.byref(h)),
                   "sieve_ctx_create")
        self._h = h
        self.device, self.rank, self.world = device, rank, world if group is None else group.world
        self._group = group

    def set_allocator(self, alloc=None, free=None):
        """sieve_ctx_set_allocator: alloc(nbytes, stream_handle) -> device pointer (int) and
        free(ptr, stream_handle), e.g. torch_caching_allocator(); None, None restores the
        library's cudaMallocAsync.  Buffers are always released by the allocator that made them."""
        if (alloc is None) != (free is None):
            raise ValueError("alloc and free must both be given or both be None")
        if alloc is None:
            self._hooks = None
            _check(_L.sieve_ctx_set_allocator(self._h, None, None, None), "sieve_ctx_set_allocator")
            return

        def _a(nbytes, stream, user):
            try:
                return int(alloc(int(nbytes), stream or 0)) or None
            except Exception:  # the library reports SIEVE_ENOMEM for a NULL result
                return None

        def _f(ptr, stream, user):
            free(int(ptr), stream or 0)

        a, f = _ALLOC_FN(_a), _FREE_FN(_f)
        # the hooks must outlive every buffer they made: keep them with the context (and with
        # any trace created while they were set, see load_trace)
        self._hooks_live = getattr(self, "_hooks_live", []) + [(a, f)]
        self._hooks = (a, f)
        _check(_L.sieve_ctx_set_allocator(self._h, ctypes.cast(a, ctypes.c_void_p),
                                          ctypes.cast(f, ctypes.c_void_p), None), "sieve_ctx_set_allocator")

    def set_term_count(self, enable=True):
        """In-window KDE term counting (strata.kde_terms); on by default."""
        _check(_L.sieve_ctx_set_term_count(self._h, 1 if enable else 0), "sieve_ctx_set_term_count")

    def set_timing(self, enable=True):
        _check(_L.sieve_ctx_set_timing(self._h, 1 if enable else 0), "sieve_ctx_set_timing")

    def timing(self):
        """{phase: (ms, calls, work)} accumulated since set_timing(True)."""
        out = {}
        for i, name in enumerate(PHASES):
            ms, calls, work = ctypes.c_double(), ctypes.c_uint64(), ctypes.c_uint64()
            _check(_L.sieve_timing_get(self._h, i, ctypes.byref(ms), ctypes.byref(calls),
                                       ctypes.byref(work)), "sieve_timing_get")
            out[name] = (ms.value, calls.value, work.value)
        return out

    def close(self):
        if getattr(self, "_h", None):
            _L.sieve_ctx_destroy(self._h)
            self._h = None

    def __del__(self):
        self.close()


_ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
_FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p)


def torch_caching_allocator(device=0):
    """(alloc, free) hooks that take device memory from PyTorch's caching allocator."""
    import torch

    def alloc(nbytes, stream):
        return torch.cuda.caching_allocator_alloc(nbytes, device, stream)

    def free(ptr, stream):
        torch.cuda.caching_allocator_delete(ptr)

    return alloc, free


def kernel_launches():
    return _L.sieve_kernel_launches()


def _is16(a):
    """a 16-bit column (numpy uint16 / torch uint16, int16): loaded with SIEVE_KID16 / CTA16"""
    if isinstance(a, np.ndarray):
        return a.dtype == np.uint16
    try:
        import torch
        return isinstance(a, torch.Tensor) and a.dtype in (torch.uint16, torch.int16)
    except ImportError:
        return False


def _col(a, dtype, device_ok=True):
    """(pointer, is_device, keepalive) for a numpy array or a CUDA tensor."""
    if a is None:
        return None, None, None
    if isinstance(a, np.ndarray):
        a = np.ascontiguousarray(a, dtype)
        return a.ctypes.data_as(ctypes.c_void_p), False, a
    import torch
    if isinstance(a, torch.Tensor):
        want = {np.uint32: (torch.uint32, torch.int32), np.uint64: (torch.uint64, torch.int64),
                np.uint16: (torch.uint16, torch.int16)}[dtype]
        if a.dtype not in want:
            raise TypeError(f"tensor dtype {a.dtype} does not match {np.dtype(dtype)}")
        if not a.is_contiguous():
            raise ValueError("tensor must be contiguous")
        if a.is_cuda:
            return ctypes.c_void_p(a.data_ptr()), True, a
        return ctypes.c_void_p(a.data_ptr()), False, a
    raise TypeError(f"unsupported column type {type(a)}")


class Trace:
    def __init__(self, h, ctx, n, keep, num_kernels=None):
        self._h, self.ctx, self.n, self._keep = h, ctx, n, keep
        self.num_kernels = num_kernels

    def close(self):
        if getattr(self, "_h", None):
            _L.sieve_trace_free(self._h)
            self._h = None

    def __del__(self):
        self.close()


def load_trace(ctx, kernel_id, instr, num_kernels, cta=None, cycles=None, first_id=0, adopt=False):
    """sieve_load_trace: columns as numpy arrays (host, copied H2D) or CUDA tensors (device).
    kernel_id / cta may be 16-bit (uint16): half the bytes copied, widened on the device."""
    k16, c16 = _is16(kernel_id), cta is not None and _is16(cta)
    cols = [_col(kernel_id, np.uint16 if k16 else np.uint32), _col(instr, np.uint64),
            _col(cta, np.uint16 if c16 else np.uint32), _col(cycles, np.uint64)]
    kinds = {c[1] for c in cols if c[1] is not None}
    if len(kinds) > 1:
        raise ValueError("all columns must be on the same side (host or device)")
    on_dev = kinds == {True}
    mem = (MEM_DEVICE if on_dev else MEM_HOST) | (ADOPT if adopt else 0) | (KID16 if k16 else 0) | \
        (CTA16 if c16 else 0)
    n = len(kernel_id)
    for name, c in zip(("instr", "cta", "cycles"), (instr, cta, cycles)):
        if c is not None and len(c) != n:  # the library reads n rows of every column
            raise ValueError(f"{name} has {len(c)} rows, kernel_id has {n}")
    if on_dev:
        import torch
        devs = {c[2].device.index for c in cols if c[2] is not None}
        if devs != {ctx.device}:
            raise ValueError(f"device columns must live on cuda:{ctx.device}")
    h = ctypes.c_void_p()
    _check(_L.sieve_load_trace(ctx._h, n, first_id, num_kernels, cols[0][0], cols[1][0], cols[2][0],
                               cols[3][0], mem, ctypes.byref(h)), "sieve_load_trace")
    t = Trace(h, ctx, n, [c[2] for c in cols] if adopt else None, num_kernels)
    t._hooks = getattr(ctx, "_hooks", None)  # the allocator that owns the copied columns
    return t


def load_csv(ctx, data, col_kernel, col_instr, col_cta=-1, col_cycles=-1, header_lines=1,
             delimiter=",", first_id=0):
    """sieve_load_csv: `data` is the CSV text (bytes / str on the host, or a CUDA uint8 tensor).
    Returns (Trace, names) with names[i] the kernel name of id i (first-appearance order)."""
    spec = CsvSpec(col_kernel, col_instr, col_cta, col_cycles, header_lines, delimiter.encode())
    keep = None
    if isinstance(data, str):
        data = data.encode()
    if isinstance(data, bytes):   # the bytes object's own buffer (no copy); kept alive below
        keep = data
        ptr, nbytes, mem = ctypes.cast(ctypes.c_char_p(data), ctypes.c_void_p), len(data), MEM_HOST
    elif isinstance(data, bytearray):
        keep = (ctypes.c_char * len(data)).from_buffer(data) if len(data) else None
        ptr = ctypes.cast(keep, ctypes.c_void_p) if keep is not None else ctypes.c_void_p(None)
        nbytes, mem = len(data), MEM_HOST
    else:
        import torch
        if not (isinstance(data, torch.Tensor) and data.is_cuda and data.dtype == torch.uint8):
            raise TypeError("data must be bytes, str or a CUDA uint8 tensor")
        ptr, nbytes, mem = ctypes.c_void_p(data.data_ptr()), data.numel(), MEM_DEVICE
    h, nk = ctypes.c_void_p(), ctypes.c_uint32()
    _check(_L.sieve_load_csv(ctx._h, ptr, nbytes, mem, ctypes.byref(spec), first_id, ctypes.byref(h),
                             ctypes.byref(nk)), "sieve_load_csv")
    n, kk = ctypes.c_uint64(), ctypes.c_uint32()
    _check(_L.sieve_trace_copy(h, None, None, None, None, ctypes.byref(n), ctypes.byref(kk)), "sieve_trace_copy")
    t = Trace(h, ctx, n.value, None, kk.value)
    need = ctypes.c_uint64()
    _check(_L.sieve_trace_kernel_names(h, None, 0, ctypes.byref(need)), "sieve_trace_kernel_names")
    buf = ctypes.create_string_buffer(max(1, need.value))
    _check(_L.sieve_trace_kernel_names(h, buf, need.value, ctypes.byref(need)), "sieve_trace_kernel_names")
    names = buf.raw[:need.value].decode(errors="replace").split("\n")[:-1] if need.value else []
    assert len(names) == nk.value
    t.names = names
    return t, names


def min_strata(trace, theta=(2, 5), max_distinct=0, num_kernels=None):
    """sieve_min_strata (NEXT-3): exact minimum strata per kernel and the canonical optimal
    cuts -> (counts uint32[K], list of per-kernel cut lists)."""
    K = num_kernels if num_kernels is not None else trace.num_kernels
    counts = np.zeros(K, np.uint32)
    nc = ctypes.c_uint64()
    cp = counts.ctypes.data_as(ctypes.c_void_p)
    _check(_L.sieve_min_strata(trace._h, theta[0], theta[1], max_distinct, cp, None, 0, ctypes.byref(nc)),
           "sieve_min_strata")
    cuts = np.zeros(max(1, nc.value), np.uint64)
    _check(_L.sieve_min_strata(trace._h, theta[0], theta[1], max_distinct, cp,
                               cuts.ctypes.data_as(ctypes.c_void_p), nc.value, ctypes.byref(nc)),
           "sieve_min_strata")
    per, o = [], 0
    for c in counts.tolist():
        k = c - 1 if 2 <= c < 0xFFFFFFFF else 0
        per.append([int(v) for v in cuts[o:o + k]])
        o += k
    return counts, per


def trace_columns(trace, cta=True, cycles=True):
    """sieve_trace_copy: the trace's columns as host numpy arrays (kid, x, cta|None, y|None)."""
    n = trace.n
    kid, x = np.zeros(n, np.uint32), np.zeros(n, np.uint64)
    c = np.zeros(n, np.uint32) if cta else None
    y = np.zeros(n, np.uint64) if cycles else None
    ptr = lambda a: None if a is None else a.ctypes.data_as(ctypes.c_void_p)
    _check(_L.sieve_trace_copy(trace._h, ptr(kid), ptr(x), ptr(c), ptr(y), None, None), "sieve_trace_copy")
    return kid, x, c, y


def default_params(**kw):
    p = Params()
    _L.sieve_params_default(ctypes.byref(p))
    if "theta" in kw:
        p.theta_num, p.theta_den = kw.pop("theta")
    for k, v in kw.items():
        setattr(p, k, v)
    return p


class Strata:
    def __init__(self, h):
        self._h = h
        n = ctypes.c_uint64()
        _check(_L.sieve_strata_count(h, ctypes.byref(n)), "sieve_strata_count")
        self._n = n.value
        self._table = None   # copied out on first use (sieve_strata_copy)
        r, t, ev = ctypes.c_uint32(), ctypes.c_uint64(), ctypes.c_uint64()
        _check(_L.sieve_strata_stats(h, ctypes.byref(r), ctypes.byref(t), ctypes.byref(ev)),
               "sieve_strata_stats")
        self.rounds, self.kde_terms, self.kde_evaluated = r.value, t.value, ev.value

    @property
    def table(self):
        """the stratum table (numpy structured array, STRATUM_DTYPE), copied on first access"""
        if self._table is None:
            tab = np.zeros(self._n, STRATUM_DTYPE)
            if self._n:
                _check(_L.sieve_strata_copy(self._h, tab.ctypes.data_as(ctypes.c_void_p), self._n),
                       "sieve_strata_copy")
            self._table = tab
        return self._table

    def __len__(self):
        return self._n

    def segments(self, G):
        n = ctypes.c_uint64()
        _check(_L.sieve_segment_count(self._h, ctypes.byref(n)), "sieve_segment_count")
        out = []
        for i in range(n.value):
            m = _Segment()
            _check(_L.sieve_segment_get(self._h, i, ctypes.byref(m), None, None, None), "sieve_segment_get")
            dlo = np.zeros(G, np.uint64)
            dhi = np.zeros(G, np.uint64)
            cuts = np.zeros(m.n_cuts, np.uint64)
            _check(_L.sieve_segment_get(self._h, i, ctypes.byref(m), dlo.ctypes.data_as(ctypes.c_void_p),
                                        dhi.ctypes.data_as(ctypes.c_void_p),
                                        cuts.ctypes.data_as(ctypes.c_void_p)), "sieve_segment_get")
            out.append({"kernel_id": m.kernel_id, "round": m.round, "split_kind": m.split_kind,
                        "n_cuts": m.n_cuts, "lo": m.lo, "hi": m.hi, "count": m.count,
                        "bandwidth": m.bandwidth, "d_lo": dlo, "d_hi": dhi, "cuts": cuts})
        return out

    def close(self):
        if getattr(self, "_h", None):
            _L.sieve_strata_free(self._h)
            self._h = None

    def __del__(self):
        self.close()


_SID_OK = {}   # (id, data_ptr, numel, dtype, id(trace), n) of the last tensor that passed _check_sid


def _check_sid(t, trace):
    """stratum ids are written / read by the kernels as a DEVICE uint32 array of n_local entries"""
    import torch
    if not isinstance(t, torch.Tensor):
        raise TypeError("stratum_of_invocation must be a contiguous CUDA int32/uint32 tensor")
    key = (id(t), t.data_ptr(), t.numel(), t.dtype, id(trace), trace.n)
    if _SID_OK.get("key") == key:   # the same tensor as last call (a bench or training loop)
        return
    if not (t.is_cuda and t.dtype in (torch.int32, torch.uint32) and t.is_contiguous()):
        raise TypeError("stratum_of_invocation must be a contiguous CUDA int32/uint32 tensor")
    if t.numel() < trace.n:
        raise ValueError(f"stratum_of_invocation has {t.numel()} entries, the trace {trace.n}")
    if t.device.index != trace.ctx.device:
        raise ValueError(f"stratum_of_invocation must live on cuda:{trace.ctx.device}")
    _SID_OK["key"] = key


_DEFAULT_PARAMS = []   # one default sieve_params, built on first use (the library only reads it)


def stratify(trace, params=None, stratum_of_invocation=None, **kw):
    """sieve_stratify; stratum_of_invocation: optional CUDA int32/uint32 tensor [n_local]."""
    if params is None and not kw:
        if not _DEFAULT_PARAMS:
            _DEFAULT_PARAMS.append(default_params())
        p = _DEFAULT_PARAMS[0]
    else:
        p = params if params is not None else default_params(**kw)
    sid_ptr = None
    if stratum_of_invocation is not None:
        _check_sid(stratum_of_invocation, trace)
        sid_ptr = ctypes.c_void_p(stratum_of_invocation.data_ptr())
    h = ctypes.c_void_p()
    _check(_L.sieve_stratify(trace._h, ctypes.byref(p), sid_ptr, ctypes.byref(h)), "sieve_stratify")
    return Strata(h)


def _thetas(thetas):
    num = np.ascontiguousarray([t[0] for t in thetas], np.uint32)
    den = np.ascontiguousarray([t[1] for t in thetas], np.uint32)
    return num, den


def stratify_sweep(trace, thetas, params=None, **kw):
    """sieve_stratify_sweep: one Strata per theta (num, den), pass A computed once."""
    p = params if params is not None else default_params(**kw)
    num, den = _thetas(thetas)
    hs = (ctypes.c_void_p * len(thetas))()
    _check(_L.sieve_stratify_sweep(trace._h, ctypes.byref(p), len(thetas),
                                   num.ctypes.data_as(ctypes.c_void_p),
                                   den.ctypes.data_as(ctypes.c_void_p), hs), "sieve_stratify_sweep")
    return [Strata(ctypes.c_void_p(h)) for h in hs]


def tier_census(trace, thetas):
    """sieve_tier_census: per theta, (kernels[3], invocations[3], instructions[3]) per tier."""
    num, den = _thetas(thetas)
    k = np.zeros((len(thetas), 3), np.uint64)
    inv = np.zeros((len(thetas), 3), np.uint64)
    ins = np.zeros((len(thetas), 3, 2), np.uint64)
    _check(_L.sieve_tier_census(trace._h, len(thetas), num.ctypes.data_as(ctypes.c_void_p),
                                den.ctypes.data_as(ctypes.c_void_p), k.ctypes.data_as(ctypes.c_void_p),
                                inv.ctypes.data_as(ctypes.c_void_p), ins.ctypes.data_as(ctypes.c_void_p)),
           "sieve_tier_census")
    instr = [[(int(ins[i, j, 1]) << 64) | int(ins[i, j, 0]) for j in range(3)] for i in range(len(thetas))]
    return k, inv, instr


def _pred_dict(out):
    return {"predicted_cycles": out.predicted_cycles, "predicted_ipc": out.predicted_ipc,
            "measured_cycles": out.measured_cycles, "error": out.error, "speedup": out.speedup,
            "total_instr": (out.total_instr_hi << 64) | out.total_instr_lo}


def predict_multi(strata, trace, rep_cycles):
    """sieve_predict_multi: rep_cycles [M][n_strata] (one row per architecture) -> M dicts."""
    rc = np.ascontiguousarray(rep_cycles, np.uint64)
    if rc.ndim != 2 or rc.shape[1] != len(strata):
        raise ValueError("rep_cycles must be [M][n_strata]")
    outs = (_Prediction * rc.shape[0])()
    _check(_L.sieve_predict_multi(strata._h, trace._h, rc.shape[0], rc.ctypes.data_as(ctypes.c_void_p),
                                  outs), "sieve_predict_multi")
    return [_pred_dict(o) for o in outs]


def cycle_cov(strata, trace, stratum_of_invocation):
    """sieve_cycle_cov: per-stratum CoV of member cycles + instruction-weighted mean (Fig. 4)."""
    _check_sid(stratum_of_invocation, trace)
    cov = np.zeros(len(strata), np.float64)
    w = ctypes.c_double()
    _check(_L.sieve_cycle_cov(strata._h, trace._h, ctypes.c_void_p(stratum_of_invocation.data_ptr()),
                              cov.ctypes.data_as(ctypes.c_void_p), ctypes.byref(w)), "sieve_cycle_cov")
    return cov, w.value


def predict(strata, trace, rep_cycles=None):
    out = _Prediction()
    rc = None
    if rep_cycles is not None:
        rc = np.ascontiguousarray(rep_cycles, np.uint64)
        if rc.ndim != 1 or len(rc) != len(strata):  # the library reads n_strata values
            raise ValueError(f"rep_cycles must have one entry per stratum ({len(strata)})")
    _check(_L.sieve_predict(strata._h, trace._h, None if rc is None else rc.ctypes.data_as(ctypes.c_void_p),
                            ctypes.byref(out)), "sieve_predict")
    return {"predicted_cycles": out.predicted_cycles, "predicted_ipc": out.predicted_ipc,
            "measured_cycles": out.measured_cycles, "error": out.error, "speedup": out.speedup,
            "total_instr": (out.total_instr_hi << 64) | out.total_instr_lo}
