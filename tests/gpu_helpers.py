"""Shared helpers of the GPU parity tests: run the CUDA path through the C-ABI binding and
compare it with the CPU oracle field by field."""
import math

import numpy as np

EXACT_FIELDS = ["kernel_id", "tier", "index_in_kernel", "rep_cta", "lo", "hi", "count",
                "instr_sum_lo", "instr_sum_hi", "rep_id", "rep_instr", "rep_cycles", "split_round"]


def run_gpu(tr, K=None, G=1024, theta=(2, 5), keep_debug=False, with_sid=True, cta=True,
            cycles=True, device_cols=False, **kw):
    import torch
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    K = tr["K"] if K is None else K
    ctx = sieve.Ctx(device=0)
    cols = dict(kernel_id=tr["kid"], instr=tr["x"], cta=tr["cta"] if cta else None,
                cycles=tr["y"] if cycles else None)
    if device_cols:
        cols = {k: (None if v is None else torch.from_numpy(v.view(np.int64 if v.dtype == np.uint64 else np.int32)).cuda())
                for k, v in cols.items()}
    trace = sieve.load_trace(ctx, num_kernels=K, **cols)
    n = len(tr["kid"])
    sid = torch.empty(max(n, 1), dtype=torch.int32, device="cuda") if with_sid else None
    st = sieve.stratify(trace, stratum_of_invocation=sid, theta=theta, grid_points=G,
                        keep_debug=1 if keep_debug else 0, **kw)
    out = {"table": st.table, "rounds": st.rounds, "terms": st.kde_terms, "strata": st,
           "trace": trace, "ctx": ctx}
    if with_sid:
        torch.cuda.synchronize()
        out["sid"] = sid[:n].cpu().numpy().view(np.uint32)
    if keep_debug:
        out["segments"] = st.segments(G)
    return out


def run_oracle(tr, K=None, G=1024, theta=(2, 5), keep_debug=False, cta=True, cycles=True, **kw):
    import oracle
    K = tr["K"] if K is None else K
    return oracle.stratify(tr["kid"], tr["x"], K, tr["cta"] if cta else None,
                           tr["y"] if cycles else None, theta=theta, G=G, keep_debug=keep_debug, **kw)


def assert_tables_equal(gpu_table, ora_table):
    assert len(gpu_table) == len(ora_table), (len(gpu_table), len(ora_table))
    for f in EXACT_FIELDS:
        a, b = gpu_table[f], ora_table[f]
        if not np.array_equal(a, b):
            bad = np.nonzero(a != b)[0][:5]
            raise AssertionError(f"field {f} differs at strata {bad.tolist()}: gpu {a[bad].tolist()} "
                                 f"oracle {b[bad].tolist()}")
    # bandwidth h: bit-identical (computed on the host by both sides from exact moments)
    assert np.array_equal(gpu_table["bandwidth"].view(np.uint64), ora_table["bandwidth"].view(np.uint64))


def assert_segments_equal(gs, os_):
    # the library lists segments round by round; the oracle kernel by kernel: compare in
    # (round, kernel, lo) order
    key = lambda s: (s["round"], s["kernel_id"], s["lo"])
    gs, os_ = sorted(gs, key=key), sorted(os_, key=key)
    assert len(gs) == len(os_)
    for a, b in zip(gs, os_):
        for k in ["kernel_id", "round", "split_kind", "n_cuts", "lo", "hi", "count"]:
            assert a[k] == b[k], (k, a[k], b[k])
        assert a["bandwidth"] == b["bandwidth"]
        assert np.array_equal(a["d_lo"], b["d_lo"]) and np.array_equal(a["d_hi"], b["d_hi"])
        assert np.array_equal(a["cuts"], b["cuts"])


def assert_predictions_close(p, q, rel=1e-9):
    for k in ["predicted_cycles", "predicted_ipc", "measured_cycles", "speedup"]:
        if math.isnan(q[k]):
            assert math.isnan(p[k]), k
        else:
            assert math.isclose(p[k], q[k], rel_tol=rel), (k, p[k], q[k])
    if math.isnan(q["error"]):
        assert math.isnan(p["error"])
    else:
        # error is a difference of two large numbers: compare in units of C_meas
        assert abs(p["error"] - q["error"]) <= rel * max(1.0, q["predicted_cycles"] / q["measured_cycles"])
    assert p["total_instr"] == q["total_instr"]
