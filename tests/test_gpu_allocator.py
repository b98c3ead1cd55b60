"""sieve_ctx_set_allocator (include/sieve.h) with PyTorch's caching allocator as the hook: every
buffer goes back to the allocator that made it, also when the hooks change between calls
(a buffer freed through the wrong allocator corrupts a caching allocator), and the
results stay identical to the oracle's."""
import numpy as np
import pytest

import gen
from tests.gpu_helpers import assert_tables_equal, run_oracle

pytestmark = pytest.mark.gpu


def test_torch_caching_allocator_hooks():
    import torch
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    base_alloc, base_free = sieve.torch_caching_allocator(0)
    live = {}
    calls = {"alloc": 0, "free": 0}

    def alloc(n, stream):
        p = base_alloc(n, stream)
        live[p] = n
        calls["alloc"] += 1
        return p

    def free(p, stream):
        assert p in live, "a buffer was freed through an allocator that did not make it"
        del live[p]
        calls["free"] += 1
        base_free(p, stream)

    tr = gen.make_trace("C1")
    o = run_oracle(tr)
    ctx = sieve.Ctx(device=0)
    ctx.set_allocator(alloc, free)
    t = sieve.load_trace(ctx, tr["kid"], tr["x"], num_kernels=tr["K"], cta=tr["cta"], cycles=tr["y"])
    assert calls["alloc"] >= 4                       # the four owned columns came from the hook
    st = sieve.stratify(t)
    assert_tables_equal(st.table, o.strata)
    sieve.predict(st, t)
    n_hook = calls["alloc"]
    # back to the library's cudaMallocAsync: the hook's arena is released through the hook
    ctx.set_allocator(None, None)
    st2 = sieve.stratify(t)
    assert calls["alloc"] == n_hook
    assert_tables_equal(st2.table, o.strata)
    # the trace's columns still belong to the hook
    t.close()
    st.close(); st2.close()
    ctx.close()
    torch.cuda.synchronize()
    assert not live, f"{len(live)} hook buffers never freed"
    assert calls["alloc"] == calls["free"]
    # and a trace loaded under the default allocator, freed after the hook is set again, goes
    # back to cudaFreeAsync (the hook never sees it)
    ctx = sieve.Ctx(device=0)
    t = sieve.load_trace(ctx, tr["kid"], tr["x"], num_kernels=tr["K"])
    ctx.set_allocator(alloc, free)
    before = dict(calls)
    t.close()
    ctx.close()
    assert calls["free"] == before["free"] and not live
