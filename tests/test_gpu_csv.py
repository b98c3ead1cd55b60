"""NEXT-4: profile CSV ingest on the GPU (sieve_load_csv) against the CPU oracle
parse (oracle/csv_ingest.py, reading A27).  Every parsed
column and the interned names must be bit-exact; a CSV-loaded trace stratifies exactly like the
oracle run on the oracle-parsed columns."""
import json
import os

import numpy as np
import pytest

import gen
from oracle import csv_ingest
from tests.gpu_helpers import assert_tables_equal

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _gpu(text, **spec):
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    ctx = sieve.Ctx(device=0)
    t, names = sieve.load_csv(ctx, text, **spec)
    kid, x, cta, y = sieve.trace_columns(t, cta=spec.get("col_cta", -1) >= 0,
                                         cycles=spec.get("col_cycles", -1) >= 0)
    return ctx, t, kid, x, cta, y, names


def _same(got, exp):
    kid, x, cta, y, names = exp
    assert got[2].tolist() == kid
    assert got[3].tolist() == x
    assert (got[4] is None and cta is None) or got[4].tolist() == cta
    assert (got[5] is None and y is None) or got[5].tolist() == y
    assert got[6] == names


def test_golden_small_csv():
    with open(os.path.join(GOLD, "csv_small.csv"), newline="") as f:
        text = f.read()
    with open(os.path.join(GOLD, "csv_small.expected.json")) as f:
        exp = json.load(f)
    got = _gpu(text, **exp["spec"])
    _same(got, (exp["kernel_id"], exp["instr"], exp["cta"], exp["cycles"], exp["names"]))


def _csv_of(name, n, delim=",", thousands=False, crlf=False, trailing=True):
    t = gen.make_trace(name, 0, n)
    K = t["K"]
    names = [f"void k{k}<{k % 7}, 128>(float const*, {delim} int)" for k in range(K)]
    text = csv_ingest.write(t["kid"], t["x"], t["cta"], t["y"], names, delimiter=delim,
                            thousands=thousands, crlf=crlf, trailing=trailing,
                            header=delim.join(["ID", "Kernel Name", "Instructions", "CTAs", "Cycles"]))
    return t, text


@pytest.mark.parametrize("name,n,delim,thousands,crlf,trailing", [
    ("C1", None, ",", False, False, True), ("C1", None, ",", True, True, False),
    ("C1", 777, ";", True, False, True), ("C1", 4097, "\t", False, True, False),
    ("C2", None, ",", True, False, True)])
def test_parse_matches_oracle(name, n, delim, thousands, crlf, trailing):
    t, text = _csv_of(name, n, delim, thousands, crlf, trailing)
    spec = dict(col_kernel=1, col_instr=2, col_cta=3, col_cycles=4, header_lines=1, delimiter=delim)
    _same(_gpu(text, **spec), csv_ingest.parse(text, 1, 2, 3, 4, 1, delim))


def test_column_subsets_and_order():
    t, text = _csv_of("C1", 5000)
    for spec in [dict(col_kernel=1, col_instr=4), dict(col_kernel=1, col_instr=2, col_cta=3),
                 dict(col_kernel=3, col_instr=0, col_cycles=2, header_lines=3)]:
        exp = csv_ingest.parse(text, spec["col_kernel"], spec["col_instr"], spec.get("col_cta", -1),
                               spec.get("col_cycles", -1), spec.get("header_lines", 1))
        _same(_gpu(text, **spec), exp)


def test_device_resident_text():
    import torch
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    t, text = _csv_of("C1", 3000, thousands=True)
    dev = torch.frombuffer(bytearray(text.encode()), dtype=torch.uint8).cuda()
    ctx = sieve.Ctx(device=0)
    tr, names = sieve.load_csv(ctx, dev, 1, 2, 3, 4)
    kid, x, cta, y = sieve.trace_columns(tr)
    exp = csv_ingest.parse(text, 1, 2, 3, 4)
    assert kid.tolist() == exp[0] and x.tolist() == exp[1] and cta.tolist() == exp[2]
    assert y.tolist() == exp[3] and names == exp[4]


@pytest.mark.parametrize("name", ["C1", "C2"])
def test_csv_trace_stratifies_like_oracle(name):
    import oracle
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    t, text = _csv_of(name, None)
    kid, x, cta, y, names = csv_ingest.parse(text, 1, 2, 3, 4)
    ctx = sieve.Ctx(device=0)
    tr, gnames = sieve.load_csv(ctx, text, 1, 2, 3, 4)
    st = sieve.stratify(tr, theta=(2, 5), grid_points=1024)
    o = oracle.stratify(np.array(kid, np.uint32), np.array(x, np.uint64), len(names),
                        np.array(cta, np.uint32), np.array(y, np.uint64), theta=(2, 5), G=1024)
    assert_tables_equal(st.table, o.strata)


@pytest.mark.parametrize("text", ["h\na,1\nb\n", "h\na,x1\n", "h\na,\n", "h\na,1\n\n",
                                  "h\na,18446744073709551616\n", "h\na,-3\n"])
def test_malformed_rows_rejected(text):
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    with pytest.raises(ValueError):
        csv_ingest.parse(text, 0, 1)
    ctx = sieve.Ctx(device=0)
    with pytest.raises(sieve.SieveError) as e:
        sieve.load_csv(ctx, text, 0, 1)
    assert e.value.code == sieve.sieve.SIEVE_EINVAL


def test_edges():
    import paper_conf_ispass_naderantahanse23_b200 as sieve
    ctx = sieve.Ctx(device=0)
    for text, hl in [("h\n", 1), ("", 0), ("", 1), ("h", 1)]:
        tr, names = sieve.load_csv(ctx, text, 0, 1, header_lines=hl)
        assert tr.n == 0 and names == []
    tr, names = sieve.load_csv(ctx, "h\nk,18446744073709551615", 0, 1)
    assert sieve.trace_columns(tr, False, False)[1].tolist() == [2**64 - 1] and names == ["k"]
    # one row, many distinct names, no header
    text = "".join(f"n{i},{i + 1}\n" for i in range(70000))
    with pytest.raises(sieve.SieveError) as e:
        sieve.load_csv(ctx, text, 0, 1, header_lines=0)
    assert e.value.code == sieve.sieve.SIEVE_ERANGE
    text = "".join(f"n{(i * 7919) % 65536},{i + 1}\n" for i in range(65536 * 2))
    tr, names = sieve.load_csv(ctx, text, 0, 1, header_lines=0)
    exp = csv_ingest.parse(text, 0, 1, header_lines=0)
    assert names == exp[4] and sieve.trace_columns(tr, False, False)[0].tolist() == exp[0]
