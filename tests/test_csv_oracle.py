"""Pins of the CSV-ingest oracle (NEXT-4, reading A27).

The golden fixture's expected arrays were derived by hand (tests/golden/csv_small.expected.json),
not by running the oracle; the round-trip and error cases pin the dialect rules independently.
"""
import json
import os

import numpy as np
import pytest

from gen import make_trace
from oracle import csv_ingest

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def test_golden_small_csv():
    with open(os.path.join(GOLD, "csv_small.csv"), newline="") as f:
        text = f.read()
    with open(os.path.join(GOLD, "csv_small.expected.json")) as f:
        exp = json.load(f)
    kid, x, cta, y, names = csv_ingest.parse(text, **exp["spec"])
    assert kid == exp["kernel_id"]
    assert x == exp["instr"]
    assert cta == exp["cta"]
    assert y == exp["cycles"]
    assert names == exp["names"]


@pytest.mark.parametrize("thousands,crlf,trailing,delim", [
    (False, False, True, ","), (True, True, False, ","), (False, True, True, ";"), (True, False, False, "\t")])
def test_round_trip_generated(thousands, crlf, trailing, delim):
    t = make_trace("C1", 0, 3000)
    K = int(t["kid"].max()) + 1
    names = [f"k{k}<{k % 3}, int>(float*, {delim} x)" for k in range(K)]
    text = csv_ingest.write(t["kid"], t["x"], t["cta"], t["y"], names, delimiter=delim,
                            thousands=thousands, crlf=crlf, trailing=trailing,
                            header=delim.join(["ID", "Kernel", "Instr", "CTAs", "Cycles"]))
    kid, x, cta, y, got = csv_ingest.parse(text, 1, 2, 3, 4, 1, delim)
    # ids are first-appearance ranks: map the original ids through their first occurrence order
    first = {}
    for k in t["kid"].tolist():
        first.setdefault(k, len(first))
    assert kid == [first[k] for k in t["kid"].tolist()]
    assert got == [names[k] for k in sorted(first, key=first.get)]
    assert x == t["x"].tolist() and cta == t["cta"].tolist() and y == t["y"].tolist()


def test_first_appearance_ids():
    text = "h\nb,5\na,6\nb,7\nc,8\na,9\n"
    kid, x, cta, y, names = csv_ingest.parse(text, 0, 1)
    assert names == ["b", "a", "c"] and kid == [0, 1, 0, 2, 1] and x == [5, 6, 7, 8, 9]
    assert cta is None and y is None


@pytest.mark.parametrize("text", ["h\na,1\nb\n", "h\na,x1\n", "h\na,\n", "h\na,1\n\n",
                                  "h\na,18446744073709551616\n", "h\na,-3\n"])
def test_malformed_rows_rejected(text):
    with pytest.raises(ValueError):
        csv_ingest.parse(text, 0, 1)


def test_u64_max_and_empty_body():
    kid, x, _, _, names = csv_ingest.parse("h\nk,18446744073709551615", 0, 1)
    assert x == [2**64 - 1] and names == ["k"]
    kid, x, _, _, names = csv_ingest.parse("h\n", 0, 1)
    assert kid == [] and names == []
    assert csv_ingest.parse("", 0, 1, header_lines=0)[0] == []
