"""CPU checks of the full-size comparison helper (tests/fullsize_oracle.py): the
parallel two-pass oracle equals ONE sequential oracle pass (including per-SA ESP
sequence numbers across range boundaries), and a single wrong field, byte or pair
is reported."""
import numpy as np
import pytest

import nfcgen
import oracle
from tests.fullsize_oracle import compare_full


def _seq(w, n):
    b = nfcgen.generate(w.traffic, w.tables, 0, n)
    orc = oracle.OracleChain(w.kinds, w.tables)
    rec, arena, (p, q), npairs = orc.run(b, match_cap=1 << 20)
    return b, rec, arena, (p, q), npairs, orc.stats.copy()


@pytest.mark.parametrize("cfg", ["C2", "C5"])
def test_parallel_oracle_equals_sequential(cfg):
    w = nfcgen.workload(cfg, small=True, k=6 if cfg == "C5" else None)
    w.traffic.pkt_len = 1
    b, rec, arena, pairs, npairs, stats = _seq(w, 6000)
    compare_full(w, rec, arena, b.off, pairs, npairs, stats, workers=3, chunk=1000)


def test_mismatches_are_reported():
    w = nfcgen.workload("C1", small=True)
    w.traffic.match_ppm = 300_000
    b, rec, arena, pairs, npairs, stats = _seq(w, 5000)
    bad = rec.copy()
    bad["acl_rule"][4321] ^= 1
    with pytest.raises(AssertionError, match="acl_rule"):
        compare_full(w, bad, arena, b.off, pairs, npairs, stats, workers=2, chunk=1000)
    a2 = arena.copy()
    i = int(np.nonzero(rec["drop_nf"] == 0xFF)[0][-1])
    a2[int(b.off[i]) + 40] ^= 0xFF
    with pytest.raises(AssertionError, match="bytes differ"):
        compare_full(w, rec, a2, b.off, pairs, npairs, stats, workers=2, chunk=1000)
    p2 = (pairs[0].copy(), pairs[1].copy())
    p2[1][0] ^= 1
    with pytest.raises(AssertionError, match="match pairs"):
        compare_full(w, rec, arena, b.off, p2, npairs, stats, workers=2, chunk=1000)
