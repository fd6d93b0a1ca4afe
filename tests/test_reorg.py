"""NEXT-2: SFC parallelization with packet copies and XOR merge
(P:L243-263 [SIV.B.1], Tables II-III, Figs. 13-14).

CPU tests: the XOR merge rule itself against brute force, the reorg
oracle against the sequential definition (same processing path, alerts
in the same packet state) for every grouping of several chains, and the
product's planner (nfc_plan_parallel) against the read/write rule of Table III
(R#16)."""
import itertools
import random

import numpy as np
import pytest

import nfcgen
import oracle


def _wl(name, **kw):
    return nfcgen.workload(name, small=True, **kw)


def test_xor_merge_rule_brute_force():
    # out = orig ^ OR_f (orig ^ f(orig)).  With disjoint write sets this is
    # the sequential application of the writers, in any order.
    rng = random.Random(5)
    for _ in range(300):
        n = rng.randrange(1, 40)
        orig = bytes(rng.randrange(256) for _ in range(n))
        m = rng.randrange(1, 5)
        owner = [rng.randrange(m + 1) for _ in range(n)]          # m = untouched
        copies = []
        for j in range(m):
            c = bytearray(orig)
            for k in range(n):
                if owner[k] == j:
                    c[k] = rng.randrange(256)
            copies.append(bytes(c))
        acc = [0] * n
        for c in copies:
            for k in range(n):
                acc[k] |= orig[k] ^ c[k]
        merged = bytes(orig[k] ^ acc[k] for k in range(n))
        seq = bytearray(orig)
        for j in range(m):
            for k in range(n):
                if owner[k] == j:
                    seq[k] = copies[j][k]
        assert merged == bytes(seq)


def _partitions(n):
    """All groupings of n positions into runs of consecutive positions."""
    for cuts in itertools.product([0, 1], repeat=n - 1):
        g, cur = [0], 0
        for c in cuts:
            cur += c
            g.append(cur)
        yield g


def _valid(kinds, g):
    for p, k in enumerate(kinds):
        if k == "IPSEC":
            if (p > 0 and g[p - 1] == g[p]) or (p + 1 < len(kinds) and g[p + 1] == g[p]):
                return False
    return True


def _compare(w, b, group):
    seq = oracle.OracleChain(w.kinds, w.tables)
    r1, a1, (mp1, mq1), n1 = seq.run(b)
    par = oracle.OracleChain(w.kinds, w.tables)
    r2, a2, (mp2, mq2), n2 = par.run_reorg(b, group)
    assert np.array_equal(r1.view(np.uint8), r2.view(np.uint8)), group
    assert n1 == n2 and np.array_equal(mp1, mp2) and np.array_equal(mq1, mq2), group
    assert np.array_equal(seq.stats, par.stats), group
    for i in np.nonzero(r1["drop_nf"] == 0xFF)[0]:
        s = int(b.off[i]) - (16 if r1["esp_sa"][i] != 0xFF else 0)
        e = s + int(r1["out_len"][i])
        assert np.array_equal(a1[s:e], a2[s:e]), (group, i)


@pytest.mark.parametrize("name", ["C1", "C3", "C4", "C5"])
def test_reorg_equals_sequential_for_every_valid_grouping(name):
    w = _wl(name)
    w.traffic.ttl1_ppm = 20_000
    w.traffic.malformed_ppm = 10_000
    b = nfcgen.generate(w.traffic, w.tables, 0, 384)
    n_checked = 0
    for g in _partitions(len(w.kinds)):
        if not _valid(w.kinds, g):
            with pytest.raises(ValueError):
                oracle.OracleChain(w.kinds, w.tables).run_reorg(b, g)
            continue
        _compare(w, b, g)
        n_checked += 1
    assert n_checked >= 1


def test_reorg_discards_side_effects_after_earliest_dropper():
    # ACL (position 0) denies a packet whose payload matches a pattern: in the fully
    # parallel grouping DPI still scans its copy, but its pairs/stats are discarded
    w = _wl("C1")
    b = nfcgen.generate(w.traffic, w.tables, 0, 4096)
    seq = oracle.OracleChain(w.kinds, w.tables)
    r1, _, _, n1 = seq.run(b)
    pats = w.tables.patterns()
    acl_denied_with_match = [i for i in np.nonzero(r1["drop_nf"] == 0)[0]
                             if any(p in b.frame(i)[42:] for p in pats)]
    assert acl_denied_with_match, "workload should contain denied packets with planted patterns"
    par = oracle.OracleChain(w.kinds, w.tables)
    r2, _, (mp2, _), n2 = par.run_reorg(b, [0, 0, 0])
    assert n2 == n1
    assert not set(acl_denied_with_match) & set(int(x) for x in mp2)
    assert np.all(r2["dpi_nmatch"][acl_denied_with_match] == 0)


@pytest.fixture(scope="module")
def nfc():
    from paper_conf_hpca_hul18_b200 import build
    build.build()
    from paper_conf_hpca_hul18_b200 import nfc as m
    return m


# Table II / III read-write sets, restated independently of the planner:
# kind -> family -> (reads, writes)
_F = dict(eth_dst=1, eth_src=2, ttl=4, csum=8, src=16, dst=32, ports=64, proto=128, payload=256, length=512)
_T = {"src", "dst", "ports", "proto"}


def _rw(kind, fam):
    if kind in ("ACL", "LB"):
        return _T, set()
    if kind == "DPI":
        return {"payload", "proto", "length"}, set()
    if kind == "LPM4":
        return ({"dst", "ttl"}, {"eth_dst", "eth_src", "ttl", "csum"}) if fam == 4 else (set(), set())
    if kind == "LPM6":
        return ({"dst", "ttl"}, {"eth_dst", "eth_src", "ttl"}) if fam == 6 else (set(), set())
    return set(_F), set(_F)   # IPSEC


def _legal(a, b_):
    if "IPSEC" in (a, b_) or "NAT" in (a, b_):   # R#29, R#30: stand alone
        return False
    for fam in (4, 6):
        ra, wa = _rw(a, fam)
        rb, wb = _rw(b_, fam)
        if wa & rb or wa & wb:
            return False
    return True


def test_planner_groups(nfc):
    assert nfc.plan_parallel(["ACL", "DPI", "LPM4"]) == [0, 0, 0]
    assert nfc.plan_parallel(nfcgen.C6_CHAIN) == [0, 0, 0, 0, 1, 2]
    assert nfc.plan_parallel(["ACL", "LPM6", "DPI", "IPSEC", "LB"]) == [0, 0, 0, 1, 2]
    assert nfc.plan_parallel(["IPSEC"]) == [0]
    kinds = list(nfcgen.KINDS)
    rng = random.Random(11)
    for _ in range(300):
        ch = rng.sample(kinds, rng.randrange(1, 7))
        g = nfc.plan_parallel(ch)
        # greedy maximal groups under the pairwise rule
        want, start, cur = [0], 0, 0
        for p in range(1, len(ch)):
            if not all(_legal(ch[q], ch[p]) for q in range(start, p)):
                cur += 1
                start = p
            want.append(cur)
        assert g == want, ch
    with pytest.raises(Exception):
        nfc.plan_parallel([])
    # repeated kinds (NEXT-2's identical NFs): the greedy rule still holds
    for ch, want in ((["ACL"] * 4, [0, 0, 0, 0]), (["DPI"] * 4, [0, 0, 0, 0]),
                     (["ACL", "DPI", "ACL", "LPM4", "LPM4"], [0, 0, 0, 0, 1]), (["LB", "ACL", "LB"], [0, 0, 0])):
        assert nfc.plan_parallel(ch) == want, ch


@pytest.mark.parametrize("kinds", [["ACL"] * 4, ["DPI"] * 4, ["ACL", "DPI", "ACL", "LPM4", "LPM4"], ["LB", "ACL", "LB"]])
def test_repeated_kinds_reorg_equals_sequential(kinds):
    """NEXT-2's identical NFs (Fig. 13 configurations a-d): a repeated kind shares
    its tables; every grouping into runs of parallel-legal NFs gives the sequential result
    (records, bytes, pairs, stats) -- including the paper's (b) one group and (c) two."""
    w = nfcgen.workload("NX2_FW")
    t = nfcgen.make_tables(9, ["ACL", "DPI", "LPM4", "LB"], n_acl=64, n_pat=100, n_r4=1000, acl_deny=0.1)
    w.traffic.pkt_len, w.traffic.match_ppm, w.traffic.tcp_pct = 1, 200_000, 40
    b = nfcgen.generate(w.traffic, t, 0, 800)
    seq = oracle.OracleChain(kinds, t)
    want, wa, (wp, wq), wn = seq.run(b)
    tried = 0
    for g in _partitions(len(kinds)):
        legal = all(_legal(kinds[p], kinds[q]) for p in range(len(kinds)) for q in range(p + 1, len(kinds))
                    if g[p] == g[q])
        if not legal:
            continue
        tried += 1
        o = oracle.OracleChain(kinds, t)
        got, ga, (gp, gq), gn = o.run_reorg(b, g)
        assert np.array_equal(got.view(np.uint8), want.view(np.uint8)), g
        assert gn == wn and sorted(zip(gp, gq)) == sorted(zip(wp, wq)), g
        assert np.array_equal(o.stats, seq.stats), g
    assert tried >= 2
