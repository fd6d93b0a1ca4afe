"""GPU parity: the fused sm_100a kernel, called through the C ABI, against the
CPU oracle on the same seeded packets.  Everything is integer, so the bar is
bit-exact equality of every per-packet record field, of the output bytes of
every forwarded packet, of the (sorted) match-pair set and of the stats vector.
"""
import numpy as np
import pytest

import nfcgen
from tests.gpu_util import check_parity, gpu_run

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def nfc():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_hpca_hul18_b200 import build
    build.build()
    from paper_conf_hpca_hul18_b200 import nfc as m
    return m


def _chain(nfc, w):
    ch = nfc.Chain(w.kinds, device=0)
    ch.load_tables(w.tables)
    return ch


def test_c1_full_batch(nfc):
    """BASELINE config C1 exactly: ACL(64)->DPI(100)->LPM4(1K), one batch of 4,096 64-B packets."""
    w = nfcgen.workload("C1")
    ch = _chain(nfc, w)
    got, want = check_parity(w, ch, 4096)
    assert (got["drop_nf"] == 0xFF).sum() > 3000
    assert (got["dpi_nmatch"] > 0).sum() > 100


@pytest.mark.parametrize("variant", ["edge", "ragged", "nomatch", "fullmatch", "tcp"])
def test_c1_variants(nfc, variant):
    w = nfcgen.workload("C1")
    t = w.traffic
    if variant == "edge":
        t.malformed_ppm, t.ttl1_ppm = 30_000, 20_000
    elif variant == "ragged":
        t.pkt_len = 1
    elif variant == "nomatch":
        t.match_ppm = 0
    elif variant == "fullmatch":
        t.match_ppm = 1_000_000
    elif variant == "tcp":
        t.tcp_pct, t.pkt_len = 40, 1
    ch = _chain(nfc, w)
    check_parity(w, ch, 3001)  # ragged tail: not a multiple of the 256-packet tile


def test_c2_ipsec(nfc):
    w = nfcgen.workload("C2")
    ch = _chain(nfc, w)
    got, _ = check_parity(w, ch, 2048)
    assert (got["esp_sa"] != 0xFF).all()


@pytest.mark.parametrize("v6,plen", [(False, 1), (True, 1), (True, 1500), (False, 0)])
def test_c2_ipsec_lengths(nfc, v6, plen):
    w = nfcgen.workload("C2")
    w.traffic.pkt_len = plen
    if v6:
        w.traffic.v6_bp = 5000
        rng = np.random.default_rng(3)
        w.tables.routes6 = nfcgen.gen_routes6(rng, 100, 16)
        w.tables.nh6, w.tables.pmac6 = nfcgen.gen_nexthops(rng, 16, 4)
    ch = _chain(nfc, w)
    check_parity(w, ch, 1500)


def test_c2_seq_across_calls_and_batches(nfc):
    """ESP sequence numbers follow global order across batches and calls."""
    w = nfcgen.workload("C2")
    w.traffic.pkt_len = 1
    ch = _chain(nfc, w)
    check_parity(w, ch, 2000, split=[300, 700, 1], compare_stats=False)
    # same chain continues: compare a second call against the oracle continuing its state
    import oracle
    orc = oracle.OracleChain(w.kinds, w.tables)
    b1 = nfcgen.generate(w.traffic, w.tables, 0, 2000)
    orc.run(b1)
    b2 = nfcgen.generate(w.traffic, w.tables, 2000, 777)
    want, _, _, _ = orc.run(b2)
    got, _, _, _ = gpu_run(ch, [b2])
    assert np.array_equal(got["esp_seq"], want["esp_seq"])


def test_c3_imix(nfc):
    w = nfcgen.workload("C3", small=True)
    ch = _chain(nfc, w)
    check_parity(w, ch, 3000)


def test_c4_small_tables(nfc):
    w = nfcgen.workload("C4", small=True)
    ch = _chain(nfc, w)
    got, _ = check_parity(w, ch, 1200)
    assert (got["drop_nf"] == 0xFF).sum() > 600


def test_c4_full_tables(nfc):
    """C4 tables at full size: 200K IPv6 prefixes, 2K patterns."""
    w = nfcgen.workload("C4")
    ch = _chain(nfc, w)
    check_parity(w, ch, 600)


@pytest.mark.parametrize("k", [1, 2, 3, 4, 5, 6])
@pytest.mark.parametrize("plen", [64, 0])
def test_c5_chain_prefixes(nfc, k, plen):
    w = nfcgen.workload("C5", k=k, pkt_len=plen, small=True)
    ch = _chain(nfc, w)
    check_parity(w, ch, 1300)


def test_dpi_many_distinct_matches(nfc):
    """> 16 distinct patterns in one payload exercises the exact bitmap path."""
    pats = [bytes([c]) for c in b"abcdefghijklmnopqrstuvwxyz"] + [b"ab", b"abc", b"xyz", b"zz"]
    w = nfcgen.workload("C1")
    off = np.zeros(len(pats) + 1, dtype=np.uint32)
    off[1:] = np.cumsum([len(p) for p in pats])
    w.tables.pat_blob = np.frombuffer(b"".join(pats), dtype=np.uint8).copy()
    w.tables.pat_off = off
    w.tables.pat_action = np.zeros(len(pats), dtype=np.uint8)
    w.traffic.pkt_len = 1
    ch = _chain(nfc, w)
    got, _ = check_parity(w, ch, 700)
    assert got["dpi_nmatch"].max() > 16


def test_match_cap_overflow(nfc):
    w = nfcgen.workload("C1")
    w.traffic.match_ppm = 1_000_000
    ch = _chain(nfc, w)
    check_parity(w, ch, 2000, match_cap=100)


def test_empty_batch(nfc):
    w = nfcgen.workload("C1")
    ch = _chain(nfc, w)
    b = nfcgen.generate(w.traffic, w.tables, 0, 0)
    before = ch.launches()
    gpu_run(ch, [b])
    assert ch.launches() == before


def test_process_host_e2e(nfc):
    """The host-buffer entry point (H2D + kernel + D2H) gives the same results."""
    import oracle
    w = nfcgen.workload("C2")
    w.traffic.pkt_len = 1
    b = nfcgen.generate(w.traffic, w.tables, 0, 1000)
    ch = _chain(nfc, w)
    arena = b.arena.copy()
    rec, (mp, mq), npairs = ch.process_host(arena, b.off, b.len)
    want, want_arena, _, _ = oracle.OracleChain(w.kinds, w.tables).run(b)
    assert np.array_equal(rec.view(np.uint8), want.view(np.uint8))
    from tests.gpu_util import compare_bytes
    compare_bytes(want, arena, b.off, want_arena, b.off, "host")


def test_missing_tables_is_estate(nfc):
    w = nfcgen.workload("C1")
    ch = nfc.Chain(w.kinds, device=0)
    ch.load_acl(w.tables.acl_rules)
    b = nfcgen.generate(w.traffic, w.tables, 0, 10)
    with pytest.raises(nfc.NfcError) as e:
        gpu_run(ch, [b])
    assert e.value.code == nfc.NFC_ESTATE


def test_malformed_specs_rejected(nfc):
    w = nfcgen.workload("C1")
    ch = nfc.Chain(w.kinds, device=0)
    r = w.tables.routes4.copy()
    r[1] = r[2]  # duplicate prefix
    with pytest.raises(nfc.NfcError) as e:
        ch.load_lpm(nfc.LPM4, r, w.tables.nh4, w.tables.pmac4)
    assert e.value.code == nfc.NFC_EINVAL
    r = w.tables.routes4.copy()
    r[1]["len"] = 33
    with pytest.raises(nfc.NfcError):
        ch.load_lpm(nfc.LPM4, r, w.tables.nh4, w.tables.pmac4)
    with pytest.raises(nfc.NfcError):
        ch.load_dpi(np.zeros(0, np.uint8), np.zeros(2, np.uint32), np.zeros(1, np.uint8))


@pytest.mark.parametrize("cfg,k", [("C1", None), ("C3", None), ("C5", 4)])
def test_unfused_baseline_parity(nfc, cfg, k):
    """NEXT-1: the per-NF kernel pipeline with device-side re-split gives the oracle's
    results exactly (records, bytes, pairs, stats), like the fused kernel."""
    w = nfcgen.workload(cfg, k=k, small=(cfg == "C3"))
    ch = nfc.Chain(w.kinds, device=0, flags=nfc.F_UNFUSED)
    ch.load_tables(w.tables)
    check_parity(w, ch, 3001)


@pytest.mark.gpu
@pytest.mark.parametrize("cfg,k,pl", [("C1", None, None), ("C3", None, None), ("C5", 4, None), ("C5", 3, 0),
                                      ("C5", 2, 1500)])
def test_parallel_sfc_parity(nfc, cfg, k, pl):
    """NEXT-2: the chain's NFs on different warps, each on its own packet copy, merged
    by XOR with the earliest dropper's later side effects discarded (P:L243-263,
    P:L269) -- the oracle's sequential results exactly (records, bytes, pairs, stats)."""
    w = nfcgen.workload(cfg, k=k, pkt_len=pl, small=(cfg == "C3"))
    w.traffic.ttl1_ppm = 10_000
    w.traffic.malformed_ppm = 5_000
    assert max(nfc.plan_parallel(w.kinds)) == 0          # one parallel-legal group
    ch = nfc.Chain(w.kinds, device=0, flags=nfc.F_PARALLEL)
    ch.load_tables(w.tables)
    check_parity(w, ch, 2999)


@pytest.mark.gpu
def test_parallel_rejects_ipsec(nfc):
    with pytest.raises(nfc.NfcError):
        nfc.Chain(["ACL", "IPSEC"], device=0, flags=nfc.F_PARALLEL)


@pytest.mark.gpu
@pytest.mark.parametrize("n_acl,pl", [(200, 64), (1000, 128), (10000, 1500), (1000, 1), (200, 0)])
def test_n3_fw_router_nat_parity(nfc, n_acl, pl):
    """NEXT-3 (Figs. 16-17): FW(200 / 1K / 10K rules) -> IPv4 router -> NAT44
    at 64 / 128 / 1500 B (and ragged / IMIX): records, rewritten bytes (SNAT / DNAT,
    IPv4 and TCP/UDP checksums) and stats equal the oracle's."""
    w = nfcgen.workload("N3", acl_rules=n_acl, pkt_len=pl)
    w.traffic.ttl1_ppm = 5_000
    w.traffic.malformed_ppm = 5_000
    ch = _chain(nfc, w)
    got, _ = check_parity(w, ch, 3001)
    assert (got["drop_nf"] == 0xFF).sum() > 2500


@pytest.mark.gpu
def test_n3_unfused_and_nat_only(nfc):
    """The unfused baseline runs the NAT stage too; a NAT-only chain (egress port 0)
    and a chain with every port Internet-facing match the oracle."""
    w = nfcgen.workload("N3", acl_rules=1000, pkt_len=1)
    ch = nfc.Chain(w.kinds, device=0, flags=nfc.F_UNFUSED)
    ch.load_tables(w.tables)
    check_parity(w, ch, 2001)
    w2 = nfcgen.workload("N3", acl_rules=200, pkt_len=1)
    w2.tables.nat_ext_ports = 1
    w2.kinds = ["NAT"]
    ch2 = _chain(nfc, w2)
    check_parity(w2, ch2, 2001)
    w3 = nfcgen.workload("N3", acl_rules=200, pkt_len=64)
    w3.tables.nat_ext_ports = 0xFFFFFFFF
    check_parity(w3, _chain(nfc, w3), 2001)


# ---------------------------------------------------------------- valid edge-case frames
# IPv4 options (IHL 6..15), fragments (ports 0, L4 not parsed), TCP data offsets 6..15 and
# Ethernet trailers (SURVEY 8(c)(i) parse cases) through the fused kernel's general parse,
# the options checksum loop, the L4-from-memory paths, the NAT memory path and ESP with
# IHL > 5.
EDGE_CASES = [("C1", None, None, False), ("C1", None, 64, False), ("C2", None, 1, False),
              ("C3", None, None, True), ("C4", None, 1, True), ("N3", None, 1, False),
              ("N3", None, 64, False), ("C5", 6, 1, True), ("C5", 3, 64, True), ("C5", 4, 0, True)]


@pytest.mark.parametrize("cfg,k,pl,small", EDGE_CASES)
def test_edge_frames_parity(nfc, cfg, k, pl, small):
    w = nfcgen.workload(cfg, k=k, pkt_len=pl, small=small, acl_rules=200 if cfg == "N3" else None)
    w.traffic.tcp_pct = 40
    w.traffic.edge(120_000)
    w.traffic.malformed_ppm = 10_000
    w.traffic.ttl1_ppm = 5_000
    ch = _chain(nfc, w)
    got, _ = check_parity(w, ch, 3001)
    assert (got["drop_nf"] == 0xFF).sum() > 1000


@pytest.mark.parametrize("flags", ["unfused", "parallel"])
def test_edge_frames_unfused_parallel(nfc, flags):
    w = nfcgen.workload("C5", k=4, pkt_len=1, small=True)
    w.traffic.tcp_pct = 40
    w.traffic.edge(120_000)
    ch = nfc.Chain(w.kinds, device=0, flags=nfc.F_UNFUSED if flags == "unfused" else nfc.F_PARALLEL)
    ch.load_tables(w.tables)
    check_parity(w, ch, 2501)


@pytest.mark.parametrize("k", [1, 2, 3, 4, 5, 6])
def test_c5_full_tables(nfc, k):
    """C5 with its full tables (200K IPv6 routes) at every chain length, IMIX, many batches."""
    w = nfcgen.workload("C5", k=k, pkt_len=0)
    ch = _chain(nfc, w)
    check_parity(w, ch, 6000, split=[4096])


def test_c1_many_batches(nfc):
    """The multi-batch descriptor path: 40 batches of 4,096 packets (ragged last) in one call."""
    w = nfcgen.workload("C1")
    ch = _chain(nfc, w)
    n = 40 * 4096 - 123
    check_parity(w, ch, n, split=[4096] * 39, match_cap=1 << 20)


@pytest.mark.parametrize("cfg,n,shuffle", [("C1", 300_000, False), ("C2", 70_000, False), ("C1", 100_000, True)])
def test_process_host_pipelined(nfc, cfg, n, shuffle):
    """nfc_process_host over many pipeline chunks (H2D / kernel / D2H on two streams,
    kernels in chunk order: ESP sequence numbers stay global), and with frames NOT laid
    out in index order (overlapping chunk ranges: one chunk) -- records, bytes and pairs
    equal the oracle's."""
    import oracle
    from tests.gpu_util import compare_bytes, sorted_pairs
    w = nfcgen.workload(cfg, small=True)
    w.traffic.pkt_len = 1 if cfg == "C2" else 64
    b = nfcgen.generate(w.traffic, w.tables, 0, n)
    if shuffle:
        perm = np.random.default_rng(1).permutation(n)
        b = nfcgen.Batch(b.arena, b.off[perm].copy(), b.len[perm].copy(), 0, b.headroom, b.tailroom)
    ch = _chain(nfc, w)
    arena = b.arena.copy()
    rec, (mp, mq), npairs = ch.process_host(arena, b.off, b.len, match_cap=1 << 20)
    want, want_arena, (wp, wq), wn = oracle.OracleChain(w.kinds, w.tables).run(b)
    assert np.array_equal(rec.view(np.uint8), want.view(np.uint8))
    compare_bytes(want, arena, b.off, want_arena, b.off, "host")
    assert npairs == wn and np.array_equal(sorted_pairs(mp, mq), sorted_pairs(wp, wq))


# ---------------------------------------------------------------- NEXT-2: identical NFs
REPEATED = [["ACL"] * 4, ["DPI"] * 4, ["ACL", "DPI", "ACL", "LPM4", "LPM4"], ["LB", "ACL", "LB"]]


def _rep_workload(kinds):
    w = nfcgen.workload("NX2_FW")
    w.tables = nfcgen.make_tables(9, ["ACL", "DPI", "LPM4", "LB"], n_acl=64, n_pat=100, n_r4=1000, acl_deny=0.1)
    w.kinds = list(kinds)
    w.traffic.pkt_len, w.traffic.match_ppm, w.traffic.tcp_pct = 1, 200_000, 40
    w.traffic.edge(50_000)
    return w


@pytest.mark.parametrize("kinds", REPEATED)
@pytest.mark.parametrize("mode", ["fused", "unfused", "parallel"])
def test_repeated_kinds_parity(nfc, kinds, mode):
    """SURVEY 8(f) NEXT-2 (Fig. 13): chains with repeated NF kinds (four identical
    FW or IDS NFs; a forwarder twice) -- fused (configuration d), one kernel per NF (a),
    parallel groups (b: nfc_plan_parallel's) -- equal the sequential oracle."""
    w = _rep_workload(kinds)
    flags = {"fused": 0, "unfused": nfc.F_UNFUSED, "parallel": nfc.F_PARALLEL}[mode]
    ch = nfc.Chain(w.kinds, device=0, flags=flags)
    ch.load_tables(w.tables)
    check_parity(w, ch, 3001)


@pytest.mark.parametrize("kinds,groups", [(["ACL"] * 4, [0, 0, 1, 1]), (["DPI"] * 4, [0, 0, 1, 1]),
                                          (["DPI"] * 4, [0, 1, 2, 3]), (["ACL", "DPI", "ACL", "LPM4", "LPM4"], [0, 1, 1, 2, 3]),
                                          (["LB", "ACL", "LB"], [0, 0, 1])])
def test_parallel_explicit_groups(nfc, kinds, groups):
    """NFC_F_PARALLEL with a chosen grouping (the paper's configuration (c): two groups of
    two identical NFs): groups run in order, members on copies of the packet that
    enters their group, XOR merge -- equal the sequential oracle."""
    w = _rep_workload(kinds)
    ch = nfc.Chain(w.kinds, device=0, flags=nfc.F_PARALLEL)
    ch.load_tables(w.tables)
    ch.set_groups(groups)
    assert ch.groups() == groups
    check_parity(w, ch, 3001)


def test_parallel_groups_validated(nfc):
    ch = nfc.Chain(["ACL", "LPM4", "LPM4"], device=0, flags=nfc.F_PARALLEL)
    assert ch.groups() == [0, 0, 1]                 # two forwarders write the same fields: apart
    for bad in ([0, 0, 0], [1, 1, 1], [0, 2, 2], [0, 1, 0]):
        with pytest.raises(nfc.NfcError) as e:
            ch.set_groups(bad)
        assert e.value.code == nfc.NFC_EINVAL
    with pytest.raises(nfc.NfcError) as e:
        nfc.Chain(["IPSEC", "ACL", "IPSEC"], device=0)
    assert e.value.code == nfc.NFC_EUNSUP


@pytest.mark.parametrize("cfg,n_acl", [("C1", None), ("N3", 10000)])
def test_c1_acl_boundary_keys(nfc, cfg, n_acl):
    """The IPv4 search image (AclImg::f4: 10-bit buckets, two or three halvings over
    padded key arrays; C1) and the 16-bit first level of large rule sets (AclImg::x4; the
    10K-rule FW of NEXT-3): 5-tuples placed exactly on, just below and just above every
    rule's interval edges, plus the extreme keys 0 / 2^32-1 and ports 0 / 65535,
    bit-exact vs the oracle's linear rule scan (DESIGN.md ACL)."""
    import oracle
    from tests.gpu_util import compare_bytes, compare_records, gpu_run, sorted_pairs
    w = nfcgen.workload(cfg, acl_rules=n_acl, pkt_len=64 if cfg == "N3" else None)
    n = 4096
    b = nfcgen.generate(w.traffic, w.tables, 0, n)
    rules = w.tables.acl_rules
    rng = np.random.default_rng(77)

    def edges(lo, hi, top):
        return [lo, hi, (lo - 1) % (top + 1), (hi + 1) % (top + 1), 0, top]

    cand_ip, cand_port = [], []
    for r in rules:
        if r["family"] != 4:
            continue
        for fld, ln in (("src", "slen"), ("dst", "dlen")):
            k = int.from_bytes(bytes(r[fld][:4]), "big")
            m = (0xFFFFFFFF << (32 - int(r[ln]))) & 0xFFFFFFFF if r[ln] else 0
            cand_ip += edges(k & m, (k & m) | (~m & 0xFFFFFFFF), 0xFFFFFFFF)
        cand_port += edges(int(r["sp_lo"]), int(r["sp_hi"]), 0xFFFF) + edges(int(r["dp_lo"]), int(r["dp_hi"]), 0xFFFF)
    ar = b.arena
    placed = 0
    for i in range(n):
        o = int(b.off[i])
        if int(b.len[i]) < 42 or ar[o + 12] != 0x08 or ar[o + 13] != 0x00 or ar[o + 14] != 0x45:
            continue
        ar[o + 26:o + 30] = np.frombuffer(int(rng.choice(cand_ip)).to_bytes(4, "big"), np.uint8)
        ar[o + 30:o + 34] = np.frombuffer(int(rng.choice(cand_ip)).to_bytes(4, "big"), np.uint8)
        ar[o + 34:o + 36] = np.frombuffer(int(rng.choice(cand_port)).to_bytes(2, "big"), np.uint8)
        ar[o + 36:o + 38] = np.frombuffer(int(rng.choice(cand_port)).to_bytes(2, "big"), np.uint8)
        placed += 1
    assert placed > 3000
    orc = oracle.OracleChain(w.kinds, w.tables)
    want, want_arena, (wp, wq), npairs = orc.run(b, match_cap=1 << 16)
    ch = _chain(nfc, w)
    got, arenas, (gp, gq), k = gpu_run(ch, [b])
    compare_records(got, want, f"{cfg} ACL edges")
    compare_bytes(want, arenas[0], b.off, want_arena, b.off, f"{cfg} ACL edges")
    assert k == npairs and np.array_equal(sorted_pairs(gp, gq), sorted_pairs(wp, wq))
    # the edges exercise many distinct rules (not just the default)
    assert len(np.unique(got["acl_rule"])) > 10


@pytest.mark.parametrize("cfg,k", [("C2", None), ("C4", None), ("C5", 5), ("C5", 6)])
def test_esp_balanced_ctr_imix(nfc, cfg, k):
    """a3 for the IPsec tiles (esp_ctr_tile): IMIX tiles take the balanced CTR pass (the
    survivors' AES blocks split evenly over the CTA, XORed in with red.xor, then MAC-only
    nf_esp).  Edge frames (IPv4 options, IPv6, fragments, malformed) and drops before IPsec
    mixed in; two batches in one call; bit-exact vs the oracle."""
    w = nfcgen.workload(cfg, k=k, pkt_len=0, small=(cfg != "C2"))
    w.traffic.tcp_pct = 30
    w.traffic.edge(80_000)
    w.traffic.malformed_ppm = 10_000
    ch = _chain(nfc, w)
    got, _ = check_parity(w, ch, 5000, split=[1700])
    assert (got["esp_sa"] != 0xFF).sum() > 2000
