"""Pins for the oracle's parse, forwarder rewrite, DPI DROP verdict and LB backend
(CPU only), with hand-built frames and expected outcomes stated in the test.

Parse cases are SURVEY.md 8(c)(i) step 1 (the validity check of the I/O loop,
P:L87 [SII.B.1]; the one header classifier): each frame below is built
byte by byte and the expected fields are written out as literals, so a wrong
offset, a dropped check or a mis-read field in oracle.c `parse` fails here.
The forwarder rewrite (R#6), the DPI DROP verdict (Table II P:L218,
R#10) and the LB range reduction (R#22) are checked against independent
formulations: a linear route scan, a naive substring search, and the MS RSS
verification vectors with a power-of-two backend count (backend = top bits of h).
"""
import struct

import numpy as np
import pytest

import nfcgen
import oracle
from tests.conftest import golden_rows

MAC_D = bytes.fromhex("020000000001")
MAC_S = bytes.fromhex("020000000002")


def eth(ethertype: int) -> bytes:
    return MAC_D + MAC_S + struct.pack(">H", ethertype)


def ipv4(total_len: int, proto: int, src=b"\x0a\x00\x00\x01", dst=b"\xc0\xa8\x01\x02", ihl=5,
         frag=0x4000, ttl=64, version=4, options=b"") -> bytes:
    assert len(options) == 4 * ihl - 20 or version != 4 or ihl < 5
    return bytes([(version << 4) | ihl, 0]) + struct.pack(">HHHBBH", total_len, 7, frag, ttl, proto, 0) + src + dst + options


def udp(sport: int, dport: int, length: int) -> bytes:
    return struct.pack(">HHHH", sport, dport, length, 0)


def tcp(sport: int, dport: int, doff: int = 5, options: bytes = b"") -> bytes:
    return struct.pack(">HHIIBBHHH", sport, dport, 1, 2, doff << 4, 0x18, 0xFFFF, 0, 0) + options


def ipv6(payload_len: int, nh: int, src=bytes(range(16)), dst=bytes(range(16, 32)), version=6) -> bytes:
    return bytes([version << 4, 0, 0, 0]) + struct.pack(">HBB", payload_len, nh, 64) + src + dst


def P(family, l4_off, ip_end, pl_off, proto, sport, dport):
    return dict(family=family, l4_off=l4_off, ip_end=ip_end, pl_off=pl_off, proto=proto, sport=sport, dport=dport)


PAY22 = bytes(range(0x41, 0x41 + 22))

CASES = [
    # name, frame, expected parse (None = dropped by the parse, drop_nf 0xFE)
    ("ipv4_udp_64", eth(0x0800) + ipv4(50, 17) + udp(1234, 80, 30) + PAY22,
     P(4, 34, 64, 42, 17, 1234, 80)),
    ("ipv4_tcp_doff5", eth(0x0800) + ipv4(60, 6) + tcp(5555, 443) + bytes(20),
     P(4, 34, 74, 54, 6, 5555, 443)),
    # IPv4 options: IHL 7 -> L4 at 14 + 28 = 42, ports read there
    ("ipv4_options_ihl7", eth(0x0800) + ipv4(28 + 8 + 10, 17, ihl=7, options=b"\x01" * 8) + udp(7, 9, 18) + bytes(10),
     P(4, 42, 60, 50, 17, 7, 9)),
    # IHL 15 (40 B of options) with TCP data offset 15 (40 B of TCP options)
    ("ipv4_ihl15_tcp_doff15", eth(0x0800) + ipv4(60 + 60 + 3, 6, ihl=15, options=bytes(40)) +
     tcp(1, 2, doff=15, options=bytes(40)) + b"xyz",
     P(4, 74, 137, 134, 6, 1, 2)),
    # fragments: MF set / non-zero offset / both -> ports 0, L4 not parsed, payload from L4 offset
    ("ipv4_frag_mf", eth(0x0800) + ipv4(50, 17, frag=0x2000) + udp(1234, 80, 30) + PAY22,
     P(4, 34, 64, 34, 17, 0, 0)),
    ("ipv4_frag_offset", eth(0x0800) + ipv4(50, 6, frag=0x00B9) + bytes(30),
     P(4, 34, 64, 34, 6, 0, 0)),
    ("ipv4_frag_mf_offset_options", eth(0x0800) + ipv4(24 + 30, 17, ihl=6, frag=0x2001, options=bytes(4)) + bytes(30),
     P(4, 38, 68, 38, 17, 0, 0)),
    # DF alone is not a fragment
    ("ipv4_df_only", eth(0x0800) + ipv4(28, 17, frag=0x4000) + udp(3, 4, 8),
     P(4, 34, 42, 42, 17, 3, 4)),
    # Ethernet trailer: bytes beyond 14 + total_len are ignored (payload ends at ip_end)
    ("ipv4_trailer", eth(0x0800) + ipv4(30, 17) + udp(10, 20, 10) + b"ab" + b"\xee" * 18,
     P(4, 34, 44, 42, 17, 10, 20)),
    # TCP options: data offset 8 -> payload at 34 + 32
    ("ipv4_tcp_doff8", eth(0x0800) + ipv4(20 + 32 + 4, 6) + tcp(80, 8080, doff=8, options=bytes(12)) + b"DATA",
     P(4, 34, 70, 66, 6, 80, 8080)),
    # other protocols: ports 0, no L4 header
    ("ipv4_icmp", eth(0x0800) + ipv4(28, 1) + bytes(8),
     P(4, 34, 42, 34, 1, 0, 0)),
    ("ipv6_udp", eth(0x86DD) + ipv6(8 + 4, 17) + udp(53, 5353, 12) + b"qqqq",
     P(6, 54, 66, 62, 17, 53, 5353)),
    ("ipv6_tcp_doff6_trailer", eth(0x86DD) + ipv6(24 + 2, 6) + tcp(9, 10, doff=6, options=bytes(4)) + b"hi" + bytes(6),
     P(6, 54, 80, 78, 6, 9, 10)),
    # IPv6 extension header numbers are taken as the L4 protocol (not parsed): 0 = hop-by-hop
    ("ipv6_ext_hdr_as_proto", eth(0x86DD) + ipv6(16, 0) + bytes(16),
     P(6, 54, 70, 54, 0, 0, 0)),
    # ---- parse drops
    ("short_frame", eth(0x0800)[:13], None),
    ("arp", eth(0x0806) + bytes(46), None),
    ("vlan_not_parsed", eth(0x8100) + bytes(50), None),
    ("ipv4_short_of_34", eth(0x0800) + ipv4(20, 17)[:19], None),
    ("ipv4_bad_version", eth(0x0800) + ipv4(50, 17, version=6) + udp(1, 2, 30) + PAY22, None),
    ("ipv4_ihl4", eth(0x0800) + bytes([0x44, 0]) + ipv4(50, 17)[2:] + udp(1, 2, 30) + PAY22, None),
    ("ipv4_total_len_below_ihl", eth(0x0800) + ipv4(24, 17, ihl=6, options=bytes(4)) + udp(1, 2, 8) + bytes(8), None),
    ("ipv4_total_len_overrun", eth(0x0800) + ipv4(51, 17) + udp(1, 2, 30) + PAY22, None),
    ("ipv4_udp_truncated", eth(0x0800) + ipv4(24, 17) + udp(1, 2, 8) + bytes(20), None),
    ("ipv4_tcp_truncated", eth(0x0800) + ipv4(20 + 16, 6) + tcp(1, 2) + bytes(10), None),
    ("ipv4_tcp_doff4", eth(0x0800) + ipv4(60, 6) + tcp(1, 2, doff=4) + bytes(20), None),
    ("ipv4_tcp_doff_overrun", eth(0x0800) + ipv4(20 + 24, 6) + tcp(1, 2, doff=7) + bytes(4), None),
    ("ipv6_short_of_54", eth(0x86DD) + ipv6(0, 17)[:39], None),
    ("ipv6_bad_version", eth(0x86DD) + ipv6(12, 17, version=4) + udp(1, 2, 12) + b"qqqq", None),
    ("ipv6_payload_overrun", eth(0x86DD) + ipv6(13, 17) + udp(1, 2, 12) + b"qqqq", None),
    ("ipv6_udp_truncated", eth(0x86DD) + ipv6(6, 17) + bytes(6), None),
]


@pytest.mark.parametrize("name,frame,want", CASES, ids=[c[0] for c in CASES])
def test_parse_hand_built(name, frame, want):
    assert oracle.parse(frame) == want


@pytest.mark.parametrize("name,frame,want", CASES, ids=[c[0] for c in CASES])
def test_parse_drop_in_chain(name, frame, want):
    """Through the chain: a parse failure drops with drop_nf 0xFE before any NF."""
    w = nfcgen.workload("C1", small=True)
    ch = oracle.OracleChain(["LB"], nfcgen.make_tables(3, ["LB"], n_r4=0))
    r, _, _ = ch.run_one(frame, 0)
    if want is None:
        assert r["drop_nf"] == 0xFE and r["port"] == 0xFFFF and r["lb_backend"] == 0xFFFF
    else:
        assert r["drop_nf"] == 0xFF and r["lb_backend"] != 0xFFFF
    del w


def test_generator_edge_frames_parse_as_built():
    """The generator's edge-case knobs produce frames whose parse is what they were built
    as (IHL, fragment, TCP data offset and trailer read back from the raw bytes)."""
    w = nfcgen.workload("C1", small=True)
    w.traffic.tcp_pct, w.traffic.pkt_len = 40, 1
    w.traffic.edge(250_000)
    b = nfcgen.generate(w.traffic, w.tables, 0, 3000)
    kinds = {"opt": 0, "frag": 0, "tcpopt": 0, "trailer": 0}
    for i in range(b.n):
        f = b.frame(i)
        v = oracle.parse(f)
        assert v is not None, i
        ihl = f[14] & 15
        tot = int.from_bytes(f[16:18], "big")
        fo = int.from_bytes(f[20:22], "big") & 0x3FFF
        assert v["l4_off"] == 14 + 4 * ihl and v["ip_end"] == 14 + tot
        kinds["opt"] += ihl > 5
        kinds["trailer"] += 14 + tot < len(f)
        if fo:
            kinds["frag"] += 1
            assert v["sport"] == v["dport"] == 0 and v["pl_off"] == v["l4_off"]
        elif v["proto"] == 6:
            doff = f[v["l4_off"] + 12] >> 4
            kinds["tcpopt"] += doff > 5
            assert v["pl_off"] == v["l4_off"] + 4 * doff
        else:
            assert v["pl_off"] == v["l4_off"] + 8
    assert min(kinds.values()) > 100, kinds


def _linear_lpm4(routes, dst: int):
    best, best_len = -1, -1
    for r in routes:
        L = int(r["len"])
        m = 0 if L == 0 else (0xFFFFFFFF << (32 - L)) & 0xFFFFFFFF
        if (dst & m) == (int(r["prefix"]) & m) and L > best_len:
            best, best_len = int(r["nh"]), L
    return best


def test_forwarder_rewrites_macs_ttl_checksum():
    """LPM4 forward (R#6): eth.dst = nh.mac, eth.src = port_mac[nh.port], TTL - 1,
    a valid RFC 1071 checksum, port = nh.port; the next hop found by a linear route scan.
    Frames with IPv4 options are included (checksum over the whole IHL)."""
    w = nfcgen.workload("C1", small=True)
    w.traffic.edge(200_000)
    w.traffic.pkt_len = 1
    t = w.tables
    b = nfcgen.generate(w.traffic, t, 0, 600)
    ch = oracle.OracleChain(["LPM4"], t)
    res, arena, _, _ = ch.run(b)
    n_opt = 0
    for i in range(b.n):
        f_in = b.frame(i)
        o = int(b.off[i])
        out = arena[o:o + len(f_in)].tobytes()
        dst = int.from_bytes(f_in[30:34], "big")
        nh = _linear_lpm4(t.routes4, dst)
        assert nh >= 0                                  # default route installed
        r = res[i]
        if f_in[22] <= 1:
            assert r["drop_nf"] == 0
            continue
        port = int(t.nh4["port"][nh])
        assert r["drop_nf"] == 0xFF and r["port"] == port
        assert out[0:6] == bytes(t.nh4["mac"][nh])
        assert out[6:12] == bytes(t.pmac4[port])
        assert out[22] == f_in[22] - 1
        ihl = f_in[14] & 15
        n_opt += ihl > 5
        assert oracle.ipv4_checksum(out[14:14 + 4 * ihl]) == 0
        # only the MACs, TTL and checksum change
        diff = {k for k in range(len(f_in)) if out[k] != f_in[k]}
        assert diff <= set(range(12)) | {22, 24, 25}
    assert n_opt > 20


def test_dpi_drop_verdict_vs_naive_search():
    """DPI in a chain (Table II, R#9/R#10): dpi_nmatch = number of distinct patterns
    occurring in the payload span (naive substring search); the packet is dropped at the
    DPI position iff one of them has action DROP; later NFs then record nothing."""
    w = nfcgen.workload("C1", small=True)
    t = w.tables
    t.pat_action = np.zeros(t.n_pat, dtype=np.uint8)
    t.pat_action[::3] = 1                               # a third of the patterns DROP
    w.traffic.match_ppm = 400_000
    w.traffic.pkt_len = 1
    w.traffic.edge(100_000)
    b = nfcgen.generate(w.traffic, t, 0, 1500)
    ch = oracle.OracleChain(["DPI", "LB"], nfcgen.Tables(pat_blob=t.pat_blob, pat_off=t.pat_off,
                                                         pat_action=t.pat_action,
                                                         lb_ports=np.arange(8, dtype=np.uint16),
                                                         lb_key=np.arange(40, dtype=np.uint8)))
    res, _, _, _ = ch.run(b)
    pats = t.patterns()
    n_drop = 0
    for i in range(b.n):
        f = b.frame(i)
        v = oracle.parse(f)
        pay = f[v["pl_off"]:v["ip_end"]]
        m = [j for j, p in enumerate(pats) if p in pay]
        r = res[i]
        assert r["dpi_nmatch"] == len(m)
        if any(t.pat_action[j] for j in m):
            n_drop += 1
            assert r["drop_nf"] == 0 and r["lb_backend"] == 0xFFFF and r["port"] == 0xFFFF
        else:
            assert r["drop_nf"] == 0xFF and r["lb_backend"] != 0xFFFF
    assert n_drop > 50


@pytest.mark.parametrize("k", [0, 1, 3, 6])
def test_lb_backend_ms_rss_vectors(k):
    """LB (R#22): h = Toeplitz(key, src|dst|sport|dport), backend = floor(h*B / 2^32).
    With the MS RSS key the hashes are the published verification values (not computed
    here), and with B = 2^k the backend is the top k bits of h."""
    rows = [r for r in golden_rows("ms_rss_toeplitz.txt") if ":" not in r[0]]
    assert len(rows) == 5
    B = 1 << k
    t = nfcgen.Tables(lb_ports=np.arange(100, 100 + B, dtype=np.uint16),
                      lb_key=np.frombuffer(oracle.MS_RSS_KEY, dtype=np.uint8).copy())
    ch = oracle.OracleChain(["LB"], t)
    for src, sp, dst, dp, _, h4 in rows:
        h = int(h4, 16)
        s = bytes(int(x) for x in src.split("."))
        d = bytes(int(x) for x in dst.split("."))
        frame = eth(0x0800) + ipv4(28, 17, src=s, dst=d) + udp(int(sp), int(dp), 8)
        r, _, _ = ch.run_one(frame, 0)
        want = h >> (32 - k) if k else 0
        assert r["lb_backend"] == want and r["port"] == 100 + want
    # a fragment hashes with ports 0 (the IP-only-with-zero-ports tuple)
    src, sp, dst, dp, h_ip, _ = rows[0]
    s = bytes(int(x) for x in src.split("."))
    d = bytes(int(x) for x in dst.split("."))
    frame = eth(0x0800) + ipv4(28, 17, src=s, dst=d, frag=0x2000) + udp(int(sp), int(dp), 8)
    r, _, _ = ch.run_one(frame, 0)
    # Toeplitz is linear over GF(2): zero port bytes add nothing, so h = the IP-only value
    assert r["lb_backend"] == (int(h_ip, 16) >> (32 - k) if k else 0)
