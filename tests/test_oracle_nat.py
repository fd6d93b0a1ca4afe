"""Pins of the oracle's NAT44 NF (R#30; "the NAT network function performs
source and destination NAT", Table II row NAT: header read + write, no drop).

Pinned against: the RFC 1624 worked example; checksum validity preserved for
packets whose TCP/UDP and IPv4 checksums are made valid here by an independent
one's-complement sum (RFC 1071 / RFC 768 / RFC 793 pseudo-header); the translation
ranges and determinism the definition fixes; and pass-through of packets the NAT
does not apply to."""
import random

import numpy as np
import pytest

import nfcgen
import oracle
from tests.conftest import golden_rows


def ocsum(data: bytes) -> int:
    """RFC 1071 one's-complement sum of 16-bit big-endian words (independent of the oracle)."""
    if len(data) % 2:
        data += b"\0"
    s = 0
    for i in range(0, len(data), 2):
        s += data[i] << 8 | data[i + 1]
        s = (s & 0xFFFF) + (s >> 16)
    return s


def l4_check(frame: bytes) -> int:
    """One's-complement sum over pseudo-header + L4 segment (0xFFFF when the checksum is valid)."""
    ihl = (frame[14] & 15) * 4
    tot = frame[16] << 8 | frame[17]
    seg = frame[14 + ihl:14 + tot]
    ph = frame[26:34] + bytes([0, frame[23]]) + len(seg).to_bytes(2, "big")
    return ocsum(ph + seg)


def make_valid(frame: bytearray) -> bytearray:
    """Fill in a valid IPv4 header checksum and TCP/UDP checksum (test-side, RFC 1071)."""
    ihl = (frame[14] & 15) * 4
    proto = frame[23]
    ck_at = 14 + ihl + (16 if proto == 6 else 6)
    frame[ck_at:ck_at + 2] = b"\0\0"
    c = (~l4_check(bytes(frame))) & 0xFFFF
    if proto == 17 and c == 0:
        c = 0xFFFF
    frame[ck_at:ck_at + 2] = c.to_bytes(2, "big")
    frame[24:26] = b"\0\0"
    frame[24:26] = ((~ocsum(bytes(frame[14:14 + ihl]))) & 0xFFFF).to_bytes(2, "big")
    return frame


@pytest.mark.parametrize("row", golden_rows("rfc1624_incremental.txt"))
def test_csum_update_rfc1624_example(row):
    hc, m, m1, want = (int(x, 16) for x in row)
    assert oracle.csum_update(hc, m, m1) == want


def test_csum_update_equals_recompute():
    """RFC 1624: updating a valid checksum per changed word == recomputing it."""
    r = random.Random(3)
    for _ in range(2000):
        words = [r.getrandbits(16) for _ in range(r.randrange(2, 20))]
        hc = (~ocsum(b"".join(w.to_bytes(2, "big") for w in words))) & 0xFFFF
        k = r.randrange(len(words))
        new = r.getrandbits(16)
        upd = oracle.csum_update(hc, words[k], new)
        words[k] = new
        full = (~ocsum(b"".join(w.to_bytes(2, "big") for w in words))) & 0xFFFF
        # one's complement has two zeros: 0x0000 and 0xFFFF encode the same sum
        assert upd == full or {upd, full} == {0, 0xFFFF}


def _n3(n_acl=200, **kw):
    w = nfcgen.workload("N3", acl_rules=n_acl, small=True, **kw)
    return w, oracle.OracleChain(["NAT"], w.tables)


def test_nat_keeps_checksums_valid_and_translates_in_range():
    w, orc = _n3()
    t = w.tables
    t.nat_ext_ports = 1          # egress port 0 (no router in front): every IPv4 L4 packet
    orc = oracle.OracleChain(["NAT"], t)
    b = nfcgen.generate(w.traffic, t, 0, 2000)
    dn = {(int(e["proto"]), int(e["ext_addr"]), int(e["ext_port"])): (int(e["int_addr"]), int(e["int_port"]))
          for e in t.nat_dnat}
    pool = set(int(x) for x in t.nat_pool)
    seen = {}
    n_s = n_d = 0
    for i in range(b.n):
        fr = make_valid(bytearray(b.frame(i)))
        r, out, _ = orc.run_one(bytes(fr), i, headroom=0)
        assert r["drop_nf"] == 0xFF and r["out_len"] == len(fr)
        proto = fr[23]
        src, dst = int.from_bytes(fr[26:30], "big"), int.from_bytes(fr[30:34], "big")
        sp, dp = int.from_bytes(fr[34:36], "big"), int.from_bytes(fr[36:38], "big")
        osrc, odst = int.from_bytes(out[26:30], "big"), int.from_bytes(out[30:34], "big")
        osp, odp = int.from_bytes(out[34:36], "big"), int.from_bytes(out[36:38], "big")
        # checksums stay valid (IPv4 header sums to 0xFFFF; L4 incl. pseudo-header too)
        assert ocsum(out[14:34]) == 0xFFFF
        ck_at = 34 + (16 if proto == 6 else 6)
        if not (proto == 17 and fr[ck_at:ck_at + 2] == b"\0\0"):
            assert l4_check(out) == 0xFFFF
        # DNAT: exact (proto, dst, dport) entries
        if (proto, dst, dp) in dn:
            assert (odst, odp) == dn[(proto, dst, dp)]
            n_d += 1
        else:
            assert (odst, odp) == (dst, dp)
        # SNAT: inside prefixes (/4 of the first nibble) -> pool address, port in range
        inside = any((src >> 28) == (int(q["prefix"]) >> 28) for q in t.nat_inside)
        if inside:
            assert osrc in pool and t.nat_port_lo <= osp <= t.nat_port_hi
            n_s += 1
            key = (src, dst, sp, dp, proto)
            assert seen.setdefault(key, (osrc, osp)) == (osrc, osp)   # a pure function of the flow
        else:
            assert (osrc, osp) == (src, sp)
        # nothing else in the frame changes
        diff = [k for k in range(len(fr)) if fr[k] != out[k]]
        assert all(k in (24, 25, 26, 27, 28, 29, 30, 31, 32, 33, 34, 35, 36, 37, ck_at, ck_at + 1) for k in diff)
    assert n_s > 500 and n_d >= 5


def test_nat_pass_through():
    """Non-Internet egress ports, IPv6 and non-TCP/UDP packets leave the NAT untouched."""
    w, _ = _n3()
    t = w.tables
    t.nat_ext_ports = 0          # no Internet-facing port
    orc = oracle.OracleChain(["NAT"], t)
    b = nfcgen.generate(w.traffic, t, 0, 500)
    res, arena, _, _ = orc.run(b)
    assert np.array_equal(arena, b.arena)
    assert orc.stats[16 + 2] == 500 and orc.stats[16 + 3] == 0       # pass-through, not applied
    tp6 = nfcgen.TrafficParams(seed=9, v6_bp=10000, pkt_len=128, l4csum=1)
    t.nat_ext_ports = 0xFFFF
    orc6 = oracle.OracleChain(["NAT"], t)
    b6 = nfcgen.generate(tp6, t, 0, 300)
    _, a6, _, _ = orc6.run(b6)
    assert np.array_equal(a6, b6.arena)
