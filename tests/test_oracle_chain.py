"""Chain-level pins for the oracle and the input generator (CPU only).

ESP framing is checked against independent crypto libraries (`cryptography`
AES-CTR, stdlib hmac); chain semantics against the sequential definition
(same processing path, alerts in the same packet state) through
invariants of the stats vector and per-packet records.
"""
import hashlib
import hmac
import random

import numpy as np
import pytest

import nfcgen
import oracle
from tests.conftest import golden_rows


def _wl(name, **kw):
    return nfcgen.workload(name, small=True, **kw)


def test_generator_deterministic_and_splittable():
    w = _wl("C1")
    a = nfcgen.generate(w.traffic, w.tables, 1000, 200)
    b1 = nfcgen.generate(w.traffic, w.tables, 1000, 77)
    b2 = nfcgen.generate(w.traffic, w.tables, 1077, 123)
    fa = [a.frame(i) for i in range(200)]
    fb = [b1.frame(i) for i in range(77)] + [b2.frame(i) for i in range(123)]
    assert fa == fb
    assert all(len(f) == 64 for f in fa)
    assert all(int(o) % 16 == 0 for o in a.off)


def test_generator_imix_histogram():
    # IMIX = 61.22% 64 B, 23.47% 536 B, 15.31% 1360 B (chi-square, 2 dof, p>1e-4)
    row = dict(x.split(":") for x in golden_rows("paper_facts.txt")[0][1:])
    w = _wl("C3")
    b = nfcgen.generate(w.traffic, w.tables, 0, 200_000)
    n = b.n
    chi = 0.0
    for L, bp in row.items():
        exp = n * int(bp) / 10000
        obs = int(np.sum(b.len == int(L)))
        chi += (obs - exp) ** 2 / exp
    assert chi < 18.4
    assert set(np.unique(b.len).tolist()) == {64, 536, 1360}


def _stats_invariants(ch, res, n):
    st = ch.stats
    assert st[oracle.ST_PKTS] == n
    assert st[oracle.ST_FWD] + st[oracle.ST_DROP] == n
    assert st[oracle.ST_FWD] == int(np.sum(res["drop_nf"] == 0xFF))
    assert st[oracle.ST_PARSE_DROP] == int(np.sum(res["drop_nf"] == 0xFE))
    prev_in = n - int(st[oracle.ST_PARSE_DROP])
    for p in range(len(ch.kinds)):
        base = oracle.ST_POS_BASE + 4 * p
        assert st[base] == prev_in
        assert st[base + 1] == int(np.sum(res["drop_nf"] == p))
        assert st[base] == st[base + 1] + st[base + 2] + st[base + 3]
        prev_in = int(st[base] - st[base + 1])


def test_c1_chain_semantics():
    w = _wl("C1")
    w.traffic.malformed_ppm = 20_000
    w.traffic.ttl1_ppm = 10_000
    b = nfcgen.generate(w.traffic, w.tables, 0, 4096)
    ch = oracle.OracleChain(w.kinds, w.tables)
    res, arena, (mp, mq), npairs = ch.run(b)
    _stats_invariants(ch, res, 4096)
    drop = res["drop_nf"]
    # early drop: NFs after the dropping position record nothing
    acl_drop = drop == 0
    assert np.all(res["dpi_nmatch"][acl_drop] == 0)
    assert np.all(res["port"][drop != 0xFF] == 0xFFFF)
    assert np.all(res["port"][drop == 0xFF] < 16)
    assert 0 < acl_drop.sum() < 4096 * 0.2
    assert (drop == 0xFE).sum() > 20
    # planted matches (5%) produce pairs, one per distinct (pkt, pattern)
    assert int(res["dpi_nmatch"].sum()) == npairs == len(mp)
    assert 100 < npairs < 400
    pairs = set(zip(mp.tolist(), mq.tolist()))
    assert len(pairs) == npairs
    pats = w.tables.patterns()
    for pk, pat in list(pairs)[:50]:
        f = b.frame(pk)
        assert pats[pat] in f[42:]
    # forwarded IPv4 packets: valid checksum, TTL decremented, MAC rewritten
    fwd = np.nonzero(drop == 0xFF)[0]
    for i in fwd[:200]:
        o = int(b.off[i])
        out = arena[o:o + 64].tobytes()
        assert oracle.ipv4_checksum(out[14:34]) == 0
        assert out[22] == b.frame(i)[22] - 1
        assert out[42:] == b.frame(i)[42:]


def test_single_nf_chain_equals_nf_alone():
    w = _wl("C1")
    b = nfcgen.generate(w.traffic, w.tables, 0, 512)
    ch = oracle.OracleChain(["ACL"], w.tables)
    res, _, _, _ = ch.run(b)
    for i in range(512):
        f = b.frame(i)
        want = ch.acl(4, f[26:30], f[30:34], int.from_bytes(f[34:36], "big"),
                      int.from_bytes(f[36:38], "big"), f[23])
        assert res["acl_rule"][i] == (0xFFFF if want < 0 else want)
        act = w.tables.acl_rules["action"][want] if want >= 0 else w.tables.acl_default
        assert (res["drop_nf"][i] == 0) == (act == 1)


def _esp_reference(frame: bytes, sa, seq: int) -> bytes:
    """ESP transport frame built with independent crypto libraries (RFC 4303/3686/2404)."""
    from cryptography.hazmat.primitives.ciphers import Cipher, algorithms, modes
    v6 = frame[12:14] == b"\x86\xdd"
    l4 = 54 if v6 else 14 + 4 * (frame[14] & 15)
    ip_end = 54 + int.from_bytes(frame[18:20], "big") if v6 else 14 + int.from_bytes(frame[16:18], "big")
    P = frame[l4:ip_end]
    p = (4 - (len(P) + 2) % 4) % 4
    nh = frame[20] if v6 else frame[23]
    pt = P + bytes(range(1, p + 1)) + bytes([p, nh])
    iv = seq.to_bytes(8, "big")
    ctr0 = bytes(sa["nonce"]) + iv + b"\x00\x00\x00\x01"
    enc = Cipher(algorithms.AES(bytes(sa["aes_key"])), modes.CTR(ctr0)).encryptor()
    C = enc.update(pt) + enc.finalize()
    esp = int(sa["spi"]).to_bytes(4, "big") + seq.to_bytes(4, "big") + iv + C
    icv = hmac.new(bytes(sa["auth_key"]), esp, hashlib.sha1).digest()[:12]
    hdr = bytearray(frame[:l4])
    if v6:
        hdr[20] = 50
        hdr[18:20] = (int.from_bytes(hdr[18:20], "big") + 30 + p).to_bytes(2, "big")
    else:
        hdr[23] = 50
        hdr[16:18] = (int.from_bytes(hdr[16:18], "big") + 30 + p).to_bytes(2, "big")
        hdr[24:26] = b"\x00\x00"
        s = sum(int.from_bytes(hdr[k:k + 2], "big") for k in range(14, l4, 2))
        while s >> 16:
            s = (s & 0xFFFF) + (s >> 16)
        hdr[24:26] = (~s & 0xFFFF).to_bytes(2, "big")
    return bytes(hdr) + esp + icv


@pytest.mark.parametrize("v6", [False, True])
def test_esp_vs_independent_crypto(v6):
    w = _wl("C2")
    w.traffic.v6_bp = 10000 if v6 else 0
    w.traffic.pkt_len = 1  # ragged lengths exercise all pad lengths
    if v6:
        w.tables.routes6 = nfcgen.gen_routes6(np.random.default_rng(1), 50, 8)
        w.tables.nh6, w.tables.pmac6 = nfcgen.gen_nexthops(np.random.default_rng(2), 8, 4)
    b = nfcgen.generate(w.traffic, w.tables, 0, 300)
    ch = oracle.OracleChain(["IPSEC"], w.tables)
    res, arena, _, _ = ch.run(b)
    seqs = {}
    pads = set()
    for i in range(b.n):
        f = b.frame(i)
        r = res[i]
        assert r["drop_nf"] == 0xFF
        al = 16 if v6 else 4
        so = 22 if v6 else 26
        tup = f[so:so + 2 * al] + f[so + 2 * al:so + 2 * al + 4]
        sa_idx = oracle.toeplitz(oracle.MS_RSS_KEY, tup) % 64
        assert r["esp_sa"] == sa_idx
        seqs[sa_idx] = seqs.get(sa_idx, 0) + 1
        assert r["esp_seq"] == seqs[sa_idx]  # seq0 = 0, ++seq in global order
        want = _esp_reference(f, w.tables.sas[sa_idx], int(r["esp_seq"]))
        o = int(b.off[i]) - 16
        assert r["out_len"] == len(want)
        assert arena[o:o + len(want)].tobytes() == want
        pads.add((len(want) - len(f)) - 30)
    assert pads == {0, 1, 2, 3}


def test_lb_backend_formula():
    w = _wl("C3")
    b = nfcgen.generate(w.traffic, w.tables, 0, 300)
    ch = oracle.OracleChain(["LB"], w.tables)
    res, _, _, _ = ch.run(b)
    for i in range(b.n):
        f = b.frame(i)
        h = oracle.toeplitz(bytes(w.tables.lb_key), f[26:34] + f[34:38])
        be = (h * 64) >> 32
        assert res["lb_backend"][i] == be
        assert res["port"][i] == w.tables.lb_ports[be]


def test_seq_override_matches_counter():
    w = _wl("C2")
    b = nfcgen.generate(w.traffic, w.tables, 0, 64)
    ch1 = oracle.OracleChain(["IPSEC"], w.tables)
    r1, a1, _, _ = ch1.run(b)
    ch2 = oracle.OracleChain(["IPSEC"], w.tables)
    r2, a2, _, _ = ch2.run(b, seq_override=r1["esp_seq"])
    assert np.array_equal(r1, r2) and np.array_equal(a1, a2)
