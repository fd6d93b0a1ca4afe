"""Pins for the CPU oracle against what the paper and external standards fix.

Each test pins oracle.c to something other than itself: published test
vectors (tests/golden/, each file citing its source), independent library
routines (hashlib/hmac, `cryptography`, `ipaddress`), brute force on tiny
inputs, closed forms and invariants.  CPU only.
"""
import hashlib
import hmac
import ipaddress
import random

import numpy as np
import pytest

import nfcgen
import oracle
from tests.conftest import golden_rows


# ------------------------------------------------------------- crypto vectors
@pytest.mark.parametrize("row", golden_rows("fips197_aes128.txt"))
def test_aes128_fips197(row):
    key, pt, ct = (bytes.fromhex(x) for x in row)
    assert oracle.aes128_block(key, pt) == ct


@pytest.mark.parametrize("row", golden_rows("rfc3686_aes_ctr.txt"))
def test_aes128_ctr_rfc3686(row):
    key, nonce, iv, pt, ct = (bytes.fromhex(x) for x in row)
    ctr0 = nonce + iv + b"\x00\x00\x00\x01"
    assert oracle.aes128_ctr(key, ctr0, pt) == ct


def test_aes_ctr_vs_cryptography_library():
    from cryptography.hazmat.primitives.ciphers import Cipher, algorithms, modes
    rng = random.Random(7)
    for n in (0, 1, 15, 16, 17, 100, 1438):
        key = bytes(rng.randrange(256) for _ in range(16))
        ctr0 = bytes(rng.randrange(256) for _ in range(12)) + b"\x00\x00\x00\x01"
        data = bytes(rng.randrange(256) for _ in range(n))
        enc = Cipher(algorithms.AES(key), modes.CTR(ctr0)).encryptor()
        assert oracle.aes128_ctr(key, ctr0, data) == enc.update(data) + enc.finalize()


@pytest.mark.parametrize("row", golden_rows("sha1.txt"))
def test_sha1_fips180(row):
    msg = {"EMPTY": b"", "MILLION_A": b"a" * 1_000_000}.get(row[0])
    if msg is None:
        msg = bytes.fromhex(row[0])
    assert oracle.sha1(msg).hex() == row[1]


def test_sha1_vs_hashlib_all_padding_lengths():
    rng = random.Random(3)
    for n in range(0, 200):
        m = bytes(rng.randrange(256) for _ in range(n))
        assert oracle.sha1(m) == hashlib.sha1(m).digest()


@pytest.mark.parametrize("row", golden_rows("rfc2202_hmac_sha1.txt"))
def test_hmac_sha1_rfc2202(row):
    key, data = bytes.fromhex(row[0]), bytes.fromhex(row[1])
    assert oracle.hmac_sha1(key, data).hex() == row[2]


def test_hmac_vs_stdlib():
    rng = random.Random(5)
    for n in (0, 1, 55, 56, 63, 64, 65, 1500):
        key = bytes(rng.randrange(256) for _ in range(20))
        m = bytes(rng.randrange(256) for _ in range(n))
        assert oracle.hmac_sha1(key, m) == hmac.new(key, m, hashlib.sha1).digest()


def _addr(s):
    return ipaddress.ip_address(s).packed


@pytest.mark.parametrize("row", golden_rows("ms_rss_toeplitz.txt"))
def test_toeplitz_ms_rss(row):
    src, sp, dst, dp, h_ip, h_l4 = row
    ip = _addr(src) + _addr(dst)
    l4 = ip + int(sp).to_bytes(2, "big") + int(dp).to_bytes(2, "big")
    assert oracle.toeplitz(oracle.MS_RSS_KEY, ip) == int(h_ip, 16)
    assert oracle.toeplitz(oracle.MS_RSS_KEY, l4) == int(h_l4, 16)


def test_toeplitz_linearity():
    # Toeplitz hashing is GF(2)-linear in its input: h(a^b) = h(a)^h(b).
    rng = random.Random(11)
    key = bytes(rng.randrange(256) for _ in range(40))
    for _ in range(50):
        a = bytes(rng.randrange(256) for _ in range(36))
        b = bytes(rng.randrange(256) for _ in range(36))
        ab = bytes(x ^ y for x, y in zip(a, b))
        assert oracle.toeplitz(key, ab) == oracle.toeplitz(key, a) ^ oracle.toeplitz(key, b)


@pytest.mark.parametrize("row", golden_rows("ipv4_checksum.txt"))
def test_ipv4_checksum(row):
    hdr = bytes.fromhex(row[0])
    ck = oracle.ipv4_checksum(hdr)
    assert ck == int(row[1], 16)
    full = hdr[:10] + ck.to_bytes(2, "big") + hdr[12:]
    assert oracle.ipv4_checksum(full) == 0  # RFC 1071: a valid header sums to 0xFFFF


def test_rfc1624_incremental_equals_full():
    # RFC 1624 eqn. 3 HC' = ~(~HC + ~m + m') equals the full recompute after a TTL decrement.
    rng = random.Random(13)
    for _ in range(2000):
        h = bytearray(rng.randrange(256) for _ in range(20))
        h[0] = 0x45
        h[8] = rng.randrange(2, 256)
        h[10] = h[11] = 0
        hc = oracle.ipv4_checksum(bytes(h))
        m = (h[8] << 8) | h[9]
        h[8] -= 1
        mp = (h[8] << 8) | h[9]
        s = (~hc & 0xFFFF) + (~m & 0xFFFF) + mp
        while s >> 16:
            s = (s & 0xFFFF) + (s >> 16)
        inc = ~s & 0xFFFF
        assert inc == oracle.ipv4_checksum(bytes(h))


# ------------------------------------------------------------- DPI vs brute force
def _tables_with_patterns(pats, actions=None):
    t = nfcgen.Tables()
    off = np.zeros(len(pats) + 1, dtype=np.uint32)
    off[1:] = np.cumsum([len(p) for p in pats])
    t.pat_blob = np.frombuffer(b"".join(pats), dtype=np.uint8).copy()
    t.pat_off = off
    t.pat_action = np.array(actions or [0] * len(pats), dtype=np.uint8)
    return t


def test_aho_corasick_vs_naive_substring():
    rng = random.Random(17)
    for trial in range(40):
        alpha = b"ab" if trial % 2 == 0 else b"abcd"
        pats = []
        while len(pats) < rng.randrange(1, 12):
            p = bytes(rng.choice(alpha) for _ in range(rng.randrange(1, 6)))
            pats.append(p)  # duplicates allowed: each ID matches independently
        ch = oracle.OracleChain(["DPI"], _tables_with_patterns(pats))
        for _ in range(30):
            text = bytes(rng.choice(alpha) for _ in range(rng.randrange(0, 40)))
            want = sorted(j for j, p in enumerate(pats) if p in text)
            assert ch.ac_match(text) == want, (pats, text)
        ch.close()


def test_aho_corasick_all_byte_values():
    rng = random.Random(19)
    pats = [bytes(rng.randrange(256) for _ in range(rng.randrange(1, 9))) for _ in range(60)]
    pats.append(b"\x00\x00")
    pats.append(b"\xff")
    ch = oracle.OracleChain(["DPI"], _tables_with_patterns(pats))
    for _ in range(200):
        text = bytes(rng.randrange(256) for _ in range(rng.randrange(0, 300)))
        if rng.random() < 0.5:
            p = rng.choice(pats)
            k = rng.randrange(0, len(text) + 1)
            text = text[:k] + p + text[k:]
        assert ch.ac_match(text) == sorted(j for j, p in enumerate(pats) if p in text)


# ------------------------------------------------------------- LPM vs linear scan
def _linear_lpm(routes, addr_int, bits):
    best, bl = -1, -1
    for r in routes:
        L = int(r["len"])
        if bits == 32:
            pv = int(r["prefix"])
        else:
            pv = int.from_bytes(bytes(r["prefix"]), "big")
        mask = ((1 << L) - 1) << (bits - L) if L else 0
        if (addr_int ^ pv) & mask == 0 and L > bl:
            best, bl = int(r["nh"]), L
    return best


def test_lpm4_trie_vs_linear_scan():
    rng = np.random.default_rng(23)
    t = nfcgen.Tables()
    t.routes4 = nfcgen.gen_routes4(rng, 300, 50, default_route=False)
    t.nh4, t.pmac4 = nfcgen.gen_nexthops(rng, 50, 4)
    ch = oracle.OracleChain(["LPM4"], t)
    r = random.Random(1)
    for k in range(3000):
        if k % 2:
            rt = t.routes4[r.randrange(len(t.routes4))]
            L = int(rt["len"])
            a = int(rt["prefix"]) | (r.getrandbits(32) & ((1 << (32 - L)) - 1))
        else:
            a = r.getrandbits(32)
        assert ch.lpm4(a) == _linear_lpm(t.routes4, a, 32)


def test_lpm6_trie_vs_linear_scan():
    rng = np.random.default_rng(29)
    t = nfcgen.Tables()
    t.routes6 = nfcgen.gen_routes6(rng, 400, 50, default_route=False)
    t.nh6, t.pmac6 = nfcgen.gen_nexthops(rng, 50, 4)
    ch = oracle.OracleChain(["LPM6"], t)
    r = random.Random(2)
    for k in range(1500):
        if k % 2:
            rt = t.routes6[r.randrange(len(t.routes6))]
            L = int(rt["len"])
            a = int.from_bytes(bytes(rt["prefix"]), "big") | (r.getrandbits(128) & ((1 << (128 - L)) - 1))
        else:
            a = r.getrandbits(128)
        assert ch.lpm6(a.to_bytes(16, "big")) == _linear_lpm(t.routes6, a, 128)


# ------------------------------------------------------------- ACL vs ipaddress
def _acl_ref(rules, fam, src, dst, sp, dp, proto):
    """First match by an independent formulation (ipaddress network containment)."""
    for i, r in enumerate(rules):
        if r["family"] != fam:
            continue
        nb = 4 if fam == 4 else 16
        sn = ipaddress.ip_network((bytes(r["src"][:nb]), int(r["slen"])))
        dn = ipaddress.ip_network((bytes(r["dst"][:nb]), int(r["dlen"])))
        if ipaddress.ip_address(src) not in sn or ipaddress.ip_address(dst) not in dn:
            continue
        if not (r["sp_lo"] <= sp <= r["sp_hi"] and r["dp_lo"] <= dp <= r["dp_hi"]):
            continue
        if not r["proto_any"] and r["proto"] != proto:
            continue
        return i
    return -1


@pytest.mark.parametrize("fam", [4, 6])
def test_acl_first_match_vs_ipaddress(fam):
    rng = np.random.default_rng(31 + fam)
    t = nfcgen.Tables()
    t.acl_rules = nfcgen.gen_acl(rng, 64, fam)
    ch = oracle.OracleChain(["ACL"], t)
    r = random.Random(fam)
    nb = 4 if fam == 4 else 16
    for _ in range(1500):
        if r.random() < 0.6:  # inside a random rule
            rule = t.acl_rules[r.randrange(64)]
            src = bytearray(r.getrandbits(8) for _ in range(nb))
            dst = bytearray(r.getrandbits(8) for _ in range(nb))
            for arr, p, L in ((src, rule["src"], int(rule["slen"])), (dst, rule["dst"], int(rule["dlen"]))):
                for k in range(nb):
                    keep = L - 8 * k
                    m = 0xFF if keep >= 8 else 0 if keep <= 0 else (0xFF << (8 - keep)) & 0xFF
                    arr[k] = (int(p[k]) & m) | (arr[k] & ~m & 0xFF)
            sp = r.randint(int(rule["sp_lo"]), int(rule["sp_hi"]))
            dp = r.randint(int(rule["dp_lo"]), int(rule["dp_hi"]))
            proto = int(rule["proto"]) if not rule["proto_any"] else r.choice([6, 17])
        else:
            src = bytearray(r.getrandbits(8) for _ in range(nb))
            dst = bytearray(r.getrandbits(8) for _ in range(nb))
            sp, dp, proto = r.getrandbits(16), r.getrandbits(16), r.choice([1, 6, 17])
        src, dst = bytes(src), bytes(dst)
        got = ch.acl(fam, src, dst, sp, dp, proto)
        assert got == _acl_ref(t.acl_rules, fam, src, dst, sp, dp, proto)
