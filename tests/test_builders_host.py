"""CPU tests of the product's table builders (include/nfc_debug.h): each device
image is walked on the host with the kernel's algorithm and compared with the
oracle, plus the paper's structural claims (IPv4 lookup takes two
memory accesses, IPv6 up to 7)."""
import math
import random

import numpy as np
import pytest

import nfcgen
import oracle
from tests.conftest import golden_rows


@pytest.fixture(scope="module")
def nfc():
    from paper_conf_hpca_hul18_b200 import build
    build.build()
    from paper_conf_hpca_hul18_b200 import nfc as m
    return m


def _pattern_tables(pats, acts=None):
    t = nfcgen.Tables()
    off = np.zeros(len(pats) + 1, dtype=np.uint32)
    off[1:] = np.cumsum([len(p) for p in pats])
    t.pat_blob = np.frombuffer(b"".join(pats), dtype=np.uint8).copy()
    t.pat_off = off
    t.pat_action = np.array(acts if acts is not None else [0] * len(pats), dtype=np.uint8)
    return t


@pytest.mark.parametrize("case", ["c1", "c4", "allbytes", "tiny"])
def test_dfa_image_vs_oracle(nfc, case):
    rng = random.Random(hash(case) & 0xFFFF)
    if case == "c1":
        t = nfcgen.workload("C1").tables
    elif case == "c4":
        t = nfcgen.workload("C4").tables
    elif case == "allbytes":  # every byte value occurs in some pattern: 256 classes, no "other" class
        pats = [bytes([b, (b * 7) & 255]) for b in range(256)] + [b"\x00\x01\x02"]
        t = _pattern_tables(pats, [rng.random() < 0.1 for _ in pats])
    else:
        pats = [bytes(rng.choice(b"ab") for _ in range(rng.randrange(1, 5))) for _ in range(12)]
        t = _pattern_tables(pats)
    img = nfc.HostImage("DPI", blob=t.pat_blob, off=t.pat_off, action=t.pat_action)
    ns, ncls, wide = img.dpi_shape()
    assert ncls <= 256
    orc = oracle.OracleChain(["DPI"], t)
    pats = t.patterns()
    for k in range(400):
        n = rng.randrange(0, 200)
        alpha = b"ab" if case == "tiny" else None
        text = bytes(rng.choice(alpha) if alpha else rng.randrange(256) for _ in range(n))
        for _ in range(rng.randrange(0, 4)):
            p = rng.choice(pats)
            i = rng.randrange(0, len(text) + 1)
            text = text[:i] + p + text[i:]
        ids, drop = img.dpi(text)
        assert ids == orc.ac_match(text)
        assert drop == any(t.pat_action[j] for j in ids)


@pytest.mark.parametrize("case", ["c3", "c1", "tiny", "allbytes"])
def test_dfa_tiered_walk_vs_oracle(nfc, case):
    """The kernel's tiered DFA placement (dense rows / sparse records / cold rows,
    DpiImg::sparse) gives the oracle's match sets for every split of the states,
    including splits where records fall back to the full table."""
    rng = random.Random(7 + len(case))
    if case == "c3":
        t = nfcgen.workload("C3").tables
    elif case == "c1":
        t = nfcgen.workload("C1").tables
    elif case == "allbytes":
        pats = [bytes([b, (b * 7) & 255, b ^ 0x55]) for b in range(256)] + [b"\x00\x01\x02"]
        t = _pattern_tables(pats, [rng.random() < 0.1 for _ in pats])
    else:
        pats = [bytes(rng.choice(b"ab") for _ in range(rng.randrange(1, 6))) for _ in range(16)]
        t = _pattern_tables(pats)
    img = nfc.HostImage("DPI", blob=t.pat_blob, off=t.pat_off, action=t.pat_action)
    ns, ncls, wide = img.dpi_shape()
    nd1, nok = img.dpi_tier_shape()
    assert 1 <= nd1 <= min(ns, 257)
    orc = oracle.OracleChain(["DPI"], t)
    pats = t.patterns()
    splits = [(nd1, ns - nd1), (nd1, (ns - nd1) // 3), (max(1, nd1 // 2), ns), (1, 0), (ns, 0)]
    used = [0, 0, 0]
    for k in range(150):
        n = rng.randrange(0, 300)
        text = bytes(rng.choice(b"ab") if case == "tiny" else rng.randrange(256) for _ in range(n))
        for _ in range(rng.randrange(0, 6)):
            p = rng.choice(pats)
            i = rng.randrange(0, len(text) + 1)
            text = text[:i] + p + text[i:]
        want = orc.ac_match(text)
        for hot, sparse in splits:
            ids, drop, ts = img.dpi_tier(text, hot, sparse)
            assert ids == want, (hot, sparse)
            assert drop == any(t.pat_action[j] for j in ids)
            used = [a + b for a, b in zip(used, ts)]
    assert used[1] > 0 and used[2] > 0          # sparse and cold paths both exercised
    if case in ("c3", "c1"):
        assert nok >= 0.99 * (ns - nd1)         # nearly every deep state has <= 2 exceptions


@pytest.mark.parametrize("case", ["c1", "c5", "tiny", "allbytes"])
def test_dfa_slot_walk_vs_oracle(nfc, case):
    """The kernel's DM_FULL slot image (DpiImg::frows: signed slots, accepting states
    negative, rows addressed relative to slot 0) gives the oracle's match sets, the
    accept-event count of a brute-force scan, and -- for walks with exactly one accept
    event -- a match summary (size, DROP flag) equal to the oracle's result."""
    rng = random.Random(11 + len(case))
    if case in ("c1", "c5"):
        t = nfcgen.workload(case.upper()).tables
    elif case == "allbytes":
        pats = [bytes([b, (b * 7) & 255, b ^ 0x55]) for b in range(256)] + [b"\x00\x01\x02"]
        t = _pattern_tables(pats, [rng.random() < 0.1 for _ in pats])
    else:
        pats = [bytes(rng.choice(b"ab") for _ in range(rng.randrange(1, 6))) for _ in range(16)]
        t = _pattern_tables(pats)
    img = nfc.HostImage("DPI", blob=t.pat_blob, off=t.pat_off, action=t.pat_action)
    orc = oracle.OracleChain(["DPI"], t)
    pats = t.patterns()
    singles = 0
    for k in range(200):
        n = rng.randrange(0, 300)
        text = bytes(rng.choice(b"ab") if case == "tiny" else rng.randrange(256) for _ in range(n))
        for _ in range(rng.randrange(0, 3)):
            p = rng.choice(pats)
            i = rng.randrange(0, len(text) + 1)
            text = text[:i] + p + text[i:]
        want = orc.ac_match(text)
        ids, drop, events, summary = img.dpi_slot(text)
        assert ids == want
        assert drop == any(t.pat_action[j] for j in ids)
        # accept events = end positions at which some pattern occurs (brute force)
        ends = sum(1 for e in range(1, len(text) + 1) if any(text[:e].endswith(p) for p in pats))
        assert events == ends
        if events == 1:
            singles += 1
            assert (summary >> 20) & 0x7FF == len(want)
            assert bool(summary >> 31) == drop
    assert singles > 0 or case == "tiny"     # binary texts always hit several patterns


def test_dir24_8_vs_oracle_and_two_accesses(nfc):
    w = nfcgen.workload("C1")
    t = w.tables
    # add /25../32 routes so TBLlong is exercised
    rng = np.random.default_rng(5)
    extra = nfcgen.gen_routes4(rng, 300, len(t.nh4), default_route=False)
    extra = extra[extra["len"] > 24]
    routes = np.concatenate([t.routes4, extra])
    _, idx = np.unique(np.stack([routes["prefix"].astype(np.int64), routes["len"].astype(np.int64)], 1),
                       axis=0, return_index=True)
    routes = routes[np.sort(idx)]
    t2 = nfcgen.Tables(routes4=routes, nh4=t.nh4, pmac4=t.pmac4)
    img = nfc.HostImage("LPM4", routes=routes, nexthops=t.nh4, port_macs=t.pmac4)
    orc = oracle.OracleChain(["LPM4"], t2)
    r = random.Random(1)
    reads_seen = set()
    max_reads = int(golden_rows("paper_facts.txt")[1][1])
    for k in range(20000):
        if k % 2:
            rt = routes[r.randrange(len(routes))]
            L = int(rt["len"])
            a = int(rt["prefix"]) | (r.getrandbits(32) & ((1 << (32 - L)) - 1))
        else:
            a = r.getrandbits(32)
        nh, reads = img.lpm4(a)
        want = orc.lpm4(a)
        assert nh == (0x7FFF if want < 0 else want)
        assert reads <= max_reads  # "two memory accesses"
        reads_seen.add(reads)
    assert reads_seen == {1, 2}


def test_lpm6_waldvogel_vs_oracle_full_c4(nfc):
    """200K IPv6 prefixes: binary search on prefix lengths, <= 7 hash-level probes."""
    t = nfcgen.workload("C4").tables
    img = nfc.HostImage("LPM6", routes=t.routes6, nexthops=t.nh6, port_macs=t.pmac6)
    orc = oracle.OracleChain(["LPM6"], t)
    levels = img.lpm6_levels()
    bound = math.ceil(math.log2(levels + 1))
    assert bound <= int(golden_rows("paper_facts.txt")[2][1])
    r = random.Random(2)
    worst = 0
    for k in range(20000):
        if k % 4:
            rt = t.routes6[r.randrange(len(t.routes6))]
            L = int(rt["len"])
            a = int.from_bytes(bytes(rt["prefix"]), "big") | (r.getrandbits(128) & ((1 << (128 - L)) - 1))
        else:
            a = r.getrandbits(128)
        dst = a.to_bytes(16, "big")
        nh, probes, _ = img.lpm6(dst)
        want = orc.lpm6(dst)
        assert nh == (0x7FFF if want < 0 else want), k
        worst = max(worst, probes)
    assert worst <= bound


def test_lpm6_adversarial_nesting(nfc):
    """Nested prefixes at many lengths (markers with and without a best-matching prefix)."""
    r = random.Random(9)
    base = r.getrandbits(128)
    routes = []
    seen = set()
    for L in [1, 3, 8, 16, 17, 31, 32, 33, 47, 48, 63, 64, 65, 96, 127, 128]:
        for j in range(3):
            v = base ^ (r.getrandbits(4) << (128 - L)) if j else base
            v &= ((1 << L) - 1) << (128 - L)
            if (v, L) in seen:
                continue
            seen.add((v, L))
            routes.append((v, L))
    rt = np.zeros(len(routes), dtype=nfcgen.ROUTE6)
    for i, (v, L) in enumerate(routes):
        rt[i]["prefix"] = np.frombuffer(v.to_bytes(16, "big"), dtype=np.uint8)
        rt[i]["len"] = L
        rt[i]["nh"] = i % 7
    nh, pm = nfcgen.gen_nexthops(np.random.default_rng(1), 7, 2)
    t = nfcgen.Tables(routes6=rt, nh6=nh, pmac6=pm)
    img = nfc.HostImage("LPM6", routes=rt, nexthops=nh, port_macs=pm)
    orc = oracle.OracleChain(["LPM6"], t)
    for k in range(5000):
        a = base ^ (r.getrandbits(128) >> r.randrange(0, 128))
        dst = a.to_bytes(16, "big")
        want = orc.lpm6(dst)
        assert img.lpm6(dst)[0] == (0x7FFF if want < 0 else want)


@pytest.mark.parametrize("fam,n", [(4, 40), (6, 40), (4, 1000), (4, 10000), (6, 1000)])
def test_acl_image_vs_oracle(nfc, fam, n):
    """Bit-vector image (one 64-bit word per field for <= 64 rules, else the aggregate
    level picks candidate words, ABV) == linear first-match scan, up to the paper's
    10K-rule ACL."""
    rng = np.random.default_rng(40 + fam + n)
    rules = np.concatenate([nfcgen.gen_acl(rng, n, 4), nfcgen.gen_acl(rng, n if fam == 6 else 40, 6)])
    rng.shuffle(rules)
    t = nfcgen.Tables(acl_rules=rules, acl_default=1)
    img = nfc.HostImage("ACL", rules=rules, default_action=1)
    orc = oracle.OracleChain(["ACL"], t)
    r = random.Random(fam + n)
    nb = 4 if fam == 4 else 16
    fam_idx = [i for i in range(len(rules)) if rules[i]["family"] == fam]
    for _ in range(3000 if n <= 1000 else 600):
        src = bytearray(r.getrandbits(8) for _ in range(nb))
        dst = bytearray(r.getrandbits(8) for _ in range(nb))
        sp, dp, proto = r.getrandbits(16), r.getrandbits(16), r.choice([1, 6, 17])
        if r.random() < 0.7:
            ru = rules[r.choice(fam_idx)]
            for arr, p, L in ((src, ru["src"], int(ru["slen"])), (dst, ru["dst"], int(ru["dlen"]))):
                for k in range(nb):
                    keep = L - 8 * k
                    m = 0xFF if keep >= 8 else 0 if keep <= 0 else (0xFF << (8 - keep)) & 0xFF
                    arr[k] = (int(p[k]) & m) | (arr[k] & ~m & 0xFF)
            sp = r.randint(int(ru["sp_lo"]), int(ru["sp_hi"]))
            dp = r.randint(int(ru["dp_lo"]), int(ru["dp_hi"]))
            proto = int(ru["proto"]) if not ru["proto_any"] else proto
        rule, act = img.acl(fam, bytes(src), bytes(dst), sp, dp, proto)
        want = orc.acl(fam, bytes(src), bytes(dst), sp, dp, proto)
        assert rule == (0xFFFF if want < 0 else want)
        assert act == (1 if want < 0 else int(rules[want]["action"]))


@pytest.mark.parametrize("row", golden_rows("fips197_aes128.txt"))
def test_ttable_aes_fips197(nfc, row):
    key, pt, ct = (bytes.fromhex(x) for x in row)
    assert nfc.dbg_aes128_block(key, pt) == ct


@pytest.mark.parametrize("row", golden_rows("ms_rss_toeplitz.txt"))
def test_nibble_toeplitz_ms_rss(nfc, row):
    import ipaddress
    src, sp, dst, dp, h_ip, h_l4 = row
    a = ipaddress.ip_address(src).packed + ipaddress.ip_address(dst).packed
    assert nfc.dbg_toeplitz(oracle.MS_RSS_KEY, a) == int(h_ip, 16)
    assert nfc.dbg_toeplitz(oracle.MS_RSS_KEY, a + int(sp).to_bytes(2, "big") + int(dp).to_bytes(2, "big")) == int(h_l4, 16)


@pytest.mark.parametrize("row", [r for r in golden_rows("rfc2202_hmac_sha1.txt") if len(r[0]) <= 40])
def test_ipad_opad_hmac_rfc2202(nfc, row):
    key = bytes.fromhex(row[0]).ljust(20, b"\x00")  # HMAC zero-pads keys shorter than the block
    assert nfc.dbg_hmac_sha1(key, bytes.fromhex(row[1])).hex() == row[2]


def test_nat_image_vs_oracle(nfc):
    """The NAT device image (DNAT open-addressing table, inside prefixes, pool, Toeplitz
    nibbles) walked with the kernel's nat_values gives the oracle's translated header
    for every packet of an N3 sample, and rejects malformed specs."""
    w = nfcgen.workload("N3", acl_rules=200, small=True, pkt_len=1)
    t = w.tables
    t.nat_ext_ports = 1
    img = nfc.HostImage("NAT", inside=t.nat_inside, pool=t.nat_pool, port_lo=t.nat_port_lo, port_hi=t.nat_port_hi,
                        dnat=t.nat_dnat, ext_ports=1, key=t.nat_key)
    orc = oracle.OracleChain(["NAT"], t)
    b = nfcgen.generate(w.traffic, t, 0, 1500)
    max_probes = 0
    for i in range(b.n):
        fr = b.frame(i)
        if fr[12:14] != b"\x08\x00" or fr[23] not in (6, 17):
            continue
        l4 = 14 + 4 * (fr[14] & 15)
        ca = l4 + (16 if fr[23] == 6 else 6)
        r, out, _ = orc.run_one(fr, i, headroom=0)
        got, probes = img.nat(fr[23], int.from_bytes(fr[26:30], "big"), int.from_bytes(fr[30:34], "big"),
                              int.from_bytes(fr[l4:l4 + 2], "big"), int.from_bytes(fr[l4 + 2:l4 + 4], "big"),
                              int.from_bytes(fr[ca:ca + 2], "big"))
        want = (int.from_bytes(out[26:30], "big"), int.from_bytes(out[30:34], "big"),
                int.from_bytes(out[l4:l4 + 2], "big"), int.from_bytes(out[l4 + 2:l4 + 4], "big"),
                int.from_bytes(out[ca:ca + 2], "big"))
        assert got == want, i
        max_probes = max(max_probes, probes)
    assert max_probes <= 16                      # load factor <= 1/2
    dup = np.concatenate([t.nat_dnat, t.nat_dnat[:1]])
    with pytest.raises(Exception):
        nfc.HostImage("NAT", inside=t.nat_inside, pool=t.nat_pool, port_lo=1, port_hi=2, dnat=dup, key=t.nat_key)
    with pytest.raises(Exception):
        nfc.HostImage("NAT", inside=t.nat_inside, pool=t.nat_pool, port_lo=9, port_hi=2, dnat=t.nat_dnat,
                      key=t.nat_key)


@pytest.mark.parametrize("n,which", [(64, 0), (40, 0), (3000, 1), (10000, 1)])
def test_acl4_fused_images_vs_oracle(nfc, n, which):
    """The fused kernel's other IPv4 ACL images, looked up as the kernel does: the search
    image of <= 64-rule sets (10-bit buckets, two or three halvings over padded keys,
    bitsets at an affine image of the key address) and the 16-bit first level of > 2K-rule
    sets (per-prefix / per-port intervals) == the oracle's linear first-match scan, on
    random 5-tuples, tuples inside rules, and tuples on every rule's interval edges
    (including 0 / 2^32-1 and ports 0 / 65535)."""
    rng = np.random.default_rng(900 + n)
    rules = nfcgen.gen_acl(rng, n, 4)
    t = nfcgen.Tables(acl_rules=rules, acl_default=1)
    img = nfc.HostImage("ACL", rules=rules, default_action=1)
    orc = oracle.OracleChain(["ACL"], t)
    assert img.acl4_image(which, 0, 0, 0, 0, 6) is not None, "the rule set should have this image"
    edges_ip, edges_port = [0, 0xFFFFFFFF], [0, 65535]
    for ru in rules:
        for fld, ln in (("src", "slen"), ("dst", "dlen")):
            k = int.from_bytes(bytes(ru[fld][:4]), "big")
            L = int(ru[ln])
            m = (0xFFFFFFFF << (32 - L)) & 0xFFFFFFFF if L else 0
            lo, hi = k & m, (k & m) | (~m & 0xFFFFFFFF)
            edges_ip += [lo, hi, (lo - 1) & 0xFFFFFFFF, (hi + 1) & 0xFFFFFFFF]
        for a, b in ((int(ru["sp_lo"]), int(ru["sp_hi"])), (int(ru["dp_lo"]), int(ru["dp_hi"]))):
            edges_port += [a, b, (a - 1) & 0xFFFF, (b + 1) & 0xFFFF]
    r = random.Random(n)
    for it in range(4000):
        mode = it % 3
        if mode == 0:
            src, dst, sp, dp = r.getrandbits(32), r.getrandbits(32), r.getrandbits(16), r.getrandbits(16)
        elif mode == 1:
            src, dst = r.choice(edges_ip), r.choice(edges_ip)
            sp, dp = r.choice(edges_port), r.choice(edges_port)
        else:
            ru = rules[r.randrange(len(rules))]
            def inside(p, L):
                k = int.from_bytes(bytes(p[:4]), "big")
                m = (0xFFFFFFFF << (32 - L)) & 0xFFFFFFFF if L else 0
                return (k & m) | (r.getrandbits(32) & ~m & 0xFFFFFFFF)
            src, dst = inside(ru["src"], int(ru["slen"])), inside(ru["dst"], int(ru["dlen"]))
            sp, dp = r.randint(int(ru["sp_lo"]), int(ru["sp_hi"])), r.randint(int(ru["dp_lo"]), int(ru["dp_hi"]))
        proto = r.choice([1, 6, 17])
        got = img.acl4_image(which, src, dst, sp, dp, proto)
        want = orc.acl(4, src.to_bytes(4, "big"), dst.to_bytes(4, "big"), sp, dp, proto)
        assert got[0] == (0xFFFF if want < 0 else want), (it, mode, hex(src), hex(dst), sp, dp, proto, got, want)
        assert got[1] == (1 if want < 0 else int(rules[want]["action"]))
