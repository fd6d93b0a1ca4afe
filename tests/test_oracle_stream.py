"""Pins of the stateful (cross-packet) DPI oracle, oracle/stream_dpi.py (NEXT-4, R#32).

The oracle is brute force over each flow's concatenated stream; it is pinned by
a hand-worked example, flow separation, agreement with the C oracle's
Aho-Corasick matcher on one-packet flows (an independent algorithm), and split
invariance (cutting a stream into packets and calls never changes the set of
occurrences in stream coordinates)."""
import random

import numpy as np
import pytest

import nfcgen
from nfcgen.stream import stream_batch
from oracle.stream_dpi import StreamDPI, parse


def _udp(payload: bytes, src=0x0A000001, dst=0x0A000002, sport=1000, dport=80, proto=17, frag=0) -> bytes:
    hl = 8 if proto == 17 else 20
    tot = 20 + hl + len(payload)
    ip = bytes([0x45, 0, tot >> 8, tot & 255, 0, 0, (frag >> 8) & 255, frag & 255, 64, proto, 0, 0]) + \
        src.to_bytes(4, "big") + dst.to_bytes(4, "big")
    if proto == 17:
        l4 = sport.to_bytes(2, "big") + dport.to_bytes(2, "big") + (8 + len(payload)).to_bytes(2, "big") + b"\0\0"
    else:
        l4 = sport.to_bytes(2, "big") + dport.to_bytes(2, "big") + bytes(8) + bytes([0x50, 0x18]) + bytes(6)
    return bytes(12) + b"\x08\x00" + ip + l4 + payload


def test_hand_example():
    # stream of one flow: "xab" | "cdd" | "d" = x a b c d d d (stream offsets 0..6)
    o = StreamDPI([b"abcd", b"cd", b"dd"], [0, 0, 1])
    occ, nocc, drop = o.process([_udp(b"xab"), _udp(b"cdd"), _udp(b"d")], first_global_index=10)
    # abcd ends at 4 (packet 11, payload offset 1); cd ends at 4; dd ends at 5 and 6
    assert occ == [(11, 0, 1), (11, 1, 1), (11, 2, 2), (12, 2, 0)]
    assert nocc == [0, 3, 1] and drop == [0, 1, 1]


def test_state_carries_across_calls_and_flows_are_separate():
    o = StreamDPI([b"hello"], [0])
    a = _udp(b"zzhel", sport=1)
    b = _udp(b"hel", sport=2)            # other flow: must not complete flow 1's prefix
    occ1, _, _ = o.process([a, b])
    assert occ1 == []
    occ2, nocc2, _ = o.process([_udp(b"lo", sport=2), _udp(b"lo!", sport=1)], first_global_index=2)
    assert occ2 == [(2, 0, 1), (3, 0, 1)]
    assert nocc2 == [1, 1] and o.n_flows() == 2


def test_parse_reading():
    assert parse(b"\0" * 13) is None
    bad = bytearray(_udp(b"abc"))
    bad[12:14] = b"\x81\x00"             # VLAN not parsed (R#24)
    assert parse(bytes(bad)) is None
    key, a, b = parse(_udp(b"abc", frag=0x2000))   # MF set: fragment, ports 0, L4 bytes are payload
    assert key[4:] == (0, 0) and b - a == 8 + 3
    key, a, b = parse(_udp(b"abc", proto=6))
    assert key[1] == 6 and b - a == 3
    # trailing bytes beyond the IP total length are not payload
    key, a, b = parse(_udp(b"abc") + b"pad")
    assert b - a == 3


def test_one_packet_flows_equal_stateless_ac():
    """Each packet its own flow: distinct pattern ids = the C oracle's Aho-Corasick set."""
    import oracle
    rng = np.random.default_rng(3)
    blob, off, act = nfcgen.gen_patterns(rng, 40, lmin=2, lmax=6)
    t = nfcgen.Tables(pat_blob=blob, pat_off=off, pat_action=act)
    pats = t.patterns()
    orc = oracle.OracleChain(["DPI"], t)
    n = 300
    sb = stream_batch(5, n, n, pats, len_choices=[64, 100, 300], plant_frac=0.0,
                      flow_of=np.arange(n))
    r = random.Random(5)
    frames = []
    for fr in sb.frames():                 # plant whole patterns inside payloads
        key, a, b = parse(fr)
        fr = bytearray(fr)
        for _ in range(r.randrange(0, 3)):
            p = r.choice(pats)
            if b - a >= len(p):
                i = r.randrange(a, b - len(p) + 1)
                fr[i:i + len(p)] = p
        frames.append(bytes(fr))
    o = StreamDPI(pats, list(act))
    occ, nocc, drop = o.process(frames)
    per = [set() for _ in frames]
    for i, j, e in occ:
        per[i].add(j)
    hits = 0
    for i, fr in enumerate(frames):
        key, a, b = parse(fr)
        want = orc.ac_match(fr[a:b])
        assert sorted(per[i]) == list(want)
        assert drop[i] == int(any(act[j] for j in want))
        hits += len(want)
    assert hits > 50


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_split_invariance(seed):
    """Any cut of a flow's stream into packets and calls gives the same occurrences."""
    r = random.Random(seed)
    pats = [bytes(r.choice(b"abc") for _ in range(r.randrange(1, 6))) for _ in range(10)]
    pats = list(dict.fromkeys(pats))
    stream = bytes(r.choice(b"abc") for _ in range(400))
    # reference: the whole stream as one packet
    o1 = StreamDPI(pats, [0] * len(pats))
    occ1, _, _ = o1.process([_udp(stream)])
    want = sorted((j, e) for _, j, e in occ1)
    # brute force count of the same thing
    brute = sorted((j, s + len(p) - 1) for j, p in enumerate(pats)
                   for s in range(len(stream) - len(p) + 1) if stream[s:s + len(p)] == p)
    assert want == brute
    # random cuts, random calls, interleaved with another flow
    cuts = sorted(r.sample(range(1, len(stream)), 60))
    pieces = [stream[a:b] for a, b in zip([0] + cuts, cuts + [len(stream)])]
    o2 = StreamDPI(pats, [0] * len(pats))
    got, base, gi, k = [], 0, 0, 0
    while k < len(pieces):
        m = r.randrange(1, 8)
        frames, bases = [], []
        for p in pieces[k:k + m]:
            frames.append(_udp(p))
            bases.append(base)
            base += len(p)
            frames.append(_udp(bytes(r.choice(b"abc") for _ in range(5)), sport=7))   # noise flow
            bases.append(None)
        occ, _, _ = o2.process(frames, first_global_index=gi)
        for i, j, e in occ:
            if bases[i - gi] is not None:
                got.append((j, bases[i - gi] + e))
        gi += len(frames)
        k += m
    assert sorted(got) == want


def test_generator_plants_cross_packet_occurrences():
    rng = np.random.default_rng(9)
    blob, off, act = nfcgen.gen_patterns(rng, 20, lmin=4, lmax=10)
    pats = nfcgen.Tables(pat_blob=blob, pat_off=off, pat_action=act).patterns()
    sb = stream_batch(11, 2000, 40, pats, plant_frac=0.2)
    occ, nocc, drop = StreamDPI(pats, list(act)).process(sb.frames())
    # an occurrence whose end offset is < len - 1 of its pattern started in an earlier packet
    cross = sum(1 for i, j, e in occ if e < len(pats[j]) - 1)
    assert cross > 100


def test_regex_oracle_hand_example():
    from oracle.stream_dpi import StreamRegexDPI
    o = StreamRegexDPI([b"a[0-9]{2}", b"(xy|z)\\.", b"q.?r"], [0, 1, 0])
    occ, nocc, drop = o.process([_udp(b"_a1"), _udp(b"2z."), _udp(b"qr q\x00r")], 0)
    # a12 ends at packet 1 offset 0; z. at packet 1 offset 2; qr at packet 2 offset 1; q\0r at offset 5
    assert occ == [(1, 0, 0), (1, 1, 2), (2, 2, 1), (2, 2, 5)]
    assert nocc == [0, 2, 2] and drop == [0, 1, 0]


def test_regex_oracle_literals_equal_string_oracle():
    """A regex set of escaped literals gives exactly the string-pattern oracle's result."""
    import re
    from oracle.stream_dpi import StreamRegexDPI
    r = random.Random(4)
    pats = list(dict.fromkeys(bytes(r.choice(b"ab.c") for _ in range(r.randrange(1, 5))) for _ in range(8)))
    frames = [_udp(bytes(r.choice(b"ab.c") for _ in range(r.randrange(0, 12))), sport=r.randrange(3))
              for _ in range(40)]
    a = StreamDPI(pats, [0] * len(pats)).process(frames)
    b = StreamRegexDPI([re.escape(p) for p in pats], [0] * len(pats)).process(frames)
    assert a == b
