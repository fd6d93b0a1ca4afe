"""oracle.stream_dpi -- TEST INFRASTRUCTURE ONLY (plain Python, small cases).

Stateful (cross-packet) DPI, reading R#32:
"stateful processing ensures the in-order processing of packet in the same
connection ... the processed data is finally resembled as traffic stream"
(PAPER.md P:L161 [SIII.B.b]); DPI "perform[s] pattern matching to select flows
or packets for stateful inspections" (P:L132 [SIII.A.2]).

Reading R#32: a flow is the exact (family, proto, src, dst, sport, dport) of a
frame that parses under R#24 (ports 0 for fragments and non-TCP/UDP).  The
payload bytes [pl_off, ip_end) of a flow's packets, in global packet order
(calls in order, packets of a call in index order), form one byte stream.  An
occurrence of pattern j is a position range [s, s + len_j) of that stream equal
to pattern j (case-sensitive, overlaps allowed); it is reported against the
packet whose payload holds its LAST byte, as (packet global index, j, offset of
that last byte within the packet's payload).  A packet is dropped iff an
occurrence of a DROP pattern ends in it.  Frames that do not parse are not
inspected.

The oracle is the definition written out: it keeps each flow's whole stream
and searches it by brute force (bytes.find at every start position).  It shares
nothing with the CUDA path (no automaton at all).
"""
from __future__ import annotations

from typing import Dict, List, Optional, Sequence, Tuple

Key = Tuple[int, int, bytes, bytes, int, int]


def _be16(f: bytes, i: int) -> int:
    return (f[i] << 8) | f[i + 1]


def parse(frame: bytes) -> Optional[Tuple[Key, int, int]]:
    """R#24 parse: returns (flow key, pl_off, ip_end) or None."""
    flen = len(frame)
    if flen < 14:
        return None
    et = _be16(frame, 12)
    frag = False
    if et == 0x0800:
        if flen < 34 or (frame[14] >> 4) != 4:
            return None
        ihl = frame[14] & 15
        if ihl < 5:
            return None
        tot = _be16(frame, 16)
        if tot < 4 * ihl or 14 + tot > flen:
            return None
        fam, l4, ip_end, proto = 4, 14 + 4 * ihl, 14 + tot, frame[23]
        src, dst = bytes(frame[26:30]), bytes(frame[30:34])
        fo = _be16(frame, 20)
        frag = bool(fo & 0x2000) or bool(fo & 0x1FFF)
    elif et == 0x86DD:
        if flen < 54 or (frame[14] >> 4) != 6:
            return None
        pl = _be16(frame, 18)
        if 54 + pl > flen:
            return None
        fam, l4, ip_end, proto = 6, 54, 54 + pl, frame[20]
        src, dst = bytes(frame[22:38]), bytes(frame[38:54])
    else:
        return None
    l4len = 0
    if not frag and proto == 17:
        if l4 + 8 > ip_end:
            return None
        l4len = 8
    elif not frag and proto == 6:
        if l4 + 20 > ip_end:
            return None
        doff = frame[l4 + 12] >> 4
        if doff < 5 or l4 + 4 * doff > ip_end:
            return None
        l4len = 4 * doff
    sport = _be16(frame, l4) if l4len else 0
    dport = _be16(frame, l4 + 2) if l4len else 0
    return (fam, proto, src, dst, sport, dport), l4 + l4len, ip_end


class StreamDPI:
    """Per-flow stream state across calls (the whole stream is kept: plain, not fast)."""

    def __init__(self, patterns: Sequence[bytes], actions: Sequence[int]):
        assert len(patterns) == len(actions) and all(len(p) > 0 for p in patterns)
        self.patterns = [bytes(p) for p in patterns]
        self.actions = list(actions)
        self.streams: Dict[Key, bytearray] = {}

    def process(self, frames: Sequence[bytes], first_global_index: int = 0):
        """One call: returns (occurrences sorted, nocc per packet, drop per packet)."""
        n = len(frames)
        nocc = [0] * n
        drop = [0] * n
        occ: List[Tuple[int, int, int]] = []
        for i, fr in enumerate(frames):
            p = parse(fr)
            if p is None:
                continue
            key, a, b = p
            st = self.streams.setdefault(key, bytearray())
            base = len(st)                     # stream offset of this payload's first byte
            st += fr[a:b]
            for j, pat in enumerate(self.patterns):
                L = len(pat)
                s = max(0, base - L + 1)       # earliest start whose last byte is in this payload
                while True:
                    s = st.find(pat, s)
                    if s < 0:
                        break
                    end = s + L - 1
                    assert end >= base
                    occ.append((first_global_index + i, j, end - base))
                    nocc[i] += 1
                    drop[i] |= self.actions[j]
                    s += 1
        occ.sort()
        return occ, nocc, drop

    def n_flows(self) -> int:
        return len(self.streams)


class StreamRegexDPI(StreamDPI):
    """Regular-expression variant ("for the regular expression we use a DFA";
    DESIGN.md R#33): an occurrence of expression j ends at stream byte x iff a
    non-empty substring of the flow's stream ending at x is in L(j).  Written with
    Python's backtracking `re` (an independent engine, no automaton of ours):
    re.search(b"(?:R)\\Z", stream[:x + 1]) at every byte, DOTALL so '.' is any byte."""

    def __init__(self, regexes: Sequence[bytes], actions: Sequence[int]):
        import re
        super().__init__([b"?"] * len(regexes), actions)
        self.res = [re.compile(b"(?:" + bytes(r) + b")\\Z", re.DOTALL) for r in regexes]

    def process(self, frames: Sequence[bytes], first_global_index: int = 0):
        n = len(frames)
        nocc, drop = [0] * n, [0] * n
        occ: List[Tuple[int, int, int]] = []
        for i, fr in enumerate(frames):
            p = parse(fr)
            if p is None:
                continue
            key, a, b = p
            st = self.streams.setdefault(key, bytearray())
            base = len(st)
            st += fr[a:b]
            view = bytes(st)
            for x in range(base, len(st)):
                for j, rx in enumerate(self.res):
                    m = rx.search(view, 0, x + 1)
                    if m is not None and m.end() > m.start():
                        occ.append((first_global_index + i, j, x - base))
                        nocc[i] += 1
                        drop[i] |= self.actions[j]
        occ.sort()
        return occ, nocc, drop
