"""Seeded synthetic traffic for stateful (cross-packet) DPI, SURVEY 8(f) NEXT-4.

Input generator only -- no DPI arithmetic.  Shared by the oracle tests, the GPU
parity tests and bench.py (R#32, input recipe "S1").

Packets are IPv4 frames (UDP, a `tcp_frac` share TCP with a 20-B header) of one
of `n_flows` flows, the flow of each packet drawn uniformly, so a flow's packets
are spread over the batch in index order.  Payload bytes are random printable.
A `plant_frac` share of packets carries the first k bytes of a random pattern at
the END of its payload and the remaining bytes at the START of the next payload
of the same flow (k uniform in [1, len-1]): occurrences that only a cross-packet
(stream) walk finds.  Frames sit in rows of `stride` bytes (offsets % 16 == 0).
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import List, Optional, Sequence

import numpy as np


@dataclass
class StreamBatch:
    arena: np.ndarray      # u8
    off: np.ndarray        # u64
    len: np.ndarray        # u16
    first_index: int = 0

    def frames(self) -> List[bytes]:
        a = self.arena
        return [a[int(o):int(o) + int(l)].tobytes() for o, l in zip(self.off, self.len)]


def stream_batch(seed: int, n_pkts: int, n_flows: int, patterns: Sequence[bytes], pkt_len=64,
                 len_choices: Optional[Sequence[int]] = None, tcp_frac: float = 0.3,
                 plant_frac: float = 0.05, first_index: int = 0, flow_seed: Optional[int] = None,
                 flow_of: Optional[np.ndarray] = None) -> StreamBatch:
    rng = np.random.default_rng(seed)
    frng = np.random.default_rng(seed if flow_seed is None else flow_seed)
    # flow 5-tuples (stable for a given flow_seed so several calls share flows)
    fsrc = frng.integers(0, 2**32, n_flows, dtype=np.uint64).astype(np.uint32)
    fdst = frng.integers(0, 2**32, n_flows, dtype=np.uint64).astype(np.uint32)
    fsp = frng.integers(1024, 65536, n_flows).astype(np.uint16)
    fdp = frng.integers(1, 65536, n_flows).astype(np.uint16)
    ftcp = frng.random(n_flows) < tcp_frac
    if flow_of is None:
        flow_of = rng.integers(0, n_flows, n_pkts)
    if len_choices is None:
        ln = np.full(n_pkts, pkt_len, dtype=np.int64)
    else:
        ln = rng.choice(np.asarray(len_choices), n_pkts).astype(np.int64)
    stride = int((ln.max() + 15) // 16 * 16) if n_pkts else 16
    A = np.zeros((max(n_pkts, 1), stride), dtype=np.uint8)
    A[:n_pkts] = rng.integers(0x20, 0x7F, (n_pkts, stride), dtype=np.uint8)
    if n_pkts:
        tcp = ftcp[flow_of]
        hl = np.where(tcp, 20, 8)
        # Ethernet: dst/src MAC, type 0x0800
        A[:n_pkts, 0:12] = rng.integers(0, 256, (n_pkts, 12), dtype=np.uint8)
        A[:n_pkts, 12], A[:n_pkts, 13] = 0x08, 0x00
        tot = ln - 14
        A[:n_pkts, 14], A[:n_pkts, 15] = 0x45, 0
        A[:n_pkts, 16], A[:n_pkts, 17] = tot >> 8, tot & 255
        A[:n_pkts, 18:20] = 0
        A[:n_pkts, 20], A[:n_pkts, 21] = 0x40, 0          # DF, offset 0
        A[:n_pkts, 22] = 64
        A[:n_pkts, 23] = np.where(tcp, 6, 17)
        A[:n_pkts, 24:26] = 0
        for k in range(4):
            A[:n_pkts, 26 + k] = (fsrc[flow_of] >> (24 - 8 * k)) & 255
            A[:n_pkts, 30 + k] = (fdst[flow_of] >> (24 - 8 * k)) & 255
        A[:n_pkts, 34], A[:n_pkts, 35] = fsp[flow_of] >> 8, fsp[flow_of] & 255
        A[:n_pkts, 36], A[:n_pkts, 37] = fdp[flow_of] >> 8, fdp[flow_of] & 255
        udp = ~tcp
        ul = tot - 20
        A[udp, 38], A[udp, 39] = (ul[udp] >> 8) & 255, ul[udp] & 255
        A[tcp, 46] = 0x50                                   # data offset 5
        A[tcp, 47] = 0x18
        # cross-packet plants: prefix at the end of i, suffix at the start of next(i)
        order = np.lexsort((np.arange(n_pkts), flow_of))
        nxt = np.full(n_pkts, -1, dtype=np.int64)
        same = flow_of[order[1:]] == flow_of[order[:-1]]
        nxt[order[:-1][same]] = order[1:][same]
        pl0 = 34 + hl
        cand = np.nonzero((rng.random(n_pkts) < plant_frac) & (nxt >= 0))[0]
        pats = [bytes(p) for p in patterns]
        pj = rng.integers(0, len(pats), len(cand)) if pats else []
        for i, j in zip(cand, pj):
            p = pats[j]
            if len(p) < 2:
                continue
            k = int(rng.integers(1, len(p)))
            a, b = p[:k], p[k:]
            e = int(ln[i])
            if e - int(pl0[i]) < len(a):
                continue
            m = int(nxt[i])
            if int(ln[m]) - int(pl0[m]) < len(b):
                continue
            A[i, e - len(a):e] = np.frombuffer(a, dtype=np.uint8)
            A[m, int(pl0[m]):int(pl0[m]) + len(b)] = np.frombuffer(b, dtype=np.uint8)
    off = (np.arange(n_pkts, dtype=np.uint64) * np.uint64(stride))
    return StreamBatch(A.reshape(-1), off, ln.astype(np.uint16), first_index)
