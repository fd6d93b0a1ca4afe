"""oracle -- TEST INFRASTRUCTURE ONLY.

ctypes wrapper around oracle.c, the plain single-threaded C oracle of the
NFCompass SFC hot path.  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this package.  It never
imports the product package and the product never imports it.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Optional

import numpy as np

import nfcgen

HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(HERE, "liboracle.so")
_P = ctypes.c_void_p


def build_lib(force: bool = False) -> str:
    src = os.path.join(HERE, "oracle.c")
    hdr = os.path.join(HERE, "oracle.h")
    newest = max(os.path.getmtime(src), os.path.getmtime(hdr))
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < newest:
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", _LIB, src])
    return _LIB


class OrSpec(ctypes.Structure):
    _fields_ = [("n_nf", ctypes.c_uint32), ("kind", ctypes.c_uint8 * 8),
                ("acl", _P), ("n_acl", ctypes.c_uint32), ("acl_default", ctypes.c_uint32),
                ("pat_blob", _P), ("pat_off", _P), ("pat_action", _P), ("n_pat", ctypes.c_uint32),
                ("r4", _P), ("n_r4", ctypes.c_uint32), ("nh4", _P), ("n_nh4", ctypes.c_uint32),
                ("pmac4", _P), ("n_port4", ctypes.c_uint32),
                ("r6", _P), ("n_r6", ctypes.c_uint32), ("nh6", _P), ("n_nh6", ctypes.c_uint32),
                ("pmac6", _P), ("n_port6", ctypes.c_uint32),
                ("sa", _P), ("n_sa", ctypes.c_uint32),
                ("lb_port", _P), ("n_lb", ctypes.c_uint32), ("lb_key", _P),
                ("nat_inside", _P), ("n_nat_inside", ctypes.c_uint32),
                ("nat_pool", _P), ("n_nat_pool", ctypes.c_uint32),
                ("nat_port_lo", ctypes.c_uint32), ("nat_port_hi", ctypes.c_uint32),
                ("nat_dnat", _P), ("n_nat_dnat", ctypes.c_uint32),
                ("nat_ext_ports", ctypes.c_uint32), ("nat_key", _P)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        build_lib()
        L = ctypes.CDLL(_LIB)
        L.oracle_create.restype = _P
        L.oracle_create.argtypes = [ctypes.POINTER(OrSpec)]
        L.oracle_destroy.argtypes = [_P]
        L.oracle_stats_len.restype = ctypes.c_size_t
        L.oracle_stats_len.argtypes = [_P]
        L.oracle_run_reorg.restype = ctypes.c_uint64
        L.oracle_run_reorg.argtypes = [_P, _P, _P, _P, _P, ctypes.c_uint32, ctypes.c_uint64, _P, _P, _P,
                                       ctypes.c_uint64, _P]
        L.oracle_run.restype = ctypes.c_uint64
        L.oracle_run.argtypes = [_P, _P, _P, _P, ctypes.c_uint32, ctypes.c_uint64, _P, _P, _P,
                                 ctypes.c_uint64, _P, _P]
        L.or_aes128_encrypt_block.argtypes = [_P, _P, _P]
        L.or_aes128_ctr.argtypes = [_P, _P, _P, _P, ctypes.c_size_t]
        L.or_sha1.argtypes = [_P, ctypes.c_size_t, _P]
        L.or_hmac_sha1.argtypes = [_P, ctypes.c_size_t, _P, ctypes.c_size_t, _P]
        L.or_toeplitz.restype = ctypes.c_uint32
        L.or_toeplitz.argtypes = [_P, _P, ctypes.c_size_t]
        L.or_ipv4_checksum.restype = ctypes.c_uint16
        L.or_ipv4_checksum.argtypes = [_P, ctypes.c_size_t]
        L.or_csum_update.restype = ctypes.c_uint16
        L.or_csum_update.argtypes = [ctypes.c_uint16, ctypes.c_uint16, ctypes.c_uint16]
        L.or_ac_match.restype = ctypes.c_uint32
        L.or_ac_match.argtypes = [_P, _P, ctypes.c_size_t, _P, ctypes.c_uint32]
        L.or_lpm4.restype = ctypes.c_int32
        L.or_lpm4.argtypes = [_P, ctypes.c_uint32]
        L.or_lpm6.restype = ctypes.c_int32
        L.or_lpm6.argtypes = [_P, _P]
        L.or_parse.restype = ctypes.c_int
        L.or_parse.argtypes = [_P, ctypes.c_int, _P]
        L.or_acl.restype = ctypes.c_int32
        L.or_acl.argtypes = [_P, ctypes.c_uint8, _P, _P, ctypes.c_uint16, ctypes.c_uint16, ctypes.c_uint8]
        _lib = L
    return _lib


def _buf(b: bytes):
    return ctypes.create_string_buffer(bytes(b), max(1, len(b)))


# ---------------------------------------------------------------- primitives
def aes128_block(key: bytes, pt: bytes) -> bytes:
    out = ctypes.create_string_buffer(16)
    lib().or_aes128_encrypt_block(_buf(key), _buf(pt), out)
    return out.raw


def aes128_ctr(key: bytes, ctr0: bytes, data: bytes) -> bytes:
    out = ctypes.create_string_buffer(max(1, len(data)))
    lib().or_aes128_ctr(_buf(key), _buf(ctr0), _buf(data), out, len(data))
    return out.raw[:len(data)]


def sha1(msg: bytes) -> bytes:
    out = ctypes.create_string_buffer(20)
    lib().or_sha1(_buf(msg), len(msg), out)
    return out.raw


def hmac_sha1(key: bytes, msg: bytes) -> bytes:
    out = ctypes.create_string_buffer(20)
    lib().or_hmac_sha1(_buf(key), len(key), _buf(msg), len(msg), out)
    return out.raw


def toeplitz(key: bytes, data: bytes) -> int:
    return int(lib().or_toeplitz(_buf(key), _buf(data), len(data)))


def ipv4_checksum(hdr: bytes) -> int:
    return int(lib().or_ipv4_checksum(_buf(hdr), len(hdr)))


def csum_update(hc: int, m: int, m1: int) -> int:
    """RFC 1624 eqn. 3 incremental checksum update (one 16-bit field m -> m1)."""
    return int(lib().or_csum_update(hc, m, m1))


def parse(frame: bytes):
    """The oracle's packet parse of one frame: None if the frame is
    dropped by the parse, else dict(family, l4_off, ip_end, pl_off, proto, sport, dport)."""
    out = (ctypes.c_int32 * 8)()
    lib().or_parse(_buf(frame), len(frame), out)
    if not out[0]:
        return None
    return dict(zip(("family", "l4_off", "ip_end", "pl_off", "proto", "sport", "dport"), list(out)[1:]))


MS_RSS_KEY = bytes.fromhex("6d5a56da255b0ec24167253d43a38fb0d0ca2bcbae7b30b477cb2da38030f20c"
                           "6a42b73bbeac01fa")

ST_PKTS, ST_BYTES_IN, ST_FWD, ST_DROP, ST_BYTES_OUT, ST_PARSE_DROP = 0, 1, 2, 3, 4, 5
ST_DPI_PAIRS, ST_MATCH_OVF, ST_ESP_PKTS, ST_ESP_BYTES, ST_ESP_BLOCKS = 6, 7, 8, 9, 10
ST_POS_BASE, ST_VAR_BASE = 16, 64


class OracleChain:
    """The sequential chain (original SFC order) over logical tables."""

    def __init__(self, kinds, t: nfcgen.Tables):
        self._keep = []
        s = OrSpec()
        s.n_nf = len(kinds)
        for i, k in enumerate(kinds):
            s.kind[i] = nfcgen.KINDS[k] if isinstance(k, str) else int(k)

        def P(a):
            if a is None:
                return None
            a = np.ascontiguousarray(a)
            self._keep.append(a)
            return a.ctypes.data if a.size else None

        ks = {nfcgen.KIND_NAMES[s.kind[i]] for i in range(len(kinds))}
        # only the chain's own tables are loaded (the stats layout depends on them)
        if "ACL" in ks and t.acl_rules is not None:
            s.acl, s.n_acl, s.acl_default = P(t.acl_rules), len(t.acl_rules), t.acl_default
        if "DPI" in ks and t.n_pat:
            s.pat_blob, s.pat_off, s.pat_action = P(t.pat_blob), P(t.pat_off), P(t.pat_action)
            s.n_pat = t.n_pat
        if "LPM4" in ks and t.routes4 is not None:
            s.r4, s.n_r4, s.nh4, s.n_nh4 = P(t.routes4), len(t.routes4), P(t.nh4), len(t.nh4)
            s.pmac4, s.n_port4 = P(t.pmac4), len(t.pmac4)
        if "LPM6" in ks and t.routes6 is not None:
            s.r6, s.n_r6, s.nh6, s.n_nh6 = P(t.routes6), len(t.routes6), P(t.nh6), len(t.nh6)
            s.pmac6, s.n_port6 = P(t.pmac6), len(t.pmac6)
        if "IPSEC" in ks and t.sas is not None:
            s.sa, s.n_sa = P(t.sas), len(t.sas)
        if "LB" in ks and t.lb_ports is not None:
            s.lb_port, s.n_lb, s.lb_key = P(t.lb_ports), len(t.lb_ports), P(t.lb_key)
        if "NAT" in ks and t.nat_pool is not None:
            s.nat_inside, s.n_nat_inside = P(t.nat_inside), len(t.nat_inside)
            s.nat_pool, s.n_nat_pool = P(t.nat_pool), len(t.nat_pool)
            s.nat_port_lo, s.nat_port_hi = t.nat_port_lo, t.nat_port_hi
            s.nat_dnat, s.n_nat_dnat = P(t.nat_dnat), len(t.nat_dnat)
            s.nat_ext_ports, s.nat_key = t.nat_ext_ports, P(t.nat_key)
        self.spec = s
        self.kinds = list(kinds)
        self.tables = t
        self.h = lib().oracle_create(ctypes.byref(s))
        self.stats_len = int(lib().oracle_stats_len(self.h))
        self.stats = np.zeros(self.stats_len, dtype=np.uint64)

    def close(self):
        if self.h:
            lib().oracle_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def run(self, b: nfcgen.Batch, arena: Optional[np.ndarray] = None, match_cap: int = 1 << 20,
            seq_override: Optional[np.ndarray] = None, sel: Optional[np.ndarray] = None):
        """Run the chain over batch b (or the packets sel of it), in order.

        Returns (results[RESULT], arena_after, (match_pkt, match_pat), n_pairs).
        The arena is copied unless given."""
        if arena is None:
            arena = b.arena.copy()
        off, ln = b.off, b.len
        first = b.first_index
        if sel is not None:
            off, ln = off[sel], ln[sel]
        off = np.ascontiguousarray(off, dtype=np.uint64)
        ln = np.ascontiguousarray(ln, dtype=np.uint16)
        n = len(off)
        res = np.zeros(n, dtype=nfcgen.RESULT)
        mp = np.zeros(max(1, match_cap), dtype=np.uint32)
        mq = np.zeros(max(1, match_cap), dtype=np.uint16)
        so = None
        if seq_override is not None:
            so = np.ascontiguousarray(seq_override, dtype=np.uint32)
        if sel is not None and n:
            # per-packet pair ids must be global indices: run one packet at a time
            raise NotImplementedError("use run_one for sampled packets")
        npairs = lib().oracle_run(self.h, arena.ctypes.data, off.ctypes.data, ln.ctypes.data, n, first,
                                  res.ctypes.data, mp.ctypes.data, mq.ctypes.data, match_cap,
                                  self.stats.ctypes.data, None if so is None else so.ctypes.data)
        k = min(int(npairs), match_cap)
        return res, arena, (mp[:k].copy(), mq[:k].copy()), int(npairs)

    def run_reorg(self, b: nfcgen.Batch, group, arena: Optional[np.ndarray] = None, match_cap: int = 1 << 20):
        """The chain re-organized into parallel groups (oracle_run_reorg: per-NF packet
        copies + XOR merge).  group[p] = group index of chain position p.
        Returns like run(); raises ValueError for an invalid grouping."""
        if arena is None:
            arena = b.arena.copy()
        off = np.ascontiguousarray(b.off, dtype=np.uint64)
        ln = np.ascontiguousarray(b.len, dtype=np.uint16)
        n = len(off)
        g = np.zeros(8, dtype=np.uint8)
        g[:len(group)] = group
        res = np.zeros(n, dtype=nfcgen.RESULT)
        mp = np.zeros(max(1, match_cap), dtype=np.uint32)
        mq = np.zeros(max(1, match_cap), dtype=np.uint16)
        npairs = lib().oracle_run_reorg(self.h, g.ctypes.data, arena.ctypes.data, off.ctypes.data, ln.ctypes.data, n,
                                        b.first_index, res.ctypes.data, mp.ctypes.data, mq.ctypes.data, match_cap,
                                        self.stats.ctypes.data)
        if npairs == (1 << 64) - 1:
            raise ValueError(f"invalid grouping {list(group)}")
        k = min(int(npairs), match_cap)
        return res, arena, (mp[:k].copy(), mq[:k].copy()), int(npairs)

    def run_one(self, frame: bytes, global_index: int, headroom=16, tailroom=64, seq=None):
        """One packet in isolation (sampled parity). Returns (result, out_frame, pattern ids)."""
        arena = np.zeros(headroom + len(frame) + tailroom + 64, dtype=np.uint8)
        arena[headroom:headroom + len(frame)] = np.frombuffer(frame, dtype=np.uint8)
        off = np.array([headroom], dtype=np.uint64)
        ln = np.array([len(frame)], dtype=np.uint16)
        res = np.zeros(1, dtype=nfcgen.RESULT)
        cap = max(1, self.tables.n_pat)
        mp = np.zeros(cap, dtype=np.uint32)
        mq = np.zeros(cap, dtype=np.uint16)
        so = None if seq is None else np.array([seq], dtype=np.uint32)
        st = np.zeros(self.stats_len, dtype=np.uint64)
        k = lib().oracle_run(self.h, arena.ctypes.data, off.ctypes.data, ln.ctypes.data, 1, global_index,
                             res.ctypes.data, mp.ctypes.data, mq.ctypes.data, cap, st.ctypes.data,
                             None if so is None else so.ctypes.data)
        r = res[0]
        start = headroom - (16 if r["esp_sa"] != 0xFF else 0)
        out = arena[start:start + int(r["out_len"])].tobytes()
        return r, out, sorted(int(x) for x in mq[:int(k)])

    # direct NF primitives (for pins)
    def ac_match(self, data: bytes):
        ids = np.zeros(max(1, self.tables.n_pat), dtype=np.uint32)
        k = lib().or_ac_match(self.h, _buf(data), len(data), ids.ctypes.data, len(ids))
        return sorted(int(x) for x in ids[:k])

    def lpm4(self, dst: int) -> int:
        return int(lib().or_lpm4(self.h, dst))

    def lpm6(self, dst: bytes) -> int:
        return int(lib().or_lpm6(self.h, _buf(dst)))

    def acl(self, family, src: bytes, dst: bytes, sport, dport, proto) -> int:
        return int(lib().or_acl(self.h, family, _buf(src), _buf(dst), sport, dport, proto))
