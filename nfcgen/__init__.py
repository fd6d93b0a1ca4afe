"""nfcgen -- seeded synthetic inputs (logical tables + packet batches).

The ONE module both the oracle and the CUDA path take their inputs from.  It
holds none of the method's arithmetic (no parsing, matching, lookup, hashing,
checksums or crypto): tables are drawn with numpy's PCG64, packets with the
counter-based generator in gen.c.  The workload recipe (shapes, sizes, value
distributions) is DESIGN.md "Synthetic inputs"; it follows SURVEY.md 8(d) and
the paper's traffic descriptions (P:L136 random IP/UDP traffic, P:L361 IMIX,
P:L383 ClassBench-style ACLs, P:L205 no-match / full-match DPI traffic).

Logical spec layouts (numpy dtypes below) are the binary interface both sides
read; see DESIGN.md "Logical spec layouts".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field
from typing import Dict, List, Optional

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(HERE, "libnfcgen.so")

# ---------------------------------------------------------------- layouts
ACL_RULE = np.dtype([("family", "u1"), ("slen", "u1"), ("dlen", "u1"), ("proto", "u1"),
                     ("proto_any", "u1"), ("action", "u1"), ("sp_lo", "<u2"), ("sp_hi", "<u2"),
                     ("dp_lo", "<u2"), ("dp_hi", "<u2"), ("pad", "u1", (2,)),
                     ("src", "u1", (16,)), ("dst", "u1", (16,))])
ROUTE4 = np.dtype([("prefix", "<u4"), ("len", "u1"), ("pad", "u1"), ("nh", "<u2")])
ROUTE6 = np.dtype([("prefix", "u1", (16,)), ("nh", "<u2"), ("len", "u1"), ("pad", "u1")])
NEXTHOP = np.dtype([("port", "<u2"), ("mac", "u1", (6,))])
SA = np.dtype([("spi", "<u4"), ("seq0", "<u4"), ("aes_key", "u1", (16,)), ("nonce", "u1", (4,)),
               ("auth_key", "u1", (20,))])
RESULT = np.dtype([("drop_nf", "u1"), ("esp_sa", "u1"), ("port", "<u2"), ("acl_rule", "<u2"),
                   ("lb_backend", "<u2"), ("dpi_nmatch", "<u2"), ("out_len", "<u2"),
                   ("esp_seq", "<u4")])
NAT_PREFIX = np.dtype([("prefix", "<u4"), ("len", "u1"), ("pad", "u1", (3,))])
NAT_DNAT = np.dtype([("ext_addr", "<u4"), ("ext_port", "<u2"), ("proto", "u1"), ("pad", "u1"),
                     ("int_addr", "<u4"), ("int_port", "<u2"), ("pad2", "<u2")])
assert NAT_PREFIX.itemsize == 8 and NAT_DNAT.itemsize == 16
assert ACL_RULE.itemsize == 48 and ROUTE4.itemsize == 8 and ROUTE6.itemsize == 20
assert NEXTHOP.itemsize == 8 and SA.itemsize == 48 and RESULT.itemsize == 16

KINDS = {"ACL": 1, "DPI": 2, "LPM4": 3, "LPM6": 4, "IPSEC": 5, "LB": 6, "NAT": 7}
KIND_NAMES = {v: k for k, v in KINDS.items()}


@dataclass
class Tables:
    acl_rules: Optional[np.ndarray] = None
    acl_default: int = 0
    pat_blob: Optional[np.ndarray] = None      # u8
    pat_off: Optional[np.ndarray] = None       # u32 [n+1]
    pat_action: Optional[np.ndarray] = None    # u8 [n]
    routes4: Optional[np.ndarray] = None
    nh4: Optional[np.ndarray] = None
    pmac4: Optional[np.ndarray] = None         # u8 [n_ports, 6]
    routes6: Optional[np.ndarray] = None
    nh6: Optional[np.ndarray] = None
    pmac6: Optional[np.ndarray] = None
    sas: Optional[np.ndarray] = None
    lb_ports: Optional[np.ndarray] = None      # u16
    lb_key: Optional[np.ndarray] = None        # u8[40]
    nat_inside: Optional[np.ndarray] = None    # NAT_PREFIX
    nat_pool: Optional[np.ndarray] = None      # u32 public addresses (host-order values)
    nat_port_lo: int = 1024
    nat_port_hi: int = 65535
    nat_dnat: Optional[np.ndarray] = None      # NAT_DNAT
    nat_ext_ports: int = 0                     # bit p: egress port p faces the Internet
    nat_key: Optional[np.ndarray] = None       # u8[40]

    @property
    def n_pat(self) -> int:
        return 0 if self.pat_off is None else len(self.pat_off) - 1

    def patterns(self) -> List[bytes]:
        if self.pat_off is None:
            return []
        b = self.pat_blob.tobytes()
        return [b[self.pat_off[i]:self.pat_off[i + 1]] for i in range(self.n_pat)]


@dataclass
class TrafficParams:
    seed: int = 1
    n_flows: int = 65536
    v6_bp: int = 0
    pkt_len: int = 64           # 0 = IMIX
    match_ppm: int = 50_000     # 5% planted DPI matches
    in_acl_pct: int = 50
    tcp_pct: int = 0
    ttl: int = 64
    ttl1_ppm: int = 0
    malformed_ppm: int = 0
    printable: int = 1
    headroom: int = 0
    tailroom: int = 0
    l4csum: int = 0             # 1: arbitrary TCP/UDP checksum values (NAT updates them)
    # valid edge-case frames (SURVEY 8(c)(i) parse cases), per million packets
    opt_ppm: int = 0            # IPv4 options (IHL 6..15)
    frag_ppm: int = 0           # IPv4 fragments (MF and/or offset): ports 0, L4 not parsed
    tcpopt_ppm: int = 0         # TCP data offset 6..15
    trailer_ppm: int = 0        # Ethernet trailer after the IP packet (1..46 B)

    def edge(self, ppm: int = 100_000):
        """Turn on every valid edge-case frame kind at `ppm` each (tests)."""
        self.opt_ppm = self.frag_ppm = self.tcpopt_ppm = self.trailer_ppm = ppm
        return self


@dataclass
class Workload:
    name: str
    kinds: List[str]
    tables: Tables
    traffic: TrafficParams
    batch_pkts: int = 4096
    note: str = ""


# ---------------------------------------------------------------- C generator
class _GenParams(ctypes.Structure):
    _fields_ = [("seed", ctypes.c_uint64), ("n_flows", ctypes.c_uint64)] + [
        (n, ctypes.c_uint32) for n in ("v6_bp", "pkt_len", "match_ppm", "in_acl_pct", "tcp_pct", "ttl",
                                       "ttl1_ppm", "malformed_ppm", "printable", "headroom", "tailroom",
                                       "l4csum", "opt_ppm", "frag_ppm", "tcpopt_ppm", "trailer_ppm")]


_P = ctypes.c_void_p


class _GenTables(ctypes.Structure):
    _fields_ = [("n_r4", ctypes.c_uint32), ("r4_prefix", _P), ("r4_len", _P),
                ("n_r6", ctypes.c_uint32), ("r6_prefix", _P), ("r6_len", _P),
                ("n_acl4", ctypes.c_uint32), ("acl4_idx", _P),
                ("n_acl6", ctypes.c_uint32), ("acl6_idx", _P),
                ("acl_rules", _P),
                ("n_pat", ctypes.c_uint32), ("pat_blob", _P), ("pat_off", _P)]


def build_lib(force: bool = False) -> str:
    src = os.path.join(HERE, "gen.c")
    newest = max(os.path.getmtime(src), os.path.getmtime(os.path.join(HERE, "gen_core.h")))
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < newest:
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", _LIB, src])
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        build_lib()
        _lib = ctypes.CDLL(_LIB)
        _lib.nfcgen_layout.restype = ctypes.c_uint64
        _lib.nfcgen_layout.argtypes = [ctypes.POINTER(_GenParams), ctypes.POINTER(_GenTables),
                                       ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint64, _P, _P]
        _lib.nfcgen_fill.restype = None
        _lib.nfcgen_fill.argtypes = [ctypes.POINTER(_GenParams), ctypes.POINTER(_GenTables),
                                     ctypes.c_uint64, ctypes.c_uint32, _P, _P, _P]
        _lib.nfcgen_flow.restype = None
        _lib.nfcgen_flow.argtypes = [ctypes.POINTER(_GenParams), ctypes.POINTER(_GenTables), ctypes.c_uint64,
                                     _P, _P, _P, _P, _P, _P]
        _lib.nfcgen_rnd.restype = ctypes.c_uint64
        _lib.nfcgen_rnd.argtypes = [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint64]
    return _lib


def _ptr(a: Optional[np.ndarray]):
    return None if a is None or a.size == 0 else a.ctypes.data


class _Keep:
    """Holds numpy buffers alive while a ctypes struct points at them."""

    def __init__(self):
        self.refs = []

    def __call__(self, a):
        if a is not None:
            a = np.ascontiguousarray(a)
            self.refs.append(a)
        return a


def _gen_structs(tp: TrafficParams, t: Tables):
    keep = _Keep()
    gp = _GenParams(tp.seed, tp.n_flows, tp.v6_bp, tp.pkt_len, tp.match_ppm, tp.in_acl_pct,
                    tp.tcp_pct, tp.ttl, tp.ttl1_ppm, tp.malformed_ppm, tp.printable,
                    tp.headroom, tp.tailroom, tp.l4csum, tp.opt_ppm, tp.frag_ppm, tp.tcpopt_ppm,
                    tp.trailer_ppm)
    gt = _GenTables()
    if t.routes4 is not None and len(t.routes4):
        r4p = keep(t.routes4["prefix"].astype(np.uint32))
        r4l = keep(t.routes4["len"].astype(np.uint8))
        gt.n_r4, gt.r4_prefix, gt.r4_len = len(r4p), _ptr(r4p), _ptr(r4l)
    if t.routes6 is not None and len(t.routes6):
        r6p = keep(t.routes6["prefix"].astype(np.uint8))
        r6l = keep(t.routes6["len"].astype(np.uint8))
        gt.n_r6, gt.r6_prefix, gt.r6_len = len(r6l), _ptr(r6p), _ptr(r6l)
    if t.acl_rules is not None and len(t.acl_rules):
        rules = keep(t.acl_rules)
        i4 = keep(np.nonzero(rules["family"] == 4)[0].astype(np.uint32))
        i6 = keep(np.nonzero(rules["family"] == 6)[0].astype(np.uint32))
        gt.n_acl4, gt.acl4_idx = len(i4), _ptr(i4)
        gt.n_acl6, gt.acl6_idx = len(i6), _ptr(i6)
        gt.acl_rules = _ptr(rules)
    if t.n_pat:
        blob = keep(t.pat_blob.astype(np.uint8))
        po = keep(t.pat_off.astype(np.uint32))
        gt.n_pat, gt.pat_blob, gt.pat_off = t.n_pat, _ptr(blob), _ptr(po)
    return gp, gt, keep


@dataclass
class Batch:
    """Host packet batch: arena bytes, frame offsets (u64) and lengths (u16)."""
    arena: np.ndarray
    off: np.ndarray
    len: np.ndarray
    first_index: int
    headroom: int
    tailroom: int

    @property
    def n(self) -> int:
        return len(self.off)

    def frame(self, i: int) -> bytes:
        o = int(self.off[i])
        return self.arena[o:o + int(self.len[i])].tobytes()


def generate(tp: TrafficParams, t: Tables, first: int, n: int) -> Batch:
    """Packets [first, first+n) of the global stream, laid out contiguously."""
    lib = _load()
    gp, gt, keep = _gen_structs(tp, t)
    off = np.zeros(n, dtype=np.uint64)
    ln = np.zeros(n, dtype=np.uint16)
    end = lib.nfcgen_layout(ctypes.byref(gp), ctypes.byref(gt), first, n, 0, _ptr(off), _ptr(ln))
    arena = np.zeros(int(end) + 64, dtype=np.uint8)
    if n:
        lib.nfcgen_fill(ctypes.byref(gp), ctypes.byref(gt), first, n, _ptr(arena), _ptr(off), _ptr(ln))
    del keep
    return Batch(arena, off, ln, first, tp.headroom, tp.tailroom)


def flow(tp: TrafficParams, t: Tables, f: int):
    """The 5-tuple of flow f: (family, src bytes, dst bytes, sport, dport, proto)."""
    lib = _load()
    gp, gt, keep = _gen_structs(tp, t)
    fam = ctypes.c_uint32()
    src, dst = (ctypes.c_uint8 * 16)(), (ctypes.c_uint8 * 16)()
    sp, dp, pr = ctypes.c_uint16(), ctypes.c_uint16(), ctypes.c_uint8()
    lib.nfcgen_flow(ctypes.byref(gp), ctypes.byref(gt), f, ctypes.byref(fam), src, dst, ctypes.byref(sp),
                    ctypes.byref(dp), ctypes.byref(pr))
    del keep
    nb = 4 if fam.value == 4 else 16
    return fam.value, bytes(src)[:nb], bytes(dst)[:nb], sp.value, dp.value, pr.value


def rnd(seed: int, stream: int, idx: int) -> int:
    return int(_load().nfcgen_rnd(seed, stream, idx))


# ---------------------------------------------------------------- tables
def _mask_bytes(a: np.ndarray, plen: int) -> np.ndarray:
    a = a.copy()
    for k in range(len(a)):
        keep = plen - 8 * k
        m = 0xFF if keep >= 8 else 0 if keep <= 0 else (0xFF << (8 - keep)) & 0xFF
        a[k] &= m
    return a


def gen_acl(rng: np.random.Generator, n: int, family: int = 4, deny_frac: float = 0.10,
            lens=None) -> np.ndarray:
    """ClassBench-like rules (SURVEY 8(d) C1 recipe)."""
    r = np.zeros(n, dtype=ACL_RULE)
    nb = 4 if family == 4 else 16
    if lens is None:
        lens = [0, 8, 16, 24, 32] if family == 4 else [0, 32, 48, 64, 128]
    for i in range(n):
        r[i]["family"] = family
        for fld, lf in (("src", "slen"), ("dst", "dlen")):
            pl = int(rng.choice(lens))
            a = np.zeros(16, dtype=np.uint8)
            a[:nb] = rng.integers(0, 256, nb, dtype=np.uint8)
            r[i][fld] = _mask_bytes(a, pl)
            r[i][lf] = pl
        for lo, hi in (("sp_lo", "sp_hi"), ("dp_lo", "dp_hi")):
            kind = int(rng.integers(0, 5))
            if kind == 0:
                a, b = 0, 65535
            elif kind == 1:
                a = b = int(rng.integers(0, 65536))
            elif kind == 2:
                a, b = 0, 1023
            elif kind == 3:
                a, b = 1024, 65535
            else:
                a, b = sorted(int(x) for x in rng.integers(0, 65536, 2))
            r[i][lo], r[i][hi] = a, b
        pk = int(rng.integers(0, 3))
        r[i]["proto_any"] = 1 if pk == 2 else 0
        r[i]["proto"] = (6, 17, 0)[pk]
        # a DENY rule names at least one address prefix (no wildcard-address deny that
        # would shadow the whole set; R#28)
        deny = rng.random() < deny_frac
        r[i]["action"] = 1 if deny and int(r[i]["slen"]) + int(r[i]["dlen"]) > 0 else 0
    # ClassBench filter sets list specific filters before general ones (a catch-all
    # last); order by specificity so a broad rule does not shadow the set (R#28)
    spec = (r["slen"].astype(np.int64) + r["dlen"]) * 2 ** 20 \
        - (r["sp_hi"].astype(np.int64) - r["sp_lo"]) - (r["dp_hi"].astype(np.int64) - r["dp_lo"]) \
        + (1 - r["proto_any"].astype(np.int64)) * 2 ** 18
    return r[np.argsort(-spec, kind="stable")].copy()


def gen_patterns(rng: np.random.Generator, n: int, lmin=4, lmax=16, printable_frac=1.0,
                 drop_frac=0.05, skew_short=False):
    """Snort-like literal patterns; unique strings."""
    seen = set()
    pats, acts = [], []
    while len(pats) < n:
        if skew_short:
            L = int(min(lmax, lmin + rng.geometric(0.12) - 1))
        else:
            L = int(rng.integers(lmin, lmax + 1))
        if rng.random() < printable_frac:
            b = bytes(int(x) for x in rng.integers(0x20, 0x7F, L))
        else:
            b = bytes(int(x) for x in rng.integers(0, 256, L))
        if b in seen:
            continue
        seen.add(b)
        pats.append(b)
        acts.append(1 if rng.random() < drop_frac else 0)
    off = np.zeros(n + 1, dtype=np.uint32)
    off[1:] = np.cumsum([len(p) for p in pats])
    blob = np.frombuffer(b"".join(pats), dtype=np.uint8).copy()
    return blob, off, np.array(acts, dtype=np.uint8)


V4_LEN_MIX = [(24, 0.55), ((16, 23), 0.35), ((8, 15), 0.05), ((25, 32), 0.05)]
V6_LEN_MIX = [(48, 0.45), (32, 0.12), (44, 0.10), (40, 0.08), (36, 0.05), (29, 0.04), (56, 0.04),
              (64, 0.04), ((20, 64), 0.08)]


def _draw_len(rng, mix):
    u = rng.random()
    acc = 0.0
    for spec, p in mix:
        acc += p
        if u < acc:
            break
    if isinstance(spec, tuple):
        return int(rng.integers(spec[0], spec[1] + 1))
    return int(spec)


def gen_routes4(rng, n: int, n_nh: int, default_route=True) -> np.ndarray:
    """BGP-like IPv4 table; unique (prefix,len); plus 0.0.0.0/0."""
    seen = set()
    out = []
    if default_route:
        out.append((0, 0, int(rng.integers(0, n_nh))))
        seen.add((0, 0))
    while len(out) < n + (1 if default_route else 0):
        L = _draw_len(rng, V4_LEN_MIX)
        v = int(rng.integers(0, 2 ** 32, dtype=np.uint64))
        v = v & ((0xFFFFFFFF << (32 - L)) & 0xFFFFFFFF) if L else 0
        if (v, L) in seen:
            continue
        seen.add((v, L))
        out.append((v, L, int(rng.integers(0, n_nh))))
    r = np.zeros(len(out), dtype=ROUTE4)
    r["prefix"] = [o[0] for o in out]
    r["len"] = [o[1] for o in out]
    r["nh"] = [o[2] for o in out]
    return r


def gen_routes6(rng, n: int, n_nh: int, default_route=True) -> np.ndarray:
    """BGP-v6-like table of prefixes <= /64; plus ::/0. Vectorised."""
    lens = np.array([_draw_len(rng, V6_LEN_MIX) for _ in range(int(n * 1.05) + 16)], dtype=np.int64)
    addr = rng.integers(0, 256, (len(lens), 16), dtype=np.uint8)
    addr[:, 0] = 0x20 | (addr[:, 0] & 0x1F)   # 2000::/3-ish global unicast look
    bitpos = np.arange(128)
    keep = bitpos[None, :] < lens[:, None]
    bits = np.unpackbits(addr, axis=1) & keep
    addr = np.packbits(bits.astype(np.uint8), axis=1)
    key = np.concatenate([addr, lens[:, None].astype(np.uint8)], axis=1)
    _, uniq = np.unique(key, axis=0, return_index=True)
    uniq = np.sort(uniq)[:n]
    m = len(uniq) + (1 if default_route else 0)
    r = np.zeros(m, dtype=ROUTE6)
    s = 1 if default_route else 0
    r["prefix"][s:] = addr[uniq]
    r["len"][s:] = lens[uniq]
    r["nh"] = rng.integers(0, n_nh, m)
    return r


def gen_nexthops(rng, n_nh: int, n_ports: int):
    nh = np.zeros(n_nh, dtype=NEXTHOP)
    nh["port"] = rng.integers(0, n_ports, n_nh)
    nh["mac"] = rng.integers(0, 256, (n_nh, 6))
    pm = rng.integers(0, 256, (n_ports, 6), dtype=np.uint8)
    return nh, pm


def gen_sas(rng, n: int) -> np.ndarray:
    s = np.zeros(n, dtype=SA)
    s["spi"] = rng.integers(0x100, 2 ** 32 - 1, n, dtype=np.uint64)
    s["seq0"] = 0
    s["aes_key"] = rng.integers(0, 256, (n, 16))
    s["nonce"] = rng.integers(0, 256, (n, 4))
    s["auth_key"] = rng.integers(0, 256, (n, 20))
    return s


def gen_lb(rng, n_backends: int, n_ports: int = 16):
    return (rng.integers(0, n_ports, n_backends).astype(np.uint16),
            rng.integers(0, 256, 40, dtype=np.uint8))


def gen_nat(rng, tp: "TrafficParams", t: Tables, n_dnat: int = 1000, n_inside: int = 8, n_pool: int = 64,
            hit_frac: float = 0.5, n_ports: int = 16):
    """NAT44 tables (R#30): n_inside distinct /4 inside prefixes (half of all source
    addresses), a pool of public addresses, source ports 1024..65535, the upper half of
    the router's ports Internet-facing, and n_dnat static DNAT entries of which
    hit_frac are (proto, dst, dport) of real flows of the traffic."""
    firsts = rng.choice(16, size=min(n_inside, 16), replace=False)
    t.nat_inside = np.zeros(len(firsts), dtype=NAT_PREFIX)
    t.nat_inside["prefix"] = firsts.astype(np.uint32) << 28
    t.nat_inside["len"] = 4
    t.nat_pool = rng.integers(0, 1 << 32, n_pool, dtype=np.uint64).astype(np.uint32)
    t.nat_port_lo, t.nat_port_hi = 1024, 65535
    t.nat_ext_ports = sum(1 << p for p in range(n_ports // 2, n_ports))
    t.nat_key = rng.integers(0, 256, 40, dtype=np.uint8)
    d = np.zeros(n_dnat, dtype=NAT_DNAT)
    seen = set()
    k = 0
    while k < n_dnat:
        if rng.random() < hit_frac:
            fam, src, dst, sp, dpt, pr = flow(tp, t, int(rng.integers(0, tp.n_flows)))
            if fam != 4 or pr not in (6, 17):
                continue
            key = (pr, int.from_bytes(dst, "big"), dpt)
        else:
            key = (int(rng.choice([6, 17])), int(rng.integers(0, 1 << 32)), int(rng.integers(0, 1 << 16)))
        if key in seen:
            continue
        seen.add(key)
        d[k]["proto"], d[k]["ext_addr"], d[k]["ext_port"] = key
        d[k]["int_addr"] = (10 << 24) | int(rng.integers(0, 1 << 24))
        d[k]["int_port"] = int(rng.integers(1, 1 << 16))
        k += 1
    t.nat_dnat = d
    return t


def make_tables(seed: int, kinds: List[str], n_acl=64, acl_family=4, n_pat=100, pat_kw=None,
                n_r4=1000, n_r6=0, n_sa=64, n_lb=64, n_nh=64, n_ports=16,
                acl_deny=0.10, acl6_extra=0) -> Tables:
    rng = np.random.default_rng(np.random.PCG64(seed))
    t = Tables()
    if "ACL" in kinds:
        rules = gen_acl(rng, n_acl, acl_family, acl_deny)
        if acl6_extra:
            rules = np.concatenate([rules, gen_acl(rng, acl6_extra, 6, acl_deny)])
        t.acl_rules = rules
        t.acl_default = 0
    if "DPI" in kinds:
        t.pat_blob, t.pat_off, t.pat_action = gen_patterns(rng, n_pat, **(pat_kw or {}))
    if "LPM4" in kinds or n_r4:
        t.nh4, t.pmac4 = gen_nexthops(rng, n_nh, n_ports)
        t.routes4 = gen_routes4(rng, n_r4, n_nh)
    if "LPM6" in kinds or n_r6:
        t.nh6, t.pmac6 = gen_nexthops(rng, n_nh, n_ports)
        t.routes6 = gen_routes6(rng, n_r6, n_nh)
    if "IPSEC" in kinds:
        t.sas = gen_sas(rng, n_sa)
    if "LB" in kinds:
        t.lb_ports, t.lb_key = gen_lb(rng, n_lb, n_ports)
    return t


# ---------------------------------------------------------------- configs
C6_CHAIN = ["ACL", "DPI", "LPM4", "LPM6", "IPSEC", "LB"]   # DESIGN.md R#20


def workload(name: str, pkt_len: Optional[int] = None, k: Optional[int] = None,
             small: bool = False, seed: Optional[int] = None, acl_rules: Optional[int] = None) -> Workload:
    """BASELINE.json configs C1..C5; small=True shrinks tables for fast tests."""
    name = name.upper()
    if name == "C1":
        kinds = ["ACL", "DPI", "LPM4"]
        sd = 1 if seed is None else seed
        t = make_tables(sd, kinds, n_acl=64, n_pat=100, n_r4=1000)
        tp = TrafficParams(seed=sd, pkt_len=64 if pkt_len is None else pkt_len)
        return Workload("C1", kinds, t, tp,
                        note="ACL(64)->DPI(100)->IPv4 LPM(1K), 64 B IPv4/UDP")
    if name == "C2":
        kinds = ["IPSEC"]
        sd = 2 if seed is None else seed
        t = make_tables(sd, kinds, n_r4=1000 if not small else 100)
        tp = TrafficParams(seed=sd, pkt_len=1500 if pkt_len is None else pkt_len, match_ppm=0,
                           in_acl_pct=0, headroom=16, tailroom=32)
        return Workload("C2", kinds, t, tp, note="IPsec AES-128-CTR + HMAC-SHA1-96, 64 SAs, 1500 B")
    if name == "C3":
        kinds = ["ACL", "DPI", "LB"]
        sd = 3 if seed is None else seed
        t = make_tables(sd, kinds, n_acl=1000 if not small else 200, n_pat=2000 if not small else 300,
                        pat_kw=dict(lmin=4, lmax=32, printable_frac=0.7, drop_frac=0.02,
                                    skew_short=True), n_r4=1000, n_lb=64)
        tp = TrafficParams(seed=sd, n_flows=1 << 20, pkt_len=0 if pkt_len is None else pkt_len)
        return Workload("C3", kinds, t, tp, note="FW(1K)->DPI(2K)->LB(64), IMIX, 1M flows")
    if name == "C4":
        kinds = ["ACL", "LPM6", "DPI", "IPSEC", "LB"]
        sd = 4 if seed is None else seed
        t = make_tables(sd, kinds, n_acl=256, acl_family=6,
                        n_pat=2000 if not small else 300,
                        pat_kw=dict(lmin=4, lmax=32, printable_frac=0.7, drop_frac=0.02,
                                    skew_short=True),
                        n_r4=0, n_r6=200_000 if not small else 5000, n_lb=64)
        tp = TrafficParams(seed=sd, v6_bp=10000, pkt_len=1500 if pkt_len is None else pkt_len,
                           headroom=16, tailroom=32)
        return Workload("C4", kinds, t, tp,
                        note="ACL(256 v6)->IPv6 LPM(200K)->DPI(2K)->IPsec->LB, 1500 B IPv6/UDP")
    if name == "C5":
        kk = 6 if k is None else k
        kinds = C6_CHAIN[:kk]
        sd = 5 if seed is None else seed
        t = make_tables(sd, C6_CHAIN, n_acl=64, acl6_extra=64, n_pat=100,
                        n_r4=1000, n_r6=200_000 if not small else 5000, n_lb=64)
        esp = "IPSEC" in kinds
        tp = TrafficParams(seed=sd, v6_bp=2500, pkt_len=64 if pkt_len is None else pkt_len,
                           headroom=16 if esp else 0, tailroom=32 if esp else 0)
        return Workload(f"C5k{kk}", kinds, t, tp,
                        note=f"C6 chain prefix k={kk}, dual-stack 75/25")
    if name == "N3":
        # SURVEY 8(f) NEXT-3 (Figs. 16-17): FW -> router -> NAT with the
        # paper's ACL sizes (200 / 1K / 10K rules) at 64 / 128 / 1500 B
        kinds = ["ACL", "LPM4", "NAT"]
        sd = 6 if seed is None else seed
        n_acl = acl_rules or (200 if small else 1000)
        t = make_tables(sd, kinds, n_acl=n_acl, n_r4=1000)
        tp = TrafficParams(seed=sd, pkt_len=64 if pkt_len is None else pkt_len, match_ppm=0, tcp_pct=30,
                           l4csum=1)
        gen_nat(np.random.default_rng(np.random.PCG64(sd + 1000)), tp, t, n_dnat=1000 if not small else 200)
        return Workload(f"N3_{n_acl}", kinds, t, tp, note=f"FW({n_acl})->IPv4 router(1K)->NAT44, SNAT+DNAT")
    if name in ("NX2", "NX2_FW", "NX2_IDS"):
        # SURVEY 8(f) NEXT-2 (Figs. 13-14): four identical NFs in sequence,
        # 64-B TCP traffic, firewall rules that never drop
        nf = "DPI" if name == "NX2_IDS" else "ACL"
        kinds = [nf] * 4
        sd = 7 if seed is None else seed
        t = make_tables(sd, ["ACL", "DPI"], n_acl=64, n_pat=100, n_r4=1000, acl_deny=0.0)
        tp = TrafficParams(seed=sd, pkt_len=64 if pkt_len is None else pkt_len, tcp_pct=100)
        return Workload(f"NX2_{'IDS' if nf == 'DPI' else 'FW'}", kinds, t, tp,
                        note=f"4 x {'IDS (Aho-Corasick, 100 patterns)' if nf == 'DPI' else 'FW (64 rules, never drop)'}, 64 B TCP")
    raise ValueError(name)
