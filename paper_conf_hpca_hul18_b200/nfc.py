"""Thin ctypes binding of libnfc.so (include/nfc.h).

Argument marshalling only: every step of the SFC hot path runs in the CUDA
kernels behind the C ABI.  There is no CPU fallback: if libnfc.so is missing
or fails to load, importing this module raises.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional, Sequence

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("NFC_LIB") or os.path.join(HERE, "libnfc.so")

NFC_OK, NFC_EINVAL, NFC_ENOMEM, NFC_ECUDA, NFC_ESTATE, NFC_ECAP, NFC_EUNSUP = 0, -1, -2, -3, -4, -5, -6
ACL, DPI, LPM4, LPM6, IPSEC, LB, NAT = 1, 2, 3, 4, 5, 6, 7
KINDS = {"ACL": ACL, "DPI": DPI, "LPM4": LPM4, "LPM6": LPM6, "IPSEC": IPSEC, "LB": LB, "NAT": NAT}
STATS_RESET = 1
STATS_ALLREDUCE = 2   # nfc_collect_stats: sum over the ranks of the attached NCCL comm
COMM_ID_BYTES = 128
F_UNFUSED = 1   # nfc_chain_opts.flags: per-NF kernels with re-split (NEXT-1 baseline)
F_PARALLEL = 2  # nfc_chain_opts.flags: the chain's NFs on different warps + XOR merge (NEXT-2)

# stats vector layout
ST_PKTS, ST_BYTES_IN, ST_FWD, ST_DROP, ST_BYTES_OUT, ST_PARSE_DROP = 0, 1, 2, 3, 4, 5
ST_DPI_PAIRS, ST_MATCH_OVF, ST_ESP_PKTS, ST_ESP_BYTES, ST_ESP_BLOCKS, ST_DPI_OVF_PKTS = 6, 7, 8, 9, 10, 11
ST_MIXED_CHUNKS = 12   # product-only diagnostic: 32-packet chunks mixing IPv4 and IPv6 (a3 regrouping)
ST_POS_BASE, ST_VAR_BASE = 16, 64

RESULT_DTYPE = np.dtype([("drop_nf", "u1"), ("esp_sa", "u1"), ("port", "<u2"), ("acl_rule", "<u2"),
                         ("lb_backend", "<u2"), ("dpi_nmatch", "<u2"), ("out_len", "<u2"),
                         ("esp_seq", "<u4")])

_P = ctypes.c_void_p
_u32 = ctypes.c_uint32


class NfcError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"nfc error {code}: {msg}")
        self.code = code


class ChainOpts(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("flags", _u32), ("max_batch_pkts", _u32)]


class AclSpec(ctypes.Structure):
    _fields_ = [("n_rules", _u32), ("default_action", _u32), ("rules", _P)]


class DpiSpec(ctypes.Structure):
    _fields_ = [("n_patterns", _u32), ("blob", _P), ("off", _P), ("action", _P)]


class LpmSpec(ctypes.Structure):
    _fields_ = [("n_routes", _u32), ("routes", _P), ("n_nexthops", _u32), ("nexthops", _P),
                ("n_ports", _u32), ("port_macs", _P)]


class IpsecSpec(ctypes.Structure):
    _fields_ = [("n_sa", _u32), ("sas", _P)]


class LbSpec(ctypes.Structure):
    _fields_ = [("n_backends", _u32), ("backend_port", _P), ("key", _P)]


class NatSpec(ctypes.Structure):
    _fields_ = [("n_inside", _u32), ("inside", _P), ("n_pool", _u32), ("pool", _P), ("port_lo", _u32),
                ("port_hi", _u32), ("n_dnat", _u32), ("dnat", _P), ("ext_ports", _u32), ("key", _P)]


class Batch(ctypes.Structure):
    _fields_ = [("arena", _P), ("off", _P), ("len", _P), ("n", _u32), ("reserved", _u32),
                ("first_global_index", ctypes.c_uint64)]


class StreamResult(ctypes.Structure):
    _fields_ = [("nocc", _P), ("drop", _P), ("occ_pkt", _P), ("occ_pat", _P), ("occ_end", _P),
                ("occ_cap", _u32), ("reserved", _u32), ("occ_count", _P)]


class Result(ctypes.Structure):
    _fields_ = [("rec", _P), ("match_pkt", _P), ("match_pat", _P), ("match_cap", _u32),
                ("reserved", _u32), ("match_count", _P)]


EXPORTS = ["nfc_build_chain", "nfc_destroy_chain", "nfc_chain_room", "nfc_load_tables",
           "nfc_process_batch", "nfc_process_host", "nfc_stats_len", "nfc_collect_stats",
           "nfc_launch_count", "nfc_last_launch", "nfc_plan_parallel", "nfc_last_error", "nfc_version", "nfc_rss_shard",
           "nfc_dpi_stream_create", "nfc_dpi_stream_create_regex", "nfc_dpi_stream_destroy", "nfc_dpi_stream_reset",
           "nfc_dpi_stream_process", "nfc_dpi_stream_flows", "nfc_comm_unique_id", "nfc_comm_init",
           "nfc_comm_destroy", "nfc_attach_comm", "nfc_measure_peaks", "nfc_set_groups", "nfc_get_groups"]
DEBUG_EXPORTS = ["nfc_dbg_build", "nfc_dbg_destroy", "nfc_dbg_dpi", "nfc_dbg_dpi_shape", "nfc_dbg_dpi_tier",
                 "nfc_dbg_dpi_tier_shape", "nfc_dbg_dpi_slot", "nfc_dbg_nat", "nfc_dbg_lpm4",
                 "nfc_dbg_lpm6", "nfc_dbg_lpm6_levels", "nfc_dbg_acl", "nfc_dbg_acl4_image", "nfc_dbg_aes128_block",
                 "nfc_dbg_toeplitz", "nfc_dbg_hmac_sha1"]


def _load_lib():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built: run __graft_entry__.build() "
                          "(no CPU fallback exists for the SFC hot path)")
    L = ctypes.CDLL(LIB_PATH)
    L.nfc_build_chain.argtypes = [_P, _u32, ctypes.POINTER(ChainOpts), ctypes.POINTER(_P)]
    L.nfc_destroy_chain.argtypes = [_P]
    L.nfc_destroy_chain.restype = None
    L.nfc_chain_room.argtypes = [_P, ctypes.POINTER(_u32), ctypes.POINTER(_u32)]
    L.nfc_load_tables.argtypes = [_P, _u32, _P, ctypes.c_size_t]
    L.nfc_process_batch.argtypes = [_P, _P, _u32, ctypes.POINTER(Result), _P]
    L.nfc_process_host.argtypes = [_P, _P, ctypes.c_uint64, _P, _P, _u32, ctypes.c_uint64, _P, _P, _P, _u32,
                                   ctypes.POINTER(_u32), _P]
    L.nfc_stats_len.argtypes = [_P, ctypes.POINTER(ctypes.c_size_t)]
    L.nfc_collect_stats.argtypes = [_P, _P, ctypes.c_size_t, _u32]
    L.nfc_launch_count.argtypes = [_P, ctypes.POINTER(ctypes.c_uint64)]
    L.nfc_last_launch.argtypes = [_P, _P]
    L.nfc_plan_parallel.argtypes = [_P, _u32, _P]
    L.nfc_rss_shard.argtypes = [ctypes.c_int, ctypes.POINTER(Batch), _u32, _P, _P]
    L.nfc_dpi_stream_create.argtypes = [ctypes.c_int, ctypes.POINTER(DpiSpec), _u32, ctypes.POINTER(_P)]
    L.nfc_dpi_stream_create_regex.argtypes = [ctypes.c_int, ctypes.POINTER(DpiSpec), _u32, _u32, ctypes.POINTER(_P)]
    L.nfc_dpi_stream_destroy.argtypes = [_P]
    L.nfc_dpi_stream_reset.argtypes = [_P, _P]
    L.nfc_dpi_stream_process.argtypes = [_P, ctypes.POINTER(Batch), ctypes.POINTER(StreamResult), _P]
    L.nfc_dpi_stream_flows.argtypes = [_P, ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64)]
    L.nfc_comm_unique_id.argtypes = [_P, ctypes.c_size_t]
    L.nfc_comm_init.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, _P, ctypes.POINTER(_P)]
    L.nfc_comm_destroy.argtypes = [_P]
    L.nfc_attach_comm.argtypes = [_P, _P]
    L.nfc_measure_peaks.argtypes = [ctypes.c_int, _P]
    L.nfc_set_groups.argtypes = [_P, _P]
    L.nfc_get_groups.argtypes = [_P, _P]
    L.nfc_last_error.restype = ctypes.c_char_p
    L.nfc_version.restype = ctypes.c_char_p
    P32 = ctypes.POINTER(_u32)
    L.nfc_dbg_build.argtypes = [_u32, _P, ctypes.c_size_t, ctypes.POINTER(_P)]
    L.nfc_dbg_destroy.argtypes = [_P]
    L.nfc_dbg_destroy.restype = None
    L.nfc_dbg_dpi.argtypes = [_P, _P, ctypes.c_size_t, _P, _u32, P32, P32]
    L.nfc_dbg_dpi_shape.argtypes = [_P, P32, P32, P32]
    L.nfc_dbg_dpi_tier.argtypes = [_P, _u32, _u32, _P, ctypes.c_size_t, _P, _u32, P32, P32, _P]
    L.nfc_dbg_dpi_tier_shape.argtypes = [_P, P32, P32]
    L.nfc_dbg_dpi_slot.argtypes = [_P, _P, ctypes.c_size_t, _P, _u32, P32, P32, P32, P32]
    L.nfc_dbg_nat.argtypes = [_P, ctypes.c_uint8, _u32, _u32, ctypes.c_uint16, ctypes.c_uint16, ctypes.c_uint16,
                              _P, P32]
    L.nfc_dbg_lpm4.argtypes = [_P, _u32, P32, P32]
    L.nfc_dbg_lpm6.argtypes = [_P, _P, P32, P32, P32]
    L.nfc_dbg_lpm6_levels.argtypes = [_P, P32]
    L.nfc_dbg_acl.argtypes = [_P, _u32, _P, _P, ctypes.c_uint16, ctypes.c_uint16, ctypes.c_uint8, P32, P32]
    L.nfc_dbg_acl4_image.argtypes = [_P, _u32, _u32, _u32, ctypes.c_uint16, ctypes.c_uint16, ctypes.c_uint8, P32, P32]
    L.nfc_dbg_aes128_block.argtypes = [_P, _P, _P]
    L.nfc_dbg_toeplitz.argtypes = [_P, _P, ctypes.c_size_t, P32]
    L.nfc_dbg_hmac_sha1.argtypes = [_P, _P, ctypes.c_size_t, _P]
    return L


lib = _load_lib()


def _check(rc: int, allow=()):
    if rc != NFC_OK and rc not in allow:
        raise NfcError(rc, lib.nfc_last_error().decode())
    return rc


def _np(a, dtype=None):
    a = np.ascontiguousarray(a if dtype is None else np.asarray(a, dtype=dtype))
    return a


class Chain:
    """A service function chain bound to one CUDA device (original SFC order)."""

    def __init__(self, kinds: Sequence, device: int = 0, max_batch_pkts: int = 0, flags: int = 0):
        ks = [KINDS[k] if isinstance(k, str) else int(k) for k in kinds]
        arr = (_u32 * len(ks))(*ks)
        h = _P()
        opts = ChainOpts(device, flags, max_batch_pkts)
        _check(lib.nfc_build_chain(arr, len(ks), ctypes.byref(opts), ctypes.byref(h)))
        self.h = h
        self.kinds = ks
        self.device = device
        self._keep = []

    def close(self):
        if getattr(self, "h", None):
            lib.nfc_destroy_chain(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def room(self):
        hr, tr = _u32(), _u32()
        _check(lib.nfc_chain_room(self.h, ctypes.byref(hr), ctypes.byref(tr)))
        return hr.value, tr.value

    # ------------------------------------------------------------ tables
    def _load(self, kind: int, spec):
        return _check(lib.nfc_load_tables(self.h, kind, ctypes.byref(spec), ctypes.sizeof(spec)))

    def load_acl(self, rules: np.ndarray, default_action: int = 0):
        r = _np(rules)
        return self._load(ACL, AclSpec(len(r), default_action, r.ctypes.data if len(r) else None))

    def load_dpi(self, blob: np.ndarray, off: np.ndarray, action: np.ndarray):
        b, o, a = _np(blob, np.uint8), _np(off, np.uint32), _np(action, np.uint8)
        return self._load(DPI, DpiSpec(len(a), b.ctypes.data, o.ctypes.data, a.ctypes.data))

    def load_lpm(self, kind: int, routes: np.ndarray, nexthops: np.ndarray, port_macs: np.ndarray):
        r, n, p = _np(routes), _np(nexthops), _np(port_macs, np.uint8)
        return self._load(kind, LpmSpec(len(r), r.ctypes.data if len(r) else None, len(n), n.ctypes.data,
                                        len(p), p.ctypes.data))

    def load_ipsec(self, sas: np.ndarray):
        s = _np(sas)
        return self._load(IPSEC, IpsecSpec(len(s), s.ctypes.data))

    def load_lb(self, ports: np.ndarray, key: np.ndarray):
        p, k = _np(ports, np.uint16), _np(key, np.uint8)
        return self._load(LB, LbSpec(len(p), p.ctypes.data, k.ctypes.data))

    def load_nat(self, inside: np.ndarray, pool: np.ndarray, port_lo: int, port_hi: int, dnat: np.ndarray,
                 ext_ports: int, key: np.ndarray):
        """NAT44 tables (nfc_nat_spec): inside prefixes (8-B records), public pool (u32),
        SNAT port range, DNAT entries (16-B records), Internet-facing port mask, 40-B key."""
        i, d = np.ascontiguousarray(inside), np.ascontiguousarray(dnat)     # 8-B / 16-B records
        assert i.itemsize == 8 and d.itemsize == 16
        p, k = _np(pool, np.uint32), _np(key, np.uint8)
        return self._load(NAT, NatSpec(len(inside), i.ctypes.data if i.size else None, len(p), p.ctypes.data,
                                       port_lo, port_hi, len(dnat), d.ctypes.data if d.size else None,
                                       ext_ports, k.ctypes.data))

    def load_tables(self, t):
        """Load every NF of the chain from an object with the nfcgen.Tables fields
        (a repeated kind shares its tables: loaded once)."""
        for k in dict.fromkeys(self.kinds):
            if k == ACL:
                self.load_acl(t.acl_rules, t.acl_default)
            elif k == DPI:
                self.load_dpi(t.pat_blob, t.pat_off, t.pat_action)
            elif k == LPM4:
                self.load_lpm(LPM4, t.routes4, t.nh4, t.pmac4)
            elif k == LPM6:
                self.load_lpm(LPM6, t.routes6, t.nh6, t.pmac6)
            elif k == IPSEC:
                self.load_ipsec(t.sas)
            elif k == LB:
                self.load_lb(t.lb_ports, t.lb_key)
            elif k == NAT:
                self.load_nat(t.nat_inside, t.nat_pool, t.nat_port_lo, t.nat_port_hi, t.nat_dnat,
                              t.nat_ext_ports, t.nat_key)

    # ------------------------------------------------------------ processing
    @staticmethod
    def batch_array(batches):
        """nfc_batch descriptor array (host) for a list of (arena_ptr, off_ptr, len_ptr, n,
        first_global_index); pass it to process() to skip rebuilding it every call."""
        arr = (Batch * max(1, len(batches)))()
        for i, (a, o, l, n, fgi) in enumerate(batches):
            arr[i] = Batch(a, o, l, n, 0, fgi)
        arr.count = len(batches)
        return arr

    def process(self, batches, rec_ptr: int, match_pkt_ptr: int = 0, match_pat_ptr: int = 0,
                match_cap: int = 0, match_count_ptr: int = 0, stream: int = 0):
        """batches: list of (arena_ptr, off_ptr, len_ptr, n, first_global_index) device pointers,
        or a batch_array() of them."""
        arr = batches if hasattr(batches, "count") and not isinstance(batches, list) else self.batch_array(batches)
        res = Result(rec_ptr, match_pkt_ptr or None, match_pat_ptr or None, match_cap, 0,
                     match_count_ptr or None)
        return _check(lib.nfc_process_batch(self.h, arr, arr.count, ctypes.byref(res), stream or None))

    def process_tensors(self, arena, off, ln, rec, match_pkt=None, match_pat=None, match_count=None,
                        first_global_index: int = 0, n: Optional[int] = None, stream=None):
        """torch CUDA tensors (arena u8, off int64/uint64, len int16/uint16, rec u8[n,16])."""
        import torch
        n = int(off.numel()) if n is None else n
        s = stream if stream is not None else torch.cuda.current_stream(arena.device)
        return self.process([(arena.data_ptr(), off.data_ptr(), ln.data_ptr(), n, first_global_index)],
                            rec.data_ptr(),
                            match_pkt.data_ptr() if match_pkt is not None else 0,
                            match_pat.data_ptr() if match_pat is not None else 0,
                            int(match_pkt.numel()) if match_pkt is not None else 0,
                            match_count.data_ptr() if match_count is not None else 0,
                            s.cuda_stream)

    def process_host(self, arena: np.ndarray, off: np.ndarray, ln: np.ndarray, first_global_index: int = 0,
                     match_cap: int = 1 << 20, stream: int = 0):
        """End-to-end call with host buffers (arena rewritten in place). Returns (rec, (pkt, pat), n_pairs)."""
        off = _np(off, np.uint64)
        ln = _np(ln, np.uint16)
        n = len(off)
        rec = np.zeros(n, dtype=RESULT_DTYPE)
        mp = np.zeros(max(1, match_cap), dtype=np.uint32)
        mq = np.zeros(max(1, match_cap), dtype=np.uint16)
        npairs = _u32()
        assert arena.flags["C_CONTIGUOUS"] and arena.dtype == np.uint8
        _check(lib.nfc_process_host(self.h, arena.ctypes.data, arena.nbytes, off.ctypes.data, ln.ctypes.data, n,
                                    first_global_index, rec.ctypes.data, mp.ctypes.data, mq.ctypes.data,
                                    match_cap, ctypes.byref(npairs), stream or None))
        k = min(npairs.value, match_cap)
        return rec, (mp[:k], mq[:k]), npairs.value

    def process_host_ptr(self, arena_ptr: int, arena_bytes: int, off_ptr: int, len_ptr: int, n: int,
                         rec_ptr: int, mp_ptr: int, mq_ptr: int, match_cap: int, first_global_index: int = 0,
                         stream: int = 0) -> int:
        npairs = _u32()
        _check(lib.nfc_process_host(self.h, arena_ptr, arena_bytes, off_ptr, len_ptr, n, first_global_index,
                                    rec_ptr, mp_ptr, mq_ptr, match_cap, ctypes.byref(npairs), stream or None))
        return npairs.value

    def stats(self, reset: bool = False, allow_cap: bool = True, allreduce: bool = False) -> np.ndarray:
        """nfc_collect_stats; allreduce=True sums over the ranks of the attached comm."""
        n = ctypes.c_size_t()
        _check(lib.nfc_stats_len(self.h, ctypes.byref(n)))
        out = np.zeros(n.value, dtype=np.uint64)
        flags = (STATS_RESET if reset else 0) | (STATS_ALLREDUCE if allreduce else 0)
        _check(lib.nfc_collect_stats(self.h, out.ctypes.data, n.value, flags),
               allow=(NFC_ECAP,) if allow_cap else ())
        return out

    def set_groups(self, group):
        """nfc_set_groups: the parallel grouping of an F_PARALLEL chain (runs of legal NFs)."""
        g = np.array(list(group) + [0] * (8 - len(group)), dtype=np.uint8)
        _check(lib.nfc_set_groups(self.h, g.ctypes.data))

    def groups(self) -> list:
        g = np.zeros(8, dtype=np.uint8)
        _check(lib.nfc_get_groups(self.h, g.ctypes.data))
        return [int(x) for x in g[:len(self.kinds)]]

    def attach_comm(self, comm: Optional["Comm"]):
        """nfc_attach_comm: the NCCL communicator NFC_STATS_ALLREDUCE sums over (None detaches)."""
        self._comm = comm
        _check(lib.nfc_attach_comm(self.h, comm.h if comm is not None else None))

    def launches(self) -> int:
        c = ctypes.c_uint64()
        _check(lib.nfc_launch_count(self.h, ctypes.byref(c)))
        return c.value

    def last_launch(self) -> dict:
        """Shape of the last fused launch (nfc_last_launch)."""
        a = np.zeros(8, dtype=np.uint32)
        _check(lib.nfc_last_launch(self.h, a.ctypes.data))
        return dict(zip(("grid", "block", "smem", "dfa_mode", "dfa_dense", "dfa_sparse", "dfa_meta_smem", "acl_smem"),
                        (int(x) for x in a)))


def plan_parallel(kinds) -> list:
    """nfc_plan_parallel: group index per chain position (SFC parallelization, NEXT-2)."""
    k = np.array([KINDS[x] if isinstance(x, str) else int(x) for x in kinds], dtype=np.uint32)
    g = np.zeros(max(1, len(k)), dtype=np.uint8)
    _check(lib.nfc_plan_parallel(k.ctypes.data, len(k), g.ctypes.data))
    return [int(x) for x in g[:len(k)]]


class DpiStream:
    """Stateful cross-packet DPI (include/nfc.h "stateful DPI", NEXT-4, R#32) on one device.

    Argument marshalling only: every step runs in dpi_stream.cu."""

    def __init__(self, blob: np.ndarray, off: np.ndarray, action: np.ndarray, max_flows: int, device: int = 0,
                 regex: bool = False, max_states: int = 0):
        """regex=True: blob/off hold regular expressions (nfc_dpi_stream_create_regex)."""
        b, o, a = _np(blob, np.uint8), _np(off, np.uint32), _np(action, np.uint8)
        h = _P()
        spec = DpiSpec(len(a), b.ctypes.data, o.ctypes.data, a.ctypes.data)
        if regex:
            _check(lib.nfc_dpi_stream_create_regex(device, ctypes.byref(spec), max_flows, max_states, ctypes.byref(h)))
        else:
            _check(lib.nfc_dpi_stream_create(device, ctypes.byref(spec), max_flows, ctypes.byref(h)))
        self.h = h
        self.device = device

    def close(self):
        if getattr(self, "h", None):
            lib.nfc_dpi_stream_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def reset(self, stream: int = 0):
        return _check(lib.nfc_dpi_stream_reset(self.h, stream or None))

    def process(self, arena_ptr: int, off_ptr: int, len_ptr: int, n: int, first_global_index: int,
                nocc_ptr: int, drop_ptr: int, occ_pkt_ptr: int, occ_pat_ptr: int, occ_end_ptr: int,
                occ_cap: int, occ_count_ptr: int, stream: int = 0):
        b = Batch(arena_ptr, off_ptr, len_ptr, n, 0, first_global_index)
        r = StreamResult(nocc_ptr, drop_ptr, occ_pkt_ptr or None, occ_pat_ptr or None, occ_end_ptr or None,
                         occ_cap, 0, occ_count_ptr)
        return _check(lib.nfc_dpi_stream_process(self.h, ctypes.byref(b), ctypes.byref(r), stream or None))

    def process_tensors(self, arena, off, ln, nocc, drop, occ_pkt, occ_pat, occ_end, occ_count,
                        first_global_index: int = 0, stream=None):
        """torch CUDA tensors: arena u8, off int64, len int16, nocc int32[n], drop u8[n],
        occ_pkt int32[cap], occ_pat int16[cap], occ_end int16[cap], occ_count int32[1] (zeroed)."""
        import torch
        s = stream if stream is not None else torch.cuda.current_stream(arena.device)
        return self.process(arena.data_ptr(), off.data_ptr(), ln.data_ptr(), int(off.numel()),
                            first_global_index, nocc.data_ptr(), drop.data_ptr(), occ_pkt.data_ptr(),
                            occ_pat.data_ptr(), occ_end.data_ptr(), int(occ_pkt.numel()),
                            occ_count.data_ptr(), s.cuda_stream)

    def flows(self):
        nf, nu = ctypes.c_uint64(), ctypes.c_uint64()
        _check(lib.nfc_dpi_stream_flows(self.h, ctypes.byref(nf), ctypes.byref(nu)))
        return nf.value, nu.value


class Peaks(ctypes.Structure):
    _fields_ = [("alu_tops", ctypes.c_double), ("issue_tops", ctypes.c_double), ("smem_glookups", ctypes.c_double),
                ("l2_gsectors", ctypes.c_double), ("sm_count", _u32), ("sm_clock_mhz", _u32)]


def measure_peaks(device: int = 0) -> dict:
    """nfc_measure_peaks: measured ALU / issue / shared-memory / L2-gather peaks."""
    p = Peaks()
    _check(lib.nfc_measure_peaks(device, ctypes.byref(p)))
    return {f: getattr(p, f) for f, _ in Peaks._fields_}


def comm_unique_id() -> bytes:
    """nfc_comm_unique_id (ncclGetUniqueId): rank 0 makes it, the others receive it out of band."""
    b = ctypes.create_string_buffer(COMM_ID_BYTES)
    _check(lib.nfc_comm_unique_id(b, COMM_ID_BYTES))
    return b.raw


class Comm:
    """An NCCL communicator made by the library (nfc_comm_init); one per rank/GPU."""

    def __init__(self, device: int, nranks: int, rank: int, uid: bytes):
        assert len(uid) == COMM_ID_BYTES
        h = _P()
        _check(lib.nfc_comm_init(device, nranks, rank, _cbuf(uid), ctypes.byref(h)))
        self.h = h.value

    def close(self):
        if getattr(self, "h", None):
            lib.nfc_comm_destroy(self.h)
            self.h = None


def rss_shard(device: int, arena_ptr: int, off_ptr: int, len_ptr: int, n: int, n_shards: int, out_ptr: int,
              stream: int = 0):
    """Device-side RSS steering: out[i] = shard of frame i (u8)."""
    b = Batch(arena_ptr, off_ptr, len_ptr, n, 0, 0)
    return _check(lib.nfc_rss_shard(device, ctypes.byref(b), n_shards, out_ptr, stream or None))


def _cbuf(b: bytes):
    return ctypes.create_string_buffer(bytes(b), max(1, len(b)))


class HostImage:
    """include/nfc_debug.h: a device table image built by the product's builders and
    walked on the host with the kernel's algorithm (diagnostics, no GPU needed)."""

    def __init__(self, kind, **tables):
        self._keep = []
        kind = KINDS[kind] if isinstance(kind, str) else kind
        if kind == ACL:
            r = _np(tables["rules"])
            self._keep.append(r)
            spec = AclSpec(len(r), tables.get("default_action", 0), r.ctypes.data)
        elif kind == DPI:
            b, o, a = _np(tables["blob"], np.uint8), _np(tables["off"], np.uint32), _np(tables["action"], np.uint8)
            self._keep += [b, o, a]
            spec = DpiSpec(len(a), b.ctypes.data, o.ctypes.data, a.ctypes.data)
        elif kind in (LPM4, LPM6):
            r, n, p = _np(tables["routes"]), _np(tables["nexthops"]), _np(tables["port_macs"], np.uint8)
            self._keep += [r, n, p]
            spec = LpmSpec(len(r), r.ctypes.data, len(n), n.ctypes.data, len(p), p.ctypes.data)
        elif kind == NAT:
            i, d = np.ascontiguousarray(tables["inside"]), np.ascontiguousarray(tables["dnat"])
            p, k = _np(tables["pool"], np.uint32), _np(tables["key"], np.uint8)
            self._keep += [i, d, p, k]
            spec = NatSpec(len(i), i.ctypes.data if i.size else None, len(p), p.ctypes.data, tables["port_lo"],
                           tables["port_hi"], len(d), d.ctypes.data if d.size else None, tables.get("ext_ports", 0),
                           k.ctypes.data)
        else:
            raise ValueError(kind)
        h = _P()
        _check(lib.nfc_dbg_build(kind, ctypes.byref(spec), ctypes.sizeof(spec), ctypes.byref(h)))
        self.h = h
        self.kind = kind

    def __del__(self):
        if getattr(self, "h", None):
            lib.nfc_dbg_destroy(self.h)
            self.h = None

    def nat(self, proto: int, src: int, dst: int, sport: int, dport: int, ck: int):
        """The kernel's NAT translation: ((src, dst, sport, dport, checksum), DNAT probes)."""
        out = np.zeros(5, dtype=np.uint32)
        pr = _u32()
        _check(lib.nfc_dbg_nat(self.h, proto, src, dst, sport, dport, ck, out.ctypes.data, ctypes.byref(pr)))
        return tuple(int(x) for x in out), pr.value

    def dpi(self, data: bytes, cap: int = 65536):
        ids = np.zeros(cap, dtype=np.uint16)
        c, d = _u32(), _u32()
        _check(lib.nfc_dbg_dpi(self.h, _cbuf(data), len(data), ids.ctypes.data, cap, ctypes.byref(c), ctypes.byref(d)))
        return [int(x) for x in ids[:min(c.value, cap)]], bool(d.value)

    def dpi_shape(self):
        a, b, c = _u32(), _u32(), _u32()
        _check(lib.nfc_dbg_dpi_shape(self.h, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c)))
        return a.value, b.value, c.value

    def dpi_tier(self, data: bytes, hot: int, sparse: int, cap: int = 65536):
        """The kernel's tiered DFA walk (dense / sparse / cold); returns (ids, drop, tier_steps)."""
        ids = np.zeros(cap, dtype=np.uint16)
        ts = np.zeros(3, dtype=np.uint32)
        c, d = _u32(), _u32()
        _check(lib.nfc_dbg_dpi_tier(self.h, hot, sparse, _cbuf(data), len(data), ids.ctypes.data, cap,
                                    ctypes.byref(c), ctypes.byref(d), ts.ctypes.data))
        return [int(x) for x in ids[:min(c.value, cap)]], bool(d.value), [int(x) for x in ts]

    def dpi_slot(self, data: bytes, cap: int = 65536):
        """The kernel's DM_FULL walk over the slot image; returns (ids, drop, events, summary)."""
        ids = np.zeros(cap, dtype=np.uint16)
        c, d, ev, sm = _u32(), _u32(), _u32(), _u32()
        _check(lib.nfc_dbg_dpi_slot(self.h, _cbuf(data), len(data), ids.ctypes.data, cap, ctypes.byref(c),
                                    ctypes.byref(d), ctypes.byref(ev), ctypes.byref(sm)))
        return [int(x) for x in ids[:min(c.value, cap)]], bool(d.value), ev.value, sm.value

    def dpi_tier_shape(self):
        a, b = _u32(), _u32()
        _check(lib.nfc_dbg_dpi_tier_shape(self.h, ctypes.byref(a), ctypes.byref(b)))
        return a.value, b.value

    def lpm4(self, dst: int):
        nh, r = _u32(), _u32()
        _check(lib.nfc_dbg_lpm4(self.h, dst, ctypes.byref(nh), ctypes.byref(r)))
        return nh.value, r.value

    def lpm6(self, dst: bytes):
        nh, p, s = _u32(), _u32(), _u32()
        _check(lib.nfc_dbg_lpm6(self.h, _cbuf(dst), ctypes.byref(nh), ctypes.byref(p), ctypes.byref(s)))
        return nh.value, p.value, s.value

    def lpm6_levels(self):
        n = _u32()
        _check(lib.nfc_dbg_lpm6_levels(self.h, ctypes.byref(n)))
        return n.value

    def acl(self, family, src: bytes, dst: bytes, sport, dport, proto):
        r, a = _u32(), _u32()
        _check(lib.nfc_dbg_acl(self.h, family, _cbuf(src), _cbuf(dst), sport, dport, proto,
                               ctypes.byref(r), ctypes.byref(a)))
        return r.value, a.value

    def acl4_image(self, which, src: int, dst: int, sport, dport, proto):
        """IPv4 lookup through the search image (which=0) or the 16-bit first level (1);
        None if the rule set has no such image."""
        r, a = _u32(), _u32()
        rc = lib.nfc_dbg_acl4_image(self.h, which, src, dst, sport, dport, proto, ctypes.byref(r), ctypes.byref(a))
        if rc == NFC_EUNSUP:
            return None
        _check(rc)
        return r.value, a.value


def dbg_aes128_block(key: bytes, block: bytes) -> bytes:
    out = ctypes.create_string_buffer(16)
    _check(lib.nfc_dbg_aes128_block(_cbuf(key), _cbuf(block), out))
    return out.raw


def dbg_toeplitz(key: bytes, data: bytes) -> int:
    h = _u32()
    _check(lib.nfc_dbg_toeplitz(_cbuf(key), _cbuf(data), len(data), ctypes.byref(h)))
    return h.value


def dbg_hmac_sha1(key20: bytes, msg: bytes) -> bytes:
    out = ctypes.create_string_buffer(20)
    _check(lib.nfc_dbg_hmac_sha1(_cbuf(key20), _cbuf(msg), len(msg), out))
    return out.raw


def version() -> str:
    return lib.nfc_version().decode()
