"""Element-wise parity at the bench's full sizes: the whole GPU pass is compared
with the CPU oracle packet by packet (records, output bytes of forwarded packets,
match pairs) and counter by counter -- nothing sampled, nothing taken from the GPU.

The oracle is the plain single-threaded definition (oracle/oracle.c); to finish a
multi-million-packet ring in seconds, index ranges of the ring run in parallel
worker processes, each a plain sequential oracle over its range.  Per-packet
results depend only on the packet, except ESP sequence numbers (per SA, global
order among packets reaching IPsec): for IPsec chains a first
pass counts each range's packets per SA (the oracle's own per-SA counter), and
the second pass starts range r's SA counters at seq0 + the counts of ranges < r --
exactly the state a single sequential pass has when it reaches range r.

Test infrastructure only (tests/): the workers import oracle/ and nfcgen/, never
the product; the GPU results are inputs to the comparison, not to the oracle.
"""
from __future__ import annotations

import multiprocessing as mp
import os
import sys
from multiprocessing import shared_memory

import numpy as np

import nfcgen
import oracle

_G = {}
_SHM = []


def _share(a: np.ndarray):
    """Put a (large) array into POSIX shared memory for spawned workers."""
    shm = shared_memory.SharedMemory(create=True, size=max(1, a.nbytes))
    v = np.ndarray(a.shape, dtype=a.dtype, buffer=shm.buf)
    v[...] = a
    _SHM.append(shm)
    return (shm.name, a.shape, a.dtype.str if a.dtype.names is None else a.dtype.descr)


def _attach(spec):
    name, shape, dt = spec
    shm = shared_memory.SharedMemory(name=name)
    _SHM.append(shm)
    return np.ndarray(shape, dtype=np.dtype(dt), buffer=shm.buf)


def _init(w, specs, first, root):
    """Spawned worker: attach the GPU results (no CUDA, no fork of a threaded parent)."""
    if root not in sys.path:
        sys.path.insert(0, root)
    recs, arena, off, gp, gq = (_attach(x) for x in specs)
    _G.update(w=w, recs=recs.view(nfcgen.RESULT).reshape(-1), arena=arena, off=off, first=first, pairs=(gp, gq))


def _var_layout(kinds, t):
    n_acl = len(t.acl_rules) if "ACL" in kinds and t.acl_rules is not None else 0
    n_lb = len(t.lb_ports) if "LB" in kinds and t.lb_ports is not None else 0
    n_sa = len(t.sas) if "IPSEC" in kinds and t.sas is not None else 0
    sa0 = oracle.ST_VAR_BASE + n_acl + 1 + n_lb
    return sa0, n_sa


def _tables_with_seq(t, seq_start):
    if seq_start is None:
        return t
    t2 = nfcgen.Tables(**{k: getattr(t, k) for k in t.__dataclass_fields__})
    sas = t.sas.copy()
    sas["seq0"] = (sas["seq0"].astype(np.uint64) + np.asarray(seq_start, dtype=np.uint64)) & 0xFFFFFFFF
    t2.sas = sas
    return t2


def _count_pass(rng_ab):
    """Pass 1 (IPsec chains): the oracle over one range; its per-SA ESP packet counts."""
    a, b = rng_ab
    w = _G["w"]
    bt = nfcgen.generate(w.traffic, w.tables, a, b - a)
    orc = oracle.OracleChain(w.kinds, w.tables)
    orc.run(bt, match_cap=1 << 22)
    sa0, n_sa = _var_layout(w.kinds, w.tables)
    return orc.stats[sa0:sa0 + n_sa].copy()


def _check_pass(job):
    """Pass 2: the oracle over one range compared element-wise with the GPU pass."""
    (a, b), seq_start = job
    w, recs, ga, goff = _G["w"], _G["recs"], _G["arena"], _G["off"]
    bt = nfcgen.generate(w.traffic, w.tables, a, b - a)
    orc = oracle.OracleChain(w.kinds, _tables_with_seq(w.tables, seq_start))
    want, wa, (wp, wq), npairs = orc.run(bt, match_cap=1 << 24)
    got = recs[a:b]
    err = []
    if not np.array_equal(got.view(np.uint8), want.view(np.uint8)):
        for f in want.dtype.names:
            bad = np.nonzero(got[f] != want[f])[0]
            if len(bad):
                i = int(bad[0])
                err.append(f"field {f}: {len(bad)} packets differ, first {a + i}: got {got[i]} want {want[i]}")
                break
    fwd = np.nonzero(want["drop_nf"] == 0xFF)[0]
    nbad = 0
    for i in fwd:
        d = 16 if want["esp_sa"][i] != 0xFF else 0
        L = int(want["out_len"][i])
        g0 = int(goff[a + i]) - d
        w0 = int(bt.off[i]) - d
        if not np.array_equal(ga[g0:g0 + L], wa[w0:w0 + L]):
            if nbad == 0:
                err.append(f"packet {a + i}: output bytes differ (len {L})")
            nbad += 1
    if nbad:
        err.append(f"{nbad} forwarded packets with differing bytes in [{a}, {b})")
    # match pairs of this range (global ids = first_index + index)
    gp, gq = _G["pairs"]
    lo, hi = np.searchsorted(gp, _G["first"] + a), np.searchsorted(gp, _G["first"] + b)
    mine = np.stack([gp[lo:hi].astype(np.int64), gq[lo:hi].astype(np.int64)], 1)
    theirs = np.stack([wp.astype(np.int64) + _G["first"], wq.astype(np.int64)], 1)   # oracle ids: a + i
    mine = mine[np.lexsort((mine[:, 1], mine[:, 0]))]
    theirs = theirs[np.lexsort((theirs[:, 1], theirs[:, 0]))]
    if npairs != len(wp) or not np.array_equal(mine, theirs):
        err.append(f"match pairs differ in [{a}, {b}): gpu {len(mine)} oracle {npairs}")
    return err, orc.stats.copy(), len(fwd)


def _free():
    while _SHM:
        shm = _SHM.pop()
        shm.close()
        try:
            shm.unlink()
        except FileNotFoundError:
            pass


def compare_full(w, recs, arena, off, pairs, n_pairs_total, stats, first=0, workers=None, chunk=None):
    """Compare the GPU pass over packets [0, n) of w's global stream (laid out as
    nfcgen.generate lays them out) with the oracle, element by element.
    recs: GPU records (nfcgen.RESULT, n); arena/off: the GPU ring after the pass (host
    copies); pairs: (pkt u32, pat u16) GPU match pairs; stats: the GPU counter vector."""
    n = len(recs)
    assert n_pairs_total == len(pairs[0]), "the GPU match-pair capacity overflowed"
    workers = workers or max(1, min(32, os.cpu_count() or 1))
    chunk = chunk or max(4096, -(-n // (4 * workers)))
    ranges = [(a, min(n, a + chunk)) for a in range(0, n, chunk)]
    order = np.lexsort((pairs[1], pairs[0]))
    specs = [_share(np.ascontiguousarray(recs).view(np.uint8)), _share(arena), _share(off),
             _share(pairs[0][order].astype(np.int64)), _share(pairs[1][order].astype(np.uint16))]
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    # spawn, not fork: the parent holds CUDA and torch threads
    ctx = mp.get_context("spawn")
    try:
        pool = ctx.Pool(workers, initializer=_init, initargs=(w, specs, first, root))
    except Exception:
        _free()
        raise
    with pool:
        seq = [None] * len(ranges)
        if "IPSEC" in w.kinds:
            counts = pool.map(_count_pass, ranges)
            acc = np.zeros_like(counts[0])
            for r, c in enumerate(counts):
                seq[r] = acc.copy()
                acc = acc + c
        out = pool.map(_check_pass, list(zip(ranges, seq)))
    _free()
    errs = [e for o in out for e in o[0]]
    assert not errs, "\n".join(errs[:10])
    tot = sum((o[1].astype(np.uint64) for o in out), np.zeros_like(out[0][1]))
    assert len(stats) == len(tot), (len(stats), len(tot))
    for i in range(len(tot)):
        if i in (11, 12):   # product-only diagnostic counters (DPI overflow, mixed chunks)
            continue
        assert int(stats[i]) == int(tot[i]), f"stats[{i}] gpu {int(stats[i])} oracle {int(tot[i])}"
    return sum(o[2] for o in out)
