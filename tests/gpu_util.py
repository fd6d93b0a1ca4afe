"""Helpers for the GPU parity tests: run a batch through the C ABI (via the
thin binding) and through the oracle, and compare everything."""
from __future__ import annotations

import numpy as np

import nfcgen
import oracle

STATS_SKIP = {11, 12}  # ST_DPI_OVF_PKTS, ST_MIXED_CHUNKS: product-only diagnostic counters


def gpu_run(chain, batches, match_cap=1 << 16):
    """batches: list of nfcgen.Batch processed in one nfc_process_batch call.
    Returns (records, [arena after per batch], (pkt, pat), match_count)."""
    import torch
    dev = torch.device("cuda", chain.device)
    keep = []
    descs = []
    n_tot = sum(b.n for b in batches)
    for b in batches:
        a = torch.from_numpy(b.arena).to(dev)
        o = torch.from_numpy(b.off.view(np.int64)).to(dev)
        ln = torch.from_numpy(b.len.view(np.int16)).to(dev)
        keep.append((a, o, ln))
        descs.append((a.data_ptr(), o.data_ptr(), ln.data_ptr(), b.n, b.first_index))
    rec = torch.zeros((max(1, n_tot), 16), dtype=torch.uint8, device=dev)
    mp = torch.zeros(max(1, match_cap), dtype=torch.int32, device=dev)
    mq = torch.zeros(max(1, match_cap), dtype=torch.int16, device=dev)
    mc = torch.zeros(1, dtype=torch.int32, device=dev)
    chain.process(descs, rec.data_ptr(), mp.data_ptr(), mq.data_ptr(), match_cap, mc.data_ptr(),
                  torch.cuda.current_stream(dev).cuda_stream)
    torch.cuda.synchronize(dev)
    recs = rec.cpu().numpy().view(nfcgen.RESULT).reshape(-1)[:n_tot]
    k = int(mc.item())
    kk = min(k, match_cap)
    pairs = (mp[:kk].cpu().numpy().view(np.uint32), mq[:kk].cpu().numpy().view(np.uint16))
    arenas = [t[0].cpu().numpy() for t in keep]
    return recs, arenas, pairs, k


def sorted_pairs(p, q):
    a = np.stack([p.astype(np.int64), q.astype(np.int64)], axis=1)
    if len(a) == 0:
        return a
    return a[np.lexsort((a[:, 1], a[:, 0]))]


def compare_records(got, want, ctx=""):
    if np.array_equal(got.view(np.uint8), want.view(np.uint8)):
        return
    for f in want.dtype.names:
        bad = np.nonzero(got[f] != want[f])[0]
        if len(bad):
            i = bad[0]
            raise AssertionError(f"{ctx}: field {f} differs at {len(bad)} packets; first {i}: "
                                 f"got {got[i]} want {want[i]}")
    raise AssertionError(f"{ctx}: records differ")


def compare_bytes(recs, got_arena, got_off, want_arena, want_off, ctx=""):
    """Output frame bytes of FORWARDED packets (dropped packets' bytes are unspecified, R#14)."""
    fwd = np.nonzero(recs["drop_nf"] == 0xFF)[0]
    for i in fwd:
        d = 16 if recs["esp_sa"][i] != 0xFF else 0
        L = int(recs["out_len"][i])
        g = got_arena[int(got_off[i]) - d:int(got_off[i]) - d + L]
        w = want_arena[int(want_off[i]) - d:int(want_off[i]) - d + L]
        if not np.array_equal(g, w):
            bad = np.nonzero(g != w)[0]
            raise AssertionError(f"{ctx}: packet {i} bytes differ at offsets {bad[:8]} (len {L})")
    return len(fwd)


def check_parity(w: nfcgen.Workload, chain, n: int, first: int = 0, split=None, match_cap=1 << 16,
                 compare_stats=True):
    b = nfcgen.generate(w.traffic, w.tables, first, n)
    orc = oracle.OracleChain(w.kinds, w.tables)
    want, want_arena, (wp, wq), npairs = orc.run(b, match_cap=max(match_cap, 1))
    if split:
        parts, s0 = [], 0
        for cnt in list(split) + [n - sum(split)]:
            parts.append(nfcgen.generate(w.traffic, w.tables, first + s0, cnt))
            s0 += cnt
        got, arenas, (gp, gq), k = gpu_run(chain, parts, match_cap)
        compare_records(got, want, w.name + " split")
        s0 = 0
        for pb, ga in zip(parts, arenas):
            compare_bytes(want[s0:s0 + pb.n], ga, pb.off, want_arena, b.off[s0:s0 + pb.n], f"{w.name} part@{s0}")
            s0 += pb.n
    else:
        got, arenas, (gp, gq), k = gpu_run(chain, [b], match_cap)
        compare_records(got, want, w.name)
        compare_bytes(want, arenas[0], b.off, want_arena, b.off, w.name)
    assert k == npairs, f"{w.name}: match_count {k} != oracle {npairs}"
    if npairs <= match_cap:
        assert np.array_equal(sorted_pairs(gp, gq), sorted_pairs(wp, wq)), f"{w.name}: match pairs differ"
    if compare_stats:
        st = chain.stats(reset=True)
        assert len(st) == len(orc.stats), (len(st), len(orc.stats))
        for i in range(len(st)):
            if i in STATS_SKIP:
                continue
            assert st[i] == orc.stats[i], f"{w.name}: stats[{i}] {st[i]} != {orc.stats[i]}"
    return got, want
