"""Parity at the bench's full sizes, in the launch configuration bench.py times
(one nfc_process_batch over a ring >> L2): sampled packets are recomputed one
by one by the oracle and compared field by field and byte by byte; properties
that hold at any size are checked on every packet (counter conservation, pair
count, per-SA ESP sequence numbers consecutive in global order)."""
import numpy as np
import pytest

import nfcgen
import oracle

pytestmark = pytest.mark.gpu


def _run_ring(w, ring_mb):
    import torch
    import bench
    from paper_conf_hpca_hul18_b200 import nfc
    n = bench.ring_packets(w, ring_mb)
    b = nfcgen.generate(w.traffic, w.tables, 0, n)
    dev = torch.device("cuda", 0)
    arena = torch.from_numpy(b.arena).to(dev)
    off = torch.from_numpy(b.off.view(np.int64)).to(dev)
    ln = torch.from_numpy(b.len.view(np.int16)).to(dev)
    rec = torch.zeros((n, 16), dtype=torch.uint8, device=dev)
    cap = 1 << 22
    mp = torch.zeros(cap, dtype=torch.int32, device=dev)
    mq = torch.zeros(cap, dtype=torch.int16, device=dev)
    mc = torch.zeros(1, dtype=torch.int32, device=dev)
    ch = nfc.Chain(w.kinds, device=0)
    ch.load_tables(w.tables)
    ch.process_tensors(arena, off, ln, rec, mp, mq, mc)
    torch.cuda.synchronize()
    recs = rec.cpu().numpy().view(nfcgen.RESULT).reshape(n)
    k = int(mc.item())
    return b, recs, arena.cpu().numpy(), k, ch.stats(), ch


def _check_samples(w, b, recs, ga, n_samples=1500, seq_from_gpu=False):
    orc = oracle.OracleChain(w.kinds, w.tables)
    rng = np.random.default_rng(7)
    sample = np.unique(np.concatenate([rng.integers(0, b.n, n_samples), [0, b.n - 1]]))
    for i in sample:
        r = recs[i]
        seq = int(r["esp_seq"]) if (seq_from_gpu and r["esp_sa"] != 0xFF) else None
        want, out, _ = orc.run_one(b.frame(i), int(i), seq=seq)
        assert bytes(r.tobytes()) == bytes(want.tobytes()), (i, r, want)
        if r["drop_nf"] == 0xFF:
            s = int(b.off[i]) - (16 if r["esp_sa"] != 0xFF else 0)
            assert ga[s:s + int(r["out_len"])].tobytes() == out, i


def _check_stats(recs, st, k):
    n = len(recs)
    assert st[0] == n
    assert st[2] == int((recs["drop_nf"] == 0xFF).sum())
    assert st[2] + st[3] == n
    assert st[6] == int(recs["dpi_nmatch"].astype(np.int64).sum()) == k


def test_c1_bench_ring_sampled():
    import bench
    w = bench.make_workload(type("A", (), {"config": "C1", "pkt_len": None, "k": None})())
    b, recs, ga, k, st, _ = _run_ring(w, 1024)
    assert b.n == 16777216
    _check_stats(recs, st, k)
    _check_samples(w, b, recs, ga)


def test_c2_bench_ring_sampled_and_seq_property():
    import bench
    w = bench.make_workload(type("A", (), {"config": "C2", "pkt_len": None, "k": None})())
    b, recs, ga, k, st, _ = _run_ring(w, 512)
    _check_stats(recs, st, k)
    # per SA: sequence numbers are 1..count in global packet order (seq0 = 0)
    sa = recs["esp_sa"].astype(np.int64)
    assert (sa != 0xFF).all()
    for s in range(64):
        q = recs["esp_seq"][sa == s].astype(np.int64)
        assert np.array_equal(q, np.arange(1, len(q) + 1)), s
    # SA selection + bytes on samples (oracle given the GPU's sequence number)
    _check_samples(w, b, recs, ga, n_samples=300, seq_from_gpu=True)


def test_c3_imix_ring_sampled():
    import bench
    w = bench.make_workload(type("A", (), {"config": "C3", "pkt_len": None, "k": None})())
    b, recs, ga, k, st, _ = _run_ring(w, 512)
    _check_stats(recs, st, k)
    _check_samples(w, b, recs, ga, n_samples=800)
