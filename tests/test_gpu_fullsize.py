"""Parity at the bench's full sizes, in the launch configuration bench.py times: the
ring (>> L2) generated in HBM, cut into 4,096-packet batch descriptors, one
nfc_process_batch call -- then EVERY packet's record, every forwarded packet's
output bytes, every match pair and every counter is compared with the CPU oracle
(tests/fullsize_oracle.py: parallel plain-oracle ranges; IPsec sequence numbers
by a two-pass per-SA prefix count, no value taken from the GPU)."""
import numpy as np
import pytest

import nfcgen
from tests.fullsize_oracle import compare_full

pytestmark = pytest.mark.gpu


def _args(config, pkt_len=None, k=None):
    return type("A", (), {"config": config, "pkt_len": pkt_len, "k": k, "acl_rules": None})()


def _run_ring(w, ring_mb, batch_pkts=4096):
    import torch
    import bench
    from paper_conf_hpca_hul18_b200 import nfc
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream(dev)
    arena, off, ln, n = bench.prepare_ring(w, ring_mb, 0, 1, 0, stream)
    rec = torch.zeros((n, 16), dtype=torch.uint8, device=dev)
    cap = 1 << 23
    mp = torch.zeros(cap, dtype=torch.int32, device=dev)
    mq = torch.zeros(cap, dtype=torch.int16, device=dev)
    mc = torch.zeros(1, dtype=torch.int32, device=dev)
    ch = nfc.Chain(w.kinds, device=0)
    ch.load_tables(w.tables)
    descs = bench.batch_descs(arena, off, ln, n, 0, batch_pkts)
    ch.process(descs, rec.data_ptr(), mp.data_ptr(), mq.data_ptr(), cap, mc.data_ptr(), stream.cuda_stream)
    torch.cuda.synchronize()
    k = int(mc.item())
    assert k <= cap
    recs = rec.cpu().numpy().view(nfcgen.RESULT).reshape(n)
    pairs = (mp[:k].cpu().numpy().view(np.uint32), mq[:k].cpu().numpy().view(np.uint16))
    return (recs, arena.cpu().numpy(), off.cpu().numpy().view(np.uint64), pairs, k, ch.stats(reset=True),
            len(descs))


@pytest.mark.parametrize("cfg,pl,k,ring_mb", [("C1", None, None, 1024), ("C2", None, None, 512),
                                              ("C3", None, None, 512), ("C4", None, None, 512),
                                              ("C5", 64, 1, 256), ("C5", 64, 2, 256), ("C5", 64, 3, 1024),
                                              ("C5", 0, 4, 256), ("C5", 512, 5, 128), ("C5", 1500, 6, 128)])
def test_full_ring_elementwise(cfg, pl, k, ring_mb):
    import bench
    w = bench.make_workload(_args(cfg, pl, k))
    recs, arena, off, pairs, npairs, stats, nb = _run_ring(w, ring_mb)
    assert nb > 1 and len(recs) == int(stats[0])
    n_fwd = compare_full(w, recs, arena, off, pairs, npairs, stats)
    assert n_fwd > 0


def test_c1_ring_one_batch_elementwise():
    """C1's ring as ONE batch descriptor (the single-batch fast path)."""
    import bench
    w = bench.make_workload(_args("C1"))
    recs, arena, off, pairs, npairs, stats, nb = _run_ring(w, 256, batch_pkts=0)
    assert nb == 1
    compare_full(w, recs, arena, off, pairs, npairs, stats)


def test_c1_ragged_batches_elementwise():
    """Batch sizes that are not multiples of 32 (chunks straddle 1-3 batch boundaries,
    empty batches in between): the chunk-record path's boundary lanes."""
    import torch
    import bench
    from paper_conf_hpca_hul18_b200 import nfc
    w = bench.make_workload(_args("C1"))
    w.traffic.match_ppm = 200_000
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream(dev)
    arena, off, ln, n = bench.prepare_ring(w, 16, 0, 1, 0, stream)
    rng = np.random.default_rng(5)
    sizes, s = [], 0
    while s < n:
        c = int(rng.choice([0, 1, 7, 13, 31, 33, 100, 4096]))
        c = min(c, n - s)
        sizes.append(c)
        s += c
    descs, s = [], 0
    for c in sizes:
        descs.append((arena.data_ptr(), off.data_ptr() + 8 * s, ln.data_ptr() + 2 * s, c, s))
        s += c
    rec = torch.zeros((n, 16), dtype=torch.uint8, device=dev)
    cap = 1 << 22
    mp = torch.zeros(cap, dtype=torch.int32, device=dev)
    mq = torch.zeros(cap, dtype=torch.int16, device=dev)
    mc = torch.zeros(1, dtype=torch.int32, device=dev)
    ch = nfc.Chain(w.kinds, device=0)
    ch.load_tables(w.tables)
    ch.process(descs, rec.data_ptr(), mp.data_ptr(), mq.data_ptr(), cap, mc.data_ptr(), stream.cuda_stream)
    torch.cuda.synchronize()
    kk = int(mc.item())
    recs = rec.cpu().numpy().view(nfcgen.RESULT).reshape(n)
    pairs = (mp[:kk].cpu().numpy().view(np.uint32), mq[:kk].cpu().numpy().view(np.uint16))
    compare_full(w, recs, arena.cpu().numpy(), off.cpu().numpy().view(np.uint64), pairs, kk, ch.stats(reset=True))
