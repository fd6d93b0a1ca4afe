"""The device traffic generator (nfcgen/gen_dev.cu: batches written straight into HBM)
is byte-identical to the host generator for every workload knob, and the dense-ring
gather keeps each selected frame's bytes."""
import numpy as np
import pytest

import nfcgen

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("cfg,k,pl,edge", [("C1", None, None, False), ("C1", None, 1, True), ("C2", None, None, False),
                                           ("C3", None, None, True), ("C4", None, 1, True), ("C5", 6, 0, True),
                                           ("N3", None, 128, False)])
def test_device_generator_equals_host(cfg, k, pl, edge):
    import torch
    from nfcgen import device as gd
    w = nfcgen.workload(cfg, k=k, pkt_len=pl, small=True)
    if edge:
        w.traffic.tcp_pct = 40
        w.traffic.edge(100_000)
        w.traffic.malformed_ppm, w.traffic.ttl1_ppm = 20_000, 10_000
    first, n = 123_457, 5000
    b = nfcgen.generate(w.traffic, w.tables, first, n)
    arena, off, ln = gd.generate(w.traffic, w.tables, first, n, device=0)
    torch.cuda.synchronize()
    assert np.array_equal(off.cpu().numpy().view(np.uint64), b.off)
    assert np.array_equal(ln.cpu().numpy().view(np.uint16), b.len)
    a = arena.cpu().numpy()
    assert np.array_equal(a[:len(b.arena) - 64], b.arena[:len(b.arena) - 64])


def test_device_gather_dense_ring():
    import torch
    from nfcgen import device as gd
    w = nfcgen.workload("C3", small=True)
    w.traffic.headroom, w.traffic.tailroom = 16, 32
    arena, off, ln = gd.generate(w.traffic, w.tables, 0, 3000, device=0)
    idx = torch.arange(1, 3000, 3, device=arena.device)
    d, doff, dl = gd.gather(arena, off, ln, idx, 16, 32)
    b = nfcgen.generate(w.traffic, w.tables, 0, 3000)
    dn, don, dln = d.cpu().numpy(), doff.cpu().numpy(), dl.cpu().numpy().view(np.uint16)
    for kk, j in enumerate(range(1, 3000, 3)):
        assert dln[kk] == b.len[j]
        assert int(don[kk]) % 16 == 0
        assert dn[don[kk]:don[kk] + dln[kk]].tobytes() == b.frame(j)
