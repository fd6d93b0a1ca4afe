"""GPU tests of the multi-GPU path on one device: nfc_rss_shard steering is
bit-exact against the RSS definition (oracle Toeplitz + RETA), and running N
independent chains on the N shards (what N GPUs do) reproduces the
single-stream oracle packet for packet -- including per-SA ESP sequence
numbers -- with the counters summing to the single-stream stats."""
import numpy as np
import pytest

import nfcgen
import oracle
from paper_conf_hpca_hul18_b200 import dist as pdist
from tests.gpu_util import compare_bytes, sorted_pairs

pytestmark = pytest.mark.gpu


def _tuple_hash(frame: bytes) -> int:
    if frame[12:14] == b"\x86\xdd":
        t = frame[22:54] + frame[54:58]
    else:
        t = frame[26:34] + frame[34:38]
    return oracle.toeplitz(oracle.MS_RSS_KEY, t)


@pytest.mark.parametrize("wl,plen", [("C2", 1), ("C5", 64), ("C5", 0)])
def test_sharded_chains_equal_single_stream(wl, plen):
    import torch
    from paper_conf_hpca_hul18_b200 import nfc
    w = nfcgen.workload(wl, small=True, pkt_len=plen)
    n = 2000
    b = nfcgen.generate(w.traffic, w.tables, 0, n)
    dev = torch.device("cuda", 0)
    arena0 = torch.from_numpy(b.arena).to(dev)
    off = torch.from_numpy(b.off.view(np.int64)).to(dev)
    ln = torch.from_numpy(b.len.view(np.int16)).to(dev)
    orc = oracle.OracleChain(w.kinds, w.tables)
    want, want_arena, (wp, wq), npairs = orc.run(b)
    want_h = np.array([_tuple_hash(b.frame(i)) for i in range(n)])
    for N in (1, 2, 4, 8):
        shard = torch.zeros(n, dtype=torch.uint8, device=dev)
        nfc.rss_shard(0, arena0.data_ptr(), off.data_ptr(), ln.data_ptr(), n, N, shard.data_ptr(),
                      torch.cuda.current_stream().cuda_stream)
        sh = shard.cpu().numpy().astype(np.int64)
        assert np.array_equal(sh, pdist.shard_of_hash(want_h, N)), N
        arena = arena0.clone()
        parts, stats, pairs = [], None, []
        for r in range(N):
            idx = pdist.shard_indices(sh, r)
            if len(idx) == 0:
                continue
            ti = torch.from_numpy(idx).to(dev)
            so, sl = off.index_select(0, ti).contiguous(), ln.index_select(0, ti).contiguous()
            ch = nfc.Chain(w.kinds, device=0)
            ch.load_tables(w.tables)
            rec = torch.zeros((len(idx), 16), dtype=torch.uint8, device=dev)
            mp = torch.zeros(1 << 14, dtype=torch.int32, device=dev)
            mq = torch.zeros(1 << 14, dtype=torch.int16, device=dev)
            mc = torch.zeros(1, dtype=torch.int32, device=dev)
            ch.process_tensors(arena, so, sl, rec, mp, mq, mc, first_global_index=0)
            torch.cuda.synchronize()
            parts.append((idx, rec.cpu().numpy().view(nfcgen.RESULT).reshape(-1)))
            k = int(mc.item())
            local = mp[:k].cpu().numpy().view(np.uint32)
            pairs.append((idx[local], mq[:k].cpu().numpy().view(np.uint16)))
            st = ch.stats()
            stats = st if stats is None else stats + st
        got = pdist.merge_by_index(parts, n, nfcgen.RESULT)
        assert np.array_equal(got.view(np.uint8), want.view(np.uint8)), N
        compare_bytes(want, arena.cpu().numpy(), b.off, want_arena, b.off, f"{wl} N={N}")
        gp = np.concatenate([p for p, _ in pairs]) if pairs else np.zeros(0)
        gq = np.concatenate([q for _, q in pairs]) if pairs else np.zeros(0)
        assert np.array_equal(sorted_pairs(gp, gq), sorted_pairs(wp, wq))
        for i in range(len(stats)):
            if i not in (11, 12):
                assert stats[i] == orc.stats[i], (N, i)


def test_library_nccl_comm_allreduce_one_rank():
    """nfc_comm_unique_id / nfc_comm_init / nfc_attach_comm / NFC_STATS_ALLREDUCE with a
    one-rank NCCL communicator (the only shape one GPU allows): the all-reduced vector is
    the local one, RESET clears the local counters, and ALLREDUCE without a comm is
    NFC_ESTATE."""
    import torch
    from paper_conf_hpca_hul18_b200 import nfc
    w = nfcgen.workload("C1", small=True)
    ch = nfc.Chain(w.kinds, device=0)
    ch.load_tables(w.tables)
    b = nfcgen.generate(w.traffic, w.tables, 0, 3000)
    dev = torch.device("cuda", 0)
    arena = torch.from_numpy(b.arena).to(dev)
    off = torch.from_numpy(b.off.view(np.int64)).to(dev)
    ln = torch.from_numpy(b.len.view(np.int16)).to(dev)
    rec = torch.zeros((b.n, 16), dtype=torch.uint8, device=dev)
    mp = torch.zeros(1 << 14, dtype=torch.int32, device=dev)
    mq = torch.zeros(1 << 14, dtype=torch.int16, device=dev)
    mc = torch.zeros(1, dtype=torch.int32, device=dev)
    ch.process_tensors(arena, off, ln, rec, mp, mq, mc)
    with pytest.raises(nfc.NfcError) as e:
        ch.stats(allreduce=True)
    assert e.value.code == nfc.NFC_ESTATE
    comm = nfc.Comm(0, 1, 0, nfc.comm_unique_id())
    ch.attach_comm(comm)
    local = ch.stats()
    red = ch.stats(allreduce=True, reset=True)
    assert np.array_equal(local, red) and local[0] == b.n
    assert ch.stats().sum() == 0
    orc = oracle.OracleChain(w.kinds, w.tables)
    orc.run(b)
    for i in range(len(red)):
        if i not in (11, 12):
            assert red[i] == orc.stats[i], i
    ch.attach_comm(None)
    comm.close()
