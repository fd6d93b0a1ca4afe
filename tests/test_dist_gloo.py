"""Multi-process (gloo, world_size 2, CPU) tests of the multi-GPU host logic:
RSS sharding keeps every ESP SA on one rank and preserves per-SA order, so the
union of the per-rank results equals the single-process run packet for packet;
the counter all-reduce equals the single-process stats; timings take the max.
The per-rank packet compute here is the oracle (CPU test infrastructure); on
GPUs the same plumbing drives nfc_rss_shard + one chain per GPU."""
import os
import socket

import numpy as np
import pytest

import nfcgen
import oracle
from paper_conf_hpca_hul18_b200 import dist as pdist


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _tuple_hash(frame: bytes) -> int:
    """Toeplitz(MS key) over src|dst|sport|dport of a parsed IPv4/IPv6 UDP frame."""
    if frame[12:14] == b"\x86\xdd":
        t = frame[22:54] + frame[54:58]
    else:
        t = frame[26:34] + frame[34:38]
    return oracle.toeplitz(oracle.MS_RSS_KEY, t)


def _worker(rank, world, port, wl_name, n, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        w = nfcgen.workload(wl_name, small=True)
        b = nfcgen.generate(w.traffic, w.tables, 0, n)
        h = np.array([_tuple_hash(b.frame(i)) for i in range(n)])
        shard = pdist.shard_of_hash(h, world)
        idx = pdist.shard_indices(shard, rank)
        orc = oracle.OracleChain(w.kinds, w.tables)
        sub = nfcgen.Batch(b.arena.copy(), b.off[idx], b.len[idx], 0, b.headroom, b.tailroom)
        res, arena, _, _ = orc.run(sub)
        stats = pdist.allreduce_stats(orc.stats)
        tmax = pdist.max_over_ranks(float(rank + 1))
        outs = [None] * world
        frames = [arena[int(o) - (16 if r["esp_sa"] != 0xFF else 0):][:int(r["out_len"])].tobytes()
                  for o, r in zip(sub.off, res)]
        dist.all_gather_object(outs, (idx, res, frames))
        if rank == 0:
            q.put((stats, tmax, outs))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("wl", ["C2", "C5"])
def test_rss_sharded_equals_single(wl):
    import torch.multiprocessing as mp
    n, world = 700, 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, wl, n, q)) for r in range(world)]
    for p in procs:
        p.start()
    stats, tmax, outs = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    w = nfcgen.workload(wl, small=True)
    b = nfcgen.generate(w.traffic, w.tables, 0, n)
    orc = oracle.OracleChain(w.kinds, w.tables)
    want, want_arena, _, _ = orc.run(b)
    got = pdist.merge_by_index([(o[0], o[1]) for o in outs], n, nfcgen.RESULT)
    assert np.array_equal(got.view(np.uint8), want.view(np.uint8))   # incl. per-SA ESP seq
    assert np.array_equal(stats, orc.stats)
    assert tmax == 2.0
    for idx, res, frames in outs:
        for i, r, fr in zip(idx, res, frames):
            if r["drop_nf"] == 0xFF:
                s = int(b.off[i]) - (16 if r["esp_sa"] != 0xFF else 0)
                assert fr == want_arena[s:s + int(r["out_len"])].tobytes()


def test_reta_and_sa_locality():
    # n_shards | 64: SA = h mod 64 determines the shard, so each SA lives on one GPU
    h = np.arange(1 << 14) * 2654435761 % (1 << 32)
    for n in (1, 2, 4, 8):
        sh = pdist.shard_of_hash(h, n)
        sa = h % 64
        for s in range(64):
            assert len(set(sh[sa == s].tolist())) == 1
    with pytest.raises(ValueError):
        pdist.reta(0)


def test_merge_by_index_checks_partition():
    a = (np.array([0, 2]), np.zeros(2, dtype=nfcgen.RESULT))
    b = (np.array([1]), np.zeros(1, dtype=nfcgen.RESULT))
    pdist.merge_by_index([a, b], 3, nfcgen.RESULT)
    with pytest.raises(ValueError):
        pdist.merge_by_index([a], 3, nfcgen.RESULT)
    with pytest.raises(ValueError):
        pdist.merge_by_index([a, a, b], 3, nfcgen.RESULT)


def _stream_worker(rank, world, port, n, q):
    """Stateful DPI sharded by the RSS hash: each rank sees whole flows (in order)."""
    import torch.distributed as dist
    from nfcgen.stream import stream_batch
    from oracle.stream_dpi import StreamDPI
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        rng = np.random.default_rng(6)
        blob, off, act = nfcgen.gen_patterns(rng, 30, lmin=2, lmax=8)
        pats = nfcgen.Tables(pat_blob=blob, pat_off=off, pat_action=act).patterns()
        outs = [None] * world
        orc = StreamDPI(pats, list(act))
        mine = []
        for call in range(2):   # two calls: flow state carried per rank
            sb = stream_batch(30 + call, n, 50, pats, plant_frac=0.3, first_index=call * n, flow_seed=3)
            frames = sb.frames()
            h = np.array([_tuple_hash(f) for f in frames])
            idx = pdist.shard_indices(pdist.shard_of_hash(h, world), rank)
            occ, nocc, drop = orc.process([frames[i] for i in idx])
            mine += [(call * n + int(idx[i]), j, e) for i, j, e in occ]
        dist.all_gather_object(outs, mine)
        if rank == 0:
            q.put(outs)
    finally:
        dist.destroy_process_group()


def test_stream_dpi_flow_sharded_equals_single():
    """NEXT-4 multi-GPU rule: sharding packets by the 5-tuple
    RSS hash keeps every flow's stream on one rank, so the union of the per-rank
    occurrences equals the single-process result -- no data-path collective."""
    import torch.multiprocessing as mp
    from nfcgen.stream import stream_batch
    from oracle.stream_dpi import StreamDPI
    n, world = 600, 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_stream_worker, args=(r, world, port, n, q)) for r in range(world)]
    for p in procs:
        p.start()
    outs = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    rng = np.random.default_rng(6)
    blob, off, act = nfcgen.gen_patterns(rng, 30, lmin=2, lmax=8)
    pats = nfcgen.Tables(pat_blob=blob, pat_off=off, pat_action=act).patterns()
    orc = StreamDPI(pats, list(act))
    want = []
    for call in range(2):
        sb = stream_batch(30 + call, n, 50, pats, plant_frac=0.3, first_index=call * n, flow_seed=3)
        occ, _, _ = orc.process(sb.frames(), call * n)
        want += occ
    assert all(len(o) > 0 for o in outs)
    assert sorted(outs[0] + outs[1]) == sorted(want)
