"""GPU parity of stateful cross-packet DPI (NEXT-4, R#32): nfc_dpi_stream_* through
the C ABI against oracle/stream_dpi.py on the same seeded S1 traffic.  Integer
work: the sorted occurrence list (packet, pattern, end offset), per-packet counts
and DROP verdicts must be identical."""
import numpy as np
import pytest

import nfcgen
from nfcgen.stream import StreamBatch, stream_batch
from oracle.stream_dpi import StreamDPI

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def nfc():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_hpca_hul18_b200 import build
    build.build()
    from paper_conf_hpca_hul18_b200 import nfc as m
    return m


def _pats(seed, n, lmin=2, lmax=8):
    rng = np.random.default_rng(seed)
    blob, off, act = nfcgen.gen_patterns(rng, n, lmin=lmin, lmax=lmax, drop_frac=0.1)
    return blob, off, act, nfcgen.Tables(pat_blob=blob, pat_off=off, pat_action=act).patterns()


def _gpu(ds, sb: StreamBatch, cap=1 << 20):
    import torch
    d = torch.device("cuda:0")
    arena = torch.from_numpy(sb.arena).to(d)
    off = torch.from_numpy(sb.off.astype(np.int64)).to(d)
    ln = torch.from_numpy(sb.len.view(np.int16)).to(d)
    n = len(sb.off)
    nocc = torch.full((n,), 0x7777, dtype=torch.int32, device=d)
    drop = torch.full((n,), 7, dtype=torch.uint8, device=d)
    op = torch.zeros(cap, dtype=torch.int32, device=d)
    oq = torch.zeros(cap, dtype=torch.int16, device=d)
    oe = torch.zeros(cap, dtype=torch.int16, device=d)
    cnt = torch.zeros(1, dtype=torch.int32, device=d)
    ds.process_tensors(arena, off, ln, nocc, drop, op, oq, oe, cnt, first_global_index=sb.first_index)
    torch.cuda.synchronize()
    k = int(cnt.item())
    m = min(k, cap)
    occ = sorted(zip(op[:m].cpu().numpy().view(np.uint32).tolist(), oq[:m].cpu().numpy().view(np.uint16).tolist(),
                     oe[:m].cpu().numpy().view(np.uint16).tolist()))
    return occ, nocc.cpu().numpy().tolist(), drop.cpu().numpy().tolist(), k


@pytest.mark.parametrize("smem", [1, 0])
def test_stream_parity_multi_call(nfc, smem, monkeypatch):
    """smem=1: the DFA staged in shared memory (k_walk<2>); 0: read through L1/L2 (k_walk<0>)."""
    if smem:
        monkeypatch.setenv("NFC_STREAM_SMEM", "1")
    blob, off, act, pats = _pats(1, 100)
    ds = nfc.DpiStream(blob, off, act, max_flows=4096)
    orc = StreamDPI(pats, list(act))
    first = 0
    total_cross = 0
    for call, n in enumerate([3000, 1, 2500, 4097]):
        sb = stream_batch(100 + call, n, 60, pats, len_choices=[64, 65, 128, 300, 1500], plant_frac=0.3,
                          first_index=first, flow_seed=42)
        want, wn, wd = orc.process(sb.frames(), first)
        got, gn, gd, k = _gpu(ds, sb)
        assert k == len(want)
        assert got == want
        assert gn == wn and gd == wd
        total_cross += sum(1 for i, j, e in want if e < len(pats[j]) - 1)
        first += n
    assert total_cross > 100
    assert ds.flows() == (orc.n_flows(), 0)
    # reset forgets every flow: the next call starts each stream afresh
    ds.reset()
    orc2 = StreamDPI(pats, list(act))
    sb = stream_batch(7, 2000, 60, pats, plant_frac=0.3, first_index=first, flow_seed=42)
    want, wn, wd = orc2.process(sb.frames(), first)
    got, gn, gd, _ = _gpu(ds, sb)
    assert got == want and gn == wn and gd == wd


def test_stream_parity_wide_dfa(nfc):
    """> 32768 DFA states: 32-bit transition entries."""
    blob, off, act, pats = _pats(2, 2600, lmin=12, lmax=16)
    ds = nfc.DpiStream(blob, off, act, max_flows=64)
    orc = StreamDPI(pats, list(act))
    sb = stream_batch(3, 400, 20, pats, len_choices=[64, 200], plant_frac=0.5)
    want, wn, wd = orc.process(sb.frames())
    got, gn, gd, _ = _gpu(ds, sb)
    assert len(want) > 20
    assert got == want and gn == wn and gd == wd


def _frame_batch(frames, first=0):
    offs, pos = [], 0
    for f in frames:
        offs.append(pos)
        pos += (len(f) + 15) // 16 * 16
    arena = np.zeros(pos + 16, dtype=np.uint8)
    for o, f in zip(offs, frames):
        arena[o:o + len(f)] = np.frombuffer(f, dtype=np.uint8)
    return StreamBatch(arena, np.array(offs, dtype=np.uint64), np.array([len(f) for f in frames], dtype=np.uint16),
                       first)


def test_stream_edge_frames(nfc):
    """IPv6, fragments, TCP options, non-parsing frames, empty payloads, capacity overflow."""
    from tests.test_oracle_stream import _udp
    pats = [b"ab", b"abc", b"b", b"cab"]
    act = [0, 1, 0, 0]
    blob = np.frombuffer(b"".join(pats), dtype=np.uint8)
    off = np.cumsum([0] + [len(p) for p in pats]).astype(np.uint32)

    def v6(payload, sport=5):
        l4 = sport.to_bytes(2, "big") + b"\x00\x35" + (8 + len(payload)).to_bytes(2, "big") + b"\0\0"
        ip = bytes([0x60, 0, 0, 0]) + (8 + len(payload)).to_bytes(2, "big") + bytes([17, 64]) + \
            bytes(range(16)) + bytes(range(16, 32))
        return bytes(12) + b"\x86\xdd" + ip + l4 + payload

    frames = [_udp(b"xxa"), v6(b"ca"), _udp(b"bcab"), v6(b"b"), _udp(b"", sport=9), _udp(b"ab", frag=0x2001),
              _udp(b"b", frag=0x2001), b"\x00" * 20, _udp(b"a", proto=6), _udp(b"bc", proto=6), v6(b"ab" * 40)]
    sb = _frame_batch(frames, first=5)
    ds = nfc.DpiStream(blob, off, np.array(act, dtype=np.uint8), max_flows=16)
    want, wn, wd = StreamDPI(pats, act).process(sb.frames(), 5)
    got, gn, gd, k = _gpu(ds, sb)
    assert got == want and gn == wn and gd == wd
    # occurrence capacity: counted, first `cap` written
    ds.reset()
    got, gn, gd, k = _gpu(ds, sb, cap=3)
    assert k == len(want) and len(got) == 3 and set(got) <= set(want) and gn == wn
    # flow table full: max_flows = 1 flow placed, packets of other flows not inspected
    small = nfc.DpiStream(blob, off, np.array(act, dtype=np.uint8), max_flows=1)
    got, gn, gd, k = _gpu(small, sb)
    nf, nu = small.flows()
    assert nf == 1 and nu > 0


def test_stream_fullsize_sampled_flows(nfc):
    """2^21 64-B packets over 64 K flows in one call (bench shape); the oracle checks
    every packet of 300 sampled flows (flows are independent streams, so the
    sample is exact), and the occurrence total is checked against the count sum."""
    n, nflows = 1 << 21, 65536
    blob, off, act, pats = _pats(4, 100, lmin=4, lmax=16)
    rng = np.random.default_rng(8)
    flow_of = rng.integers(0, nflows, n)
    sb = stream_batch(9, n, nflows, pats, plant_frac=0.05, flow_of=flow_of)
    ds = nfc.DpiStream(blob, off, act, max_flows=1 << 17)
    got, gn, gd, k = _gpu(ds, sb, cap=1 << 22)
    assert k == sum(gn) and len(got) == k
    assert ds.flows() == (len(np.unique(flow_of)), 0)
    sample = rng.choice(nflows, 300, replace=False)
    sel = np.nonzero(np.isin(flow_of, sample))[0]
    orc = StreamDPI(pats, list(act))
    frames = sb.frames_of(sel) if hasattr(sb, "frames_of") else \
        [sb.arena[int(sb.off[i]):int(sb.off[i]) + int(sb.len[i])].tobytes() for i in sel]
    want, wn, wd = orc.process(frames)
    want = sorted((int(sel[i]), j, e) for i, j, e in want)
    selset = set(sel.tolist())
    assert [o for o in got if o[0] in selset] == want
    assert [gn[i] for i in sel] == wn and [gd[i] for i in sel] == wd
    assert sum(1 for i, j, e in want if e < len(pats[j]) - 1) > 10


REGEXES = [b"[a-f][0-9]", b"(ab|cd)[^a-z]", b"\\.[A-Z]{2}", b"q.{3,5}z", b"[0-4]{3}", b"(x|y)?[kK]{2}",
           b"\\x41\\x42?C", b"G(o|oo|ooo)gle"]
EXAMPLES = [b"a7", b"cdX", b".QZ", b"q1234z", b"012", b"ykK", b"AC", b"Gooogle"]


@pytest.mark.parametrize("calls", [[300, 1, 300]])
def test_regex_stream_parity(nfc, calls):
    """Regex DFA (host subset construction) walked by the stream kernels vs Python re."""
    from oracle.stream_dpi import StreamRegexDPI
    blob = np.frombuffer(b"".join(REGEXES), dtype=np.uint8).copy()
    off = np.cumsum([0] + [len(r) for r in REGEXES]).astype(np.uint32)
    act = np.array([0, 0, 1, 0, 0, 0, 1, 0], dtype=np.uint8)
    ds = nfc.DpiStream(blob, off, act, max_flows=256, regex=True)
    orc = StreamRegexDPI(REGEXES, list(act))
    first = 0
    for c, n in enumerate(calls):
        sb = stream_batch(200 + c, n, 40, EXAMPLES, len_choices=[64, 96, 160], plant_frac=0.4,
                          first_index=first, flow_seed=77)
        want, wn, wd = orc.process(sb.frames(), first)
        got, gn, gd, k = _gpu(ds, sb)
        assert k == len(want) and got == want
        assert gn == wn and gd == wd
        first += n
    assert len(want) > 50


def test_stream_long_empty_payload_runs(nfc):
    """runs of zero-payload packets in one flow (the ACK direction of a bulk
    transfer) -- exact results and no quadratic warm-up walk-back: 60 K empty packets
    of one flow between payload-carrying ones take about as long as 60 K packets of
    60 K flows."""
    import time
    import torch
    from tests.test_oracle_stream import _udp
    pats = [b"abcdefgh", b"hab", b"zz"]
    act = [0, 1, 0]
    blob = np.frombuffer(b"".join(pats), dtype=np.uint8)
    off = np.cumsum([0] + [len(p) for p in pats]).astype(np.uint32)
    rng = np.random.default_rng(3)
    frames = []
    for k in range(60000):
        if k % 20000 == 0:
            frames.append(_udp(b"xyzabcd"))
        elif k % 20000 == 1:
            frames.append(_udp(b"efgh" + bytes(rng.integers(97, 123, 5))))
        else:
            frames.append(_udp(b""))
    frames.append(_udp(b"ab"))
    sb = _frame_batch(frames, first=3)
    ds = nfc.DpiStream(blob, off, np.array(act, dtype=np.uint8), max_flows=16)
    want, wn, wd = StreamDPI(pats, act).process(sb.frames(), 3)
    got, gn, gd, k = _gpu(ds, sb)
    assert got == want and gn == wn and gd == wd
    # timing against the same packet count spread over distinct flows
    spread = _frame_batch([_udp(b"", sport=1000 + (j % 60000), src=0x0B000000 + j) for j in range(len(frames))])
    ds2 = nfc.DpiStream(blob, off, np.array(act, dtype=np.uint8), max_flows=1 << 17)
    ts = []
    for dsx, sbx in ((ds, sb), (ds2, spread)):
        dsx.reset()
        _gpu(dsx, sbx)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(3):
            _gpu(dsx, sbx)
        torch.cuda.synchronize()
        ts.append(time.perf_counter() - t0)
    assert ts[0] < 3 * ts[1] + 0.05, ts


def test_stream_rss_sharded_equals_single(nfc):
    """the multi-GPU stateful path as N GPUs run it -- frames steered by
    nfc_rss_shard, one DpiStream (own flow table) per shard, several calls -- equals the
    single-stream oracle, with fragments, IPv4 options and TCP options in the traffic
    (a fragment's flow key has ports 0, so all fragments of a (src, dst, proto) share a
    flow and a shard)."""
    import torch
    from oracle.stream_dpi import StreamDPI as SD
    from paper_conf_hpca_hul18_b200 import dist as pdist
    blob, off, act, pats = _pats(5, 40, lmin=2, lmax=6)
    w = nfcgen.workload("C1", small=True)
    w.traffic.n_flows, w.traffic.tcp_pct, w.traffic.pkt_len = 300, 40, 1
    w.traffic.edge(150_000)
    w.traffic.match_ppm = 0
    d = torch.device("cuda:0")
    want_all, got_all = [], {}
    orc = SD(pats, list(act))
    for N in (2, 4):
        got_all[N] = []
        streams = [nfc.DpiStream(blob, off, act, max_flows=1024) for _ in range(N)]
        for call in range(3):
            b = nfcgen.generate(w.traffic, w.tables, 2000 * call, 2000)
            if N == 2:
                occ, _, _ = orc.process([b.frame(i) for i in range(b.n)], 2000 * call)
                want_all += occ
            arena = torch.from_numpy(b.arena).to(d)
            o_t = torch.from_numpy(b.off.view(np.int64)).to(d)
            l_t = torch.from_numpy(b.len.view(np.int16)).to(d)
            sh = torch.zeros(b.n, dtype=torch.uint8, device=d)
            nfc.rss_shard(0, arena.data_ptr(), o_t.data_ptr(), l_t.data_ptr(), b.n, N, sh.data_ptr())
            torch.cuda.synchronize()
            shn = sh.cpu().numpy()
            for r in range(N):
                idx = pdist.shard_indices(shn, r)
                if not len(idx):
                    continue
                sub = StreamBatch(b.arena, b.off[idx], b.len[idx], 0)
                occ, _, _, _ = _gpu(streams[r], sub)
                got_all[N] += [(int(2000 * call + idx[p]), q, e) for p, q, e in occ]
    assert len(want_all) > 100
    for N in (2, 4):
        assert sorted(got_all[N]) == sorted(want_all), N


UNB_REGEXES = [b"ab+c", b"x[0-9]*y", b"(GET|POST) /[a-z]+\\?", b"k{3,}!", b"<[a-z]+>", b"(ab|cd)*ef", b"Q.{2,}Z"]
UNB_EXAMPLES = [b"abbbbbbc", b"x0123456789y", b"GET /index?", b"kkkkk!", b"<script>", b"abcdabef", b"Qhello worldZ"]


@pytest.mark.parametrize("calls", [[250, 1, 250]])
def test_regex_unbounded_stream_parity(nfc, calls):
    """NEXT-4: regexes with '*', '+' and {m,} (unbounded matches, walked flow-serially
    from the carried state: no bounded re-walk reconstructs the start) vs Python re,
    with occurrences spanning packets and calls."""
    from oracle.stream_dpi import StreamRegexDPI
    blob = np.frombuffer(b"".join(UNB_REGEXES), dtype=np.uint8).copy()
    off = np.cumsum([0] + [len(r) for r in UNB_REGEXES]).astype(np.uint32)
    act = np.array([0, 1, 0, 0, 1, 0, 0], dtype=np.uint8)
    ds = nfc.DpiStream(blob, off, act, max_flows=128, regex=True)
    orc = StreamRegexDPI(UNB_REGEXES, list(act))
    first, total = 0, 0
    for c, n in enumerate(calls):
        sb = stream_batch(300 + c, n, 25, UNB_EXAMPLES, len_choices=[64, 96], plant_frac=0.4,
                          first_index=first, flow_seed=78)
        want, wn, wd = orc.process(sb.frames(), first)
        got, gn, gd, k = _gpu(ds, sb)
        assert k == len(want) and got == want
        assert gn == wn and gd == wd
        first += n
        total += len(want)
    assert total > 30
