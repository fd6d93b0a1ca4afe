#!/usr/bin/env python
"""bench.py -- throughput of the fused B200 SFC kernel (BASELINE.json metric).

A step is one nfc_process_batch call (one persistent kernel launch) over a
ring of synthetic packets resident in HBM that is much larger than the 126 MB
L2.  Default workload: BASELINE config C1's chain ACL(64)->DPI(100)->LPM4(1K)
on 64-B packets -- the DPI+LPM chain the north-star's HBM-roofline target is
stated on.  Other configs: --config C2..C5.

    python bench.py [--gpus N --steps K --warmup W] [--config C1] [--impl reference]

Multi-GPU: one process per GPU (torchrun), flows sharded across ranks, no
data-path collective (weak scaling); the per-rank counters are summed with
one NCCL all-reduce after the timed region.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = json.load(open(os.path.join(ROOT, "BASELINE.json")))["metric"]
RESTORE_KINDS = {"IPSEC"}    # chains whose in-place rewrite changes the next step's work
BATCH = 4096                  # one batch (C1: "one batch of 4,096 synthetic 64-B packets")


def parse_args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C1")
    ap.add_argument("--pkt-len", type=int, default=None, help="frame length (0 = IMIX)")
    ap.add_argument("--k", type=int, default=None, help="C5 chain length")
    ap.add_argument("--acl-rules", type=int, default=None, help="N3 (NEXT-3) ACL size: 200 / 1000 / 10000")
    ap.add_argument("--match-ppm", type=int, default=None, help="planted DPI matches per million packets (experiments)")
    ap.add_argument("--v6-bp", type=int, default=None, help="IPv6 share in basis points (experiments)")
    ap.add_argument("--ring-mb", type=int, default=1024, help="HBM ring size per GPU (>> 126 MB L2)")
    ap.add_argument("--batch-pkts", type=int, default=BATCH,
                    help="packets per nfc_batch descriptor (SURVEY 8(c)(ii)#4: 4,096); 0 = the ring as one batch")
    ap.add_argument("--cpu-seconds", type=float, default=10.0, help="oracle baseline budget")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-unfused", action="store_true", help="skip the NEXT-1 unfused baseline timing")
    ap.add_argument("--unfused", action="store_true", help="time the unfused baseline as the main arm")
    return ap.parse_args()


# ------------------------------------------------------------------ workload
def make_workload(args):
    import nfcgen
    w = nfcgen.workload(args.config, pkt_len=args.pkt_len, k=args.k, acl_rules=getattr(args, "acl_rules", None))
    w.traffic.ttl = 255  # steps re-process the same ring: keep TTL/hop limit from expiring
    if getattr(args, "match_ppm", None) is not None:
        w.traffic.match_ppm = args.match_ppm
    if getattr(args, "v6_bp", None) is not None:
        w.traffic.v6_bp = args.v6_bp
    return w


def ring_packets(w, ring_mb):
    import nfcgen
    probe = nfcgen.generate(w.traffic, w.tables, 0, 4096)
    slot = (len(probe.arena) - 64) / 4096.0
    n = int(ring_mb * (1 << 20) / slot)
    return max(4096, (n // 4096) * 4096)


def prepare_ring(w, ring_mb, rank, world, local_dev, stream):
    """This rank's packets, resident in HBM: its RSS shard (nfc_rss_shard, the P:L87 Receive
    Side Steering model: Toeplitz(MS key, 5-tuple) -> RETA) of the global packet stream, in
    global order, written on the device by the traffic generator (nfcgen.device) one window
    of the global stream at a time and packed into a dense ring.  World 1: the stream itself.
    Returns (arena u8, off i64, len i16) device tensors and the packet count."""
    import torch

    from nfcgen import device as gd
    from paper_conf_hpca_hul18_b200 import nfc
    dev = torch.device("cuda", local_dev)
    n = ring_packets(w, ring_mb)
    dtab = gd.DeviceTables(w.traffic, w.tables, dev)
    if world == 1:
        a, o, l_ = gd.generate(w.traffic, w.tables, 0, n, device=dev, dtab=dtab)
        return a, o, l_, n
    hr, tr = w.traffic.headroom, w.traffic.tailroom
    pieces, have, s0 = [], 0, 0
    shard = torch.empty(n, dtype=torch.uint8, device=dev)
    while have < n:
        a, o, l_ = gd.generate(w.traffic, w.tables, s0, n, device=dev, dtab=dtab)
        nfc.rss_shard(local_dev, a.data_ptr(), o.data_ptr(), l_.data_ptr(), n, world, shard.data_ptr(),
                      stream.cuda_stream)
        idx = torch.nonzero(shard == rank).flatten()[: n - have]
        pieces.append(gd.gather(a, o, l_, idx, hr, tr))
        have += int(idx.numel())
        s0 += n
        del a, o, l_
    base, arenas, offs = 0, [], []
    for a, o, _ in pieces:
        arenas.append(a[:-64])
        offs.append(o + base)
        base += a.numel() - 64
    arenas.append(torch.zeros(64, dtype=torch.uint8, device=dev))
    return torch.cat(arenas), torch.cat(offs), torch.cat([p_[2] for p_ in pieces]), n


def host_view(arena, off, ln, first, w):
    """nfcgen.Batch view (host copies) of a device ring, for the byte accounting and the e2e leg."""
    import nfcgen
    return nfcgen.Batch(arena.cpu().numpy(), off.cpu().numpy().view(np.uint64), ln.cpu().numpy().view(np.uint16),
                        first, w.traffic.headroom, w.traffic.tailroom)


def batch_descs(arena, off, ln, n, first, bp):
    """nfc_batch descriptors: the ring cut into batches of bp packets (bp = 0: one batch)."""
    bp = bp or n
    return [(arena.data_ptr(), off.data_ptr() + 8 * s_, ln.data_ptr() + 2 * s_, min(bp, n - s_), first + s_)
            for s_ in range(0, n, bp)]


def alg_bytes_per_step(kinds, lens, fam, rec):
    """Algorithmic HBM bytes of one pass: per packet the header bytes
    min(len, 64) [+ the rest of the frame if a payload NF (DPI/IPSEC) is reached in
    original order] + 16 B record + 32 B header sector if a forwarder rewrote it + the
    ESP output frame if IPsec ran (descriptors and match pairs: other_bytes_per_step)."""
    lens = lens.astype(np.int64)
    n = len(lens)
    drop = rec["drop_nf"].astype(np.int64)
    parsed = drop != 0xFE

    def reached(p):
        return parsed & ((drop == 0xFF) | (drop >= p))

    def passed(p):
        return parsed & ((drop == 0xFF) | (drop > p))

    payload = np.zeros(n, dtype=bool)
    rewritten = np.zeros(n, dtype=bool)
    for p, k in enumerate(kinds):
        if k in ("DPI", "IPSEC"):
            payload |= reached(p)
        if k == "LPM4":
            rewritten |= passed(p) & (fam == 4)
        if k == "LPM6":
            rewritten |= passed(p) & (fam == 6)
        if k == "NAT":      # address/port/checksum sector [32, 64) of IPv4 packets past the NAT
            natw = passed(p) & (fam == 4)
    rd = int(np.where(payload, lens, np.minimum(lens, 64)).sum())
    wr = 16 * n + 32 * int(rewritten.sum())
    if "NAT" in kinds:
        wr += 32 * int(natw.sum())
    esp = rec["esp_sa"] != 0xFF
    wr += int(rec["out_len"][esp].astype(np.int64).sum())
    return rd + wr, rd, wr


def other_bytes_per_step(n, rec):
    """Bytes the kernel also moves that SURVEY 8(d)'s per-packet count leaves out: the
    descriptors (off u64 + len u16 = 10 B per packet) and the match pairs (6 B each)."""
    return 10 * n + 6 * int(rec["dpi_nmatch"].astype(np.int64).sum())


# Algorithmic integer work of IPsec ESP: a textbook
# T-table AES-128 block (10 rounds x 16 lookups, each byte-extract + lookup + xor,
# plus key additions) and a SHA-1 compression (80 rounds of rotate/boolean/4 adds,
# 64 message-schedule words of 3 xors + rotate), counted as 32-bit integer ops.
AES_BLOCK_OPS = 560
SHA1_BLOCK_OPS = 816


def esp_alg_ops(rec, l4_off):
    """Integer ops of the ESP packets of one pass: AES-CTR blocks over the ciphertext,
    HMAC-SHA1 = inner hash (ipad state precomputed) over ESP hdr+IV+C, outer hash 1 block."""
    esp = rec["esp_sa"] != 0xFF
    if not esp.any():
        return 0
    out_len = rec["out_len"][esp].astype(np.int64)
    l4 = l4_off[esp].astype(np.int64)
    clen = out_len - 12 - (l4 + 16)            # ciphertext = payload + trailer
    aes = (clen + 15) // 16
    msg = 16 + clen                             # ESP header + IV + ciphertext
    sha = (msg + 9 + 63) // 64 + 1
    return int((aes * AES_BLOCK_OPS + sha * SHA1_BLOCK_OPS).sum())


def l4_offsets(b):
    o = b.off.astype(np.int64)
    fam = frame_family(b)
    ihl = (b.arena[o + 14] & 15).astype(np.int64)
    return np.where(fam == 6, 54, 14 + 4 * ihl)


def frame_family(b):
    et = b.arena[b.off.astype(np.int64) + 12].astype(np.int64) << 8 | b.arena[b.off.astype(np.int64) + 13]
    return np.where(et == 0x86DD, 6, np.where(et == 0x0800, 4, 0))


# ------------------------------------------------------------------ clocks
class ClockSampler:
    REASONS = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x2: "applications_clocks",
               0x10: "sync_boost"}

    def __init__(self, torch_dev: int):
        self.samples, self.reasons, self.ok = [], set(), False
        self.max_mhz = None
        try:
            import pynvml
            pynvml.nvmlInit()
            import torch
            pr = torch.cuda.get_device_properties(torch_dev)
            h = None
            try:
                bus = f"{pr.pci_domain_id:08x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
                h = pynvml.nvmlDeviceGetHandleByPciBusId(bus)
            except Exception:
                h = pynvml.nvmlDeviceGetHandleByIndex(torch_dev)
            self.h, self.nv = h, pynvml
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # noqa: BLE001
            self.err = repr(e)
        self._stop = threading.Event()

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.005)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.ok:
            self.t.join()

    def summary(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "note": getattr(self, "err", "")}
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ------------------------------------------------------------------ oracle baseline
def oracle_rate(w, first, budget_s, chunk=8192, max_chunks=100000):
    """Plain C oracle, single-threaded, on consecutive chunks of the same workload."""
    import nfcgen
    import oracle
    orc = oracle.OracleChain(w.kinds, w.tables)
    t_work, pk, by = 0.0, 0, 0
    i = 0
    while t_work < budget_s and i < max_chunks:
        b = nfcgen.generate(w.traffic, w.tables, first + pk, chunk)
        t0 = time.perf_counter()
        orc.run(b, match_cap=1 << 20)
        t_work += time.perf_counter() - t0
        pk += b.n
        by += int(b.len.astype(np.int64).sum())
        i += 1
    return pk / t_work / 1e6, by * 8 / t_work / 1e9, pk, t_work


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


_ALLCORE = {}


def _allcore_worker(p):
    """One single-threaded oracle process on its RSS shard of the sample (timed alone)."""
    import oracle
    w, b, shard = _ALLCORE["w"], _ALLCORE["b"], _ALLCORE["shard"]
    import nfcgen
    idx = np.nonzero(shard == p)[0]
    sub = nfcgen.Batch(b.arena.copy(), b.off[idx], b.len[idx], 0, b.headroom, b.tailroom)
    orc = oracle.OracleChain(w.kinds, w.tables)
    t0 = time.perf_counter()
    orc.run(sub, match_cap=1 << 22)
    return len(idx), int(b.len[idx].astype(np.int64).sum()), time.perf_counter() - t0


def oracle_all_cores(w, local_dev, rate_1core_mpps, budget_s):
    """All host cores: nproc independent single-threaded oracle processes, each on the RSS
    shard it would own: the sample's shard ids come from nfc_rss_shard with
    n_shards = nproc; a sample sized for ~budget_s of work per process."""
    import multiprocessing as mp

    import torch

    import nfcgen
    from paper_conf_hpca_hul18_b200 import nfc
    ncores = os.cpu_count() or 1
    n = int(max(4096, min(8_000_000, rate_1core_mpps * 1e6 * budget_s * ncores)))
    b = nfcgen.generate(w.traffic, w.tables, 1 << 40, n)
    dev = torch.device("cuda", local_dev)
    a_d = torch.from_numpy(b.arena).to(dev)
    o_d = torch.from_numpy(b.off.view(np.int64)).to(dev)
    l_d = torch.from_numpy(b.len.view(np.int16)).to(dev)
    sh = torch.empty(n, dtype=torch.uint8, device=dev)
    nfc.rss_shard(local_dev, a_d.data_ptr(), o_d.data_ptr(), l_d.data_ptr(), n, min(ncores, 128), sh.data_ptr(),
                  torch.cuda.current_stream(dev).cuda_stream)
    shard = sh.cpu().numpy()
    del a_d, o_d, l_d
    _ALLCORE.update(w=w, b=b, shard=shard)
    ctx = mp.get_context("fork")
    with ctx.Pool(ncores) as pool:
        t0 = time.perf_counter()
        res = pool.map(_allcore_worker, range(min(ncores, 128)))
        wall = time.perf_counter() - t0
    _ALLCORE.clear()
    pk = sum(r[0] for r in res)
    by = sum(r[1] for r in res)
    return {"value": round(pk / wall / 1e6, 6), "unit": "Mpps", "cores": ncores, "kind": "oracle",
            "gbps": round(by * 8 / wall / 1e9, 6),
            "sample": f"{pk} packets of {w.name}, {ncores} processes of the single-threaded oracle, each on its "
                      f"RSS shard (nfc_rss_shard, n_shards = nproc); wall {wall:.1f} s, slowest shard "
                      f"{max(r[2] for r in res):.1f} s"}


def pcie_peaks(torch, dev, nbytes, reps=3):
    """Measured pinned-host <-> HBM copy rates (GB/s) on this box: H2D alone, D2H alone,
    and both directions at once on two streams (the full-duplex bound the pipelined
    nfc_process_host can reach).  The denominator of the e2e roofline."""
    nbytes = int(min(nbytes, 1 << 30))
    hs = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    hd = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d1 = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    d2 = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    s1, s2 = torch.cuda.Stream(dev), torch.cuda.Stream(dev)

    def timed(h2d, d2h):
        best = float("inf")
        for _ in range(reps):
            torch.cuda.synchronize(dev)
            t0 = time.perf_counter()
            if h2d:
                with torch.cuda.stream(s1):
                    d1.copy_(hs, non_blocking=True)
            if d2h:
                with torch.cuda.stream(s2):
                    hd.copy_(d2, non_blocking=True)
            torch.cuda.synchronize(dev)
            best = min(best, time.perf_counter() - t0)
        return best

    th, td, tb = timed(True, False), timed(False, True), timed(True, True)
    del hs, hd, d1, d2
    return {"h2d_gbs": round(nbytes / th / 1e9, 1), "d2h_gbs": round(nbytes / td / 1e9, 1),
            "duplex_each_gbs": round(nbytes / tb / 1e9, 1), "bytes": nbytes,
            "method": "torch pinned copies, best of %d; duplex = both directions on two streams" % reps}


def payload_bytes(b):
    """Payload bytes [pl_off, ip_end) per packet by a vectorised read of the headers
    (bench accounting only: the DPI work per packet; 0 if not parsed)."""
    o = b.off.astype(np.int64)
    A = b.arena
    L = b.len.astype(np.int64)
    et = A[o + 12].astype(np.int64) << 8 | A[o + 13]
    v4, v6 = et == 0x0800, et == 0x86DD
    ihl = (A[o + 14] & 15).astype(np.int64)
    l4 = np.where(v6, 54, 14 + 4 * ihl)
    ip_end = np.where(v6, 54 + (A[o + 18].astype(np.int64) << 8 | A[o + 19]),
                      14 + (A[o + 16].astype(np.int64) << 8 | A[o + 17]))
    proto = np.where(v6, A[o + 20], A[o + 23]).astype(np.int64)
    frag = v4 & (((A[o + 20].astype(np.int64) << 8 | A[o + 21]) & 0x3FFF) != 0)
    lim = np.minimum(o + np.minimum(l4 + 12, L - 1), len(A) - 1)
    doff = (A[lim] >> 4).astype(np.int64)
    hl = np.where(frag, 0, np.where(proto == 17, 8, np.where(proto == 6, 4 * doff, 0)))
    pl = l4 + hl
    ver = (A[o + 14] >> 4).astype(np.int64)
    ok = (v4 & (ver == 4) & (ihl >= 5) & (L >= 34) & (ip_end - 14 >= 4 * ihl)) | (v6 & (ver == 6) & (L >= 54))
    ok &= (ip_end <= L) & (pl <= ip_end) & ~(~frag & (proto == 6) & ((doff < 5) | (l4 + 20 > ip_end)))
    return np.where(ok, ip_end - pl, 0)


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    w = make_workload(args)
    # calibrate a per-step sample of ~1 s of oracle work
    rate, _, _, _ = oracle_rate(w, 0, 0.5, chunk=2048, max_chunks=50)
    per_step = max(2048, int(rate * 1e6 * 1.0) // 2048 * 2048)
    ts, pk, by = [], 0, 0
    import nfcgen
    import oracle
    orc = oracle.OracleChain(w.kinds, w.tables)
    for s in range(args.warmup + args.steps):
        b = nfcgen.generate(w.traffic, w.tables, s * per_step, per_step)
        t0 = time.perf_counter()
        orc.run(b, match_cap=1 << 20)
        dt = time.perf_counter() - t0
        if s >= args.warmup:
            ts.append(dt)
            pk += b.n
            by += int(b.len.astype(np.int64).sum())
    tot = sum(ts)
    mpps = pk / tot / 1e6
    sample = f"{args.steps} steps x {per_step} packets of {w.name} (same generator/tables), 1 thread"
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": round(mpps, 6), "unit": "Mpps",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(tot / args.steps * 1e3, 3), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "gbps": round(by * 8 / tot / 1e9, 6),
        "config": {"workload": f"{w.name}: {w.note}", "chain": w.kinds, "packets_per_step": per_step},
        "cpu_baseline": {"value": round(mpps, 6), "unit": "Mpps", "cores": 1, "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": round(mpps, 6), "unit": "Mpps", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }))


# ------------------------------------------------------------------ our arm
# ------------------------------------------------------------------ NEXT-4: stateful DPI
def run_stream(args):
    """--config S1: stateful cross-packet DPI (nfc_dpi_stream_process, NEXT-4, R#32) over a
    ring of 64-B IPv4 frames of 64 K flows resident in HBM; a step = one call over the
    whole ring (flow state carries from step to step, as a continuing stream)."""
    import torch
    import torch.distributed as dist

    import nfcgen
    from nfcgen.stream import stream_batch
    from paper_conf_hpca_hul18_b200 import nfc

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    local_dev = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local_dev)
    dev = torch.device("cuda", local_dev)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    pkt_len = args.pkt_len or 64
    n = (args.ring_mb << 20) // ((pkt_len + 15) // 16 * 16)
    n_flows = 65536
    regex = args.config == "S1R"
    if regex:   # S1R: regular expressions (R#33); plants are example words of each expression
        rx = [b"[a-f][0-9]{2}", b"(ab|cd)[^a-z]", b"\\.[A-Z]{2}", b"q.{3,5}z", b"[0-4]{4}", b"(x|y)?[kK]{3}",
              b"\\x41\\x42?C[0-9]", b"G(o|oo|ooo)gle", b"(GET|POST) /[a-z]{1,8}", b"[Uu]ser-[Aa]gent: [A-Z]",
              b"\\x90{4,8}", b"(cmd|exe)\\.[a-z]{3}", b"id=[0-9]{4,6}&", b"<scr(i|1)pt", b"%[0-9A-F]{2}%",
              b"pass(wd|word)="]
        ex = [b"a12", b"cdX", b".QZ", b"q1234z", b"0123", b"ykKk", b"AC7", b"Gooogle", b"GET /index",
              b"User-Agent: M", b"\x90\x90\x90\x90", b"cmd.exe", b"id=12345&", b"<scr1pt", b"%2F%", b"password="]
        blob = np.frombuffer(b"".join(rx), dtype=np.uint8).copy()
        poff = np.cumsum([0] + [len(r) for r in rx]).astype(np.uint32)
        act = np.array([0] * 13 + [1, 0, 1], dtype=np.uint8)
        pats, plants = rx, ex
    else:
        rng = np.random.default_rng(4)
        blob, poff, act = nfcgen.gen_patterns(rng, 100, lmin=4, lmax=16, drop_frac=0.05)
        pats = nfcgen.Tables(pat_blob=blob, pat_off=poff, pat_action=act).patterns()
        plants = pats
    sb = stream_batch(9 + rank, n, n_flows, plants, pkt_len=pkt_len, plant_frac=0.05, flow_seed=1000 + rank)
    ds = nfc.DpiStream(blob, poff, act, max_flows=2 * n_flows, device=local_dev, regex=regex)
    arena = torch.from_numpy(sb.arena).to(dev)
    off = torch.from_numpy(sb.off.astype(np.int64)).to(dev)
    ln = torch.from_numpy(sb.len.view(np.int16)).to(dev)
    nocc = torch.empty(n, dtype=torch.int32, device=dev)
    drop = torch.empty(n, dtype=torch.uint8, device=dev)
    cap = 1 << 22
    op = torch.empty(cap, dtype=torch.int32, device=dev)
    oq = torch.empty(cap, dtype=torch.int16, device=dev)
    oe = torch.empty(cap, dtype=torch.int16, device=dev)
    cnt = torch.zeros(1, dtype=torch.int32, device=dev)
    stream = torch.cuda.current_stream(dev)

    def step():
        cnt.zero_()
        ds.process_tensors(arena, off, ln, nocc, drop, op, oq, oe, cnt, first_global_index=rank * n, stream=stream)

    for _ in range(max(3, args.warmup)):
        step()
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local_dev) as clk:
        e0.record(stream)
        for _ in range(args.steps):
            step()
        e1.record(stream)
        torch.cuda.synchronize(dev)
    ms = e0.elapsed_time(e1)
    ms_t = torch.tensor([ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
    ms_max = float(ms_t.item())
    mpps = n * args.steps * world / (ms_max / 1e3) / 1e6
    n_occ = int(cnt.item())
    # algorithmic bytes per packet: the frame read once (64 B) + nocc (4) + drop (1) +
    # 6 B per occurrence written; the call is bound by dependent DFA steps
    alg = n * (pkt_len + 5) + n_occ * 8
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    peak = peaks.get("hbm_gbs", 6650.0)
    achieved = alg / (ms / args.steps / 1e3) / 1e9
    traffic = None
    tfile = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tfile) and not regex:
        tj = json.load(open(tfile)).get("S1")
        if tj and tj.get("packets"):
            traffic = int(tj["dram_bytes_per_launch"] * n / tj["packets"])
    roof = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
            "frac": round(achieved / peak, 4), "traffic": traffic, "alg_bytes_per_launch": alg,
            "alg_bytes_per_packet": round(alg / n, 2), "scope": "whole call (k_flow + radix sort + k_walk + k_commit)",
            "peak_source": "MEASURED_PEAKS.json hbm_gbs" if "hbm_gbs" in peaks else "B200_PROFILING fallback"}
    # end to end: pinned host frames -> device, the call, per-packet verdicts + occurrences back
    e2e = None
    if not args.no_e2e:
        h_arena = torch.from_numpy(sb.arena).pin_memory()
        h_off = torch.from_numpy(sb.off.astype(np.int64)).pin_memory()
        h_len = torch.from_numpy(sb.len.view(np.int16)).pin_memory()
        h_nocc = torch.empty(n, dtype=torch.int32, pin_memory=True)
        h_drop = torch.empty(n, dtype=torch.uint8, pin_memory=True)
        times, d2h = [], 0
        for s_ in range(4):
            torch.cuda.synchronize(dev)
            t0 = time.perf_counter()
            arena.copy_(h_arena, non_blocking=True)
            off.copy_(h_off, non_blocking=True)
            ln.copy_(h_len, non_blocking=True)
            step()
            h_nocc.copy_(nocc, non_blocking=True)
            h_drop.copy_(drop, non_blocking=True)
            torch.cuda.synchronize(dev)
            k = min(int(cnt.item()), cap)
            occ_h = (op[:k].cpu(), oq[:k].cpu(), oe[:k].cpu())
            dt = time.perf_counter() - t0
            d2h = n * 5 + 4 + k * 8
            if s_:
                times.append(dt)
        e2e = {"value": round(n * len(times) * world / sum(times) / 1e6, 3), "unit": "Mpps",
               "h2d_bytes_per_step": len(sb.arena) + n * 10, "d2h_bytes_per_step": d2h, "steps": len(times),
               "api": "DpiStream.process_tensors (nfc_dpi_stream_process) + pinned host copies"}
    cpu = None
    if not args.no_cpu and rank == 0 and world == 1:
        from oracle.stream_dpi import StreamDPI, StreamRegexDPI
        orc = StreamRegexDPI(pats, list(act)) if regex else StreamDPI(pats, list(act))
        ns = 6000 if regex else 60000
        frames = [sb.arena[int(o):int(o) + int(l)].tobytes() for o, l in zip(sb.off[:ns], sb.len[:ns])]
        t0 = time.perf_counter()
        orc.process(frames)
        t = time.perf_counter() - t0
        cpu = {"value": round(len(frames) / t / 1e6, 6), "unit": "Mpps", "cores": 1, "kind": "oracle",
               "sample": f"first {len(frames)} packets of {args.config} (brute-force Python stream oracle{' with re' if regex else ''}), {t:.1f} s, 1 thread"}
    if rank == 0:
        print(json.dumps({
            "metric": METRIC, "value": round(mpps, 3), "unit": "Mpps", "n_gpus": world, "steps": args.steps,
            "warmup": max(3, args.warmup), "ms_per_step": round(ms_max / args.steps, 4), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
            "gbps": round(n * pkt_len * 8 * args.steps * world / (ms_max / 1e3) / 1e9, 2),
            "config": {"workload": f"S1R: stateful cross-packet regex DPI (NEXT-4, R#33), {len(pats)} expressions, {pkt_len} B IPv4 "
                                   f"(30 % TCP), {n_flows} flows, 5 % cross-packet plants" if regex else
                                   f"S1: stateful cross-packet DPI (NEXT-4), 100 patterns, {pkt_len} B IPv4 "
                                   f"(30 % TCP), {n_flows} flows, 5 % cross-packet plants",
                       "packets_per_step_per_gpu": n, "ring_bytes_per_gpu": len(sb.arena),
                       "l2": "ring >> 126 MB L2 (no flush needed)",
                       "timing": "CUDA events on the launch stream; max over ranks",
                       "parallelism": f"flow-sharded x{world}, no data-path collective",
                       "occurrences_per_step": n_occ},
            "roofline": roof, "cpu_baseline": cpu, "e2e": e2e,
            "gpu_launches": 3 * args.steps, "gpu_launches_note": "k_flow + k_walk + k_commit per step (+ cub sort)",
            "clocks": clk.summary()}))
    if world > 1:
        dist.destroy_process_group()


def run_next2(args):
    """--config NX2_FW / NX2_IDS (Figs. 13-14): four identical
    NFs on 64-B TCP traffic, the paper's configurations on B200 -- (a) sequential: one kernel
    per NF (NFC_F_UNFUSED), (b) one parallel group of four (NFC_F_PARALLEL), (c) two parallel
    groups of two, (d) synthesized: the fused kernel -- throughput over the ring and the
    latency of one 4,096-packet batch (median of 30 launches)."""
    import torch

    from paper_conf_hpca_hul18_b200 import nfc
    local_dev = int(os.environ.get("LOCAL_RANK", "0")) % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local_dev)
    dev = torch.device("cuda", local_dev)
    w = make_workload(args)
    stream = torch.cuda.current_stream(dev)
    arena, off, ln, n = prepare_ring(w, args.ring_mb, 0, 1, local_dev, stream)
    rec = torch.empty((n, 16), dtype=torch.uint8, device=dev)
    cap = 1 << 22
    mp = torch.empty(cap, dtype=torch.int32, device=dev)
    mq = torch.empty(cap, dtype=torch.int16, device=dev)
    mc = torch.zeros(1, dtype=torch.int32, device=dev)
    descs = nfc.Chain.batch_array(batch_descs(arena, off, ln, n, 0, args.batch_pkts))
    one = nfc.Chain.batch_array([(arena.data_ptr(), off.data_ptr(), ln.data_ptr(), min(n, BATCH), 0)])
    cfgs = {"a_sequential": (nfc.F_UNFUSED, None), "b_parallel_1group": (nfc.F_PARALLEL, [0, 0, 0, 0]),
            "c_parallel_2groups": (nfc.F_PARALLEL, [0, 0, 1, 1]), "d_synthesized_fused": (0, None)}
    out, main = {}, None
    for name, (flags, groups) in cfgs.items():
        ch = nfc.Chain(w.kinds, device=local_dev, flags=flags)
        ch.load_tables(w.tables)
        if groups:
            ch.set_groups(groups)

        def step(d=descs):
            mc.zero_()
            ch.process(d, rec.data_ptr(), mp.data_ptr(), mq.data_ptr(), cap, mc.data_ptr(), stream.cuda_stream)
        for _ in range(max(3, args.warmup)):
            step()
        torch.cuda.synchronize(dev)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with ClockSampler(local_dev) as clk:
            e0.record(stream)
            for _ in range(args.steps):
                step()
            e1.record(stream)
            torch.cuda.synchronize(dev)
        ms = e0.elapsed_time(e1)
        lat = []
        for it in range(40):
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            step(one)
            a1.record(stream)
            torch.cuda.synchronize(dev)
            if it >= 10:
                lat.append(a0.elapsed_time(a1) * 1e3)
        out[name] = {"mpps": round(n * args.steps / (ms / 1e3) / 1e6, 3), "ms_per_step": round(ms / args.steps, 4),
                     "batch_latency_us": round(float(np.median(lat)), 2), "groups": ch.groups() if flags == nfc.F_PARALLEL else None}
        if flags == 0:
            main = (ms, clk.summary(), ch.launches())
        ch.close()
    ms, clocks, _ = main
    print(json.dumps({
        "metric": METRIC, "value": out["d_synthesized_fused"]["mpps"], "unit": "Mpps", "n_gpus": 1, "steps": args.steps,
        "warmup": max(3, args.warmup), "ms_per_step": round(ms / args.steps, 4), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": f"{w.name}: {w.note} (NEXT-2, configurations a-d of Fig. 13)", "chain": w.kinds,
                   "packets_per_step_per_gpu": n, "batch_pkts": args.batch_pkts, "latency_batch_pkts": min(n, BATCH)},
        "next2_configs": out,
        "paper_context": "P:L330-353: parallelization cuts latency (GPU 24 ms -> 5 ms, a -> b); synthesis (d) "
                         "raises throughput over (b) by 13-21 % on GPU",
        "clocks": clocks}))


def main():
    args = parse_args()
    if args.impl == "reference":
        return run_reference(args)
    if args.config in ("S1", "S1R"):
        return run_stream(args)
    if args.config in ("NX2_FW", "NX2_IDS"):
        return run_next2(args)
    import torch
    import torch.distributed as dist

    import nfcgen
    from paper_conf_hpca_hul18_b200 import dist as pdist
    from paper_conf_hpca_hul18_b200 import nfc

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    ndev = torch.cuda.device_count()
    local_dev = local % max(1, ndev)     # == local on a real N-GPU node
    torch.cuda.set_device(local_dev)
    dev = torch.device("cuda", local_dev)
    backend = os.environ.get("NFC_DIST_BACKEND", "nccl")   # gloo: test the N>1 path on fewer GPUs
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    cdev = dev if backend == "nccl" else torch.device("cpu")   # where collectives run

    w = make_workload(args)
    stream = torch.cuda.current_stream(dev)
    arena, off, ln, n = prepare_ring(w, args.ring_mb, rank, world, local_dev, stream)
    first = rank * n                       # match-pair ids: rank-local numbering of the shard
    b = host_view(arena, off, ln, first, w)
    chain = nfc.Chain(w.kinds, device=local_dev, flags=nfc.F_UNFUSED if args.unfused else 0)
    chain.load_tables(w.tables)
    hr, tr = chain.room()
    assert hr <= w.traffic.headroom and tr <= w.traffic.tailroom
    comm = None
    if world > 1 and backend == "nccl":
        comm = pdist.library_comm(local_dev)      # the library's own NCCL comm: counters only
        chain.attach_comm(comm)

    restore = bool(RESTORE_KINDS & set(w.kinds))
    pristine = arena.clone() if restore else None
    rec = torch.empty((n, 16), dtype=torch.uint8, device=dev)
    cap = 1 << 22
    mp = torch.empty(cap, dtype=torch.int32, device=dev)
    mq = torch.empty(cap, dtype=torch.int16, device=dev)
    mc = torch.zeros(1, dtype=torch.int32, device=dev)
    descs = batch_descs(arena, off, ln, n, first, args.batch_pkts)
    desc = nfc.Chain.batch_array(descs)

    def step():
        mc.zero_()
        chain.process(desc, rec.data_ptr(), mp.data_ptr(), mq.data_ptr(), cap, mc.data_ptr(), stream.cuda_stream)

    for _ in range(args.warmup):
        if restore:
            arena.copy_(pristine)
        step()
    torch.cuda.synchronize(dev)
    chain.stats(reset=True)
    launches0 = chain.launches()

    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    t_wall0 = time.perf_counter()
    with ClockSampler(local_dev) as clk:
        if restore:   # restore the pristine ring between steps, outside the timed intervals
            for s in range(args.steps):
                arena.copy_(pristine)
                ev[s][0].record(stream)
                step()
                ev[s][1].record(stream)
        else:         # back-to-back launches; the 1 GiB ring evicts L2 between passes
            ev[0][0].record(stream)
            for s in range(args.steps):
                step()
            ev[-1][1].record(stream)
        torch.cuda.synchronize(dev)
    t_wall = time.perf_counter() - t_wall0
    if world > 1:
        dist.barrier()
    if restore:
        ms = sum(a.elapsed_time(b_) for a, b_ in ev)
    else:
        ms = ev[0][0].elapsed_time(ev[-1][1])
    launches = chain.launches() - launches0
    launch_info = chain.last_launch()
    # the only data collective: the counters, summed over ranks inside the library
    # (nfc_collect_stats(NFC_STATS_ALLREDUCE): one ncclAllReduce on the chain's stream)
    stats = chain.stats(reset=True, allreduce=comm is not None)
    ms_t = torch.tensor([ms], dtype=torch.float64, device=cdev)
    st_t = torch.from_numpy(stats.view(np.int64).copy()).to(cdev)
    if world > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
        if comm is None:   # gloo test plumbing (several ranks on one GPU): host-side sum
            dist.all_reduce(st_t, op=dist.ReduceOp.SUM)
    ms_max = float(ms_t.item())
    tot_pkts = n * args.steps * world
    tot_bytes = int(b.len.astype(np.int64).sum()) * args.steps * world
    mpps = tot_pkts / (ms_max / 1e3) / 1e6
    gbps = tot_bytes * 8 / (ms_max / 1e3) / 1e9

    # measured integer / shared-memory / L2 peaks of this GPU (the integer rooflines)
    mpk = nfc.measure_peaks(local_dev)
    # roofline of the (only) kernel: algorithmic bytes per launch / avg launch duration
    rec_h = rec.cpu().numpy().view(nfcgen.RESULT).reshape(n)
    alg, rd, wr = alg_bytes_per_step(w.kinds, b.len, frame_family(b), rec_h)
    launch_ms = ms / args.steps
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    peak = peaks.get("hbm_gbs", 6650.0)
    achieved = alg / (launch_ms / 1e3) / 1e9
    traffic = None
    tfile = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tfile):
        tj = json.load(open(tfile)).get(w.name)
        if tj and tj.get("packets"):
            traffic = int(tj["dram_bytes_per_launch"] * n / tj["packets"])
    roof = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
            "frac": round(achieved / peak, 4), "traffic": traffic,
            "alg_bytes_per_launch": alg, "alg_bytes_per_packet": round(alg / n, 2),
            "alg_bytes": "SURVEY 8(d): header (+ payload if a payload NF is reached) + 16 B record + 32 B rewrite + ESP output",
            "other_bytes_per_packet": round(other_bytes_per_step(n, rec_h) / n, 2),
            "peak_source": "MEASURED_PEAKS.json hbm_gbs" if "hbm_gbs" in peaks else "B200_PROFILING fallback"}
    ops = esp_alg_ops(rec_h, l4_offsets(b)) if "IPSEC" in w.kinds else 0
    if ops:
        # integer-bound chains: the measured integer issue peak (nfc_measure_peaks: LOP3/SHF
        # chains interleaved with IMAD, one instruction per scheduler per clock)
        alu_peak = mpk["issue_tops"]
        alu_ach = ops / (launch_ms / 1e3) / 1e12
        if alu_ach / alu_peak > achieved / peak:
            roof = {"bound": "alu", "achieved": round(alu_ach, 3), "peak": round(alu_peak, 2), "unit": "Tops/s",
                    "frac": round(alu_ach / alu_peak, 4), "traffic": traffic,
                    "alg_ops_per_launch": ops, "alg_ops_per_packet": round(ops / n, 1),
                    "peak_source": "measured on this GPU: nfc_measure_peaks issue_tops (integer ALU + IMAD issue)",
                    "alu_pipe_frac": round(alu_ach / mpk["alu_tops"], 4),
                    "hbm": {"achieved": round(achieved, 1), "peak": peak, "frac": round(achieved / peak, 4),
                            "alg_bytes_per_packet": round(alg / n, 2)}}
    if "DPI" in w.kinds:
        # DPI work: one dependent DFA lookup per payload byte of every packet reaching DPI
        # in original order (SURVEY 8(d) "report both fractions")
        dpos = w.kinds.index("DPI")
        dr = rec_h["drop_nf"].astype(np.int64)
        reach = (dr != 0xFE) & ((dr == 0xFF) | (dr >= dpos))
        lk = int(payload_bytes(b)[reach].sum())
        roof["dpi_lookups"] = {"per_packet": round(lk / n, 1), "achieved_g_per_s": round(lk / (launch_ms / 1e3) / 1e9, 1),
                               "smem_peak_g_per_s": round(mpk["smem_glookups"], 1),
                               "frac": round(lk / (launch_ms / 1e3) / 1e9 / mpk["smem_glookups"], 4)}

    # end to end through the host-buffer C-ABI call (H2D + kernel + D2H every step)
    e2e = None
    if not args.no_e2e:
        host = torch.empty(len(b.arena), dtype=torch.uint8, pin_memory=True)
        hnp = host.numpy()
        hoff = torch.from_numpy(b.off.view(np.int64)).pin_memory()
        hlen = torch.from_numpy(b.len.view(np.int16)).pin_memory()
        hrec = torch.empty((n, 16), dtype=torch.uint8, pin_memory=True)
        hmp = torch.empty(cap, dtype=torch.int32, pin_memory=True)
        hmq = torch.empty(cap, dtype=torch.int16, pin_memory=True)
        e2e_steps = max(2, min(args.steps, 5))
        times = []
        npairs = 0
        for s in range(1 + e2e_steps):
            hnp[:] = b.arena
            torch.cuda.synchronize(dev)
            t0 = time.perf_counter()
            npairs = chain.process_host_ptr(host.data_ptr(), len(b.arena), hoff.data_ptr(), hlen.data_ptr(), n,
                                            hrec.data_ptr(), hmp.data_ptr(), hmq.data_ptr(), cap, first,
                                            stream.cuda_stream)
            dt = time.perf_counter() - t0
            if s:
                times.append(dt)
        e2e_t = torch.tensor([sum(times)], dtype=torch.float64, device=cdev)
        if world > 1:
            dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
        e2e = {"value": round(n * len(times) * world / float(e2e_t.item()) / 1e6, 3), "unit": "Mpps",
               "h2d_bytes_per_step": len(b.arena) + n * 10,
               "d2h_bytes_per_step": len(b.arena) + n * 16 + 4 + min(npairs, cap) * 6,
               "steps": len(times), "api": "nfc_process_host (pinned host buffers)"}
        del host, hrec
        pk = pcie_peaks(torch, dev, len(b.arena))
        # copy roofline: both directions overlapped at the measured duplex rate
        bound_s = max(e2e["h2d_bytes_per_step"], e2e["d2h_bytes_per_step"]) / (pk["duplex_each_gbs"] * 1e9)
        step_s = float(e2e_t.item()) / len(times)
        e2e["pcie"] = dict(pk, bound_mpps=round(n / bound_s / 1e6, 1), frac=round(bound_s / step_s, 3))
        chain.stats(reset=True)

    # the general multi-batch path: the same batches in shuffled order, so the descriptors
    # are not one run and the kernel locates packets through per-chunk records
    general = None
    if not args.no_unfused and len(descs) > 1 and not restore:
        perm = np.random.default_rng(11).permutation(len(descs))
        gdesc = nfc.Chain.batch_array([descs[i] for i in perm])

        def gstep():
            mc.zero_()
            chain.process(gdesc, rec.data_ptr(), mp.data_ptr(), mq.data_ptr(), cap, mc.data_ptr(), stream.cuda_stream)
        for _ in range(args.warmup):
            gstep()
        torch.cuda.synchronize(dev)
        ge0, ge1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ge0.record(stream)
        for _ in range(args.steps):
            gstep()
        ge1.record(stream)
        torch.cuda.synchronize(dev)
        g_t = torch.tensor([ge0.elapsed_time(ge1)], dtype=torch.float64, device=cdev)
        if world > 1:
            dist.all_reduce(g_t, op=dist.ReduceOp.MAX)
        general = {"value": round(n * args.steps * world / (float(g_t.item()) / 1e3) / 1e6, 3), "unit": "Mpps",
                   "what": "the same batches in shuffled order: not one descriptor run, so packets are located "
                           "through per-chunk records (k_chunk_recs + the staged record path)"}
        chain.stats(reset=True)

    # NEXT-1: the same chain as one kernel per NF with a device-side
    # re-split between NFs, timed on the same ring -- the fusion benefit on B200
    unfused = None
    if not args.no_unfused and not args.unfused and "IPSEC" not in w.kinds:
        uch = nfc.Chain(w.kinds, device=local_dev, flags=nfc.F_UNFUSED)
        uch.load_tables(w.tables)

        def ustep():
            mc.zero_()
            uch.process(desc, rec.data_ptr(), mp.data_ptr(), mq.data_ptr(), cap, mc.data_ptr(), stream.cuda_stream)
        for _ in range(args.warmup):
            ustep()
        torch.cuda.synchronize(dev)
        l0 = uch.launches()
        ue0, ue1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ue0.record(stream)
        for _ in range(args.steps):
            ustep()
        ue1.record(stream)
        torch.cuda.synchronize(dev)
        ums = ue0.elapsed_time(ue1)
        u_t = torch.tensor([ums], dtype=torch.float64, device=cdev)
        if world > 1:
            dist.all_reduce(u_t, op=dist.ReduceOp.MAX)
        u_mpps = n * args.steps * world / (float(u_t.item()) / 1e3) / 1e6
        unfused = {"value": round(u_mpps, 3), "unit": "Mpps",
                   "kernels_per_step": (uch.launches() - l0) // args.steps,
                   "fused_speedup": round(mpps / u_mpps, 3),
                   "what": "NFC_F_UNFUSED: one kernel per NF + device-side re-split, same ring and tables"}
        uch.close()

    # NEXT-2: SFC parallelization -- the chain's NFs on different warps,
    # each on its own packet copy, XOR-merged -- on the same ring, and the
    # latency of ONE batch (the paper's Fig. 14 metric) for fused / parallel / unfused
    parallel = None
    if not args.no_unfused and not args.unfused and "IPSEC" not in w.kinds and "NAT" not in w.kinds:
        pch = nfc.Chain(w.kinds, device=local_dev, flags=nfc.F_PARALLEL)
        pch.load_tables(w.tables)

        def pstep():
            mc.zero_()
            pch.process(desc, rec.data_ptr(), mp.data_ptr(), mq.data_ptr(), cap, mc.data_ptr(), stream.cuda_stream)
        for _ in range(args.warmup):
            pstep()
        torch.cuda.synchronize(dev)
        pe0, pe1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        pe0.record(stream)
        for _ in range(args.steps):
            pstep()
        pe1.record(stream)
        torch.cuda.synchronize(dev)
        p_t = torch.tensor([pe0.elapsed_time(pe1)], dtype=torch.float64, device=cdev)
        if world > 1:
            dist.all_reduce(p_t, op=dist.ReduceOp.MAX)
        p_mpps = n * args.steps * world / (float(p_t.item()) / 1e3) / 1e6
        # one batch of BATCH packets (C1's 4,096): median of 30 launches per arm
        nb = min(n, BATCH)
        bdesc = [(arena.data_ptr(), off.data_ptr(), ln.data_ptr(), nb, first)]
        uch2 = nfc.Chain(w.kinds, device=local_dev, flags=nfc.F_UNFUSED)
        uch2.load_tables(w.tables)
        lat = {}
        for name, ch in (("fused", chain), ("parallel", pch), ("unfused", uch2)):
            ts = []
            for it in range(40):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                mc.zero_()
                e0.record(stream)
                ch.process(bdesc, rec.data_ptr(), mp.data_ptr(), mq.data_ptr(), cap, mc.data_ptr(), stream.cuda_stream)
                e1.record(stream)
                torch.cuda.synchronize(dev)
                if it >= 10:
                    ts.append(e0.elapsed_time(e1) * 1e3)
            lat[name + "_us"] = round(float(np.median(ts)), 2)
        parallel = {"value": round(p_mpps, 3), "unit": "Mpps", "groups": nfc.plan_parallel(w.kinds),
                    "fused_speedup": round(mpps / p_mpps, 3), "batch_pkts": nb, "batch_latency": lat,
                    "what": "NFC_F_PARALLEL: NFs on different warps of a team, per-warp packet copies, XOR merge"}
        uch2.close()
        pch.close()
        chain.stats(reset=True)

    cpu = None
    if not args.no_cpu and rank == 0 and world == 1:
        r_mpps, r_gbps, r_pk, r_t = oracle_rate(w, first, args.cpu_seconds)
        cpu = {"value": round(r_mpps, 6), "unit": "Mpps", "cores": 1, "kind": "oracle",
               "sample": f"{r_pk} packets of {w.name} (same generator and tables), {r_t:.1f} s, 1 thread",
               "gbps": round(r_gbps, 6), "cpu_model": cpu_model(), "nproc": os.cpu_count()}
        try:
            cpu["all_cores"] = oracle_all_cores(w, local_dev, r_mpps, args.cpu_seconds)
        except Exception as e:  # noqa: BLE001 -- reported, never fatal to the GPU line
            cpu["all_cores"] = {"error": repr(e)[:300]}

    if rank == 0:
        st = st_t.cpu().numpy().view(np.uint64)
        out = {
            "metric": METRIC, "value": round(mpps, 3), "unit": "Mpps", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms_max / args.steps, 4), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
            "gbps": round(gbps, 2),
            "config": {"workload": f"{w.name}: {w.note}", "chain": w.kinds,
                       "pkt_len": "IMIX" if w.traffic.pkt_len == 0 else w.traffic.pkt_len,
                       "packets_per_step_per_gpu": n, "ring_bytes_per_gpu": len(b.arena),
                       "batch_pkts": args.batch_pkts or n, "batches_per_step_per_gpu": len(descs),
                       "sharding": "RSS: nfc_rss_shard (Toeplitz MS key -> RETA) of the global stream, device-generated"
                                   if world > 1 else "single GPU: the global stream, device-generated",
                       "l2": "ring >> 126 MB L2 (no flush needed)" if not restore else
                             "pristine ring restored between steps (1 GiB-class copy, evicts L2), outside timed intervals",
                       "timing": "CUDA events on the launch stream; max over ranks",
                       "parallelism": f"RSS flow-sharded x{world}, no data-path collective; counters summed by "
                                      f"one ncclAllReduce inside the library",
                       "fwd_frac": round(float(st[2]) / max(1, float(st[0])), 4),
                       "launch": launch_info},
            "roofline": roof,
            "measured_peaks": {k_: (round(v_, 2) if isinstance(v_, float) else v_) for k_, v_ in mpk.items()},
            "cpu_baseline": cpu,
            "general_batch_path": general,
            "unfused_baseline": unfused,
            "sfc_parallel": parallel,
            "e2e": e2e,
            "gpu_launches": int(launches),
            "clocks": clk.summary(),
            "wall_s_timed_region": round(t_wall, 4),
        }
        print(json.dumps(out))
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
