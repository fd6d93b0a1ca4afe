"""Quick device timing of stateful DPI (NEXT-4) on S1 traffic: python tools/stream_time.py [n_pkts] [n_flows]."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import nfcgen
from nfcgen.stream import stream_batch
from paper_conf_hpca_hul18_b200 import nfc

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 22
nflows = int(sys.argv[2]) if len(sys.argv) > 2 else 65536
rng = np.random.default_rng(4)
blob, off, act = nfcgen.gen_patterns(rng, 100, lmin=4, lmax=16, drop_frac=0.05)
pats = nfcgen.Tables(pat_blob=blob, pat_off=off, pat_action=act).patterns()
sb = stream_batch(9, n, nflows, pats, plant_frac=0.05)
d = torch.device("cuda:0")
arena = torch.from_numpy(sb.arena).to(d)
o = torch.from_numpy(sb.off.astype(np.int64)).to(d)
ln = torch.from_numpy(sb.len.view(np.int16)).to(d)
nocc = torch.zeros(n, dtype=torch.int32, device=d)
drop = torch.zeros(n, dtype=torch.uint8, device=d)
cap = 1 << 22
op = torch.zeros(cap, dtype=torch.int32, device=d)
oq = torch.zeros(cap, dtype=torch.int16, device=d)
oe = torch.zeros(cap, dtype=torch.int16, device=d)
cnt = torch.zeros(1, dtype=torch.int32, device=d)
ds = nfc.DpiStream(blob, off, act, max_flows=max(2 * nflows, 1024))
for _ in range(3):
    cnt.zero_()
    ds.process_tensors(arena, o, ln, nocc, drop, op, oq, oe, cnt)
torch.cuda.synchronize()
K = 20
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(K):
    ds.process_tensors(arena, o, ln, nocc, drop, op, oq, oe, cnt)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / K
print(f"stream DPI: {n} pkts x 64 B, {nflows} flows: {ms:.3f} ms/call, {n / ms / 1e3:.1f} Mpps, "
      f"{n * 64 / ms / 1e6:.1f} GB/s of frames, occurrences/call {int(cnt.item()) // (K + 3)}, flows {ds.flows()}")
