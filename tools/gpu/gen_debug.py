"""Debug: first differences between the device and host traffic generators."""
import sys
import numpy as np
sys.path.insert(0, ".")
import torch
import nfcgen
from nfcgen import device as gd

w = nfcgen.workload("C1", small=True)
first, n = 123_457, 5000
b = nfcgen.generate(w.traffic, w.tables, first, n)
arena, off, ln = gd.generate(w.traffic, w.tables, first, n, device=0)
torch.cuda.synchronize()
a = arena.cpu().numpy()
bad = np.nonzero(a[:len(b.arena) - 64] != b.arena[:len(b.arena) - 64])[0]
print("n bad bytes", len(bad))
offs = b.off.astype(np.int64)
seen = 0
for x in bad[:2000]:
    k = int(np.searchsorted(offs, x, side="right") - 1)
    if seen < 12:
        print("pkt", k, "byte", x - offs[k], "dev", a[x], "host", b.arena[x])
    seen += 1
pk = np.unique(np.searchsorted(offs, bad, side="right") - 1)
print("packets with diffs", len(pk), pk[:20])
print("bytes-in-frame histogram", np.bincount((bad - offs[np.searchsorted(offs, bad, side='right') - 1]).astype(np.int64))[:64])
