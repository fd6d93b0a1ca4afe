"""Debug: which route the device generator picked for the first differing packets."""
import sys
import numpy as np
sys.path.insert(0, ".")
import torch
import nfcgen
from nfcgen import device as gd

w = nfcgen.workload("C1", small=True)
first, n = 123_457, 64
b = nfcgen.generate(w.traffic, w.tables, first, n)
dt = gd.DeviceTables(w.traffic, w.tables, torch.device("cuda", 0))
for tt in dt._t:
    print("dev table bytes", tt.numel(), tt.data_ptr() % 16)
gp, gt, keep = nfcgen._gen_structs(w.traffic, w.tables)
for name, _ in gt._fields_:
    print(name, getattr(gt, name), getattr(dt.gt, name))
arena, off, ln = gd.generate(w.traffic, w.tables, first, n, device=0, dtab=dt)
a = arena.cpu().numpy()
r = w.tables.routes4
pre = r["prefix"].astype(np.int64)
for k in range(8):
    o = int(b.off[k])
    hd = bytes(b.arena[o + 30:o + 34]); dd = bytes(a[o + 30:o + 34])
    if hd == dd:
        continue
    hv, dv = int.from_bytes(hd, "big"), int.from_bytes(dd, "big")
    cand = [(j, int(r["len"][j])) for j in range(len(r)) if int(r["len"][j]) and ((dv ^ pre[j]) >> (32 - int(r["len"][j]))) == 0]
    hc = [(j, int(r["len"][j])) for j in range(len(r)) if int(r["len"][j]) and ((hv ^ pre[j]) >> (32 - int(r["len"][j]))) == 0]
    print("pkt", k, hd.hex(), dd.hex(), "dev-matching routes", cand[:5], "host-matching", hc[:5])
# table contents back
for tt, name in zip(dt._t, [nm for nm, c in gt._fields_ if c is nfcgen._P and getattr(gt, nm)]):
    src = next(x for x in keep.refs if x.ctypes.data == getattr(gt, name))
    print(name, np.array_equal(tt.cpu().numpy(), src.view(np.uint8).reshape(-1)))
