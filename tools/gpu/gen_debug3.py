import sys, ctypes, subprocess
import numpy as np
sys.path.insert(0, ".")
import torch
import nfcgen
from nfcgen import device as gd
for flags in (["-O3"], ["-G"]):
    so = f"/tmp/gdbg{len(flags[0])}.so"
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", *flags, "-Xcompiler", "-fPIC", "-shared",
                           "-o", so, "tools/gpu/gen_dbg.cu"])
    L = ctypes.CDLL(so)
    w = nfcgen.workload("C1", small=True)
    dt = gd.DeviceTables(w.traffic, w.tables, torch.device("cuda", 0))
    out = torch.zeros(8 * 8, dtype=torch.int64, device="cuda")
    rc = L.dbg(ctypes.byref(dt.gp), ctypes.byref(dt.gt), ctypes.c_uint64(123457), ctypes.c_uint32(8), ctypes.c_void_p(out.data_ptr()))
    o = out.cpu().numpy().reshape(8, 8)
    print(flags, "rc", rc)
    for k in range(8):
        f = nfcgen.rnd(1, 1, 123457 + k) % 65536
        kr = nfcgen.rnd(1, 10, f) % 1001
        print(list(o[k][:7]), hex(o[k][7]), "host f", f, "kr", kr, "prefix", int(w.tables.routes4["prefix"][kr]), "len", int(w.tables.routes4["len"][kr]))
