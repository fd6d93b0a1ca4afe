"""nfcgen.device -- the traffic generator on the GPU (gen_dev.cu): packet batches
written straight into HBM, byte-identical to nfcgen.generate() (same per-packet
body, gen_core.h).  Input infrastructure only; torch provides device memory."""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from . import HERE, Tables, TrafficParams, _GenTables, _gen_structs

_LIB = os.path.join(HERE, "libnfcgen_dev.so")
_P = ctypes.c_void_p
_lib = None


def build_lib(force: bool = False) -> str:
    srcs = [os.path.join(HERE, f) for f in ("gen_dev.cu", "gen_core.h")]
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(os.path.getmtime(s) for s in srcs):
        nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
        subprocess.check_call([nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo",
                               "-Xcompiler", "-fPIC", "-shared", "-o", _LIB + ".tmp", srcs[0]])
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build_lib()
        L = ctypes.CDLL(_LIB)
        L.nfcgen_dev_lengths.argtypes = [_P, _P, ctypes.c_uint64, ctypes.c_uint32, _P, _P, _P]
        L.nfcgen_dev_fill.argtypes = [_P, _P, ctypes.c_uint64, ctypes.c_uint32, _P, _P, _P, _P]
        L.nfcgen_dev_gather.argtypes = [_P, _P, _P, _P, ctypes.c_uint32, _P, _P, _P]
        _lib = L
    return _lib


class DeviceTables:
    """The generator's view of the logical tables, copied to `device` once."""

    def __init__(self, tp: TrafficParams, t: Tables, device):
        import torch
        gp, gt, keep = _gen_structs(tp, t)
        self._t = []
        dt = _GenTables()
        for name, ctype in gt._fields_:
            v = getattr(gt, name)
            if ctype is _P and v:
                src = next(a for a in keep.refs if a.ctypes.data == v)
                d = torch.from_numpy(src.view(np.uint8).reshape(-1).copy()).to(device)
                self._t.append(d)
                setattr(dt, name, d.data_ptr())
            else:
                setattr(dt, name, v)
        self.gp, self.gt, self.device = gp, dt, device


def generate(tp: TrafficParams, t: Tables, first: int, n: int, device=0, dtab: DeviceTables = None,
             stream=None):
    """Packets [first, first+n) of the global stream in HBM: (arena u8, off i64, len i16)
    torch tensors on `device`, laid out exactly as nfcgen.generate() lays them out."""
    import torch
    dev = torch.device("cuda", device) if isinstance(device, int) else device
    lib = _load()
    dtab = dtab or DeviceTables(tp, t, dev)
    st = (stream or torch.cuda.current_stream(dev)).cuda_stream
    ln = torch.empty(max(1, n), dtype=torch.int16, device=dev)
    slot = torch.empty(max(1, n), dtype=torch.int32, device=dev)
    if n:
        assert lib.nfcgen_dev_lengths(ctypes.byref(dtab.gp), ctypes.byref(dtab.gt), first, n, ln.data_ptr(),
                                      slot.data_ptr(), st) == 0
    cs = torch.cumsum(slot[:n].to(torch.int64), 0)
    total = int(cs[-1].item()) if n else 0
    off = torch.zeros(max(1, n), dtype=torch.int64, device=dev)
    if n > 1:
        off[1:n] = cs[:-1]
    off += tp.headroom
    arena = torch.zeros(total + 64, dtype=torch.uint8, device=dev)
    if n:
        assert lib.nfcgen_dev_fill(ctypes.byref(dtab.gp), ctypes.byref(dtab.gt), first, n, arena.data_ptr(),
                                   off.data_ptr(), ln.data_ptr(), st) == 0
    return arena, off[:n], ln[:n]


def gather(arena, off, ln, idx, headroom: int, tailroom: int):
    """Frames idx (i64 device tensor) of (arena, off, ln) packed into a new dense ring with
    the same headroom/tailroom slots: (arena, off, ln) of the selected packets in order."""
    import torch
    lib = _load()
    n = int(idx.numel())
    sel_len = ln.index_select(0, idx)
    slot = ((sel_len.to(torch.int64) & 0xFFFF) + headroom + tailroom + 15) // 16 * 16
    cs = torch.cumsum(slot, 0)
    total = int(cs[-1].item()) if n else 0
    doff = torch.zeros(max(1, n), dtype=torch.int64, device=arena.device)
    if n > 1:
        doff[1:n] = cs[:-1]
    doff += headroom
    dst = torch.zeros(total + 64, dtype=torch.uint8, device=arena.device)
    if n:
        st = torch.cuda.current_stream(arena.device).cuda_stream
        assert lib.nfcgen_dev_gather(arena.data_ptr(), off.data_ptr(), ln.data_ptr(), idx.data_ptr(), n,
                                     dst.data_ptr(), doff.data_ptr(), st) == 0
    return dst, doff[:n], sel_len
