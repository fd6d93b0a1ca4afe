import sys
sys.path.insert(0, ".")
import numpy as np
from tests.test_gpu_stream import _pats, _gpu
from nfcgen.stream import stream_batch
from oracle.stream_dpi import StreamDPI
from paper_conf_hpca_hul18_b200 import nfc
for npat, lmin, lmax in ((2600, 12, 16), (300, 12, 16), (300, 2, 8), (2600, 2, 8)):
    blob, off, act, pats = _pats(2, npat, lmin=lmin, lmax=lmax)
    ds = nfc.DpiStream(blob, off, act, max_flows=64)
    orc = StreamDPI(pats, list(act))
    sb = stream_batch(3, 400, 20, pats, len_choices=[64, 200], plant_frac=0.5)
    want, wn, wd = orc.process(sb.frames())
    got, gn, gd, _ = _gpu(ds, sb)
    print(npat, lmin, lmax, "want", len(want), "got", len(got), "equal", got == want, "nocc equal", gn == wn)
