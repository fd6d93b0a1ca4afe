"""paper_conf_hpca_hul18_b200 -- B200-native NFCompass SFC hot path.

The product is libnfc.so (C ABI in include/nfc.h: nfc_build_chain /
nfc_load_tables / nfc_process_batch / nfc_collect_stats) whose fused
persistent sm_100a kernel runs the service function chain; `nfc` is the thin
ctypes binding.  Importing the binding fails loudly if the library is not
built -- there is no CPU fallback.
"""
from . import nfc  # noqa: F401
from .nfc import Chain, NfcError  # noqa: F401
