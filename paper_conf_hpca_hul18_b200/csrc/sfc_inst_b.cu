// sfc_inst_b.cu -- kernel instantiations (split across files for parallel compilation)
#include "sfc_kernel.cuh"
namespace nfc {
NFC_INSTANTIATE_LAUNCH(SIG_K2, DM_FULL)
NFC_INSTANTIATE_LAUNCH(SIG_K2, DM_HOT)
NFC_INSTANTIATE_LAUNCH(SIG_K1, DM_HOT)
} // namespace nfc
