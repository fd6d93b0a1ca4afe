// sfc_inst_a.cu -- kernel instantiations (split across files for parallel compilation)
#include "sfc_kernel.cuh"
namespace nfc {
NFC_INSTANTIATE_LAUNCH(SIG_C1, DM_FULL)
NFC_INSTANTIATE_LAUNCH(SIG_C1, DM_HOT)
} // namespace nfc
