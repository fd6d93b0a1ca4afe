// sfc_inst_c.cu -- kernel instantiations (split across files for parallel compilation)
#include "sfc_kernel.cuh"
namespace nfc {
NFC_INSTANTIATE_LAUNCH(SIG_K4, DM_FULL)
NFC_INSTANTIATE_LAUNCH(SIG_K4, DM_HOT)
} // namespace nfc
