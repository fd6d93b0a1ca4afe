// sfc_inst_d.cu -- kernel instantiations (split across files for parallel compilation)
#include "sfc_kernel.cuh"
namespace nfc {
NFC_INSTANTIATE_LAUNCH(SIG_C2, DM_HOT)
NFC_INSTANTIATE_LAUNCH(SIG_C3, DM_HOT)
} // namespace nfc
