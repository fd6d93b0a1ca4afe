// sfc_inst_h.cu -- kernel instantiations (split across files for parallel compilation)
#include "sfc_kernel.cuh"
namespace nfc {
NFC_INSTANTIATE_LAUNCH(SIG_ANY, DM_HOT)
} // namespace nfc
