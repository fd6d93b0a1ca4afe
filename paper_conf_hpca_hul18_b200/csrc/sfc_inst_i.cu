// sfc_inst_i.cu -- kernel instantiations (split across files for parallel compilation)
#include "sfc_kernel.cuh"
namespace nfc {
NFC_INSTANTIATE_LAUNCH(SIG_N3, DM_HOT)   // NEXT-3: FW -> router -> NAT
} // namespace nfc
