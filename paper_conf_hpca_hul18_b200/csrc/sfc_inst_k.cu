// sfc_inst_k.cu -- kernel instantiations (split across files for parallel compilation):
// the a3 regrouping variants of the C5 k=2 and k=4 chains
#include "sfc_kernel.cuh"
namespace nfc {
#if NFC_REGROUP
NFC_INSTANTIATE_LAUNCH_RG(SIG_K2, DM_FULL)
NFC_INSTANTIATE_LAUNCH_RG(SIG_K4, DM_FULL)
#endif
} // namespace nfc
