// sfc_inst_j.cu -- kernel instantiations (split across files for parallel compilation):
// the a3 regrouping variant of the C1 chain (also C5 k=3)
#include "sfc_kernel.cuh"
namespace nfc {
#if NFC_REGROUP
NFC_INSTANTIATE_LAUNCH_RG(SIG_C1, DM_FULL)
#endif
} // namespace nfc
