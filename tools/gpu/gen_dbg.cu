// debug: intermediate values of make_flow on the device
#include <cuda_runtime.h>
#include <stdint.h>
#include "../../nfcgen/gen_core.h"
static __global__ void k_dbg(gen_params p, gen_tables t, uint64_t first, uint32_t n, uint64_t *out)
{
    const uint32_t k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= n) return;
    const uint64_t i = first + k;
    const gen_params *pp = &p;
    uint64_t f = gen_rnd(pp->seed, S_FLOW, i) % pp->n_flows;
    flow_t fl;
    make_flow(pp, &t, f, &fl);
    uint64_t kr = gen_rnd(pp->seed, S_ROUTE, f) % t.n_r4;
    out[8 * k + 0] = f;
    out[8 * k + 1] = kr;
    out[8 * k + 2] = t.n_r4;
    out[8 * k + 3] = t.r4_prefix[kr];
    out[8 * k + 4] = t.r4_len[kr];
    out[8 * k + 5] = (uint64_t)fl.dst[0] << 24 | fl.dst[1] << 16 | fl.dst[2] << 8 | fl.dst[3];
    out[8 * k + 6] = gen_rnd(pp->seed, S_INACL, f) % 100;
    out[8 * k + 7] = (uint64_t)(uintptr_t)t.r4_prefix;
}
extern "C" int dbg(const gen_params *p, const gen_tables *t, uint64_t first, uint32_t n, uint64_t *out)
{
    k_dbg<<<(n + 127) / 128, 128>>>(*p, *t, first, n, out);
    return cudaDeviceSynchronize();
}
