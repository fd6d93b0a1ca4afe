/*
 * nfcgen/gen_dev.cu -- the synthetic traffic generator on the GPU: packet
 * batches written straight into HBM (north_star "a synthetic traffic generator
 * writing packet batches straight into HBM").  Input generator only (see
 * gen_core.h): it runs the same per-packet body as the host generator gen.c,
 * so a batch generated here is byte-identical to nfcgen.generate(); it is not
 * part of the product library and holds none of the method's arithmetic.
 *
 * Layout: k_len writes each packet's frame length and slot size (headroom +
 * frame + tailroom, 16-B aligned); the caller's exclusive scan of the slots
 * gives the offsets (torch.cumsum in nfcgen/device.py); k_fill writes the bytes.
 * k_gather copies selected frames into a dense ring (per-rank RSS shards).
 */
#include <cuda_runtime.h>
#include <stdint.h>

#include "gen_core.h"

static __global__ void k_len(gen_params p, gen_tables t, uint64_t first, uint32_t n, uint16_t *len, uint32_t *slot)
{
    const uint32_t k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= n) return;
    const uint32_t L = gen_len_one(&p, &t, first + k);
    len[k] = (uint16_t)L;
    slot[k] = (uint32_t)round16((uint64_t)p.headroom + L + p.tailroom);
}

static __global__ void k_fill(gen_params p, gen_tables t, uint64_t first, uint32_t n, uint8_t *arena,
                              const uint64_t *off, const uint16_t *len)
{
    const uint32_t k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= n) return;
    gen_fill_one(&p, &t, first + k, arena + off[k], len[k]);
}

// dst frame k = src frame idx[k] (16-B words; offsets are 16-B aligned, arenas padded)
static __global__ void k_gather(const uint8_t *src, const uint64_t *src_off, const uint16_t *len, const int64_t *idx,
                                uint32_t n, uint8_t *dst, const uint64_t *dst_off)
{
    const uint32_t k = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32, lane = threadIdx.x & 31;
    if (k >= n) return;
    const int64_t j = idx[k];
    const uint4 *s = reinterpret_cast<const uint4 *>(src + src_off[j]);
    uint4 *d = reinterpret_cast<uint4 *>(dst + dst_off[k]);
    const uint32_t words = (len[j] + 15u) / 16u;
    for (uint32_t w = lane; w < words; w += 32) d[w] = s[w];
}

extern "C" {

int nfcgen_dev_lengths(const gen_params *p, const gen_tables *t, uint64_t first, uint32_t n, uint16_t *len,
                       uint32_t *slot, void *stream)
{
    if (n) k_len<<<(n + 255) / 256, 256, 0, (cudaStream_t)stream>>>(*p, *t, first, n, len, slot);
    return cudaGetLastError() == cudaSuccess ? 0 : -3;
}

int nfcgen_dev_fill(const gen_params *p, const gen_tables *t, uint64_t first, uint32_t n, uint8_t *arena,
                    const uint64_t *off, const uint16_t *len, void *stream)
{
    if (n) k_fill<<<(n + 127) / 128, 128, 0, (cudaStream_t)stream>>>(*p, *t, first, n, arena, off, len);
    return cudaGetLastError() == cudaSuccess ? 0 : -3;
}

int nfcgen_dev_gather(const uint8_t *src, const uint64_t *src_off, const uint16_t *len, const int64_t *idx,
                      uint32_t n, uint8_t *dst, const uint64_t *dst_off, void *stream)
{
    if (n) k_gather<<<(n + 7) / 8, 256, 0, (cudaStream_t)stream>>>(src, src_off, len, idx, n, dst, dst_off);
    return cudaGetLastError() == cudaSuccess ? 0 : -3;
}

} // extern "C"
