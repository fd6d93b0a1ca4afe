// peaks.cu -- measured integer, shared-memory and L2-gather peaks of the device
// (SURVEY.md 8(d) "Integer and shared-memory peaks: a repo microbenchmark measures
// them on the box"): the denominators of the integer-bound rooflines (IPsec ESP:
// AES T-table lookups + SHA-1 rounds; DPI: dependent shared-memory DFA steps).
//
//   alu     -- independent chains of LOP3 / SHF / PRMT (the ALU pipe only)
//   issue   -- the same chains interleaved with IMAD (ALU + FMA pipes: the
//              one-instruction-per-scheduler-per-clock issue limit)
//   smem    -- conflict-free 32-bit shared-memory loads (every lane its own bank)
//   l2      -- random 32-B sectors gathered from an L2-resident 64 MiB buffer
//
// Each kernel is timed with CUDA events after a warm-up launch; the counts are of
// the SASS instructions the loops issue (checked with cuobjdump: the loop bodies
// are fully unrolled straight-line code), times 32 lanes.
#include <cuda_runtime.h>

#include <string>

#include "nfc_internal.h"

namespace {

constexpr int CH = 8;          // independent chains per thread
constexpr int UNR = 8;         // unrolled steps per loop iteration

__device__ __forceinline__ uint32_t lop3(uint32_t a, uint32_t b, uint32_t c)
{
    uint32_t d;
    asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}
__device__ __forceinline__ uint32_t shf(uint32_t a, uint32_t b)
{
    uint32_t d;
    asm volatile("shf.l.wrap.b32 %0, %1, %2, 7;" : "=r"(d) : "r"(a), "r"(b));
    return d;
}
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b)
{
    uint32_t d;
    asm volatile("prmt.b32 %0, %1, %2, 0x2107;" : "=r"(d) : "r"(a), "r"(b));
    return d;
}
__device__ __forceinline__ uint32_t lop3b(uint32_t a, uint32_t b, uint32_t c)
{
    uint32_t d;
    asm volatile("lop3.b32 %0, %1, %2, %3, 0xE8;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}
__device__ __forceinline__ uint32_t imad(uint32_t a, uint32_t b, uint32_t c)
{
    uint32_t d;
    asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}

// 4 ALU-pipe ops per chain step (LOP3, LOP3, SHF, PRMT): CH * UNR * 4 per loop iteration
__global__ void __launch_bounds__(512) k_alu(uint32_t *out, uint32_t iters, uint32_t kk)
{
    const uint32_t k = kk ^ (threadIdx.x >> 10);   // a register, not a constant-bank operand
    uint32_t a[CH];
#pragma unroll
    for (int c = 0; c < CH; c++) a[c] = threadIdx.x * 0x9E3779B9u + c;
    for (uint32_t it = 0; it < iters; it++) {
#pragma unroll
        for (int u = 0; u < UNR; u++)
#pragma unroll
            for (int c = 0; c < CH; c++) {
                a[c] = lop3(a[c], k, a[(c + 1) % CH]);
                a[c] = lop3b(a[c], k, a[(c + 2) % CH]);
                a[c] = shf(a[c], a[c]);
                a[c] = prmt(a[c], k);
            }
    }
    uint32_t x = 0;
#pragma unroll
    for (int c = 0; c < CH; c++) x ^= a[c];
    if (x == 0x12345678u) out[threadIdx.x] = x;   // keeps the chains live
}

// 2 ALU-pipe + 2 FMA-pipe (IMAD) ops per chain step
__global__ void __launch_bounds__(512) k_issue(uint32_t *out, uint32_t iters, uint32_t kk)
{
    const uint32_t k = kk ^ (threadIdx.x >> 10), m = 0x01000193u ^ (threadIdx.x >> 10);
    uint32_t a[CH];
#pragma unroll
    for (int c = 0; c < CH; c++) a[c] = threadIdx.x * 0x9E3779B9u + c;
    for (uint32_t it = 0; it < iters; it++) {
#pragma unroll
        for (int u = 0; u < UNR; u++)
#pragma unroll
            for (int c = 0; c < CH; c++) {
                a[c] = lop3(a[c], k, a[(c + 1) % CH]);
                a[c] = imad(a[c], k, a[(c + 3) % CH]);
                a[c] = shf(a[c], a[c]);
                a[c] = imad(a[c], m, k);
            }
    }
    uint32_t x = 0;
#pragma unroll
    for (int c = 0; c < CH; c++) x ^= a[c];
    if (x == 0x12345678u) out[threadIdx.x] = x;
}

// conflict-free LDS.32: table[i] = (i + 32 * 7) & mask keeps every lane in its own bank
__global__ void __launch_bounds__(1024) k_smem(uint32_t *out, uint32_t iters, uint32_t mask)
{
    extern __shared__ uint32_t tab[];
    for (uint32_t i = threadIdx.x; i <= mask; i += blockDim.x) tab[i] = (i + 32 * 7) & mask;
    __syncthreads();
    const uint32_t lane = threadIdx.x & 31;
    uint32_t x[4];
#pragma unroll
    for (int c = 0; c < 4; c++) x[c] = (lane + 32 * (threadIdx.x / 32 + 11 * c)) & mask;
    for (uint32_t it = 0; it < iters; it++) {
#pragma unroll
        for (int u = 0; u < UNR; u++)
#pragma unroll
            for (int c = 0; c < 4; c++) x[c] = tab[x[c]];
    }
    if ((x[0] ^ x[1] ^ x[2] ^ x[3]) == 0xFFFFFFFFu) out[threadIdx.x] = 1;
}

// random 32-B sectors of an L2-resident buffer (ld.global.cg: not cached in L1)
__global__ void __launch_bounds__(512) k_l2(const uint32_t *buf, uint32_t *out, uint32_t iters, uint32_t sectors_mask)
{
    uint32_t h = (blockIdx.x * blockDim.x + threadIdx.x) * 0x9E3779B9u, acc = 0;
    for (uint32_t it = 0; it < iters; it++) {
#pragma unroll
        for (int u = 0; u < UNR; u++) {
            h = h * 1664525u + 1013904223u;
            acc += __ldcg(buf + 8 * ((h >> 5) & sectors_mask));
        }
    }
    if (acc == 0x12345678u) out[0] = acc;
}

__global__ void k_touch(uint32_t *buf, size_t n)
{
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
        buf[i] = (uint32_t)i;
}

template <class F>
float time_ms(F launch, cudaEvent_t e0, cudaEvent_t e1)
{
    launch();   // warm-up
    cudaEventRecord(e0);
    launch();
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    return ms;
}

}  // namespace

extern "C" int nfc_measure_peaks(int device, nfc_peaks *out)
{
    if (!out) return nfc::set_fail(NFC_EINVAL, "nfc_measure_peaks: out is NULL");
    if (cudaSetDevice(device) != cudaSuccess) return nfc::set_fail(NFC_ECUDA, "cudaSetDevice failed");
    int sms = 0, clk_khz = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, device);
    uint32_t *d_out = nullptr, *buf = nullptr;
    const size_t l2_bytes = 64ull << 20;
    cudaEvent_t e0, e1;
    if (cudaMalloc(&d_out, 1 << 16) != cudaSuccess || cudaMalloc(&buf, l2_bytes) != cudaSuccess)
        return nfc::set_fail(NFC_ENOMEM, "nfc_measure_peaks: cudaMalloc failed");
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const uint32_t iters = 4096, k = 0x5bd1e995u;
    const int grid = sms * 4, block = 512;
    const double threads = (double)grid * block;
    float ms = time_ms([&] { k_alu<<<grid, block>>>(d_out, iters, k); }, e0, e1);
    out->alu_tops = threads * iters * UNR * CH * 4 / (ms * 1e-3) / 1e12;
    ms = time_ms([&] { k_issue<<<grid, block>>>(d_out, iters, k); }, e0, e1);
    out->issue_tops = threads * iters * UNR * CH * 4 / (ms * 1e-3) / 1e12;
    const uint32_t mask = 16384 - 1;   // 64 KiB table
    cudaFuncSetAttribute(k_smem, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
    const int sgrid = sms * 2, sblock = 1024;
    ms = time_ms([&] { k_smem<<<sgrid, sblock, 65536>>>(d_out, iters, mask); }, e0, e1);
    out->smem_glookups = (double)sgrid * sblock * iters * UNR * 4 / (ms * 1e-3) / 1e9;
    k_touch<<<sms * 4, 512>>>(buf, l2_bytes / 4);
    const uint32_t smask = (uint32_t)(l2_bytes / 32) - 1;
    const uint32_t l2it = 256;
    ms = time_ms([&] { k_l2<<<grid, block>>>(buf, d_out, l2it, smask); }, e0, e1);
    out->l2_gsectors = threads * l2it * UNR / (ms * 1e-3) / 1e9;
    out->sm_count = (uint32_t)sms;
    out->sm_clock_mhz = (uint32_t)(clk_khz / 1000);
    cudaError_t e = cudaDeviceSynchronize();
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(d_out);
    cudaFree(buf);
    if (e != cudaSuccess) return nfc::set_fail(NFC_ECUDA, std::string("nfc_measure_peaks: ") + cudaGetErrorString(e));
    return NFC_OK;
}
