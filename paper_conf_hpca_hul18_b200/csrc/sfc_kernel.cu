// sfc_kernel.cu -- variant selection and dispatch for the fused SFC kernel
// (sfc_kernel.cuh), plus the RSS steering kernel for multi-GPU sharding.
// The kernel instantiations live in sfc_inst_*.cu (compiled in parallel).
#include "sfc_kernel.cuh"

namespace nfc {

NFC_DECLARE_LAUNCH(SIG_C1, DM_FULL)
NFC_DECLARE_LAUNCH(SIG_C1, DM_HOT)
NFC_DECLARE_LAUNCH(SIG_K2, DM_FULL)
NFC_DECLARE_LAUNCH(SIG_K2, DM_HOT)
NFC_DECLARE_LAUNCH(SIG_K4, DM_FULL)
NFC_DECLARE_LAUNCH(SIG_K4, DM_HOT)
NFC_DECLARE_LAUNCH(SIG_C2, DM_HOT)
NFC_DECLARE_LAUNCH(SIG_C3, DM_HOT)
NFC_DECLARE_LAUNCH(SIG_K1, DM_HOT)
NFC_DECLARE_LAUNCH(SIG_C4, DM_HOT)
NFC_DECLARE_LAUNCH(SIG_K5, DM_HOT)
NFC_DECLARE_LAUNCH(SIG_K6, DM_HOT)
NFC_DECLARE_LAUNCH(SIG_N3, DM_HOT)
NFC_DECLARE_LAUNCH(SIG_ANY, DM_HOT)
#if NFC_REGROUP
NFC_DECLARE_LAUNCH_RG(SIG_C1, DM_FULL)
NFC_DECLARE_LAUNCH_RG(SIG_K2, DM_FULL)
NFC_DECLARE_LAUNCH_RG(SIG_K4, DM_FULL)
#define NFC_RG_OR(S) (v.rg ? launch_t<S, DM_FULL, true>(p, dev, stream, err, cfg, q) : launch_t<S, DM_FULL, false>(p, dev, stream, err, cfg, q))
#else
#define NFC_RG_OR(S) launch_t<S, DM_FULL, false>(p, dev, stream, err, cfg, q)
#endif

// chains with a DM_FULL instantiation (no IPsec: the DFA takes the whole CTA's shared memory)
static bool has_full(uint32_t sig) { return sig == SIG_C1 || sig == SIG_K2 || sig == SIG_K4; }
static bool known(uint32_t sig)
{
    return has_full(sig) || sig == SIG_C2 || sig == SIG_C3 || sig == SIG_K1 || sig == SIG_C4 || sig == SIG_K5 ||
           sig == SIG_K6 || sig == SIG_N3;
}

Variant sfc_variant(const uint32_t *kinds, uint32_t n, bool dfa_full)
{
    uint32_t sig = n << 28;
    bool esp = false;
    for (uint32_t i = 0; i < n; i++) {
        sig |= kinds[i] << (4 * i);
        esp |= kinds[i] == NFC_IPSEC;
    }
    Variant v{};
    if (!known(sig)) sig = SIG_ANY;
    v.sig = sig;
    v.dm = (dfa_full && has_full(sig)) ? DM_FULL : DM_HOT;
    v.esp = esp;
    v.threads = kcfg_threads(sig, v.dm);
    return v;
}

size_t sfc_smem_bytes(const Variant &v, const KParams &p)
{
    return smem_layout(p.present & sig_mask(v.sig), v.threads / 32, p, kcfg_nws(v.sig), v.dm).total;
}

size_t sfc_smem_limit(int device)
{
    int v = 0;
    cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, device);
    return (size_t)v;
}

static int dispatch(const Variant &v, const KParams &p, int dev, void *stream, std::string &err, LaunchCfg *cfg,
                    bool q)
{
#define NFC_CASE(S)                                                                                        \
    if (v.sig == S) return v.dm == DM_FULL ? NFC_RG_OR(S) : launch_t<S, DM_HOT, false>(p, dev, stream, err, cfg, q);
    NFC_CASE(SIG_C1)
    NFC_CASE(SIG_K2)
    NFC_CASE(SIG_K4)
#undef NFC_CASE
#define NFC_CASE(S) if (v.sig == S) return launch_t<S, DM_HOT, false>(p, dev, stream, err, cfg, q);
    NFC_CASE(SIG_C2)
    NFC_CASE(SIG_C3)
    NFC_CASE(SIG_K1)
    NFC_CASE(SIG_C4)
    NFC_CASE(SIG_K5)
    NFC_CASE(SIG_K6)
    NFC_CASE(SIG_N3)
#undef NFC_CASE
    return launch_t<SIG_ANY, DM_HOT, false>(p, dev, stream, err, cfg, q);
}

int sfc_launch(const Variant &v, const KParams &p, int device, void *stream, std::string &err, LaunchCfg *cfg_out)
{
    return dispatch(v, p, device, stream, err, cfg_out, false);
}

int sfc_query(const Variant &v, const KParams &p, int device, LaunchCfg *cfg_out)
{
    std::string err;
    return dispatch(v, p, device, nullptr, err, cfg_out, true);
}

// ---------------------------------------------------------------- multi-batch chunk records
// One thread per 32-packet chunk: the batch holding the chunk's first packet (binary
// search over the batch starts; among equal starts the last batch, i.e. the non-empty
// one), its descriptor pointers rebased so that packet g of the call indexes them
// directly, and where the next batch begins inside the chunk (ChunkRec).
__global__ void k_chunk_recs(const BatchDev *B, uint32_t nb, uint32_t n, ChunkRec *out)
{
    const uint32_t c = blockIdx.x * blockDim.x + threadIdx.x;
    const uint32_t g0 = c * 32;
    if (g0 >= n) return;
    uint32_t lo = 0, hi = nb - 1;
    while (lo < hi) {
        const uint32_t mid = (lo + hi + 1) >> 1;
        if (B[mid].start <= g0) lo = mid; else hi = mid - 1;
    }
    const BatchDev b = B[lo];
    const uint32_t end = min(g0 + 32, n);
    uint32_t split = 0, cnt = 0;
    for (uint32_t j = lo + 1; j < nb && B[j].start < end; j++)
        if (B[j].n) {
            if (!cnt) split = B[j].start - g0;
            cnt++;
        }
    ChunkRec r;
    r.offp = b.off - b.start;
    r.lenp = b.len - b.start;
    r.arena = b.arena;
    r.gb_lo = (uint32_t)b.first - b.start;
    r.meta = split | (cnt > 1 ? 32u : 0u);
    out[c] = r;
}

int chunk_recs_launch(const BatchDev *batches, uint32_t n_batches, uint32_t n_pkts, ChunkRec *out, void *stream,
                      std::string &err)
{
    const uint32_t chunks = (n_pkts + 31) / 32;
    if (!chunks) return NFC_OK;
    k_chunk_recs<<<(chunks + 255) / 256, 256, 0, (cudaStream_t)stream>>>(batches, n_batches, n_pkts, out);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) { err = std::string("k_chunk_recs: ") + cudaGetErrorString(e); return NFC_ECUDA; }
    return NFC_OK;
}

// ---------------------------------------------------------------- RSS steering
// Receive Side Steering: shard = RETA[Toeplitz(MS key, src|dst|sport|dport) & 127]
// with RETA[i] = i mod n_shards.  For n_shards | 64 every ESP SA (hash mod n_sa, n_sa = 64)
// maps to exactly one shard.  Frames that fail to parse go to shard 0.
__global__ void rss_shard_kernel(const uint8_t *arena, const uint64_t *off, const uint16_t *len, uint32_t n,
                                 const uint32_t *nib, uint32_t n_shards, uint8_t *out)
{
    __shared__ uint32_t snib[72 * 16];
    for (uint32_t i = threadIdx.x; i < 72 * 16; i += blockDim.x) snib[i] = __ldg(nib + i);
    __syncthreads();
    const uint64_t pol = pol_first();
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
        const uint8_t *f = arena + off[i];
        const uint32_t fl = len[i];
        uint32_t h[16];
        load_header(f, fl, h, pol);
        PV v;
        uint32_t hsh = 0;
        if (parse(h, f, fl, v)) hsh = toeplitz(snib, v);
        out[i] = (uint8_t)((hsh & 127) % n_shards);
    }
}

int rss_shard_launch(const uint8_t *arena, const uint64_t *off, const uint16_t *len, uint32_t n, const uint32_t *nib,
                     uint32_t n_shards, uint8_t *out, void *stream, std::string &err)
{
    if (!n) return NFC_OK;
    const uint32_t grid = min((n + 255) / 256, 148u * 8u);
    rss_shard_kernel<<<grid, 256, 0, (cudaStream_t)stream>>>(arena, off, len, n, nib, n_shards, out);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) { err = cudaGetErrorString(e); return NFC_ECUDA; }
    return NFC_OK;
}

} // namespace nfc
