// sfc_kernel.cuh -- the fused, persistent SFC kernel for sm_100a (device code and
// the launch template; instantiated per chain signature in sfc_inst_*.cu).
//
// One launch drains all packets of an nfc_process_batch call.  Every thread
// carries one packet through the whole chain in registers:
//   parse once (the de-duplicated header classifier)
//   -> NFs in original SFC order, a dropped packet skipping every later NF
//      (early drop; no batch re-split or per-NF launch)
//   -> one 16 B result record; counters in per-warp private shared memory.
// NF synthesis is done at compile time: the chain's kinds are a
// template "signature", so the NF sequence is straight-line code with no
// per-packet dispatch; one SIG_ANY instantiation interprets any other chain.
// Scheduling (persistent kernel, P:L112, P:L235 [SIV]): without IPsec each warp
// claims 32-packet chunks from a global atomic counter (no CTA barriers); with
// IPsec each CTA claims tiles in order and assigns per-SA ESP sequence numbers
// in global packet order by a decoupled look-back.
// Tables stay on chip where they fit: the ACL bit-vector image, the Aho-Corasick
// DFA (entirely, DM_FULL; or its hot rows, DM_HOT), AES T-tables and Toeplitz
// nibble tables live in shared memory; DIR-24-8 / IPv6 hash levels are read
// through L2 with an evict-last policy while the packet stream is evict-first.
// Packet bytes are read from HBM once and rewritten in place.  No tensor cores:
// nothing here is a dense contraction.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "nfc_internal.h"

namespace nfc {

static constexpr int DPI_LIST = 16;     // distinct matches kept in a list before the bitmap path
static constexpr int NFIX = ST_VAR_BASE;
static constexpr int NWS = ST_POS_BASE + 4 * NFC_MAX_CHAIN;   // per-warp counter slots

// ---------------------------------------------------------------- chain signatures
// n_nf in bits 28..31, the NF kind of position p in bits 4p..4p+3; SIG_ANY = 0
// interprets P.kind at run time.
static constexpr uint32_t SIG_ANY = 0;
__host__ __device__ constexpr uint32_t sig_n(uint32_t s) { return s >> 28; }
__host__ __device__ constexpr uint32_t sig_kind(uint32_t s, int p) { return (s >> (4 * p)) & 15u; }
__host__ __device__ constexpr uint32_t sig_mask(uint32_t s)
{
    if (s == SIG_ANY) return (1u << NFC_ACL) | (1u << NFC_DPI) | (1u << NFC_LPM4) | (1u << NFC_LPM6) |
                             (1u << NFC_IPSEC) | (1u << NFC_LB) | (1u << NFC_NAT);
    uint32_t m = 0;
    for (int p = 0; p < (int)sig_n(s); p++) m |= 1u << sig_kind(s, p);
    return m;
}
__host__ __device__ constexpr uint32_t sig_pos(uint32_t s, uint32_t kind)
{
    for (int p = 0; p < (int)sig_n(s); p++)
        if (sig_kind(s, p) == kind) return (uint32_t)p;
    return 0xFF;
}
__host__ __device__ constexpr uint32_t make_sig(uint32_t n, uint32_t k0, uint32_t k1 = 0, uint32_t k2 = 0, uint32_t k3 = 0, uint32_t k4 = 0,
                            uint32_t k5 = 0)
{
    return n << 28 | k0 | k1 << 4 | k2 << 8 | k3 << 12 | k4 << 16 | k5 << 20;
}


// ---------------------------------------------------------------- tuning knobs (compile-time; defaults = measured best)
#ifndef NFC_EARLY_T24
#define NFC_EARLY_T24 0       // issue the DIR-24-8 first read right after parse, use it at LPM4
#endif
#ifndef NFC_DEFER_PAIRS
#define NFC_DEFER_PAIRS 0     // 1: claim match-pair slots at DPI, write the pairs at the end of the chunk
#endif
#ifndef NFC_LOOKBACK_WIN
#define NFC_LOOKBACK_WIN 1    // ESP sequence look-back over 32 predecessor tiles per step
#endif
#ifndef NFC_TIE
#define NFC_TIE 1             // DM_HOT: order class lookups after the walk state (register pressure)
#endif
#ifndef NFC_CLAIM
#define NFC_CLAIM 4           // 32-packet chunks a warp claims per atomic (DM_FULL; DM_HOT: 1)
#endif
#ifndef NFC_SPEC
#define NFC_SPEC 1            // speculative ACL || DPI head walk || TBL24 block (spec_ok)
#endif
#ifndef NFC_T24_NA
#define NFC_T24_NA 1          // DIR-24-8 reads bypass L1
#endif
#ifndef NFC_PF_LATE
#define NFC_PF_LATE 1         // frame L2 prefetch of the next chunk issued after the chain's head part
#endif
#ifndef NFC_ESP_PF
#define NFC_ESP_PF 1          // prefetch the whole frame into L2 when ESP starts on it (+1 %)
#endif
#ifndef NFC_ESP_MINB
#define NFC_ESP_MINB 2        // IPsec chains: resident 256-thread tiles per SM (launch bounds)
#endif
#ifndef NFC_ESP_RK_SMEM
#define NFC_ESP_RK_SMEM 1     // ESP reads AES round keys from shared memory (one out-of-line block cipher; C2 +11 %)
#endif
#ifndef NFC_SPEC_V6
#define NFC_SPEC_V6 0         // 1: dual-stack warps take the speculative block in every chain (IPv6 lanes re-classified)
#endif
#ifndef NFC_HOT_FAST
#define NFC_HOT_FAST 0        // 1: DM_HOT split walk takes the unconditional 16-byte step too
#endif
#ifndef NFC_CARRY_DESC
#define NFC_CARRY_DESC 1      // carry the next chunk's off/len in registers from the loop top (C1 +2 %)
#endif
#ifndef NFC_DESC_L1
#define NFC_DESC_L1 1         // descriptors prefetched into L1 two chunks ahead instead of held in registers (C1 +11 %)
#endif
#ifndef NFC_RGQ
#define NFC_RGQ 48            // per-warp queue words in shared memory (47 packet indices + the length)
#endif
#ifndef NFC_T24_L2_EARLY
#define NFC_T24_L2_EARLY 0    // 1: the DIR-24-8 second-level read issued right after the speculative block
#endif
#ifndef NFC_FWD_DERIVED
#define NFC_FWD_DERIVED 0     // 1: the forwarded count derived at the flush (pkts - parse drops - NF drops)
#endif
#ifndef NFC_LD256
#define NFC_LD256 1           // 256-bit header loads / rewrite stores for 32-B aligned frames
#endif
#ifndef NFC_WALK_AHEAD
#define NFC_WALK_AHEAD 0      // 1: split-walk payload words loaded one 16-B step ahead
#endif
#ifndef NFC_HDR_AHEAD
#define NFC_HDR_AHEAD 0       // 1: load the next chunk's header at the tail of the current one
#endif
#ifndef NFC_FULL_THREADS
#define NFC_FULL_THREADS 640   // DPI chains without IPsec: one CTA per SM (640: no spills at 96 regs)
#endif
#ifndef NFC_HOTBIG_THREADS
#define NFC_HOTBIG_THREADS 768 // DPI chains without IPsec whose DFA is tiered (DM_HOT)
#endif
#ifndef NFC_HOT_MINB
#define NFC_HOT_MINB 3         // DM_HOT chains without IPsec: resident 256-thread CTAs per SM
#endif
// Launch shape: DPI chains without IPsec run one big CTA per SM (the DFA -- all of it,
// or as many hot rows as fit -- is staged once per SM); IPsec chains run 256-thread
// tiles (ESP sequence order), the rest 256-thread CTAs at NFC_HOT_MINB per SM.
__host__ __device__ constexpr bool kcfg_big(uint32_t S)
{
    return S != SIG_ANY && !(sig_mask(S) & (1u << NFC_IPSEC)) && (sig_mask(S) & (1u << NFC_DPI));
}
#ifndef NFC_ESP_DPI_THREADS
#define NFC_ESP_DPI_THREADS 512   // IPsec chains with DPI: one 512-packet tile per SM (the DFA tiers get the SM's shared memory)
#endif
__host__ __device__ constexpr bool kcfg_esp_dpi(uint32_t S)
{
    return S != SIG_ANY && (sig_mask(S) & (1u << NFC_IPSEC)) && (sig_mask(S) & (1u << NFC_DPI));
}
__host__ __device__ constexpr int kcfg_threads(uint32_t S, int dm)
{
    return kcfg_big(S) ? (dm == DM_FULL ? NFC_FULL_THREADS : NFC_HOTBIG_THREADS) : kcfg_esp_dpi(S) ? NFC_ESP_DPI_THREADS : 256;
}
// per-warp counter slots: the fixed counters + 4 per chain position
__host__ __device__ constexpr int kcfg_nws(uint32_t S) { return ST_POS_BASE + 4 * (S == SIG_ANY ? NFC_MAX_CHAIN : (int)sig_n(S)); }
// chains whose warp loop regroups mixed IPv4/IPv6 chunks (NFC_REGROUP): the ones with the
// IPv4 speculative ACL || DPI block, i.e. ACL -> DPI first with the whole DFA on chip
__host__ __device__ constexpr bool rg_sig(uint32_t S, int dm)
{
    return S != SIG_ANY && dm == DM_FULL && sig_n(S) >= 2 && sig_kind(S, 0) == NFC_ACL && sig_kind(S, 1) == NFC_DPI;
}
template <uint32_t S, int DM> struct KCfg {
    static constexpr int nws = kcfg_nws(S);
    static constexpr bool esp = (sig_mask(S) & (1u << NFC_IPSEC)) != 0;
    static constexpr int threads = kcfg_threads(S, DM);
    static constexpr int minb = esp ? (kcfg_threads(S, DM) > 256 ? 1 : NFC_ESP_MINB) : (kcfg_big(S) ? 1 : NFC_HOT_MINB);
    static constexpr int nwarp = threads / 32;
    static constexpr uint32_t claim = DM == DM_FULL ? NFC_CLAIM : 1;   // chunks per warp claim
};

// ---------------------------------------------------------------- shared memory layout
// the kernels' dynamic shared memory (one symbol: device functions address it directly,
// with region offsets from P.lay in the constant bank -- no per-thread base registers)
extern __shared__ __align__(16) uint8_t nfc_smem[];
__host__ __device__ inline SmemLayout smem_layout(uint32_t mask, int nwarp, const KParams &p, int nws = NWS, int dm = DM_HOT)
{
    SmemLayout L{};
    uint32_t o = 0;
    // the DPI byte-class table first: offset 0 is a compile-time address for the walk
    if (mask & MASK_DPI) { L.cls = o; o += dm == DM_FULL ? 256 : 256 * 4; }
    L.wst = o; o += nwarp * nws * 8;                                // per-warp private counters (u64)
    L.vst = o; o += (p.smem_stats ? p.stats_len - NFIX : 0) * 4;  // ACL/LB/SA hit counters (u32)
    o = (o + 15) & ~15u;
    if (mask & MASK_IPSEC) {
        L.te = o; o += 256 * 32 * 4; L.ms_nib = o; o += 72 * 16 * 4;
#if NFC_ESP_RK_SMEM
        L.rk = o; o += ((p.esp.n_sa * ESP_RK_STRIDE * 4) + 15) & ~15u;
#endif
    }
    if (mask & MASK_LB) { L.lb_nib = o; o += 72 * 16 * 4; }
    if (mask & MASK_NAT) { L.nat_nib = o; o += 72 * 16 * 4; }
    if (mask & MASK_DPI) {
        // L.cls (byte -> 2 * class, u8 / u32) sits at offset 0 (above)
        L.hot = o; o += (p.dpi.hot_states * p.dpi.ncls * 2 + 15) & ~15u;
        L.frow0 = L.hot + p.dpi.n_acc * p.dpi.ncls * 2;            // DM_FULL slot rows
        L.sp = o; o += p.dpi.sparse_states * 8;
        // match summaries: DM_FULL of the accepting slots only, else of every state
        L.meta = o; o += p.dpi.meta_smem ? ((dm == DM_FULL ? p.dpi.n_acc : p.dpi.n_states) * 4 + 15) & ~15u : 0;
        L.seg = o; o += nwarp * 64 * 4;                             // split-walk accumulators (cnt, mx) x 32
    }
    o = (o + 15) & ~15u;
    if (mask & MASK_ACL) {
        const uint32_t s4 = p.acl.smem_words ? (p.acl.fast ? p.acl.words_f4 : p.acl.words4) : 0,
                       s6 = p.acl.smem_words ? p.acl.words6 : 0;
        L.acl4 = o; o += s4 * 4;
        L.acl6 = o; o += s6 * 4;
    }
    o = (o + 15) & ~15u;
    if ((mask & MASK_LPM4) && p.l4.nh_smem) { L.nh4 = o; o += p.l4.n_nh * 16; }
    if (p.n_batches > 1 && !(mask & MASK_IPSEC)) { L.crs = o; o += nwarp * 64; }
    if (NFC_REGROUP && dm == DM_FULL && (mask & MASK_ACL) && (mask & MASK_DPI) && !(mask & MASK_IPSEC)) { L.rgq = o; o += nwarp * NFC_RGQ * 4; }
    if (mask & MASK_IPSEC) {
        L.wcnt = o; o += nwarp * 256 * 2;
        L.prefix = o; o += (max(256, nwarp * 32) + 64) * 4;   // esp_assign prefixes; esp_ctr_tile block prefix + warp totals
    }
    L.total = o;
    return L;
}

// ---------------------------------------------------------------- small helpers
__device__ __forceinline__ uint32_t bswap32(uint32_t x) { return __byte_perm(x, 0, 0x0123); }
__device__ __forceinline__ uint32_t ld_acquire(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(uint32_t *p, uint32_t v)
{
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t mask32d(int len) { return len <= 0 ? 0u : len >= 32 ? 0xFFFFFFFFu : 0xFFFFFFFFu << (32 - len); }

// L2 eviction policies: the packet stream is touched once (evict-first); lookup
// tables are re-used by every packet (evict-last).
__device__ __forceinline__ uint64_t pol_first()
{
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t pol_last()
{
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint4 ld_stream16(const void *a, uint64_t pol)
{
    uint4 v;
    asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(a), "l"(pol));
    return v;
}
// 32-B (256-bit) versions: one L1TEX data-pipe wavefront per 128-B line for twice the
// bytes of a 16-B access -- the fused kernel's header loads and rewrite stores touch
// 16 lines per warp instruction (32 frames), so they cost half the wavefronts (needs a
// 32-B aligned address)
__device__ __forceinline__ void ld_stream32(const void *a, uint64_t pol, uint32_t *v)
{
    asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
                 : "l"(a), "l"(pol));
}
__device__ __forceinline__ void st_stream32(void *a, const uint32_t *v, uint64_t pol)
{
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8}, %9;"
                 ::"l"(a), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ void st_stream16(void *a, uint4 v, uint64_t pol)
{
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.u32 [%0], {%1,%2,%3,%4}, %5;"
                 ::"l"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "l"(pol) : "memory");
}
__device__ __forceinline__ uint32_t ld_tab16(const uint16_t *a, uint64_t pol)
{
    uint16_t v;
#if NFC_T24_NA
    // DIR-24-8 reads are random over 32 MB: keep them out of L1 (the descriptors and the
    // next-hop records live there)
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.u16 %0, [%1], %2;" : "=h"(v) : "l"(a), "l"(pol));
#else
    asm("ld.global.nc.L2::cache_hint.u16 %0, [%1], %2;" : "=h"(v) : "l"(a), "l"(pol));
#endif
    return v;
}
// predicated read-only u16 load: returns `dflt` when !p (no memory access)
__device__ __forceinline__ uint32_t ld_u16_if(bool p, const uint16_t *a, uint32_t dflt)
{
    uint32_t v = dflt;
    asm("{\n\t.reg .pred q;\n\t.reg .u16 t;\n\tsetp.ne.u32 q, %2, 0;\n\t@q ld.global.nc.u16 t, [%1];\n\t@q cvt.u32.u16 %0, t;\n\t}"
        : "+r"(v) : "l"(a), "r"((uint32_t)p));
    return v;
}

// A DPI walk is a dependent chain of shared-memory lookups, so the bytes ahead of it are
// prefetched into L2 (NFC_PF_DIST bytes ahead, one 128-B line at a time).
#ifndef NFC_PF_DIST
#define NFC_PF_DIST 512       // split walk: L2 prefetch distance (bytes) ahead of each lane
#endif
__device__ __forceinline__ void prefetch_l2(const void *a) { asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(a)); }

// byte k (0..63) of the 64 B header cache; k compile-time in hot paths
__device__ __forceinline__ uint32_t hbyte(const uint32_t h[16], uint32_t k) { return (h[k >> 2] >> ((k & 3) * 8)) & 0xFF; }
// big-endian 32/16-bit fields at byte k: one PRMT of the two words spanning them (k
// compile-time at every call site, so the word indices and the selector fold)
__device__ __forceinline__ uint32_t hbe32(const uint32_t h[16], uint32_t k)
{
    const uint32_t i = k >> 2, r = k & 3;
    const uint32_t hi = i + 1 < 16 ? h[i + 1] : 0u;
    return __byte_perm(h[i], hi, r << 12 | (r + 1) << 8 | (r + 2) << 4 | (r + 3));
}
__device__ __forceinline__ uint32_t hbe16(const uint32_t h[16], uint32_t k) { return hbe32(h, k) >> 16; }
// ---------------------------------------------------------------- per-packet state
struct PV {
    uint32_t fam;                 // 4 or 6
    uint32_t l4_off, ip_end, pl_off;
    uint32_t proto, sport, dport;
    uint32_t src[4], dst[4];      // big-endian-valued words
};

__device__ __forceinline__ void load_header(const uint8_t *f, uint32_t flen, uint32_t h[16], uint64_t pol)
{
    const uint32_t nch = min(4u, (flen + 15) >> 4);
#if NFC_LD256
    // frames of >= 64 B at 32-B aligned offsets (every 64-B-multiple ring): two 256-bit loads
    if (nch == 4 && (reinterpret_cast<uintptr_t>(f) & 31) == 0) {
        ld_stream32(f, pol, h);
        ld_stream32(f + 32, pol, h + 8);
        return;
    }
#endif
#pragma unroll
    for (int c = 0; c < 4; c++) {
        uint4 v = c < (int)nch ? ld_stream16(f + 16 * c, pol) : make_uint4(0, 0, 0, 0);
        h[4 * c] = v.x; h[4 * c + 1] = v.y; h[4 * c + 2] = v.z; h[4 * c + 3] = v.w;
    }
}

// L4 fields outside the 64-B header cache (IPv4 options): rare, from memory
static __device__ __noinline__ uint32_t l4_fields_mem(const uint8_t *f, uint32_t l4, uint32_t tcp)
{
    const uint32_t ports = (uint32_t)f[l4] << 24 | (uint32_t)f[l4 + 1] << 16 | (uint32_t)f[l4 + 2] << 8 | f[l4 + 3];
    (void)tcp;
    return ports;
}
static __device__ __noinline__ uint32_t tcp_doff_mem(const uint8_t *f, uint32_t l4) { return (uint32_t)f[l4 + 12] >> 4; }

// Parse (P:L87 validity check): Ethernet -> IPv4/IPv6 -> UDP/TCP.
__device__ __forceinline__ bool parse(const uint32_t h[16], const uint8_t *f, uint32_t flen, PV &v)
{
    // fast path, the common frames: Ethernet / IPv4 (IHL 5, not a fragment) / UDP or TCP
    // with the L4 header in the header cache (words are little-endian: byte 12 is the
    // low byte of h[3]); anything else, valid or not, takes the general parse below
    {
        const uint32_t pr = h[5] >> 24;
        if ((h[3] & 0x00FFFFFFu) == 0x00450008u && (h[5] & 0x0000FF3Fu) == 0 && (pr == 17 || pr == 6)) {
            const uint32_t tot = __byte_perm(h[4], 0, 0x4401);
            const uint32_t doff = (h[11] >> 20) & 15;                  // TCP data offset, byte 46
            const uint32_t l4len = pr == 6 ? 4 * doff : 8;
            if (14 + tot <= flen && l4len + 20 <= tot && (pr == 17 || doff >= 5)) {
                v.fam = 4;
                v.l4_off = 34;
                v.ip_end = 14 + tot;
                v.pl_off = 34 + l4len;
                v.proto = pr;
                v.src[0] = __byte_perm(h[6], h[7], 0x2345);
                v.dst[0] = __byte_perm(h[7], h[8], 0x2345);
                v.src[1] = v.src[2] = v.src[3] = v.dst[1] = v.dst[2] = v.dst[3] = 0;
                const uint32_t ports = __byte_perm(h[8], h[9], 0x2345);
                v.sport = ports >> 16;
                v.dport = ports & 0xFFFF;
                return true;
            }
        }
    }
    if (flen < 14) return false;
    const uint32_t et = hbe16(h, 12);
    bool frag = false;
    if (et == 0x0800) {
        if (flen < 34) return false;
        const uint32_t vi = hbyte(h, 14);
        if ((vi >> 4) != 4) return false;
        const uint32_t ihl = vi & 15;
        if (ihl < 5) return false;
        const uint32_t tot = hbe16(h, 16);
        if (tot < 4 * ihl || 14 + tot > flen) return false;
        v.fam = 4;
        v.l4_off = 14 + 4 * ihl;
        v.ip_end = 14 + tot;
        v.proto = hbyte(h, 23);
        v.src[0] = hbe32(h, 26);
        v.dst[0] = hbe32(h, 30);
        v.src[1] = v.src[2] = v.src[3] = v.dst[1] = v.dst[2] = v.dst[3] = 0;
        const uint32_t fo = hbe16(h, 20);
        frag = (fo & 0x3FFF) != 0;       // MF set or non-zero offset
    } else if (et == 0x86DD) {
        if (flen < 54) return false;
        if ((hbyte(h, 14) >> 4) != 6) return false;
        const uint32_t pl = hbe16(h, 18);
        if (54 + pl > flen) return false;
        v.fam = 6;
        v.l4_off = 54;
        v.ip_end = 54 + pl;
        v.proto = hbyte(h, 20);
#pragma unroll
        for (int k = 0; k < 4; k++) { v.src[k] = hbe32(h, 22 + 4 * k); v.dst[k] = hbe32(h, 38 + 4 * k); }
    } else {
        return false;
    }
    uint32_t l4len = 0;
    v.sport = v.dport = 0;
    if (!frag && (v.proto == 17 || v.proto == 6)) {
        const uint32_t l4 = v.l4_off;
        const bool tcp = v.proto == 6;
        if (l4 + (tcp ? 20u : 8u) > v.ip_end) return false;
        l4len = 8;
        if (tcp) {
            // data offset: byte 46 sits in the header cache; other offsets are rare -> memory
            const uint32_t doff = l4 == 34 ? hbyte(h, 46) >> 4 : tcp_doff_mem(f, l4);
            if (doff < 5 || l4 + 4 * doff > v.ip_end) return false;
            l4len = 4 * doff;
        }
        uint32_t ports;
        if (l4 == 34) ports = hbe32(h, 34);
        else if (l4 == 54) ports = hbe32(h, 54);
        else ports = l4_fields_mem(f, l4, tcp);
        v.sport = ports >> 16;
        v.dport = ports & 0xFFFF;
    }
    v.pl_off = v.l4_off + l4len;
    return true;
}

// ---------------------------------------------------------------- ACL
// Bit-vector first match: five interval lookups, AND of the five rule bitsets,
// lowest set bit.  Each interval lookup is a bucket read on the top 8 key bits
// followed by a fixed-depth window search whose depth is a table property
// (warp-uniform trip count, no per-key divergence).  Header words come from the
// kernel parameters (constant bank), not from the image.
__device__ __forceinline__ bool le128(const uint4 b, const uint32_t k[4])
{
    if (b.x != k[0]) return b.x < k[0];
    if (b.y != k[1]) return b.y < k[1];
    if (b.z != k[2]) return b.z < k[2];
    return b.w <= k[3];
}

// bucket t of a field's 257-entry u16 bucket table at word offset o
__device__ __forceinline__ uint32_t acl_bucket(const uint32_t *A, uint32_t o, uint32_t t)
{
    return reinterpret_cast<const uint16_t *>(A + o)[t];
}

// returns global rule index (0xFFFF none) | action << 31
__device__ __forceinline__ uint32_t acl_match(const uint32_t *A, const uint32_t *hd, uint32_t default_action,
                                              uint32_t js, uint32_t jd, uint32_t jsp, uint32_t jdp, uint32_t proto)
{
    const uint32_t W = hd[1];
    js = min(js, hd[2] - 1);
    jd = min(jd, hd[3] - 1);
    jsp = min(jsp, hd[4] - 1);
    jdp = min(jdp, hd[5] - 1);
    const uint64_t *vs = reinterpret_cast<const uint64_t *>(A + hd[9]) + (size_t)js * W;
    const uint64_t *vd = reinterpret_cast<const uint64_t *>(A + hd[11]) + (size_t)jd * W;
    const uint64_t *vsp = reinterpret_cast<const uint64_t *>(A + hd[13]) + (size_t)jsp * W;
    const uint64_t *vdp = reinterpret_cast<const uint64_t *>(A + hd[15]) + (size_t)jdp * W;
    const uint64_t *vpr = reinterpret_cast<const uint64_t *>(A + hd[16]) + (size_t)proto * W;
    if (W == 1) {
        const uint64_t x = vs[0] & vd[0] & vsp[0] & vdp[0] & vpr[0];
        return x ? A[hd[17] + (__ffsll((long long)x) - 1)] : 0xFFFFu | default_action << 31;
    }
    // aggregate level: only words whose five rows are all non-zero are examined, in order
    const uint32_t WA = hd[29];
    const uint64_t *as = reinterpret_cast<const uint64_t *>(A + hd[24]) + (size_t)js * WA;
    const uint64_t *ad = reinterpret_cast<const uint64_t *>(A + hd[25]) + (size_t)jd * WA;
    const uint64_t *asp = reinterpret_cast<const uint64_t *>(A + hd[26]) + (size_t)jsp * WA;
    const uint64_t *adp = reinterpret_cast<const uint64_t *>(A + hd[27]) + (size_t)jdp * WA;
    const uint64_t *apr = reinterpret_cast<const uint64_t *>(A + hd[28]) + (size_t)proto * WA;
    for (uint32_t a = 0; a < WA; a++) {
        uint64_t cand = as[a] & ad[a] & asp[a] & adp[a] & apr[a];
        while (cand) {
            const uint32_t w = 64 * a + (__ffsll((long long)cand) - 1);
            const uint64_t x = vs[w] & vd[w] & vsp[w] & vdp[w] & vpr[w];
            if (x) return A[hd[17] + 64 * w + (__ffsll((long long)x) - 1)];
            cand &= cand - 1;
        }
    }
    return 0xFFFFu | default_action << 31;
}

// The four interval lookups (src, dst, sport, dport) run jointly: one bucket read
// each on the top 8 key bits, then one loop of the image's max window depth
// (a table property: warp-uniform trip count) with four independent compare
// steps per iteration.  Header words come from the constant bank.  Generic version
// (any image pointer; used by the unfused and parallel kernels).
__device__ __forceinline__ uint32_t nf_acl(const uint32_t *A4, const uint32_t *A6, const AclImg &ai, const PV &v)
{
    if (v.fam == 4) {
        const uint32_t *hd = ai.hdr4;
        if (hd[0] == 0) return 0xFFFFu | ai.default_action << 31;
        const uint32_t *A = A4;
        const uint32_t *Bs = A + hd[8], *Bd = A + hd[10], *Bsp = A + hd[12], *Bdp = A + hd[14];
        const uint32_t ks = v.src[0], kd = v.dst[0];
        uint32_t js = acl_bucket(A, hd[18], ks >> 24), jd = acl_bucket(A, hd[19], kd >> 24);
        uint32_t jsp = acl_bucket(A, hd[20], v.sport >> 8), jdp = acl_bucket(A, hd[21], v.dport >> 8);
        for (uint32_t h = (1u << hd[23]) >> 1; h; h >>= 1) {
            js = Bs[js + h] <= ks ? js + h : js;
            jd = Bd[jd + h] <= kd ? jd + h : jd;
            jsp = Bsp[jsp + h] <= v.sport ? jsp + h : jsp;
            jdp = Bdp[jdp + h] <= v.dport ? jdp + h : jdp;
        }
        return acl_match(A, hd, ai.default_action, js, jd, jsp, jdp, v.proto);
    }
    const uint32_t *hd = ai.hdr6;
    if (hd[0] == 0) return 0xFFFFu | ai.default_action << 31;
    const uint32_t *A = A6;
    const uint4 *Bs = reinterpret_cast<const uint4 *>(A + hd[8]), *Bd = reinterpret_cast<const uint4 *>(A + hd[10]);
    const uint32_t *Bsp = A + hd[12], *Bdp = A + hd[14];
    uint32_t js = acl_bucket(A, hd[18], v.src[0] >> 24), jd = acl_bucket(A, hd[19], v.dst[0] >> 24);
    uint32_t jsp = acl_bucket(A, hd[20], v.sport >> 8), jdp = acl_bucket(A, hd[21], v.dport >> 8);
    for (uint32_t h = (1u << hd[23]) >> 1; h; h >>= 1) {
        js = le128(Bs[js + h], v.src) ? js + h : js;
        jd = le128(Bd[jd + h], v.dst) ? jd + h : jd;
        jsp = Bsp[jsp + h] <= v.sport ? jsp + h : jsp;
        jdp = Bdp[jdp + h] <= v.dport ? jdp + h : jdp;
    }
    return acl_match(A, hd, ai.default_action, js, jd, jsp, jdp, v.proto);
}

// Fused-kernel version: the image is addressed in one known space -- shared memory
// (SM: 32-bit shared addresses, the image base a compile-time symbol plus a
// constant-bank offset) or global (read-only path, 32-bit byte offsets from one
// base) -- never through generic pointers.  The window search keeps byte offsets
// into the key arrays and is unrolled up to 8 halvings, each guarded by the image
// depth (constant bank, warp-uniform): a step is one load at a constant offset, a
// compare and a predicated add.
template <bool SM> struct AclMem {
    const uint8_t *g;     // global image (SM == false)
    uint32_t s;           // shared-memory byte offset of the image (SM == true)
    template <typename T> __device__ __forceinline__ T at(uint32_t o) const
    {
        if constexpr (SM) return *reinterpret_cast<const T *>(nfc_smem + s + o);
        else return __ldg(reinterpret_cast<const T *>(g + o));
    }
};
template <bool SM>
__device__ __forceinline__ uint32_t acl_match_w(const AclMem<SM> &M, const uint32_t *hd, uint32_t default_action,
                                                uint32_t js, uint32_t jd, uint32_t jsp, uint32_t jdp, uint32_t proto)
{
    js = min(js, hd[2] - 1);
    jd = min(jd, hd[3] - 1);
    jsp = min(jsp, hd[4] - 1);
    jdp = min(jdp, hd[5] - 1);
    const uint32_t W = hd[1];
    auto word = [&](uint32_t w, uint32_t &lo, uint32_t &hi) {
        const uint2 a = M.template at<uint2>(4 * hd[9] + 8 * (js * W + w));
        const uint2 b = M.template at<uint2>(4 * hd[11] + 8 * (jd * W + w));
        const uint2 c = M.template at<uint2>(4 * hd[13] + 8 * (jsp * W + w));
        const uint2 d = M.template at<uint2>(4 * hd[15] + 8 * (jdp * W + w));
        const uint2 e = M.template at<uint2>(4 * hd[16] + 8 * (proto * W + w));
        lo = a.x & b.x & c.x & d.x & e.x;
        hi = a.y & b.y & c.y & d.y & e.y;
    };
    uint32_t lo, hi;
    if (W == 1) {                 // up to 64 rules of the family
        word(0, lo, hi);
        if (lo | hi) return M.template at<uint32_t>(4 * (hd[17] + (lo ? __ffs(lo) - 1 : 31 + __ffs(hi))));
        return 0xFFFFu | default_action << 31;
    }
    // aggregate level (builders.cpp "ABV"): only words whose five rows are non-zero
    const uint32_t WA = hd[29];
    for (uint32_t a = 0; a < WA; a++) {
        const uint2 s0 = M.template at<uint2>(4 * hd[24] + 8 * (js * WA + a));
        const uint2 s1 = M.template at<uint2>(4 * hd[25] + 8 * (jd * WA + a));
        const uint2 s2 = M.template at<uint2>(4 * hd[26] + 8 * (jsp * WA + a));
        const uint2 s3 = M.template at<uint2>(4 * hd[27] + 8 * (jdp * WA + a));
        const uint2 s4 = M.template at<uint2>(4 * hd[28] + 8 * (proto * WA + a));
        uint64_t cand = (uint64_t)(s0.x & s1.x & s2.x & s3.x & s4.x) | (uint64_t)(s0.y & s1.y & s2.y & s3.y & s4.y) << 32;
        while (cand) {
            const uint32_t w = 64 * a + (__ffsll((long long)cand) - 1);
            word(w, lo, hi);
            if (lo | hi) return M.template at<uint32_t>(4 * (hd[17] + 64 * w + (lo ? __ffs(lo) - 1 : 31 + __ffs(hi))));
            cand &= cand - 1;
        }
    }
    return 0xFFFFu | default_action << 31;
}
__device__ __forceinline__ uint32_t lds_u32(uint32_t a)
{
    uint32_t v;
    asm("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint32_t lds_u16z(uint32_t a)
{
    uint32_t v;
    asm("{\n\t.reg .u16 t;\n\tld.shared.u16 t, [%1];\n\tcvt.u32.u16 %0, t;\n\t}" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint2 lds_u64(uint32_t a)
{
    uint2 v;
    asm("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
    return v;
}
// shared-memory window search over absolute 32-bit shared addresses: D halvings
// (compile-time), each a load at an immediate offset, a compare and a predicated add
template <uint32_t H4>
__device__ __forceinline__ void acl_step_s(uint32_t &a, uint32_t key)
{
    uint32_t v;
    asm("ld.shared.u32 %0, [%1+%2];" : "=r"(v) : "r"(a), "n"(H4));
    a += v <= key ? H4 : 0u;
}
template <int D>
__device__ __forceinline__ void acl_search4_s(uint32_t &as, uint32_t &ad, uint32_t &asp, uint32_t &adp, const PV &v)
{
    if constexpr (D > 0) {
        constexpr uint32_t H4 = 4u << (D - 1);
        acl_step_s<H4>(as, v.src[0]);
        acl_step_s<H4>(ad, v.dst[0]);
        acl_step_s<H4>(asp, v.sport);
        acl_step_s<H4>(adp, v.dport);
        acl_search4_s<D - 1>(as, ad, asp, adp, v);
    }
}
// IPv4 ACL from the search image (AclImg::f4) in shared memory at byte offset `img`:
// per field one bucket read and two or three window halvings at immediate offsets over the
// 4-B keys (the pad keys make overshooting the last interval harmless), then the
// bitset at the key's affine image; returns as acl_core.  Any key stays in bounds
// (dead lanes included).
__device__ __forceinline__ uint32_t acl4_fast(uint32_t img, const AclImg &ai, const PV &v)
{
    const uint32_t B = (uint32_t)__cvta_generic_to_shared(nfc_smem) + img;
    const uint32_t ks = v.src[0], kd = v.dst[0], ksp = v.sport & 0xFFFF, kdp = v.dport & 0xFFFF;
    constexpr uint32_t NB2 = 2 * ACLF_NB;
    uint32_t as = B + lds_u16z(B + ACLF_BK + 2 * (ks >> (32 - NFC_ACLF_BITS)));
    uint32_t ad = B + lds_u16z(B + ACLF_BK + NB2 + 2 * (kd >> (32 - NFC_ACLF_BITS)));
    uint32_t asp = B + lds_u16z(B + ACLF_BK + 2 * NB2 + 2 * (ksp >> (16 - NFC_ACLF_BITS)));
    uint32_t adp = B + lds_u16z(B + ACLF_BK + 3 * NB2 + 2 * (kdp >> (16 - NFC_ACLF_BITS)));
    if (ai.f4_d3) { acl_step_s<16>(as, ks); acl_step_s<16>(ad, kd); acl_step_s<16>(asp, ksp); acl_step_s<16>(adp, kdp); }
    acl_step_s<8>(as, ks); acl_step_s<8>(ad, kd); acl_step_s<8>(asp, ksp); acl_step_s<8>(adp, kdp);
    acl_step_s<4>(as, ks); acl_step_s<4>(ad, kd); acl_step_s<4>(asp, ksp); acl_step_s<4>(adp, kdp);
    // bitset address = 2 * key address + (bv - 2 key - B) per field
    const uint2 a = lds_u64(2 * as + (ai.f4_bv[0] - 2 * ai.f4_key[0] - B));
    const uint2 b = lds_u64(2 * ad + (ai.f4_bv[1] - 2 * ai.f4_key[1] - B));
    const uint2 c = lds_u64(2 * asp + (ai.f4_bv[2] - 2 * ai.f4_key[2] - B));
    const uint2 d = lds_u64(2 * adp + (ai.f4_bv[3] - 2 * ai.f4_key[3] - B));
    const uint2 e = lds_u64(B + ACLF_PROTO + 8 * (v.proto & 255));
    const uint32_t lo = a.x & b.x & c.x & d.x & e.x, hi = a.y & b.y & c.y & d.y & e.y;
    const uint32_t bit = lo ? __ffs(lo) - 1 : 31 + __ffs(hi);
    uint32_t r = 0xFFFFu | ai.default_action << 31;
    if (lo | hi) r = lds_u32(B + ACLF_RULE + 4 * bit);
    return r;
}
template <bool SM>
__device__ __forceinline__ uint32_t acl_core(const AclMem<SM> &M4, const AclMem<SM> &M6, const AclImg &ai, const PV &v)
{
    if (v.fam == 4) {
        const uint32_t *hd = ai.hdr4;
        if (hd[0] == 0) return 0xFFFFu | ai.default_action << 31;
        if constexpr (SM)
            if (ai.fast) return acl4_fast(M4.s, ai, v);
        const AclMem<SM> &M = M4;
        if constexpr (!SM)
            if (ai.x4 != nullptr) {          // 16-bit first level (large rule sets, global image)
                const uint32_t ks = v.src[0], kd = v.dst[0];
                uint32_t js = __ldg(ai.x4 + (ks >> 16)), jd = __ldg(ai.x4 + 65536 + (kd >> 16));
                const uint32_t jsp = __ldg(ai.x4 + 131072 + (v.sport & 0xFFFF)), jdp = __ldg(ai.x4 + 196608 + (v.dport & 0xFFFF));
                for (int i = (int)(ai.d16 & 255) - 1; i >= 0; i--) {
                    const uint32_t h = 1u << i;
                    js += M.template at<uint32_t>(4 * (hd[8] + js + h)) <= ks ? h : 0u;
                }
                for (int i = (int)(ai.d16 >> 8) - 1; i >= 0; i--) {
                    const uint32_t h = 1u << i;
                    jd += M.template at<uint32_t>(4 * (hd[10] + jd + h)) <= kd ? h : 0u;
                }
                return acl_match_w<SM>(M, hd, ai.default_action, js, jd, jsp, jdp, v.proto);
            }
        const uint32_t ks = v.src[0], kd = v.dst[0], ksp = v.sport, kdp = v.dport;
        // window starts (bucket reads on the top 8 key bits), as byte offsets
        uint32_t os = 4 * hd[8] + 4 * M.template at<uint16_t>(4 * hd[18] + 2 * (ks >> 24));
        uint32_t od = 4 * hd[10] + 4 * M.template at<uint16_t>(4 * hd[19] + 2 * (kd >> 24));
        uint32_t osp = 4 * hd[12] + 4 * M.template at<uint16_t>(4 * hd[20] + 2 * (ksp >> 8));
        uint32_t odp = 4 * hd[14] + 4 * M.template at<uint16_t>(4 * hd[21] + 2 * (kdp >> 8));
        const uint32_t D = hd[23];
        if constexpr (SM) {
            // absolute shared addresses; one straight-line search per image depth
            const uint32_t base = (uint32_t)__cvta_generic_to_shared(nfc_smem) + M.s;
            uint32_t as = base + os, ad = base + od, asp = base + osp, adp = base + odp;
            // (a uniform if-chain, not a switch: no indexed jump per packet)
            if (D == 3) acl_search4_s<3>(as, ad, asp, adp, v);
            else if (D == 2) acl_search4_s<2>(as, ad, asp, adp, v);
            else if (D == 4) acl_search4_s<4>(as, ad, asp, adp, v);
            else if (D == 1) acl_search4_s<1>(as, ad, asp, adp, v);
            else if (D == 5) acl_search4_s<5>(as, ad, asp, adp, v);
            else if (D > 5) {
                for (int i = (int)D - 1; i >= 5; i--) {
                    const uint32_t h4 = 4u << i;
                    as += M.template at<uint32_t>(as - base + h4) <= ks ? h4 : 0u;
                    ad += M.template at<uint32_t>(ad - base + h4) <= kd ? h4 : 0u;
                    asp += M.template at<uint32_t>(asp - base + h4) <= ksp ? h4 : 0u;
                    adp += M.template at<uint32_t>(adp - base + h4) <= kdp ? h4 : 0u;
                }
                acl_search4_s<5>(as, ad, asp, adp, v);
            }
            os = as - base; od = ad - base; osp = asp - base; odp = adp - base;
        } else {
            for (int i = (int)D - 1; i >= 0; i--) {
                const uint32_t h4 = 4u << i;
                os += M.template at<uint32_t>(os + h4) <= ks ? h4 : 0u;
                od += M.template at<uint32_t>(od + h4) <= kd ? h4 : 0u;
                osp += M.template at<uint32_t>(osp + h4) <= ksp ? h4 : 0u;
                odp += M.template at<uint32_t>(odp + h4) <= kdp ? h4 : 0u;
            }
        }
        return acl_match_w<SM>(M, hd, ai.default_action, (os >> 2) - hd[8], (od >> 2) - hd[10], (osp >> 2) - hd[12],
                               (odp >> 2) - hd[14], v.proto);
    }
    const uint32_t *hd = ai.hdr6;
    if (hd[0] == 0) return 0xFFFFu | ai.default_action << 31;
    const AclMem<SM> &M = M6;
    uint32_t js = M.template at<uint16_t>(4 * hd[18] + 2 * (v.src[0] >> 24));
    uint32_t jd = M.template at<uint16_t>(4 * hd[19] + 2 * (v.dst[0] >> 24));
    uint32_t jsp = M.template at<uint16_t>(4 * hd[20] + 2 * (v.sport >> 8));
    uint32_t jdp = M.template at<uint16_t>(4 * hd[21] + 2 * (v.dport >> 8));
    for (uint32_t h = (1u << hd[23]) >> 1; h; h >>= 1) {
        js = le128(M.template at<uint4>(4 * hd[8] + 16 * (js + h)), v.src) ? js + h : js;
        jd = le128(M.template at<uint4>(4 * hd[10] + 16 * (jd + h)), v.dst) ? jd + h : jd;
        jsp = M.template at<uint32_t>(4 * hd[12] + 4 * (jsp + h)) <= v.sport ? jsp + h : jsp;
        jdp = M.template at<uint32_t>(4 * hd[14] + 4 * (jdp + h)) <= v.dport ? jdp + h : jdp;
    }
    return acl_match_w<SM>(M, hd, ai.default_action, js, jd, jsp, jdp, v.proto);
}
// the fused kernel's entry: image staged in shared memory (P.lay offsets) or global
__device__ __forceinline__ uint32_t nf_acl_fused(const KParams &P, const PV &v)
{
    if (P.acl.smem_words)
        return acl_core<true>(AclMem<true>{nullptr, P.lay.acl4}, AclMem<true>{nullptr, P.lay.acl6}, P.acl, v);
    return acl_core<false>(AclMem<false>{reinterpret_cast<const uint8_t *>(P.acl.bv4), 0u},
                           AclMem<false>{reinterpret_cast<const uint8_t *>(P.acl.bv6), 0u}, P.acl, v);
}

// ---------------------------------------------------------------- DPI
// Aho-Corasick DFA walk over byte classes.  Transition entries are u16: next
// state | ACCEPT << 15 (ACCEPT: the next state has a non-empty output set); u32
// with ACCEPT << 31 above 32K states ("wide").
//   DM_FULL: all rows in shared memory; cls8[b] = 2*class(b) (u8, ncls <= 128),
//            so a step is PRMT (byte) + LDS.U8 (class) + IMAD + LDS.U16.
//   DM_HOT:  the first H states (BFS order) in shared memory, cls[b] = 2*class(b);
//            cold states read the global table (predicated load).
// A walk keeps three registers: s (state), cnt (accept events), mx (max entry
// seen).  Accept entries are >= 0x8000 > any other entry, so when cnt == 1 the
// state after the only accept event is mx & 0x7FFF and the match set is its
// output closure; cnt > 1 takes the exact re-walk (dpi_slow).
// DM_FULL walks the slot image (DpiImg::frows) instead: s is a signed slot, an
// entry is the next slot sign-extended to 32 bits, cnt += e >> 31, and the
// accepting entries (negative) are the largest as u32, so with cnt == 1 the only
// accepting slot is mx and ~mx indexes the accept tables.  The class table sits
// at shared offset 0: a step is PRMT + LDS.U8 + IMAD + LDS.S16 (+ 2 ALU).
struct DpiCtx {
    const uint32_t *cls;    // smem, 256 entries (DM_HOT)
    const uint8_t *cls8;    // smem, 256 entries (DM_FULL)
    const uint8_t *gcls;    // global byte -> class table (exact re-walk)
    const uint8_t *sm;      // smem base (DM_FULL addressing)
    const uint8_t *hot;     // smem hot rows (DM_HOT)
    const uint2 *sp;        // smem sparse records (DM_HOT), states [H, H + S)
    uint32_t row2;          // bytes per row = 2 * ncls
    uint32_t H, HK2, S;     // DM_HOT: hot states, byte offset of the last hot entry, sparse records
    uint32_t ncls, wide;
    const void *trans;
    const uint32_t *out_off;
    const uint16_t *out_ids;
    const uint8_t *pat_action;
    const uint32_t *acc_id;   // DM_FULL: accepting slot -> state id
};

struct Walk { uint32_t s, cnt, mx; };

// byte k (compile-time) of a little-endian word, zero-extended: one PRMT
__device__ __forceinline__ uint32_t byte_of(uint32_t w, int k) { return __byte_perm(w, 0, 0x4440 + k); }

template <int DM>
__device__ __forceinline__ uint32_t dfa_entry(const KParams &P, uint32_t s, uint32_t byte)
{
    if (DM == DM_FULL) {     // slot image; class table at shared offset 0
        // (uniform row base) + (per-lane offset): one LDS [R + UR] after the IMAD
        const uint32_t rb = (uint32_t)__cvta_generic_to_shared(nfc_smem) + P.lay.frow0;
        const uint32_t t = s * P.dpi.row2 + nfc_smem[byte];
        int32_t e;
        asm("{\n\t.reg .s16 h;\n\tld.shared.s16 h, [%1];\n\tcvt.s32.s16 %0, h;\n\t}" : "=r"(e) : "r"(rb + t));
        return (uint32_t)e;
    }
    // tiered rows (DpiImg::sparse): dense row, or a sparse record's base row with <= 2
    // exceptions, or (cold) the global table.  Branch-free: the sparse-record, dense-row
    // and cold loads are predicated.  cls[byte] = class (u32).
    const uint32_t c = reinterpret_cast<const uint32_t *>(nfc_smem + P.lay.cls)[byte];
    const uint32_t H = P.dpi.hot_states;
    uint32_t rx, ry;
    {
        const uint32_t ra = (uint32_t)__cvta_generic_to_shared(nfc_smem + P.lay.sp) + 8u * (s - H);
        asm("{\n\t.reg .pred q;\n\tsetp.lt.u32 q, %2, %3;\n\tmov.b32 %0, -1;\n\tmov.b32 %1, 0;\n\t"
            "@q ld.shared.v2.u32 {%0, %1}, [%4];\n\t}"
            : "=r"(rx), "=r"(ry) : "r"(s - H), "r"(P.dpi.sparse_states), "r"(ra));
    }
    const bool sp = s >= H;
    const uint32_t b = sp ? (rx & 0xFFFFu) : s;
    uint32_t e;
    {
        const uint32_t da = (uint32_t)__cvta_generic_to_shared(nfc_smem + P.lay.hot) + 2u * (b * P.dpi.ncls + c);
        asm("{\n\t.reg .pred q;\n\tsetp.lt.u32 q, %1, %2;\n\tmov.b32 %0, 0;\n\t@q ld.shared.u16 %0, [%3];\n\t}"
            : "=r"(e) : "r"(b), "r"(H), "r"(da));
    }
    e = (sp && c == __byte_perm(rx, 0, 0x4442)) ? (ry & 0xFFFFu) : e;
    e = (sp && c == __byte_perm(rx, 0, 0x4443)) ? (ry >> 16) : e;
    // cold rows (deep states beyond the on-chip tiers): predicated load
    const bool cold = b >= H;
    {
        const uint16_t *ga = reinterpret_cast<const uint16_t *>(P.dpi.trans) + (s * P.dpi.ncls + c);
        uint32_t o;
        asm("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %1, 0;\n\tmov.b32 %0, %2;\n\t@q ld.global.nc.u16 %0, [%3];\n\t}"
            : "=r"(o) : "r"((uint32_t)cold), "r"(e), "l"(ga));
        e = o;
    }
    return e;
}
template <int DM>
__device__ __forceinline__ void dfa_step(const KParams &P, Walk &w, uint32_t byte)
{
    const uint32_t e = dfa_entry<DM>(P, w.s, byte);
    if (DM == DM_FULL) {
        w.s = e;
        w.cnt += e >> 31;
    } else {
        w.s = e & 0x7FFFu;
        w.cnt += e >> 15;
    }
    w.mx = max(w.mx, e);
}
// step only if `in` (bytes outside the payload leave the walk unchanged: s <= mx always)
template <int DM>
__device__ __forceinline__ void dfa_step_if(const KParams &P, Walk &w, uint32_t byte, bool in)
{
    // branch-free: the entry is looked up for any state (all loads stay in bounds) and
    // discarded when the byte is outside the span
    uint32_t e = dfa_entry<DM>(P, w.s, byte);
    asm("" : "+r"(e));
    if (DM == DM_FULL) {     // the state keeps its sign: count only bytes inside the span
        w.cnt += in ? e >> 31 : 0u;
        e = in ? e : w.s;
        w.s = e;
    } else {
        e = in ? e : w.s;
        w.s = e & 0x7FFFu;
        w.cnt += e >> 15;
    }
    w.mx = max(w.mx, e);
}
__device__ __forceinline__ void dfa_step_wide(const DpiCtx &c, Walk &w, uint32_t byte, bool in)
{
    const uint32_t k = w.s * c.ncls + c.cls[byte];
    const uint32_t e = in ? __ldg(reinterpret_cast<const uint32_t *>(c.trans) + k) : w.s;
    w.s = e & 0x7FFFFFFFu;
    w.cnt += e >> 31;
    w.mx = max(w.mx, e);
}

// DM_HOT: make a payload word depend on the walk state so the class lookups of its
// bytes are not hoisted far ahead of the walk (that raises register pressure past the
// occupancy budget and spills); DM_FULL has the registers to spare
template <int DM>
__device__ __forceinline__ uint32_t tie(uint32_t word, const Walk &w)
{
    if (DM == DM_HOT && NFC_TIE) asm("" : "+r"(word) : "r"(w.s));
    return word;
}

// payload bytes [A, 64) of the header cache, A compile-time: no per-byte guards
template <int DM, int A>
__device__ __forceinline__ void walk_cached(const KParams &P, const uint32_t h[16], Walk &w)
{
    uint32_t wd = tie<DM>(h[A >> 2], w);
#pragma unroll
    for (int idx = A; idx < 64; idx++) {
        if ((idx & 3) == 0) wd = tie<DM>(h[idx >> 2], w);
        dfa_step<DM>(P, w, byte_of(wd, idx & 3));
    }
}

// walk of a DFA with > 32K states (u32 entries, all rows in global memory); not inlined
static __device__ __noinline__ Walk dpi_walk_wide(const DpiCtx &c, const uint8_t *f, uint32_t a, uint32_t b,
                                                  uint64_t pol)
{
    // payload bytes come from memory here (the header cache stays in registers in the caller)
    Walk w{0, 0, 0};
    for (uint32_t ch = a & ~15u; ch < b; ch += 16) {
        const uint4 q = ld_stream16(f + ch, pol);
        const uint32_t wd[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
        for (int k = 0; k < 16; k++) dfa_step_wide(c, w, (wd[k >> 2] >> ((k & 3) * 8)) & 0xFF, ch + k - a < b - a);
    }
    return w;
}

// Fast walk over payload [a, b): counts accept events (see DpiCtx).  Bytes 32..63
// come from the header cache (a payload never starts before byte 34), the rest
// from memory in 16-B chunks.
template <int DM>
__device__ __forceinline__ Walk dpi_walk(const KParams &P, const DpiCtx &c, const uint32_t h[16], const uint8_t *f,
                                         uint32_t a, uint32_t b, uint64_t pol)
{
    if (DM != DM_FULL && P.dpi.wide) return dpi_walk_wide(c, f, a, b, pol);
    for (uint32_t l = 128; l < min(b, 64u + NFC_PF_DIST); l += 128) prefetch_l2(f + l);
    Walk w{0, 0, 0};
    if (b >= 64 && a == 42) walk_cached<DM, 42>(P, h, w);        // IPv4 UDP
    else if (b >= 64 && a == 62) walk_cached<DM, 62>(P, h, w);   // IPv6 UDP
    else if (b >= 64 && a == 54) walk_cached<DM, 54>(P, h, w);   // IPv4 TCP
    else {
        uint32_t wd = 0;
#pragma unroll
        for (int idx = 32; idx < 64; idx++) {
            if ((idx & 3) == 0) wd = tie<DM>(h[idx >> 2], w);
            dfa_step_if<DM>(P, w, byte_of(wd, idx & 3), (uint32_t)idx - a < b - a);
        }
    }
    for (uint32_t ch = max(64u, a & ~15u); ch < b; ch += 16) {
        if ((ch & 127) == 0 && ch + NFC_PF_DIST < b) prefetch_l2(f + ch + NFC_PF_DIST);
        const uint4 q = ld_stream16(f + ch, pol);
        uint32_t wd[4] = {q.x, q.y, q.z, q.w};
        if (ch >= a && ch + 16 <= b) {
#pragma unroll
            for (int k = 0; k < 16; k++) {
                const uint32_t x = (k & 3) == 0 ? tie<DM>(wd[k >> 2], w) : wd[k >> 2];
                if ((k & 3) == 0) wd[k >> 2] = x;
                dfa_step<DM>(P, w, byte_of(x, k & 3));
            }
        } else {
#pragma unroll
            for (int k = 0; k < 16; k++) {
                const uint32_t x = (k & 3) == 0 ? tie<DM>(wd[k >> 2], w) : wd[k >> 2];
                if ((k & 3) == 0) wd[k >> 2] = x;
                dfa_step_if<DM>(P, w, byte_of(x, k & 3), ch + k - a < b - a);
            }
        }
    }
    return w;
}

// Payload bytes [a, min(b, 64)) from the header cache (the owner lane's registers).
template <int DM>
__device__ __forceinline__ Walk dpi_walk_head(const KParams &P, const uint32_t h[16], uint32_t a, uint32_t b)
{
    Walk w{0, 0, 0};
    if (b >= 64 && a == 42) walk_cached<DM, 42>(P, h, w);        // IPv4 UDP
    else if (DM == DM_FULL && b >= 64 && a == 62) walk_cached<DM, 62>(P, h, w);   // IPv6 UDP
    else if (DM == DM_FULL && b >= 64 && a == 54) walk_cached<DM, 54>(P, h, w);   // IPv4 TCP
    else if (a < 64) {
        uint32_t wd = 0;
#pragma unroll
        for (int idx = 32; idx < 64; idx++) {
            if ((idx & 3) == 0) wd = tie<DM>(h[idx >> 2], w);
            dfa_step_if<DM>(P, w, byte_of(wd, idx & 3), (uint32_t)idx - a < b - a);
        }
    }
    return w;
}

// Exact match set of a packet whose walk hit more than one accept event (rare
// path, not inlined): re-walk the payload from memory collecting distinct pattern
// ids in a register list, or -- beyond DPI_LIST ids -- in a per-thread global
// bitmap; emit the (packet, pattern) pairs.  Returns nmatch | any_drop << 31.
struct DpiOvf {
    uint32_t *bitmap;
    uint32_t words;
    uint32_t *match_count, *match_pkt;
    uint16_t *match_pat;
    uint32_t match_cap;
    unsigned long long *stats;
    uint32_t emit;          // 0: count ids and the DROP flag only (no pairs, no counters)
};
// one exact DFA step (state -> next, accept flag): the on-chip tiers as in dfa_entry
// (DM_FULL: all rows; DM_HOT: dense rows / sparse records / global), or the global
// table for > 32K-state DFAs
template <int DM>
__device__ __forceinline__ uint32_t dfa_step_global(const DpiCtx &c, uint32_t s, uint32_t b, bool &acc)
{
    if (!c.wide) {
        uint32_t e;
        if (DM == DM_FULL) {     // slot image: s and the result are slots (c.hot = row of slot 0)
            const int32_t x = *reinterpret_cast<const int16_t *>(c.hot + (int32_t)s * (int32_t)c.row2 + c.cls8[b]);
            acc = x < 0;
            return (uint32_t)x;
        } else {
            const uint32_t cl = c.cls[b];
            const bool sp = s >= c.H;
            uint2 r = make_uint2(0xFFFFFFFFu, 0u);
            if (sp && s - c.H < c.S) r = c.sp[s - c.H];
            const uint32_t bs = sp ? (r.x & 0xFFFFu) : s;
            e = bs < c.H ? *reinterpret_cast<const uint16_t *>(c.hot + 2 * (bs * c.ncls + cl)) : 0u;
            if (sp && cl == ((r.x >> 16) & 0xFFu)) e = r.y & 0xFFFFu;
            if (sp && cl == (r.x >> 24)) e = r.y >> 16;
            if (bs >= c.H) e = __ldg(reinterpret_cast<const uint16_t *>(c.trans) + s * c.ncls + cl);
        }
        acc = (e >> 15) & 1;
        return e & 0x7FFFu;
    }
    const uint32_t k = s * c.ncls + __ldg(c.gcls + b);
    if (c.wide) {
        const uint32_t e = __ldg(reinterpret_cast<const uint32_t *>(c.trans) + k);
        acc = e >> 31;
        return e & 0x7FFFFFFFu;
    }
    const uint32_t e = __ldg(reinterpret_cast<const uint16_t *>(c.trans) + k);
    acc = (e >> 15) & 1;
    return e & 0x7FFFu;
}
// BFS state id of an accepting walk state (DM_FULL walks slots)
template <int DM>
__device__ __forceinline__ uint32_t dfa_out_state(const DpiCtx &c, uint32_t s)
{
    if (DM == DM_FULL && !c.wide) return __ldg(c.acc_id + ~s);
    return s;
}
template <int DM>
static __device__ __noinline__ uint32_t dpi_slow(DpiCtx c, const uint8_t *f, uint32_t a, uint32_t b, uint32_t gtid,
                                          DpiOvf o, uint32_t pkt_id)
{
    uint16_t ids[DPI_LIST];
    uint32_t n = 0, drop = 0;
    bool ovf = false;
    uint32_t s = 0;
    uint4 q = make_uint4(0, 0, 0, 0);
    for (uint32_t i = a; i < b && !ovf; i++) {
        if (i == a || (i & 15) == 0) q = *reinterpret_cast<const uint4 *>(f + (i & ~15u));
        const uint32_t wd = (i & 8) ? ((i & 4) ? q.w : q.z) : ((i & 4) ? q.y : q.x);
        bool acc;
        s = dfa_step_global<DM>(c, s, (wd >> ((i & 3) * 8)) & 0xFF, acc);
        if (!acc) continue;
        const uint32_t so = dfa_out_state<DM>(c, s);
        const uint32_t e = __ldg(c.out_off + so + 1);
        for (uint32_t x = __ldg(c.out_off + so); x < e; x++) {
            const uint32_t id = __ldg(c.out_ids + x);
            drop |= __ldg(c.pat_action + id);
            bool seen = false;
            for (uint32_t k = 0; k < n; k++) seen |= ids[k] == id;
            if (seen) continue;
            if (n == DPI_LIST) { ovf = true; break; }
            ids[n++] = (uint16_t)id;
        }
    }
    if (!ovf) {
        if (n && o.emit) {
            const uint32_t slot = atomicAdd(o.match_count, n);
            for (uint32_t k = 0; k < n; k++)
                if (slot + k < o.match_cap) { o.match_pkt[slot + k] = pkt_id; o.match_pat[slot + k] = ids[k]; }
            if (slot + n > o.match_cap)
                atomicAdd(&o.stats[ST_MATCH_OVF], (unsigned long long)(slot + n - max(slot, o.match_cap)));
        }
        return n | drop << 31;
    }
    // more than DPI_LIST distinct ids: exact bitmap pass
    if (o.emit) atomicAdd(&o.stats[ST_DPI_OVF_PKTS], 1ull);
    uint32_t *bm = o.bitmap + (size_t)gtid * o.words;
    for (uint32_t k = 0; k < o.words; k++) bm[k] = 0;
    uint32_t cnt = 0;
    s = 0;
    drop = 0;
    for (uint32_t i = a; i < b; i++) {
        if (i == a || (i & 15) == 0) q = *reinterpret_cast<const uint4 *>(f + (i & ~15u));
        const uint32_t wd = (i & 8) ? ((i & 4) ? q.w : q.z) : ((i & 4) ? q.y : q.x);
        bool acc;
        s = dfa_step_global<DM>(c, s, (wd >> ((i & 3) * 8)) & 0xFF, acc);
        if (!acc) continue;
        const uint32_t so = dfa_out_state<DM>(c, s);
        const uint32_t e = __ldg(c.out_off + so + 1);
        for (uint32_t x = __ldg(c.out_off + so); x < e; x++) {
            const uint32_t id = __ldg(c.out_ids + x);
            drop |= __ldg(c.pat_action + id);
            const uint32_t bit = 1u << (id & 31);
            if (bm[id >> 5] & bit) continue;
            bm[id >> 5] |= bit;
            cnt++;
            if (!o.emit) continue;
            const uint32_t slot = atomicAdd(o.match_count, 1u);
            if (slot < o.match_cap) { o.match_pkt[slot] = pkt_id; o.match_pat[slot] = (uint16_t)id; }
            else atomicAdd(&o.stats[ST_MATCH_OVF], 1ull);
        }
    }
    return cnt | drop << 31;
}

// ---------------------------------------------------------------- LPM
__device__ __forceinline__ uint32_t lpm6_lookup(const Lpm6Img &t, const uint32_t dst[4])
{
    uint32_t best = t.def_nh;
    int lo = 0, hi = (int)t.n_levels - 1;
    while (lo <= hi) {
        int mid = (lo + hi) >> 1;
        int L = __ldg(t.lens + mid);
        uint32_t k0 = dst[0] & mask32d(L), k1 = dst[1] & mask32d(L - 32);
        uint32_t k2 = dst[2] & mask32d(L - 64), k3 = dst[3] & mask32d(L - 96);
        uint32_t m = __ldg(t.mask + mid), base = __ldg(t.base + mid);
        uint32_t hsh = l6_hash(k0, k1, k2, k3) & m;
        bool found = false;
        uint32_t info = 0;
        for (;;) {
            const uint4 *e = t.ent + 2 * (size_t)(base + hsh);
            uint4 key = __ldg(e);
            uint32_t inf = __ldg(reinterpret_cast<const uint32_t *>(e + 1));
            if (!(inf & L6_VALID)) break;
            if (key.x == k0 && key.y == k1 && key.z == k2 && key.w == k3) { found = true; info = inf; break; }
            hsh = (hsh + 1) & m;
        }
        if (found) {
            if ((info & 0xFFFF) != 0x7FFF) best = info & 0xFFFF;
            lo = mid + 1;
        } else {
            hi = mid - 1;
        }
    }
    return best;
}

// L2/L3 rewrite after an LPM hit (R#6): dst MAC = nh MAC, src MAC = port MAC,
// TTL / hop limit - 1, IPv4 header checksum recomputed (RFC 1071, byte-order independent
// sum over little-endian halves).  Writes the first 32 B of the frame.
__device__ __forceinline__ void forward_words(uint8_t *f, uint32_t h[16], const PV &v, uint2 nh, uint2 pm)
{
    h[0] = nh.x;
    h[1] = (nh.y & 0xFFFF) | (pm.x << 16);
    h[2] = (pm.x >> 16) | (pm.y << 16);
    if (v.fam == 4) {
        h[5] -= 1u << 16;                     // TTL: byte 22
        h[6] &= 0xFFFF0000u;                  // checksum bytes 24..25 := 0
        uint32_t sum;
        if (v.l4_off == 34) {
            sum = (h[3] >> 16) + (h[4] & 0xFFFF) + (h[4] >> 16) + (h[5] & 0xFFFF) + (h[5] >> 16) +
                  (h[6] >> 16) + (h[7] & 0xFFFF) + (h[7] >> 16) + (h[8] & 0xFFFF);
        } else {                              // IPv4 options (rare): bytes >= 32 from memory
            sum = (h[3] >> 16) + (h[4] & 0xFFFF) + (h[4] >> 16) + (h[5] & 0xFFFF) + (h[5] >> 16) +
                  (h[6] >> 16) + (h[7] & 0xFFFF) + (h[7] >> 16);
            for (uint32_t k = 32; k < v.l4_off; k += 2) sum += (uint32_t)f[k] | (uint32_t)f[k + 1] << 8;
        }
        sum = (sum & 0xFFFF) + (sum >> 16);
        sum = (sum & 0xFFFF) + (sum >> 16);
        h[6] |= (~sum) & 0xFFFF;
    } else {
        h[5] -= 1u << 8;                      // hop limit: byte 21
    }
}
__device__ __forceinline__ void forward_rewrite(uint8_t *f, uint32_t h[16], const PV &v, uint2 nh, uint2 pm, uint64_t pol)
{
    forward_words(f, h, v, nh, pm);
#if NFC_LD256
    if ((reinterpret_cast<uintptr_t>(f) & 31) == 0) {
        st_stream32(f, h, pol);
        return;
    }
#endif
    st_stream16(f, make_uint4(h[0], h[1], h[2], h[3]), pol);
    st_stream16(f + 16, make_uint4(h[4], h[5], h[6], h[7]), pol);
}

// ---------------------------------------------------------------- Toeplitz flow hash
__device__ __forceinline__ uint32_t toeplitz(const uint32_t *nib, const PV &v)
{
    uint32_t w[9];
    uint32_t nw;
    if (v.fam == 4) { w[0] = v.src[0]; w[1] = v.dst[0]; w[2] = v.sport << 16 | v.dport; nw = 3; }
    else {
#pragma unroll
        for (int k = 0; k < 4; k++) { w[k] = v.src[k]; w[4 + k] = v.dst[k]; }
        w[8] = v.sport << 16 | v.dport;
        nw = 9;
    }
    uint32_t hsh = 0;
#pragma unroll
    for (int i = 0; i < 9; i++) {
        if (i < (int)nw) {
#pragma unroll
            for (int n = 0; n < 8; n++) hsh ^= nib[(8 * i + n) * 16 + ((w[i] >> (28 - 4 * n)) & 15)];
        }
    }
    return hsh;
}

// ---------------------------------------------------------------- NAT44 (Table II; R#30)
// The translation as values: DNAT by the open-addressing table, SNAT by the inside
// prefixes (constant bank) and the flow hash h; the L4 checksum updated per changed
// 16-bit word (RFC 1624 eqn. 3).  Returns the new (src, dst, ports, l4 checksum).
struct NatOut { uint32_t src, dst, ports, ck; };
__device__ __forceinline__ uint32_t oc_add16(uint32_t a, uint32_t b)
{
    const uint32_t x = a + b;
    return (x & 0xFFFF) + (x >> 16);
}
// RFC 1624 eqn. 3 for one field m -> m1 (identity when m == m1: ~(~HC + ~m + m) = HC
// except that 0xFFFF and 0x0000 are the two zeros -- skipped explicitly)
__device__ __forceinline__ uint32_t csum_upd(uint32_t hc, uint32_t m, uint32_t m1)
{
    const uint32_t x = oc_add16(oc_add16(~hc & 0xFFFF, ~m & 0xFFFF), m1);
    return m == m1 ? hc : (~x & 0xFFFF);
}
__device__ __forceinline__ NatOut nat_values(const KParams &P, const uint32_t *nat_nib, const PV &v, uint32_t ck)
{
    const NatImg &N = P.nat;
    const uint32_t h = toeplitz(nat_nib, v);
    const uint32_t src = v.src[0], dst = v.dst[0], sp = v.sport, dp = v.dport;
    uint32_t nsrc = src, ndst = dst, nsp = sp, ndp = dp;
    // DNAT: (proto, dst, dport) exact match, linear probing
    const uint32_t key1 = dp | v.proto << 16;
    for (uint32_t slot = nat_slot(dst, key1) & N.dnat_mask;; slot = (slot + 1) & N.dnat_mask) {
        const uint4 e = __ldg(N.dnat + slot);
        if (!(e.y & NAT_VALID)) break;
        if (e.x == dst && (e.y & 0xFFFFFF) == key1) { ndst = e.z; ndp = e.w; break; }
    }
    // SNAT: first inside prefix (constant bank, uniform loop)
    for (uint32_t q = 0; q < N.n_inside; q++)
        if ((src & N.in_mask[q]) == N.in_pref[q]) {
            nsrc = __ldg(N.pool + (h & 0xFFFF) % N.n_pool);
            nsp = N.port_lo + (h >> 16) % N.port_range;
            break;
        }
    if (!(v.proto == 17 && ck == 0)) {
        ck = csum_upd(ck, src >> 16, nsrc >> 16);
        ck = csum_upd(ck, src & 0xFFFF, nsrc & 0xFFFF);
        ck = csum_upd(ck, dst >> 16, ndst >> 16);
        ck = csum_upd(ck, dst & 0xFFFF, ndst & 0xFFFF);
        ck = csum_upd(ck, sp, nsp);
        ck = csum_upd(ck, dp, ndp);
        if (v.proto == 17 && ck == 0) ck = 0xFFFF;
    }
    return NatOut{nsrc, ndst, nsp << 16 | ndp, ck};
}
__device__ __forceinline__ uint32_t bswap16w(uint32_t x) { return __byte_perm(x, 0, 0x4401); }   // 16-bit value <-> 2 LE bytes
// Applies the NAT to a packet (v.fam == 4, TCP/UDP, egress port Internet-facing):
// header-cache fast path for a 20-B IPv4 header (bytes 24..63 written back), memory
// path otherwise.  Updates v (and h) for the NFs after it.
__device__ __forceinline__ void nf_nat(const KParams &P, const uint32_t *nat_nib, uint8_t *f, uint32_t h[16], PV &v,
                                       uint64_t pol)
{
    const bool tcp = v.proto == 6;
    if (v.l4_off == 34) {
        // UDP checksum: bytes 40..41 (h[10] low half); TCP: bytes 50..51 (h[12] high half)
        const uint32_t ckw = tcp ? h[12] >> 16 : h[10] & 0xFFFF;
        const NatOut o = nat_values(P, nat_nib, v, bswap16w(ckw));
        const uint32_t sb = bswap32(o.src), db = bswap32(o.dst), pb = bswap32(o.ports);   // network-order words
        // bytes 26..29 src, 30..33 dst, 34..37 ports (word-straddling: byte_perm)
        h[6] = __byte_perm(h[6], sb, 0x5410);            // bytes 24,25 keep; 26,27 = src[0..1]
        h[7] = __byte_perm(sb, db, 0x5432);              // 28,29 = src[2..3]; 30,31 = dst[0..1]
        h[8] = __byte_perm(db, pb, 0x5432);              // 32,33 = dst[2..3]; 34,35 = sport
        h[9] = __byte_perm(pb, h[9], 0x7632);            // 36,37 = dport; 38,39 keep
        if (tcp) h[12] = (h[12] & 0xFFFFu) | bswap16w(o.ck) << 16;
        else h[10] = (h[10] & 0xFFFF0000u) | bswap16w(o.ck);
        // IPv4 header checksum (RFC 1071 over bytes 14..33, field 24..25 zeroed)
        h[6] &= 0xFFFF0000u;
        uint32_t sum = (h[3] >> 16) + (h[4] & 0xFFFF) + (h[4] >> 16) + (h[5] & 0xFFFF) + (h[5] >> 16) +
                       (h[6] >> 16) + (h[7] & 0xFFFF) + (h[7] >> 16) + (h[8] & 0xFFFF);
        sum = (sum & 0xFFFF) + (sum >> 16);
        sum = (sum & 0xFFFF) + (sum >> 16);
        h[6] |= (~sum) & 0xFFFF;
        st_stream16(f + 16, make_uint4(h[4], h[5], h[6], h[7]), pol);
        st_stream16(f + 32, make_uint4(h[8], h[9], h[10], h[11]), pol);
        if (tcp) st_stream16(f + 48, make_uint4(h[12], h[13], h[14], h[15]), pol);
        v.src[0] = o.src; v.dst[0] = o.dst; v.sport = o.ports >> 16; v.dport = o.ports & 0xFFFF;
        return;
    }
    // IPv4 options (rare): bytes from memory
    const uint32_t l4 = v.l4_off, ca = l4 + (tcp ? 16 : 6);
    const NatOut o = nat_values(P, nat_nib, v, (uint32_t)f[ca] << 8 | f[ca + 1]);
    for (int k = 0; k < 4; k++) { f[26 + k] = (uint8_t)(o.src >> (24 - 8 * k)); f[30 + k] = (uint8_t)(o.dst >> (24 - 8 * k)); }
    for (int k = 0; k < 4; k++) f[l4 + k] = (uint8_t)(o.ports >> (24 - 8 * k));
    f[ca] = (uint8_t)(o.ck >> 8); f[ca + 1] = (uint8_t)o.ck;
    f[24] = f[25] = 0;
    uint32_t sum = 0;
    for (uint32_t k = 14; k < l4; k += 2) sum += (uint32_t)f[k] << 8 | f[k + 1];
    sum = (sum & 0xFFFF) + (sum >> 16);
    sum = (sum & 0xFFFF) + (sum >> 16);
    f[24] = (uint8_t)(~sum >> 8); f[25] = (uint8_t)~sum;
    load_header(f, 64, h, pol);     // refresh the cache (frames here are >= 64 B: IHL > 5 + L4)
    v.src[0] = o.src; v.dst[0] = o.dst; v.sport = o.ports >> 16; v.dport = o.ports & 0xFFFF;
}

// ---------------------------------------------------------------- AES-128 / SHA-1
// AES-128 encryption with one T-table replicated 32 times in shared memory: lane l
// reads copy l, which lives in bank l, so the 160 random lookups per block are free
// of bank conflicts.  T1..T3 are byte rotations of T0; the S-box is byte 1 of T0.
// tl = this lane's column of the replicated table (tl[x * 32] = T0[x]).
__device__ __forceinline__ uint32_t T(const uint32_t *tl, uint32_t x) { return tl[x << 5]; }
__device__ __forceinline__ uint32_t ror8(uint32_t x) { return __funnelshift_r(x, x, 8); }
__device__ __forceinline__ uint32_t ror16(uint32_t x) { return __funnelshift_r(x, x, 16); }
__device__ __forceinline__ uint32_t ror24(uint32_t x) { return __funnelshift_r(x, x, 24); }

__device__ __forceinline__ void aes128_encrypt(const uint32_t *tl, const uint32_t rk[44], uint32_t in0, uint32_t in1,
                                               uint32_t in2, uint32_t in3, uint32_t out[4])
{
    uint32_t s0 = in0 ^ rk[0], s1 = in1 ^ rk[1], s2 = in2 ^ rk[2], s3 = in3 ^ rk[3];
#pragma unroll
    for (int r = 1; r < 10; r++) {
        const uint32_t t0 = T(tl, s0 >> 24) ^ ror8(T(tl, (s1 >> 16) & 255)) ^ ror16(T(tl, (s2 >> 8) & 255)) ^ ror24(T(tl, s3 & 255)) ^ rk[4 * r];
        const uint32_t t1 = T(tl, s1 >> 24) ^ ror8(T(tl, (s2 >> 16) & 255)) ^ ror16(T(tl, (s3 >> 8) & 255)) ^ ror24(T(tl, s0 & 255)) ^ rk[4 * r + 1];
        const uint32_t t2 = T(tl, s2 >> 24) ^ ror8(T(tl, (s3 >> 16) & 255)) ^ ror16(T(tl, (s0 >> 8) & 255)) ^ ror24(T(tl, s1 & 255)) ^ rk[4 * r + 2];
        const uint32_t t3 = T(tl, s3 >> 24) ^ ror8(T(tl, (s0 >> 16) & 255)) ^ ror16(T(tl, (s1 >> 8) & 255)) ^ ror24(T(tl, s2 & 255)) ^ rk[4 * r + 3];
        s0 = t0; s1 = t1; s2 = t2; s3 = t3;
    }
    // final round: S[x] = byte 1 of T0[x]
#define SB(x) ((T(tl, (x)) >> 8) & 255u)
    out[0] = (SB(s0 >> 24) << 24 | SB((s1 >> 16) & 255) << 16 | SB((s2 >> 8) & 255) << 8 | SB(s3 & 255)) ^ rk[40];
    out[1] = (SB(s1 >> 24) << 24 | SB((s2 >> 16) & 255) << 16 | SB((s3 >> 8) & 255) << 8 | SB(s0 & 255)) ^ rk[41];
    out[2] = (SB(s2 >> 24) << 24 | SB((s3 >> 16) & 255) << 16 | SB((s0 >> 8) & 255) << 8 | SB(s1 & 255)) ^ rk[42];
    out[3] = (SB(s3 >> 24) << 24 | SB((s0 >> 16) & 255) << 16 | SB((s1 >> 8) & 255) << 8 | SB(s2 & 255)) ^ rk[43];
#undef SB
}

// the same cipher with round keys in shared memory (rk: this SA's 44 words), out of line:
// one copy of the 10 rounds in the kernel instead of four inlined per 16-word SHA block
static __device__ __noinline__ uint4 aes128_encrypt_s(const uint32_t *tl, const uint32_t *rk, uint32_t in0, uint32_t in1,
                                                      uint32_t in2, uint32_t in3)
{
    uint32_t s0 = in0 ^ rk[0], s1 = in1 ^ rk[1], s2 = in2 ^ rk[2], s3 = in3 ^ rk[3];
#pragma unroll
    for (int r = 1; r < 10; r++) {
        const uint32_t t0 = T(tl, s0 >> 24) ^ ror8(T(tl, (s1 >> 16) & 255)) ^ ror16(T(tl, (s2 >> 8) & 255)) ^ ror24(T(tl, s3 & 255)) ^ rk[4 * r];
        const uint32_t t1 = T(tl, s1 >> 24) ^ ror8(T(tl, (s2 >> 16) & 255)) ^ ror16(T(tl, (s3 >> 8) & 255)) ^ ror24(T(tl, s0 & 255)) ^ rk[4 * r + 1];
        const uint32_t t2 = T(tl, s2 >> 24) ^ ror8(T(tl, (s3 >> 16) & 255)) ^ ror16(T(tl, (s0 >> 8) & 255)) ^ ror24(T(tl, s1 & 255)) ^ rk[4 * r + 2];
        const uint32_t t3 = T(tl, s3 >> 24) ^ ror8(T(tl, (s0 >> 16) & 255)) ^ ror16(T(tl, (s1 >> 8) & 255)) ^ ror24(T(tl, s2 & 255)) ^ rk[4 * r + 3];
        s0 = t0; s1 = t1; s2 = t2; s3 = t3;
    }
#define SB(x) ((T(tl, (x)) >> 8) & 255u)
    uint4 o;
    o.x = (SB(s0 >> 24) << 24 | SB((s1 >> 16) & 255) << 16 | SB((s2 >> 8) & 255) << 8 | SB(s3 & 255)) ^ rk[40];
    o.y = (SB(s1 >> 24) << 24 | SB((s2 >> 16) & 255) << 16 | SB((s3 >> 8) & 255) << 8 | SB(s0 & 255)) ^ rk[41];
    o.z = (SB(s2 >> 24) << 24 | SB((s3 >> 16) & 255) << 16 | SB((s0 >> 8) & 255) << 8 | SB(s1 & 255)) ^ rk[42];
    o.w = (SB(s3 >> 24) << 24 | SB((s0 >> 16) & 255) << 16 | SB((s1 >> 8) & 255) << 8 | SB(s2 & 255)) ^ rk[43];
#undef SB
    return o;
}

__device__ __forceinline__ uint32_t rotl(uint32_t x, int n) { return __funnelshift_l(x, x, n); }

__device__ __forceinline__ void sha1_compress(uint32_t H[5], uint32_t W[16])
{
    uint32_t a = H[0], b = H[1], c = H[2], d = H[3], e = H[4];
#pragma unroll
    for (int t = 0; t < 80; t++) {
        uint32_t w;
        if (t < 16) w = W[t];
        else {
            w = rotl(W[(t - 3) & 15] ^ W[(t - 8) & 15] ^ W[(t - 14) & 15] ^ W[t & 15], 1);
            W[t & 15] = w;
        }
        uint32_t f, k;
        if (t < 20) { f = d ^ (b & (c ^ d)); k = 0x5a827999u; }
        else if (t < 40) { f = b ^ c ^ d; k = 0x6ed9eba1u; }
        else if (t < 60) { f = (b & c) | (d & (b | c)); k = 0x8f1bbcdcu; }
        else { f = b ^ c ^ d; k = 0xca62c1d6u; }
        uint32_t tmp = rotl(a, 5) + f + e + k + w;
        e = d; d = c; c = rotl(b, 30); b = a; a = tmp;
    }
    H[0] += a; H[1] += b; H[2] += c; H[3] += d; H[4] += e;
}

// IPsec ESP transport mode (RFC 4303 + RFC 3686 + RFC 2404; R#8), in place:
// the header [0,l4) moves to f-16, ESP header + IV fill [l4-16, l4) of the new frame,
// the L4 bytes are encrypted where they lie, trailer and ICV are appended.
// Returns the new frame length.  Stream bytes are handled as 32-bit words; memory
// words are 4-B aligned and related to stream words by a funnel shift of r = A & 3.
// ESP encapsulation of one packet, everything but the payload cipher and the MAC:
// the header moves 16 B left (the frame now starts at f - 16), the IP header is
// fixed up (proto 50, lengths, IPv4 checksum), the ESP header {SPI, seq, IV = 0 || seq}
// goes to [l4 - 16, l4) of the old frame, and (trailer) the pad bytes 1..p, the pad
// length and the next header are written as plaintext after the payload
__device__ __forceinline__ void esp_header(uint8_t *f, const PV &v, uint32_t spi, uint32_t seq, uint32_t p, bool trailer)
{
    const uint32_t l4 = v.l4_off;
    uint32_t *src = reinterpret_cast<uint32_t *>(f);
    uint32_t *dst = reinterpret_cast<uint32_t *>(f - 16);
    uint32_t nw = (l4 + 3) >> 2;
    for (uint32_t i = 0; i < nw; i++) dst[i] = src[i];
    uint8_t *g = f - 16;
    if (v.fam == 4) {
        g[23] = 50;
        uint32_t tot = ((uint32_t)g[16] << 8 | g[17]) + 30 + p;
        g[16] = (uint8_t)(tot >> 8); g[17] = (uint8_t)tot;
        g[24] = 0; g[25] = 0;
        uint32_t sum = 0;
        for (uint32_t k = 14; k < l4; k += 2) sum += (uint32_t)g[k] << 8 | g[k + 1];
        sum = (sum & 0xFFFF) + (sum >> 16);
        sum = (sum & 0xFFFF) + (sum >> 16);
        sum = ~sum;
        g[24] = (uint8_t)(sum >> 8); g[25] = (uint8_t)sum;
    } else {
        g[20] = 50;
        uint32_t pl = ((uint32_t)g[18] << 8 | g[19]) + 30 + p;
        g[18] = (uint8_t)(pl >> 8); g[19] = (uint8_t)pl;
    }
    // the new frame starts at f-16, so its ESP header bytes [l4, l4+16) are f+[l4-16, l4)
    uint8_t *e = f + l4 - 16;
    const uint32_t hw[4] = {spi, seq, 0u, seq};
#pragma unroll
    for (int i = 0; i < 4; i++) {
        e[4 * i] = (uint8_t)(hw[i] >> 24); e[4 * i + 1] = (uint8_t)(hw[i] >> 16);
        e[4 * i + 2] = (uint8_t)(hw[i] >> 8); e[4 * i + 3] = (uint8_t)hw[i];
    }
    if (trailer) {
        const uint32_t plen = v.ip_end - l4;
        uint8_t *t = f + l4 + plen;
        for (uint32_t b = 0; b < p; b++) t[b] = (uint8_t)(b + 1);
        t[p] = (uint8_t)p;
        t[p + 1] = (uint8_t)v.proto;
    }
}
// HMAC-SHA1-96 of an encapsulated packet whose [A, A + clen) is already ciphertext in
// memory (the balanced pass XORed it in at L2): message = ESP header {spi, seq, 0, seq}
// || ciphertext, keyed by the SA's precomputed ipad / opad states; the 12-B ICV is
// written at A + clen.  Only the lines holding header bytes (below A) can sit in L1
// (esp_header read them), so words below `l1` are read L2-only (ld.cg), the rest
// through L1 (one L2 request per line).
__device__ __forceinline__ void esp_mac_mem(uint8_t *A, uint32_t clen, const EspSa *sap, uint32_t seq)
{
    const uint32_t spi = __ldg(&sap->spi), nK = clen >> 2;
    const uint32_t r = (uint32_t)(reinterpret_cast<uintptr_t>(A) & 3);
    uint32_t *W0 = reinterpret_cast<uint32_t *>(A - r);
    const uint32_t sh = 32 - 8 * r;
    const uint32_t *l1 = reinterpret_cast<const uint32_t *>((reinterpret_cast<uintptr_t>(A - 1) | (uintptr_t)127) + 1);
    uint32_t Mcur = __ldcg(W0);
    uint32_t Cprev = r ? (Mcur << (8 * (4 - r))) : 0u;
    uint32_t H[5];
#pragma unroll
    for (int i = 0; i < 5; i++) H[i] = __ldg(&sap->ipad[i]);
    uint32_t W[16];
    const uint32_t nmsg = 4 + nK;
    const uint32_t total_bits = (64u + 4u * nmsg) * 8u;
    const uint32_t nblk = (4 * nmsg + 9 + 63) / 64;
    for (uint32_t blk = 0; blk < nblk; blk++) {
#pragma unroll
        for (int w = 0; w < 16; w++) {
            const uint32_t i = blk * 16 + w;
            uint32_t m;
            if (i < 4) {
                m = (w == 0) ? spi : (w == 2) ? 0u : seq;
            } else if (i < nmsg) {
                const uint32_t k = i - 4;
                const uint32_t Mnext = W0 + k + 1 < l1 ? __ldcg(W0 + k + 1) : W0[k + 1];
                const uint32_t C = __funnelshift_rc(Mcur, Mnext, 8 * r);
                Cprev = C;
                Mcur = Mnext;
                m = bswap32(C);
            } else if (i == nmsg) {
                m = 0x80000000u;
            } else if (i == nblk * 16 - 1) {
                m = total_bits;
            } else {
                m = 0;
            }
            W[w] = m;
        }
        sha1_compress(H, W);
    }
    uint32_t G[5];
#pragma unroll
    for (int i = 0; i < 5; i++) G[i] = __ldg(&sap->opad[i]);
#pragma unroll
    for (int i = 0; i < 16; i++) W[i] = i < 5 ? H[i] : (i == 5 ? 0x80000000u : (i == 15 ? (64u + 20u) * 8u : 0u));
    sha1_compress(G, W);
    const uint32_t icv[3] = {bswap32(G[0]), bswap32(G[1]), bswap32(G[2])};
    W0[nK] = __funnelshift_rc(Cprev, icv[0], sh);
    W0[nK + 1] = __funnelshift_rc(icv[0], icv[1], sh);
    W0[nK + 2] = __funnelshift_rc(icv[1], icv[2], sh);
    if (r) W0[nK + 3] = __funnelshift_rc(icv[2], 0u, sh);
}
// pre: the packet was encapsulated, encrypted and MACed by its tile's balanced pass
// (esp_ctr_tile): only the new frame length is returned
template <bool pre>
__device__ __forceinline__ uint32_t nf_esp(uint8_t *f, const PV &v, const EspSa *sap, uint32_t seq, const uint32_t *te,
                                           const uint32_t *rk_smem)
{
    const uint32_t l4 = v.l4_off, plen = v.ip_end - l4;
#if NFC_ESP_PF
    if constexpr (!pre)
        for (uint32_t o = 128; o < v.ip_end; o += 128) prefetch_l2(f + o);
#endif
    const uint32_t p = (4 - ((plen + 2) & 3)) & 3;
    const uint32_t clen = plen + p + 2;          // multiple of 4
    const uint32_t nK = clen >> 2;
#if NFC_ESP_RK_SMEM
    const uint32_t *rks = rk_smem;
#else
    uint32_t rk[44];
    {
        const uint4 *q = reinterpret_cast<const uint4 *>(sap->rk);
#pragma unroll
        for (int i = 0; i < 11; i++) { uint4 x = __ldg(q + i); rk[4 * i] = x.x; rk[4 * i + 1] = x.y; rk[4 * i + 2] = x.z; rk[4 * i + 3] = x.w; }
    }
#endif
    if constexpr (pre) return v.ip_end + 30 + p;
    const uint32_t spi = __ldg(&sap->spi), nonce = __ldg(&sap->nonce);
    // 1. move the header 16 B left and fix up the IP header
    esp_header(f, v, spi, seq, p, false);
    // 2. encrypt [A, A+clen) in place and MAC [A-16, A+clen), A = f + l4
    uint8_t *A = f + l4;
    const uint32_t r = (uint32_t)(reinterpret_cast<uintptr_t>(A) & 3);
    uint32_t *W0 = reinterpret_cast<uint32_t *>(A - r);   // aligned word 0 (contains stream bytes -r..3-r)
    const uint32_t sh = 32 - 8 * r;                       // funnel amount memory<-stream
    uint32_t Mcur = W0[0];                                // memory word k (plaintext side)
    uint32_t Cprev = r ? (Mcur << (8 * (4 - r))) : 0u;    // carries the IV bytes below A
    uint32_t H[5];
#pragma unroll
    for (int i = 0; i < 5; i++) H[i] = __ldg(&sap->ipad[i]);
    uint32_t W[16];
    const uint32_t nmsg = 4 + nK;                         // message words (ESP hdr + C)
    const uint32_t total_bits = (64u + 4u * nmsg) * 8u;
    const uint32_t nblk = (4 * nmsg + 9 + 63) / 64;       // SHA blocks after the ipad block
    const uint32_t trailer_nh = v.proto;
    uint32_t ks[4] = {0, 0, 0, 0};
    for (uint32_t blk = 0; blk < nblk; blk++) {
#pragma unroll
        for (int w = 0; w < 16; w++) {
            const uint32_t i = blk * 16 + w;              // message word index
            uint32_t m;
            if (i < 4) {
                m = (w == 0) ? spi : (w == 2) ? 0u : seq;
            } else if (i < nmsg) {
                const uint32_t k = i - 4;                 // stream word
                if ((w & 3) == 0) {                       // new AES counter block every 4 words
#if NFC_ESP_RK_SMEM
                    const uint4 o = aes128_encrypt_s(te, rks, nonce, 0u, seq, (k >> 2) + 1);
                    ks[0] = bswap32(o.x); ks[1] = bswap32(o.y); ks[2] = bswap32(o.z); ks[3] = bswap32(o.w);
#else
                    uint32_t o[4];
                    aes128_encrypt(te, rk, nonce, 0u, seq, (k >> 2) + 1, o);
                    ks[0] = bswap32(o[0]); ks[1] = bswap32(o[1]); ks[2] = bswap32(o[2]); ks[3] = bswap32(o[3]);
#endif
                }
                uint32_t Mnext = W0[k + 1];
                uint32_t P = __funnelshift_rc(Mcur, Mnext, 8 * r);   // stream bytes 4k..4k+3 (LE)
                if (4 * k + 4 > plen) {                   // trailer: pad 1..p, p, next header
                    uint32_t pw = 0;
#pragma unroll
                    for (int b = 0; b < 4; b++) {
                        uint32_t s = 4 * k + b, byte;
                        if (s < plen) byte = (P >> (8 * b)) & 0xFF;
                        else if (s < plen + p) byte = s - plen + 1;
                        else if (s == plen + p) byte = p;
                        else byte = trailer_nh;
                        pw |= byte << (8 * b);
                    }
                    P = pw;
                }
                uint32_t C = P ^ ks[w & 3];
                W0[k] = __funnelshift_rc(Cprev, C, sh);   // memory word k (LE)
                Cprev = C;
                Mcur = Mnext;
                m = bswap32(C);
            } else if (i == nmsg) {
                m = 0x80000000u;
            } else if (i == nblk * 16 - 1) {
                m = total_bits;
            } else {
                m = 0;
            }
            W[w] = m;
        }
        sha1_compress(H, W);
    }
    // outer hash: opad state, message = inner digest (20 B)
    uint32_t G[5];
#pragma unroll
    for (int i = 0; i < 5; i++) G[i] = __ldg(&sap->opad[i]);
#pragma unroll
    for (int i = 0; i < 16; i++) W[i] = i < 5 ? H[i] : (i == 5 ? 0x80000000u : (i == 15 ? (64u + 20u) * 8u : 0u));
    sha1_compress(G, W);
    // 3. ICV = first 12 bytes; memory words nK .. nK+3
    const uint32_t icv[3] = {bswap32(G[0]), bswap32(G[1]), bswap32(G[2])};
    W0[nK] = __funnelshift_rc(Cprev, icv[0], sh);
    W0[nK + 1] = __funnelshift_rc(icv[0], icv[1], sh);
    W0[nK + 2] = __funnelshift_rc(icv[1], icv[2], sh);
    if (r) W0[nK + 3] = __funnelshift_rc(icv[2], 0u, sh);
    return v.ip_end + 30 + p;
}

// ---------------------------------------------------------------- the kernel
struct Pkt {
    uint8_t *f;
    uint32_t flen, orig_len;
    uint32_t g;               // index of the packet within the call (global index: pkt_gidx)
    uint32_t h[16];
    PV v;
    uint32_t drop, esp_sa, port, acl_rule, lb_b, nmatch, esp_seq, passmask, esp_bytes, out_len;
    uint32_t npairs;          // pairs of every DPI applied (a chain may repeat DPI; SIG_ANY)
    uint32_t t24;             // TBL24 entry, loaded right after parse (NFC_EARLY_T24)
    uint32_t mmeta, mslot;    // deferred match-pair emission: closure meta, first pair slot
    uint32_t mbase;           // deferred warp-aggregated claim: base slot (lane 0)
    uint32_t esp_pre;         // 1: encapsulated and encrypted by the tile's balanced CTR pass (esp_ctr_tile)
    bool alive;
};


struct Ctx {
    const uint32_t *acl4, *acl6;
    DpiCtx dpi;
    const uint32_t *te, *ms_nib, *lb_nib, *nat_nib;
    const uint32_t *meta;     // per-state match summary (smem or global)
    uint32_t *vst;            // smem u32 hit counters (nullptr: global atomics)
    uint64_t pol_f, pol_l;
    uint32_t gtid;
};

__device__ __forceinline__ void var_stat(const KParams &P, const Ctx &C, uint32_t idx)
{
    if (C.vst) atomicAdd(&C.vst[idx - NFIX], 1u);
    else atomicAdd(&P.stats[idx], 1ull);
}

struct Loc { uint8_t *f; uint32_t len; uint32_t g; };
struct Raw { uint64_t off; uint32_t len, bi; };   // a packet's descriptor loads (issued early)

// batch of packet g (binary search over batch starts) and its off/len loads
__device__ __forceinline__ Raw pkt_raw(const KParams &P, uint32_t g, bool valid)
{
    Raw r{0, 0, 0};
    if (!valid) return r;
    if (P.n_batches == 1) {
        r.off = P.b0.off[g];
        r.len = P.b0.len[g];
        return r;
    }
    uint32_t lo = 0, hi = P.n_batches - 1;
    while (lo < hi) {
        const uint32_t mid = (lo + hi + 1) >> 1;
        if (P.batches[mid].start <= g) lo = mid; else hi = mid - 1;
    }
    const BatchDev &B = P.batches[lo];
    r.off = B.off[g - B.start];
    r.len = B.len[g - B.start];
    r.bi = lo;
    return r;
}
__device__ __forceinline__ Loc pkt_loc(const KParams &P, const Raw &r, uint32_t g, bool valid)
{
    Loc l{nullptr, 0, 0};
    if (!valid) return l;
    if (P.n_batches == 1) {
        l.f = P.b0.arena + r.off;
    } else {
        const BatchDev &B = P.batches[r.bi];
        l.f = B.arena + r.off;
    }
    l.len = r.len;
    l.g = g;
    return l;
}
// Global packet index (low 32 bits: match-pair packet ids) of packet g of the call;
// only lanes that emit match pairs ask, so it is looked up instead of carried
static __device__ __noinline__ uint32_t gidx_search(const BatchDev *bs, uint32_t nb, uint32_t g)
{
    uint32_t lo = 0, hi = nb - 1;
    while (lo < hi) {
        const uint32_t mid = (lo + hi + 1) >> 1;
        if (bs[mid].start <= g) lo = mid; else hi = mid - 1;
    }
    return (uint32_t)bs[lo].first + (g - bs[lo].start);
}
__device__ __forceinline__ uint32_t pkt_gidx(const KParams &P, uint32_t g)
{
    if (P.n_batches == 1) return (uint32_t)P.b0.first + g;
    if (P.crec) {   // the chunk record's batch, unless g lies past a batch boundary in the chunk
        const uint2 m = __ldg(reinterpret_cast<const uint2 *>(&P.crec[g >> 5].gb_lo));
        const uint32_t split = m.y & 31;
        if (!(m.y & 32) && !(split && (g & 31) >= split)) return m.x + g;
    }
    return gidx_search(P.batches, P.n_batches, g);
}

// descriptors of packet g for the pipelined loop: frame offset relative to the arena
// of batch 0 (P.b0.arena, a kernel constant: frame = P.b0.arena + off for every
// batch, 64-bit wrap-around), and length; single batch from the constant bank,
// multi-batch from the chunk record (ChunkRec) -- lanes past a batch boundary in the
// chunk take the binary search.  The rebase add is skipped (warp-uniform branch) when
// the chunk's batch shares batch 0's arena, so the loop top never waits for the
// descriptor loads.
__device__ __forceinline__ void desc_get(const KParams &P, uint32_t g, uint64_t &off, uint32_t &len)
{
    if (P.n_batches == 1) {
        off = P.b0.off[g];
        len = P.b0.len[g];
        return;
    }
    const uint4 *r = reinterpret_cast<const uint4 *>(P.crec + (g >> 5));
    const uint4 a = __ldg(r), b = __ldg(r + 1);
    const uint32_t split = b.w & 31, lane = g & 31;
    if ((b.w & 32) || (split && lane >= split)) {
        const Raw w = pkt_raw(P, g, true);
        off = (uint64_t)P.batches[w.bi].arena + w.off - (uint64_t)P.b0.arena;
        len = w.len;
        return;
    }
    const uint64_t *offp = reinterpret_cast<const uint64_t *>((uint64_t)a.x | (uint64_t)a.y << 32);
    const uint16_t *lenp = reinterpret_cast<const uint16_t *>((uint64_t)a.z | (uint64_t)a.w << 32);
    off = offp[g];
    len = lenp[g];
    const uint64_t delta = ((uint64_t)b.x | (uint64_t)b.y << 32) - (uint64_t)P.b0.arena;
    if (delta != 0) off += delta;   // same record for every lane here: uniform
}

// shared-memory word the warp itself rewrites (volatile: never hoisted or merged)
__device__ __forceinline__ uint32_t lds_u32_v(uint32_t a)
{
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
    return v;
}

// multi-batch: the chunk record of chunk c copied into this warp's shared-memory slot
// (cp.async by lanes 0-1: no registers held; consumed a chunk later)
__device__ __forceinline__ void crec_stage(const KParams &P, uint32_t c, uint32_t slot_addr, uint32_t lane)
{
    if (lane < 2 && c < P.n_pkts) {
        const char *src = reinterpret_cast<const char *>(P.crec + (c >> 5)) + 16 * lane;
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(slot_addr + 16 * lane), "l"(src) : "memory");
        asm volatile("cp.async.commit_group;" ::: "memory");
    }
}
// desc_get (above) with the chunk record read from its staging slot (after cp.async.wait_all
// and __syncwarp by the whole warp)
__device__ __forceinline__ void desc_get_s(const KParams &P, uint32_t g, uint64_t &off, uint32_t &len, uint32_t slot_addr)
{
    uint4 a, b;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(a.x), "=r"(a.y), "=r"(a.z), "=r"(a.w) : "r"(slot_addr));
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(b.x), "=r"(b.y), "=r"(b.z), "=r"(b.w) : "r"(slot_addr + 16));
    const uint32_t split = b.w & 31, lane = g & 31;
    if ((b.w & 32) || (split && lane >= split)) {
        const Raw w = pkt_raw(P, g, true);
        off = (uint64_t)P.batches[w.bi].arena + w.off - (uint64_t)P.b0.arena;
        len = w.len;
        return;
    }
    const uint64_t *offp = reinterpret_cast<const uint64_t *>((uint64_t)a.x | (uint64_t)a.y << 32);
    const uint16_t *lenp = reinterpret_cast<const uint16_t *>((uint64_t)a.z | (uint64_t)a.w << 32);
    off = offp[g];
    len = lenp[g];
    const uint64_t delta = ((uint64_t)b.x | (uint64_t)b.y << 32) - (uint64_t)P.b0.arena;
    if (delta != 0) off += delta;   // same record for every lane here: uniform
}

__device__ __forceinline__ Loc pkt_locate(const KParams &P, uint32_t g, bool valid)
{
    return pkt_loc(P, pkt_raw(P, g, valid), g, valid);
}

__device__ __forceinline__ void pkt_begin(const Ctx &C, const Loc &l, bool valid, Pkt &k)
{
    k.drop = 0xFF; k.esp_sa = 0xFF; k.port = 0; k.acl_rule = 0xFFFF; k.lb_b = 0xFFFF; k.nmatch = 0;
    k.esp_seq = 0; k.passmask = 0; k.esp_bytes = 0; k.alive = false; k.t24 = 0xFFFFFFFFu; k.mmeta = 0; k.mbase = 0;
    k.esp_pre = 0;
    k.npairs = 0;
    k.f = l.f; k.flen = k.orig_len = l.len; k.g = l.g;
    k.out_len = k.flen;
    if (!valid) return;
    load_header(k.f, k.flen, k.h, C.pol_f);
    k.alive = parse(k.h, k.f, k.flen, k.v);
    if (!k.alive) k.drop = 0xFE;
}

// pkt_begin with the header words already loaded (NFC_HDR_AHEAD)
__device__ __forceinline__ void pkt_begin_h(const Loc &l, bool valid, Pkt &k, const uint32_t hn[16])
{
    k.drop = 0xFF; k.esp_sa = 0xFF; k.port = 0; k.acl_rule = 0xFFFF; k.lb_b = 0xFFFF; k.nmatch = 0;
    k.esp_seq = 0; k.passmask = 0; k.esp_bytes = 0; k.alive = false; k.t24 = 0xFFFFFFFFu; k.mmeta = 0; k.mbase = 0;
    k.esp_pre = 0;
    k.npairs = 0;
    k.f = l.f; k.flen = k.orig_len = l.len; k.g = l.g;
    k.out_len = k.flen;
    if (!valid) return;
#pragma unroll
    for (int i = 0; i < 16; i++) k.h[i] = hn[i];
    k.alive = parse(k.h, k.f, k.flen, k.v);
    if (!k.alive) k.drop = 0xFE;
}

// (packet, pattern) pairs of an output closure [o0, o0+nm) at slots [slot, slot+nm)
__device__ __forceinline__ void emit_pairs(const KParams &P, uint32_t o0, uint32_t nm, uint32_t slot, uint32_t pkt)
{
    // o0: CSR offset of the closure, or (nm == 1) the pattern id itself (DpiHost::out_meta)
    for (uint32_t q = 0; q < nm; q++)
        if (slot + q < P.match_cap) {
            P.match_pkt[slot + q] = pkt;
            P.match_pat[slot + q] = nm == 1 ? o0 : __ldg(P.dpi.out_ids + o0 + q);
        }
    if (slot + nm > P.match_cap)
        atomicAdd(&P.stats[ST_MATCH_OVF], (unsigned long long)(slot + nm - max(slot, P.match_cap)));
}

// DPI result of a packet from its walk summary (R#9/R#10): no accept
// event -> no match; exactly one -> the output closure of that state (per-state summary:
// size + DROP flag); more -> exact re-walk (dpi_slow).  Returns true if a DROP pattern matched.
template <int DM>
__device__ __forceinline__ bool dpi_finish(const KParams &P, const Ctx &C, Pkt &k, const Walk w)
{
    bool dropped = false;
    k.nmatch = 0;                 // this DPI's count (a chain may repeat DPI: no earlier count carried)
    // DM_FULL: C.meta holds the accepting slots' summaries (index ~slot)
    const uint32_t st = DM == DM_FULL ? ~w.mx : C.dpi.wide ? (w.mx & 0x7FFFFFFFu) : (w.mx & 0x7FFFu);
    const uint32_t meta = w.cnt == 1 ? C.meta[st] : 0u;
    if (w.cnt == 1 && meta != DPI_META_NONE) {
        // exactly one accept event: the match set is the output closure of that state
        // (distinct ids); its size and DROP flag come from the per-state summary.  The
        // pair slots are claimed now and the pairs written at the end of the chunk, so
        // the atomic's latency overlaps the rest of the chain.
        const uint32_t nm = (meta >> 20) & 0x7FF;
        k.nmatch = nm;
        dropped = (meta >> 31) != 0;
        // (per-lane path: emitted at once -- the unfused and parallel kernels have no pkt_end)
        emit_pairs(P, meta & 0xFFFFF, nm, atomicAdd(P.match_count, nm), pkt_gidx(P, k.g));
    } else if (w.cnt >= 1) {
        const DpiOvf ov{P.dpi.ovf_bitmap, P.dpi.bitmap_words, P.match_count, P.match_pkt, P.match_pat,
                        P.match_cap, P.stats, 1u};
        const uint32_t r = dpi_slow<DM>(C.dpi, k.f, k.v.pl_off, k.v.ip_end, C.gtid, ov, pkt_gidx(P, k.g));
        k.nmatch = r & 0x7FFFFFFFu;
        dropped = (r >> 31) != 0;
    }
    return dropped;
}

// dpi_finish for a whole warp (all lanes call it): the match-pair slots of the lanes whose
// walk had exactly one accept event are claimed with ONE atomic per warp (sum of the
// closure sizes, exclusive prefix by ballot/popc when every closure has one pattern, else
// by a shuffle scan); lanes with several events take the exact re-walk as in dpi_finish.
template <int DM>
__device__ __forceinline__ bool dpi_finish_warp(const KParams &P, const Ctx &C, Pkt &k, const Walk w, bool act)
{
    const uint32_t FULL = 0xFFFFFFFFu, lane = threadIdx.x & 31;
    const uint32_t st = DM == DM_FULL ? ~w.mx : C.dpi.wide ? (w.mx & 0x7FFFFFFFu) : (w.mx & 0x7FFFu);
    const uint32_t meta = act && w.cnt == 1 ? C.meta[st] : DPI_META_NONE;
    const bool single = meta != DPI_META_NONE;
    const uint32_t nm = single ? (meta >> 20) & 0x7FF : 0u;
    bool dropped = false;
    if (__any_sync(FULL, nm != 0)) {
        uint32_t excl, total;
        if (__all_sync(FULL, nm <= 1)) {
            const uint32_t b = __ballot_sync(FULL, nm != 0);
            excl = __popc(b & ((1u << lane) - 1));
            total = __popc(b);
        } else {
            uint32_t incl = nm;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t y = __shfl_up_sync(FULL, incl, d);
                if (lane >= (uint32_t)d) incl += y;
            }
            total = __shfl_sync(FULL, incl, 31);
            excl = incl - nm;
        }
        uint32_t base = 0;
        if (lane == 0) base = atomicAdd(P.match_count, total);
#if NFC_DEFER_PAIRS
        // the atomic's result is consumed at the end of the chunk (pkt_end): its round trip
        // overlaps the NFs after the DPI
        k.mbase = base;
        k.mslot = excl;
        k.mmeta = nm ? meta & 0x7FFFFFFFu : 0u;
#else
        base = __shfl_sync(FULL, base, 0);
        if (nm) emit_pairs(P, meta & 0xFFFFF, nm, base + excl, pkt_gidx(P, k.g));
#endif
    }
    if (single) {
        k.nmatch = nm;
        dropped = (meta >> 31) != 0;
    } else if (act && w.cnt >= 1) {
        const DpiOvf ov{P.dpi.ovf_bitmap, P.dpi.bitmap_words, P.match_count, P.match_pkt, P.match_pat,
                        P.match_cap, P.stats, 1u};
        const uint32_t r = dpi_slow<DM>(C.dpi, k.f, k.v.pl_off, k.v.ip_end, C.gtid, ov, pkt_gidx(P, k.g));
        k.nmatch = r & 0x7FFFFFFFu;
        dropped = (r >> 31) != 0;
    }
    return dropped;
}

// DPI for the 32 packets of a warp, called by all lanes (compile-time chains).  With
// the whole DFA on chip (DM_FULL) each lane first walks its own packet's payload bytes
// below 64 from the header cache.  The rest of the 32 payloads ([base, b) per packet,
// base = 64 or the 16-B line of the payload start, padded to 16 B) is concatenated into one virtual byte stream and cut
// into 32 equal 16-B-aligned ranges, one per lane, so IMIX lengths do not leave lanes
// idle.  All lanes advance one 16-B chunk per iteration (a convergent loop); a lane
// whose piece ends fetches the next piece's packet by warp shuffles.  A piece that
// starts inside a payload re-walks the maxlen - 1 bytes before it from the root
// without counting (the Aho-Corasick state depends only on the last maxlen bytes, so
// the state at the piece start is exact); a piece at the start of a remainder
// continues the owner's walk.  Piece results (accept-event count, largest entry) are
// combined into the owner's summary through shared memory, so the owner ends with
// exactly the (cnt, mx) of a sequential walk, evaluated by dpi_finish.
template <int DM>
__device__ __forceinline__ bool nf_dpi_warp(const KParams &P, const Ctx &C, Pkt &k, const Walk *head = nullptr)
{
    const uint32_t FULL = 0xFFFFFFFFu, lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (DM != DM_FULL && P.dpi.wide)          // > 32K states: per-lane walk from L2
        return k.alive ? dpi_finish<DM>(P, C, k, dpi_walk<DM>(P, C.dpi, k.h, k.f, k.v.pl_off, k.v.ip_end, C.pol_f))
                       : false;
    const bool act = k.alive;
    const uint32_t a = k.v.pl_off, b = k.v.ip_end;
    Walk w{0, 0, 0};
    // DM_FULL: bytes below 64 from the header cache (registers); DM_HOT: everything
    // through the stream (one copy of the walk loop keeps the kernel's code small)
    if (DM == DM_FULL && head) w = *head;     // walked speculatively with the ACL (spec_acl_dpi)
    else if (DM == DM_FULL && act) w = dpi_walk_head<DM>(P, k.h, a, b);
    const uint32_t base = (DM != DM_FULL || a >= 64) ? (a & ~15u) : 64u;
    // (an empty payload past byte 64 -- e.g. IPv6/TCP frames of 74 B -- has nothing to walk)
    const uint32_t rem = act && b > max(a, base) ? (b - base + 15) & ~15u : 0u;
    if (__any_sync(FULL, rem != 0)) {         // warp-uniform (64-B frames: never)
        uint32_t incl = rem;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(FULL, incl, d);
            if (lane >= (uint32_t)d) incl += y;
        }
        const uint32_t total = __shfl_sync(FULL, incl, 31);
        const uint32_t excl = incl - rem;
        uint32_t *acc = reinterpret_cast<uint32_t *>(nfc_smem + P.lay.seg) + warp * 64;
        acc[lane] = 0;
        acc[32 + lane] = 0;
        __syncwarp();
        const uint32_t per = ((total + 31) / 32 + 15) & ~15u;
        uint32_t lo = min(lane * per, total);
        const uint32_t hi = min(lo + per, total);
        const uint32_t O = P.dpi.maxlen - 1;
        const uint64_t fa = reinterpret_cast<uint64_t>(k.f);
        uint32_t x = 0, e0 = 0, v0 = 0, sc = 0, own = 0;
        const uint8_t *f = nullptr;
        Walk pw{0, 0, 0};
#if NFC_WALK_AHEAD
        uint4 qn = make_uint4(0, 0, 0, 0);     // the next 16 payload bytes, loaded one step ahead
        bool have = false;
#endif
        for (;;) {
            const bool need = x >= e0 && lo < hi;
            if (__any_sync(FULL, need)) {
                // next piece: the packet owning virtual byte lo (the last whose range starts at or before it)
                uint32_t p = 0;
#pragma unroll
                for (uint32_t bit = 16; bit; bit >>= 1)
                    if (__shfl_sync(FULL, excl, p + bit) <= lo) p += bit;
                const uint32_t pe = __shfl_sync(FULL, incl, p), px = __shfl_sync(FULL, excl, p);
                const uint32_t pb = __shfl_sync(FULL, base, p), pa = __shfl_sync(FULL, a, p);
                const uint32_t pend = __shfl_sync(FULL, b, p), ps = __shfl_sync(FULL, w.s, p);
                const uint64_t pf = __shfl_sync(FULL, fa, p);
                if (need) {
                    const uint32_t ev = min(hi, pe);
                    const uint32_t s0 = pb + (lo - px);
                    e0 = min(pb + (ev - px), pend);
                    own = p;
                    f = reinterpret_cast<const uint8_t *>(pf);
                    if (s0 == pb) {               // continues the owner's walk
                        pw = Walk{ps, 0, 0};
                        v0 = max(pa, s0);
                        x = s0;
                        sc = s0;
                    } else {                      // warm-up from the root, counting from s0
                        pw = Walk{0, 0, 0};
                        v0 = max(pa, s0 - min(O, s0));
                        x = v0 & ~15u;
                        sc = s0;
                    }
                    for (uint32_t l = x & ~127u; l < min(e0, x + NFC_PF_DIST); l += 128) prefetch_l2(f + l);
                    lo = ev;
#if NFC_WALK_AHEAD
                    have = false;
#endif
                }
            }
            const bool run = x < e0;
            if (!__any_sync(FULL, run)) break;
            if (run) {
                if (x == sc) { pw.cnt = 0; pw.mx = 0; }
                if ((x & 127) == 0 && x + NFC_PF_DIST < e0) prefetch_l2(f + x + NFC_PF_DIST);
#if NFC_WALK_AHEAD
                // software-pipelined payload loads: this step's 16 bytes were loaded during the
                // previous step; the next 16 go out now, so the walk never waits on the L2
                const uint4 q = have ? qn : ld_stream16(f + x, C.pol_f);
                have = x + 16 < e0;
                if (have) qn = ld_stream16(f + x + 16, C.pol_f);
#else
                const uint4 q = ld_stream16(f + x, C.pol_f);
#endif
                uint32_t wd[4] = {q.x, q.y, q.z, q.w};
                if ((DM == DM_FULL || NFC_HOT_FAST) && x >= v0 && x + 16 <= e0) {
#pragma unroll
                    for (int kk = 0; kk < 16; kk++) {
                        const uint32_t y = (kk & 3) == 0 ? tie<DM>(wd[kk >> 2], pw) : wd[kk >> 2];
                        if ((kk & 3) == 0) wd[kk >> 2] = y;
                        dfa_step<DM>(P, pw, byte_of(y, kk & 3));
                    }
                } else {
#pragma unroll
                    for (int kk = 0; kk < 16; kk++) {
                        const uint32_t y = (kk & 3) == 0 ? tie<DM>(wd[kk >> 2], pw) : wd[kk >> 2];
                        if ((kk & 3) == 0) wd[kk >> 2] = y;
                        dfa_step_if<DM>(P, pw, byte_of(y, kk & 3), x + kk - v0 < e0 - v0);
                    }
                }
                x += 16;
                if (x >= e0 && pw.cnt) {          // piece done: into the owner's summary
                    atomicAdd(&acc[own], pw.cnt);
                    atomicMax(&acc[32 + own], pw.mx);
                }
            }
        }
        __syncwarp();
        if (rem) {
            w.cnt += acc[lane];
            w.mx = max(w.mx, acc[32 + lane]);
        }
    }
    return dpi_finish_warp<DM>(P, C, k, w, act);
}

// ---------------------------------------------------------------- speculative ACL || DPI || TBL24
// Chains that open with ACL -> DPI (C1, C3, the C5 prefixes) on a whole-DFA launch:
// the ACL classification, the DPI walk over the payload bytes in the header cache
// and (if LPM4 follows) the DIR-24-8 first-level read are pure functions of the
// parsed packet, so they are computed together in ONE basic block -- no branches,
// the ACL window search with predicated steps -- and the scheduler interleaves the
// ACL's shared-memory chain and the TBL24 read with the DFA chain.  Their effects are
// then applied in chain order (nf_apply / nf_dpi_warp), so results equal the
// sequential chain (effects in original-order packet state).  Taken when
// warp-uniformly: IPv4 ACL image with rules, <= 64 rules, depth <= 3, staged in
// shared memory; otherwise the sequential path runs.
// DPI walk of payload bytes [a, min(b, 64)) from the header cache for a >= 42, every
// step predicated (UDP and TCP payload starts in one code path)
__device__ __forceinline__ Walk dpi_head_spec(const KParams &P, const uint32_t h[16], uint32_t a, uint32_t b)
{
    Walk w{0, 0, 0};
#pragma unroll
    for (int idx = 42; idx < 64; idx++)
        dfa_step_if<DM_FULL>(P, w, byte_of(h[idx >> 2], idx & 3), (uint32_t)idx - a < b - a);
    return w;
}
// the same walk when every lane's payload starts at byte 42 (UDP) or 54 (TCP) and runs
// past byte 64: unconditional steps, a TCP lane restarting from the root at byte 54
__device__ __forceinline__ Walk dpi_head_fast(const KParams &P, const uint32_t h[16], bool tcp)
{
    Walk w{0, 0, 0};
#pragma unroll
    for (int idx = 42; idx < 64; idx++) {
        if (idx == 54 && tcp) w = Walk{0, 0, 0};
        dfa_step<DM_FULL>(P, w, byte_of(h[idx >> 2], idx & 3));
    }
    return w;
}
template <uint32_t S>
__device__ __forceinline__ bool spec_ok(const KParams &P)
{
    return S != SIG_ANY && sig_kind(S, 0) == NFC_ACL && sig_n(S) >= 2 && sig_kind(S, 1) == NFC_DPI &&
           P.acl.smem_words && P.acl.fast;
}

// one NF of kind KIND at chain position pos (KIND compile-time)
template <uint32_t KIND, int DM>
__device__ __forceinline__ void nf_apply(const KParams &P, const Ctx &C, Pkt &k, uint32_t pos)
{
    bool dropped = false;
    if constexpr (KIND == NFC_ACL) {
        const uint32_t r = nf_acl_fused(P, k.v);
        const uint32_t rule = r & 0xFFFF;
        k.acl_rule = rule;
        var_stat(P, C, P.st_acl + (rule == 0xFFFF ? P.acl.n_rules : rule));
        dropped = (r >> 31) != 0;
    } else if constexpr (KIND == NFC_DPI) {
        dropped = dpi_finish<DM>(P, C, k, dpi_walk<DM>(P, C.dpi, k.h, k.f, k.v.pl_off, k.v.ip_end, C.pol_f));
        k.npairs += k.nmatch;
    } else if constexpr (KIND == NFC_LPM4) {
        // DIR-24-8: at most two dependent table reads ("two memory accesses")
        if (k.v.fam != 4) { k.passmask |= 1u << pos; return; }
        uint32_t nh = k.t24 != 0xFFFFFFFFu ? k.t24 : ld_tab16(P.l4.tbl24 + (k.v.dst[0] >> 8), C.pol_l);
        if (nh & 0x8000) nh = ld_tab16(P.l4.tbllong + ((nh & 0x7FFF) << 8) + (k.v.dst[0] & 0xFF), C.pol_l);
        if (nh == 0x7FFF || hbyte(k.h, 22) <= 1) dropped = true;
        else if (P.l4.nh_smem) {          // {nh, pmac[nh.port]} in one shared-memory record
            const uint4 r = reinterpret_cast<const uint4 *>(nfc_smem + P.lay.nh4)[nh];
            forward_rewrite(k.f, k.h, k.v, make_uint2(r.x, r.y), make_uint2(r.z, r.w), C.pol_f);
            k.port = r.y >> 16;
        } else {
            const uint2 n = __ldg(P.l4.nh + nh);
            const uint32_t pt = n.y >> 16;
            forward_rewrite(k.f, k.h, k.v, n, __ldg(P.l4.pmac + pt), C.pol_f);
            k.port = pt;
        }
    } else if constexpr (KIND == NFC_LPM6) {
        if (k.v.fam != 6) { k.passmask |= 1u << pos; return; }
        const uint32_t nh = lpm6_lookup(P.l6, k.v.dst);
        if (nh == 0x7FFF || hbyte(k.h, 21) <= 1) dropped = true;
        else {
            const uint2 n = __ldg(P.l6.nh + nh);
            const uint32_t pt = n.y >> 16;
            forward_rewrite(k.f, k.h, k.v, n, __ldg(P.l6.pmac + pt), C.pol_f);
            k.port = pt;
        }
    } else if constexpr (KIND == NFC_IPSEC) {
        const uint32_t *rks = reinterpret_cast<const uint32_t *>(nfc_smem + P.lay.rk) + k.esp_sa * ESP_RK_STRIDE;
        // (two instances: the MAC-only one after the tile's balanced CTR pass, tile-uniform)
        const uint32_t nl = k.esp_pre ? nf_esp<true>(k.f, k.v, P.esp.sa + k.esp_sa, k.esp_seq, C.te, rks)
                                      : nf_esp<false>(k.f, k.v, P.esp.sa + k.esp_sa, k.esp_seq, C.te, rks);
        k.esp_bytes = nl - 28 - k.v.l4_off;      // ciphertext bytes |C|
        k.f -= 16;
        k.flen = nl;
        k.out_len = nl;
        load_header(k.f, k.flen, k.h, C.pol_f);
        parse(k.h, k.f, k.flen, k.v);             // later NFs see proto 50, ports 0
    } else if constexpr (KIND == NFC_NAT) {
        const bool l4 = k.v.fam == 4 && (k.v.proto == 6 || k.v.proto == 17) && k.v.pl_off != k.v.l4_off;
        if (!l4 || k.port >= 32 || !((P.nat.ext_ports >> k.port) & 1)) { k.passmask |= 1u << pos; return; }
        nf_nat(P, C.nat_nib, k.f, k.h, k.v, C.pol_f);
    } else if constexpr (KIND == NFC_LB) {
        const uint32_t hsh = toeplitz(C.lb_nib, k.v);
        const uint32_t b = (uint32_t)(((uint64_t)hsh * P.lb.n_backends) >> 32);
        k.lb_b = b;
        k.port = __ldg(P.lb.port + b);
        var_stat(P, C, P.st_lb + b);
    }
    if (dropped) { k.drop = pos; k.alive = false; }
}

// positions [POS, END) of a compile-time chain; SIG_ANY interprets P.kind
template <uint32_t S, int DM, int POS, int END>
__device__ __forceinline__ void run_fixed(const KParams &P, const Ctx &C, Pkt &k)
{
    if constexpr (POS < END) {
        if constexpr (sig_kind(S, POS) == NFC_DPI) {
            // warp-cooperative (all lanes): payload bytes split evenly over the lanes
            if (nf_dpi_warp<DM>(P, C, k)) { k.drop = POS; k.alive = false; }
        } else {
            if (k.alive) nf_apply<sig_kind(S, POS), DM>(P, C, k, POS);
        }
        run_fixed<S, DM, POS + 1, END>(P, C, k);
    }
}
template <int DM>
__device__ __forceinline__ void run_any(const KParams &P, const Ctx &C, Pkt &k, uint32_t from, uint32_t to)
{
    for (uint32_t pos = from; pos < to && k.alive; pos++) {
        switch (P.kind[pos]) {
        case NFC_ACL: nf_apply<NFC_ACL, DM>(P, C, k, pos); break;
        case NFC_DPI: nf_apply<NFC_DPI, DM>(P, C, k, pos); break;
        case NFC_LPM4: nf_apply<NFC_LPM4, DM>(P, C, k, pos); break;
        case NFC_LPM6: nf_apply<NFC_LPM6, DM>(P, C, k, pos); break;
        case NFC_IPSEC: nf_apply<NFC_IPSEC, DM>(P, C, k, pos); break;
        case NFC_LB: nf_apply<NFC_LB, DM>(P, C, k, pos); break;
        case NFC_NAT: nf_apply<NFC_NAT, DM>(P, C, k, pos); break;
        }
    }
}
// chain positions [0, esp) or [esp, n) (esp = n for chains without IPsec)
template <uint32_t S, int DM, bool HEAD>
__device__ __forceinline__ void run_part(const KParams &P, const Ctx &C, Pkt &k)
{
    if constexpr (HEAD && NFC_EARLY_T24 && S != SIG_ANY && sig_pos(S, NFC_LPM4) != 0xFF && sig_pos(S, NFC_LPM4) != 0) {
        // header-phase read of the DIR-24-8 first level: its latency overlaps the NFs
        // before LPM4 (a later NF may rewrite only the IPsec-moved header, and IPsec is
        // never placed before LPM4 in the instantiated signatures)
        static_assert(sig_pos(S, NFC_IPSEC) == 0xFF || sig_pos(S, NFC_IPSEC) > sig_pos(S, NFC_LPM4), "");
        if (k.alive && k.v.fam == 4) k.t24 = ld_tab16(P.l4.tbl24 + (k.v.dst[0] >> 8), C.pol_l);
    }
    if constexpr (NFC_SPEC && HEAD && S != SIG_ANY && DM == DM_FULL && sig_n(S) >= 2 && sig_kind(S, 0) == NFC_ACL &&
                  sig_kind(S, 1) == NFC_DPI) {
        // speculative ACL || DPI head walk || TBL24 (see spec_ok), warp-uniform choice
        // every payload starts at byte 42 or later; IPv6 lanes (dual-stack traffic) take the
        // IPv4 classification speculatively too and are re-classified below
        // dual-stack warps too for ACL -> DPI and ACL -> DPI -> LPM4 -> LPM6 (measured: +12 % and
        // +4 % on C5 k2 / k4 64 B; -2 % on k3 and -6 % on C1, whose instance keeps the IPv4 gate)
        constexpr bool V6 = NFC_SPEC_V6 || S == make_sig(2, NFC_ACL, NFC_DPI) ||
                            S == make_sig(4, NFC_ACL, NFC_DPI, NFC_LPM4, NFC_LPM6);
        const bool v4 = !k.alive || ((k.v.fam == 4 || V6) && k.v.pl_off >= 42);
        if (spec_ok<S>(P) && __all_sync(0xFFFFFFFFu, v4)) {
            constexpr bool T24 = sig_pos(S, NFC_LPM4) != 0xFF &&
                                 (sig_pos(S, NFC_IPSEC) == 0xFF || sig_pos(S, NFC_IPSEC) > sig_pos(S, NFC_LPM4));
            // UDP/TCP payloads from byte 42/54 past byte 64 (64-B-class frames): unconditional
            // DFA steps; else every step predicated.  Each branch is one basic block.
            const bool fastw = __all_sync(0xFFFFFFFFu, !k.alive || ((k.v.pl_off == 42 || k.v.pl_off == 54) &&
                                                                    k.v.ip_end >= 64));
            uint32_t r;
            Walk wh;
            if (fastw) {
                r = acl4_fast(P.lay.acl4, P.acl, k.v);
                wh = dpi_head_fast(P, k.h, k.v.pl_off == 54);
                if constexpr (T24) k.t24 = ld_tab16(P.l4.tbl24 + (k.v.dst[0] >> 8), C.pol_l);
            } else {
                r = acl4_fast(P.lay.acl4, P.acl, k.v);
                wh = dpi_head_spec(P, k.h, k.v.pl_off, k.v.ip_end);
                if constexpr (T24) k.t24 = ld_tab16(P.l4.tbl24 + (k.v.dst[0] >> 8), C.pol_l);
            }
#if NFC_T24_L2_EARLY
            // the DIR-24-8 second level right after the block (its first level has arrived):
            // the read overlaps the DPI finish and the match-pair atomic instead of the LPM
            if constexpr (T24)
                if (k.t24 & 0x8000) k.t24 = ld_tab16(P.l4.tbllong + ((k.t24 & 0x7FFF) << 8) + (k.v.dst[0] & 0xFF), C.pol_l);
#endif
            if (V6 && k.alive && k.v.fam != 4) r = nf_acl_fused(P, k.v);   // IPv6 lanes
            if (k.alive) {                     // ACL effects (position 0)
                const uint32_t rule = r & 0xFFFF;
                k.acl_rule = rule;
                var_stat(P, C, P.st_acl + (rule == 0xFFFF ? P.acl.n_rules : rule));
                if (r >> 31) { k.drop = 0; k.alive = false; }
            }
            if (nf_dpi_warp<DM>(P, C, k, &wh)) { k.drop = 1; k.alive = false; }
            constexpr int E = sig_pos(S, NFC_IPSEC) == 0xFF ? (int)sig_n(S) : (int)sig_pos(S, NFC_IPSEC);
            run_fixed<S, DM, 2, E>(P, C, k);
            return;
        }
    }
    if constexpr (S == SIG_ANY) {
        const uint32_t e = min(P.esp_pos, P.n_nf);
        if (HEAD) run_any<DM>(P, C, k, 0, e);
        else run_any<DM>(P, C, k, e, P.n_nf);
    } else {
        constexpr int N = (int)sig_n(S);
        constexpr int E = sig_pos(S, NFC_IPSEC) == 0xFF ? N : (int)sig_pos(S, NFC_IPSEC);
        if constexpr (HEAD) run_fixed<S, DM, 0, E>(P, C, k);
        else run_fixed<S, DM, E, N>(P, C, k);
    }
}

// Record store + counters of one warp's 32 packets into the warp's private slot.
// Only independent counts are kept per warp (chain-position "in", "applied" and
// the total drop count are derived at the flush).
template <uint32_t S>
__device__ __forceinline__ void pkt_end(const KParams &P, const Ctx &C, Pkt &k, bool valid, uint32_t g,
                                        unsigned long long *ws, uint32_t lane)
{
    constexpr uint32_t M = sig_mask(S);
    if constexpr ((M & MASK_DPI) != 0 && NFC_DEFER_PAIRS) {
        // warp-aggregated claims keep the base in lane 0 (k.mbase) and the lane's offset in
        // k.mslot; per-lane claims keep the absolute slot in k.mslot and k.mbase = 0
        if (__any_sync(0xFFFFFFFFu, k.mmeta != 0)) {
            const uint32_t b0 = __shfl_sync(0xFFFFFFFFu, k.mbase, 0);
            if (k.mmeta) emit_pairs(P, k.mmeta & 0xFFFFF, k.mmeta >> 20, b0 + k.mslot, pkt_gidx(P, k.g));
        }
    }
    if (valid) {
        if (k.drop != 0xFF) k.port = 0xFFFF;
        const uint4 rec = make_uint4(k.drop | k.esp_sa << 8 | k.port << 16, k.acl_rule | k.lb_b << 16,
                                     k.nmatch | k.out_len << 16, k.esp_seq);
        st_stream16(reinterpret_cast<uint4 *>(P.rec) + g, rec, C.pol_f);
    }
    const uint32_t FULL = 0xFFFFFFFFu;
    const bool fwd = valid && k.drop == 0xFF;
    const uint32_t nv = __popc(__ballot_sync(FULL, valid));
    const uint32_t nparse = __popc(__ballot_sync(FULL, valid && k.drop == 0xFE));
    const uint32_t nfwd = NFC_FWD_DERIVED ? 0u : __popc(__ballot_sync(FULL, fwd));
    const uint32_t bin = __reduce_add_sync(FULL, valid ? k.orig_len : 0u);
    const uint32_t bout = __reduce_add_sync(FULL, fwd ? k.out_len : 0u);
    uint32_t pairs = 0, nesp = 0, eb = 0, eblk = 0;
    if constexpr ((M & MASK_DPI) != 0) pairs = __reduce_add_sync(FULL, S == SIG_ANY ? k.npairs : k.nmatch);
    if constexpr ((M & MASK_IPSEC) != 0) {
        const bool esp = k.esp_sa != 0xFF;
        nesp = __popc(__ballot_sync(FULL, esp));
        eb = __reduce_add_sync(FULL, esp ? k.esp_bytes : 0u);
        eblk = __reduce_add_sync(FULL, esp ? (k.esp_bytes + 15) >> 4 : 0u);
    }
    if (lane == 0) {
        ws[ST_PKTS] += nv;
        if (!NFC_FWD_DERIVED) ws[ST_FWD] += nfwd;
        ws[ST_PARSE_DROP] += nparse;
        ws[ST_BYTES_IN] += bin;
        ws[ST_BYTES_OUT] += bout;
        if constexpr ((M & MASK_DPI) != 0) ws[ST_DPI_PAIRS] += pairs;
        if constexpr ((M & MASK_IPSEC) != 0) {
            ws[ST_ESP_PKTS] += nesp;
            ws[ST_ESP_BYTES] += eb;
            ws[ST_ESP_BLOCKS] += eblk;
        }
    }
    constexpr int NP = S == SIG_ANY ? NFC_MAX_CHAIN : (int)sig_n(S);
#pragma unroll
    for (int p = 0; p < NP; p++) {
        if (S == SIG_ANY && (uint32_t)p >= P.n_nf) break;          // uniform
        const uint32_t nd = __popc(__ballot_sync(FULL, valid && k.drop == (uint32_t)p));
        const uint32_t kd = S == SIG_ANY ? P.kind[p] : sig_kind(S, p);
        uint32_t np = 0;
        if (kd == NFC_LPM4 || kd == NFC_LPM6 || kd == NFC_NAT) np = __popc(__ballot_sync(FULL, (k.passmask >> p) & 1));
        if (lane == 0) {
            ws[ST_POS_BASE + 4 * p + 1] += nd;
            ws[ST_POS_BASE + 4 * p + 2] += np;
        }
    }
}

// ESP sequence numbers for one CTA tile: per SA, global packet order (decoupled look-back)
template <int NW>
__device__ __forceinline__ void esp_assign(const KParams &P, const Ctx &C, uint8_t *smem, const SmemLayout &L,
                                           uint32_t tile, Pkt &k)
{
    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t nsa = P.esp.n_sa;
    uint16_t *wcnt = reinterpret_cast<uint16_t *>(smem + L.wcnt);
    uint32_t *pref = reinterpret_cast<uint32_t *>(smem + L.prefix);
    for (uint32_t i = tid; i < NW * 256; i += NW * 32) wcnt[i] = 0;
    uint32_t sa = 0xFFFF;
    if (k.alive) sa = toeplitz(C.ms_nib, k.v) % nsa;
    __syncthreads();
    const uint32_t key = k.alive ? sa : (0x10000u + lane);
    const uint32_t grp = __match_any_sync(0xFFFFFFFFu, key);
    const uint32_t rank = __popc(grp & ((1u << lane) - 1));
    if (k.alive && rank == 0) wcnt[warp * 256 + sa] = (uint16_t)__popc(grp);
    __syncthreads();
    if (warp == 0) {
        uint32_t *vec = P.tile_vec + (size_t)tile * 2 * nsa;
        for (uint32_t s = lane; s < nsa; s += 32) {
            uint32_t run = 0;
#pragma unroll
            for (int w = 0; w < NW; w++) { const uint32_t c = wcnt[w * 256 + s]; wcnt[w * 256 + s] = (uint16_t)run; run += c; }
            vec[s] = run;
            pref[s] = 0;
        }
        __syncwarp();
        if (tile > 0) {
            if (lane == 0) { __threadfence(); st_release(P.tile_flag + tile, P.epoch << 2 | 1u); }
#if NFC_LOOKBACK_WIN
            // windowed decoupled look-back: lane j watches tile base-j; the window stops at
            // the nearest tile with an inclusive prefix (or before tile 0); the aggregates
            // of the tiles in front of it are summed in parallel
            int base = (int)tile - 1;
            for (;;) {
                const int pt = base - (int)lane;
                uint32_t fl = 2;
                if (pt >= 0)
                    do { fl = ld_acquire(P.tile_flag + pt); } while ((fl >> 2) != P.epoch || (fl & 3) == 0);
                const uint32_t stop = __ballot_sync(0xFFFFFFFFu, pt < 0 || (fl & 3) == 2);
                const int d = stop ? __ffs(stop) - 1 : 32;          // aggregates before the stop lane
                const bool incl = stop && base - d >= 0;            // stop lane holds an inclusive prefix
                for (uint32_t s = lane; s < nsa; s += 32) {
                    uint32_t acc = 0;
                    for (int j = 0; j < d; j++) acc += __ldcg(P.tile_vec + (size_t)(base - j) * 2 * nsa + s);
                    if (incl) acc += __ldcg(P.tile_vec + (size_t)(base - d) * 2 * nsa + nsa + s);
                    pref[s] += acc;
                }
                if (stop) break;
                base -= 32;
            }
#else
            int pt = (int)tile - 1;
            for (;;) {
                uint32_t fl;
                do { fl = ld_acquire(P.tile_flag + pt); } while ((fl >> 2) != P.epoch || (fl & 3) == 0);
                const uint32_t *pv = P.tile_vec + (size_t)pt * 2 * nsa;
                const bool incl = (fl & 3) == 2;
                for (uint32_t s = lane; s < nsa; s += 32) pref[s] += __ldcg(pv + (incl ? nsa : 0) + s);
                if (incl) break;
                pt--;
            }
#endif
        }
        __syncwarp();
        for (uint32_t s = lane; s < nsa; s += 32) vec[nsa + s] = pref[s] + vec[s];
        __syncwarp();
        if (lane == 0) { __threadfence(); st_release(P.tile_flag + tile, P.epoch << 2 | 2u); }
        if (tile == P.n_tiles - 1)
            for (uint32_t s = lane; s < nsa; s += 32) P.seq_out[s] = P.seq_in[s] + pref[s] + vec[s];
    }
    __syncthreads();
    if (k.alive) {
        k.esp_sa = sa;
        k.esp_seq = __ldg(P.seq_in + sa) + pref[sa] + wcnt[warp * 256 + sa] + rank + 1;
        var_stat(P, C, P.st_sa + sa);
    }
}

#ifndef NFC_ESP_BALANCE
#define NFC_ESP_BALANCE 2     // balanced CTR pass when the tile's largest packet has > this x the mean AES blocks (0: off)
#endif
// a3 for the IPsec tiles: the AES-CTR keystream blocks of the tile's
// SURVIVORS (packets alive at the IPsec position; dropped packets contribute none) are
// concatenated into one block list and split evenly over the CTA's threads.  With
// mixed sizes (IMIX) a thread-per-packet cipher runs every warp as long as its longest
// packet; here each thread encrypts ~total/NT blocks whatever the mix.  Each packet's
// own thread first writes its ESP header and plaintext trailer (esp_header); after a
// barrier the block owners XOR the keystream into the frames with fire-and-forget
// red.global.xor on the aligned words a block touches (a word shared by two blocks gets
// both halves, in either order); after a second barrier each thread MACs its own packet
// over the ciphertext (nf_esp, pre).  Tiles whose sizes are balanced (the largest
// packet within NFC_ESP_BALANCE x the mean) keep the fused per-thread cipher + MAC.
// AES blocks of this thread's packet (0 unless it reaches IPsec); the warp's inclusive
// prefix is returned and the warp's total and largest count go to shared memory --
// before esp_assign, whose barriers publish them (no barrier of its own)
template <int NW>
__device__ __forceinline__ uint32_t esp_blocks_scan(uint8_t *smem, const SmemLayout &L, const Pkt &k)
{
    constexpr uint32_t NT = NW * 32, FULL = 0xFFFFFFFFu;
    const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t nb = 0;
    if (k.alive) {
        const uint32_t plen = k.v.ip_end - k.v.l4_off;
        nb = (plen + ((4 - ((plen + 2) & 3)) & 3) + 2 + 15) >> 4;
    }
    uint32_t incl = nb;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, incl, d);
        if (lane >= (uint32_t)d) incl += y;
    }
    const uint32_t wmax = __reduce_max_sync(FULL, nb);
    uint32_t *wtot = reinterpret_cast<uint32_t *>(smem + L.prefix) + NT;
    if (lane == 31) { wtot[warp] = incl; wtot[NW + warp] = wmax; }
    return incl;
}
template <int NW>
__device__ __forceinline__ void esp_ctr_tile(const KParams &P, const Ctx &C, uint8_t *smem, const SmemLayout &L, Pkt &k,
                                             uint32_t incl)
{
    constexpr uint32_t NT = NW * 32;
    const uint32_t tid = threadIdx.x, warp = tid >> 5;
    const bool e = k.alive;                 // alive at the IPsec position: ESP applies
    uint32_t *pref = reinterpret_cast<uint32_t *>(smem + L.prefix), *wtot = pref + NT, *wmx = pref + NT + NW;
    uint32_t off = 0, T = 0, mx = 0;
#pragma unroll
    for (int w = 0; w < NW; w++) {
        const uint32_t t = wtot[w];
        off += (uint32_t)w < warp ? t : 0u;
        T += t;
        mx = max(mx, wmx[w]);
    }
    if (NFC_ESP_BALANCE == 0 || T == 0 || (uint64_t)mx * NT <= (uint64_t)NFC_ESP_BALANCE * T) return;   // CTA-uniform
    incl += off;
    uint4 *rec = reinterpret_cast<uint4 *>(smem + L.wcnt);   // NT records over esp_assign's scratch
    __syncthreads();                        // esp_assign's readers of its scratch are done
    pref[tid] = incl;
    if (e) {
        const uint32_t plen = k.v.ip_end - k.v.l4_off, p = (4 - ((plen + 2) & 3)) & 3, clen = plen + p + 2;
        esp_header(k.f, k.v, __ldg(&P.esp.sa[k.esp_sa].spi), k.esp_seq, p, true);
        const uint64_t A = reinterpret_cast<uint64_t>(k.f) + k.v.l4_off;
        rec[tid] = make_uint4((uint32_t)A, (uint32_t)(A >> 32), clen | k.esp_sa << 16, k.esp_seq);
    }
    k.esp_pre = 1;
    __threadfence();                        // the header / trailer bytes are performed at L2 before the XORs
    __syncthreads();                        // headers, trailers, records and prefixes visible
    const uint32_t per = (T + NT - 1) / NT;
    uint32_t q = min(tid * per, T);
    const uint32_t qe = min(q + per, T);
    if (q < qe) {
        uint32_t i = 0;                     // the packet owning block q: first i with pref[i] > q
#pragma unroll
        for (uint32_t bit = NT / 2; bit; bit >>= 1)
            if (pref[i + bit - 1] <= q) i += bit;
        const uint32_t *rk0 = reinterpret_cast<const uint32_t *>(nfc_smem + P.lay.rk);
        // one flat loop with one block per iteration: the lanes of a warp stay converged at
        // the cipher call whatever the packet boundaries inside their ranges
        for (; q < qe; q++) {
            while (pref[i] <= q) i++;       // next packet (packets without blocks skipped)
            const uint32_t j = q - (i ? pref[i - 1] : 0u);
            const uint4 R = rec[i];
            const uint32_t cl = R.z & 0xFFFF, sa = R.z >> 16, seq = R.w;
            const uint64_t A = (uint64_t)R.x | (uint64_t)R.y << 32;
            const uint32_t r = (uint32_t)(A & 3), sh = 8 * r;
            uint32_t *Wj = reinterpret_cast<uint32_t *>(A - r) + 4 * j;
            const uint4 o = aes128_encrypt_s(C.te, rk0 + sa * ESP_RK_STRIDE, __ldg(&P.esp.sa[sa].nonce), 0u, seq, j + 1);
            const uint32_t ks[4] = {bswap32(o.x), bswap32(o.y), bswap32(o.z), bswap32(o.w)};
            const uint32_t nw = min(4u, (cl - 16 * j) >> 2);          // clen is a multiple of 4
            uint32_t carry = 0;
#pragma unroll
            for (int w = 0; w < 4; w++)
                if ((uint32_t)w < nw) {
                    atomicXor(Wj + w, (ks[w] << sh) | carry);
                    carry = r ? ks[w] >> (32 - sh) : 0u;
                }
            if (r) atomicXor(Wj + nw, carry);
        }
    }
    __threadfence();                        // every XOR performed at L2 ...
    __syncthreads();                        // ... before the MACs read the ciphertext (ld.cg)
    // the MACs: one packet per thread, the survivors ordered by length (counting sort on
    // 64-B buckets, longest first) so that each warp's packets take about as many SHA-1
    // blocks; the packet's own thread then only re-parses (nf_esp<true>)
    uint32_t *perm = pref, *hist = pref + NT, *cur = pref + NT + 32;
    uint32_t nb = 0;
    if (e) {
        const uint32_t plen = k.v.ip_end - k.v.l4_off;
        nb = (plen + ((4 - ((plen + 2) & 3)) & 3) + 2 + 15) >> 4;
    }
    const uint32_t b = 31u - min(nb >> 2, 31u);   // longest first
    if (tid < 64) hist[tid] = 0;            // hist and cur
    __syncthreads();
    if (e) atomicAdd(&hist[b], 1u);
    __syncthreads();
    if (warp == 0) {
        const uint32_t lane = tid & 31, h = hist[lane];
        uint32_t x = h;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
            if (lane >= (uint32_t)d) x += y;
        }
        cur[lane] = x - h;                  // bucket bases
        if (lane == 31) hist[0] = x;        // survivors
    }
    __syncthreads();
    const uint32_t ns = hist[0];
    if (e) perm[atomicAdd(&cur[b], 1u)] = tid;
    __syncthreads();
    if (tid < ns) {
        const uint4 R = rec[perm[tid]];
        uint8_t *A = reinterpret_cast<uint8_t *>((uint64_t)R.x | (uint64_t)R.y << 32);
        esp_mac_mem(A, R.z & 0xFFFF, P.esp.sa + (R.z >> 16), R.w);
    }
    __syncthreads();                        // every ICV written before the packets move on
}

// Per-CTA context: pointers into the tables, staged into shared memory for the NFs of
// SMASK (compile-time) that the chain uses (mask).  No barrier: the caller syncs.
template <uint32_t SMASK, int DM, int NT>
__device__ __forceinline__ void setup_ctx(const KParams &P, uint8_t *smem, const SmemLayout &L, uint32_t mask,
                                          bool has_esp, uint32_t *vst, Ctx &C)
{
    const uint32_t tid = threadIdx.x, lane = tid & 31;
    C.gtid = blockIdx.x * NT + tid;
    C.vst = P.smem_stats ? vst : nullptr;
    C.pol_f = pol_first();
    C.pol_l = pol_last();
    C.acl4 = C.acl6 = nullptr;
    C.te = C.ms_nib = C.lb_nib = nullptr;
    C.dpi.cls = reinterpret_cast<const uint32_t *>(smem + L.cls);
    C.dpi.cls8 = smem + L.cls;
    C.dpi.gcls = P.dpi.cls;
    C.dpi.sm = smem;
    C.dpi.hot = smem + (DM == DM_FULL ? L.frow0 : L.hot);   // DM_FULL: row of slot 0
    C.dpi.row2 = 2 * P.dpi.ncls;
    C.dpi.ncls = P.dpi.ncls;
    C.dpi.wide = DM == DM_FULL ? 0 : P.dpi.wide;
    C.dpi.trans = P.dpi.trans;
    C.dpi.out_off = P.dpi.out_off;
    C.dpi.out_ids = P.dpi.out_ids;
    C.dpi.pat_action = P.dpi.pat_action;
    C.dpi.acc_id = P.dpi.acc_id;
    C.dpi.H = 0;
    C.dpi.HK2 = 0;
    C.meta = P.dpi.meta_smem ? reinterpret_cast<const uint32_t *>(smem + L.meta)
                             : DM == DM_FULL ? P.dpi.acc_meta : P.dpi.out_meta;
    if ((SMASK & MASK_ACL) && (mask & MASK_ACL)) {
        if (P.acl.smem_words) {
            uint4 *d4 = reinterpret_cast<uint4 *>(smem + L.acl4);
            uint4 *d6 = reinterpret_cast<uint4 *>(smem + L.acl6);
            if (P.acl.fast)       // the record image (acl4_fast)
                for (uint32_t i = tid; i < P.acl.words_f4 / 4; i += NT) d4[i] = __ldg(reinterpret_cast<const uint4 *>(P.acl.f4) + i);
            else
                for (uint32_t i = tid; i < P.acl.words4 / 4; i += NT) d4[i] = __ldg(reinterpret_cast<const uint4 *>(P.acl.bv4) + i);
            for (uint32_t i = tid; i < P.acl.words6 / 4; i += NT) d6[i] = __ldg(reinterpret_cast<const uint4 *>(P.acl.bv6) + i);
            C.acl4 = reinterpret_cast<const uint32_t *>(d4);
            C.acl6 = reinterpret_cast<const uint32_t *>(d6);
        } else {
            C.acl4 = P.acl.bv4;
            C.acl6 = P.acl.bv6;
        }
    }
    if ((SMASK & MASK_DPI) && (mask & MASK_DPI)) {
        // 2 * class as u8 for DM_FULL (ncls <= 128), class as u32 for DM_HOT
        if (DM == DM_FULL) {
            for (uint32_t i = tid; i < 256; i += NT) smem[L.cls + i] = (uint8_t)(2u * __ldg(P.dpi.cls + i));
        } else {
            uint32_t *cls = reinterpret_cast<uint32_t *>(smem + L.cls);
            for (uint32_t i = tid; i < 256; i += NT) cls[i] = __ldg(P.dpi.cls + i);
        }
        const uint32_t H = C.dpi.wide ? 0 : P.dpi.hot_states;
        uint16_t *hot = reinterpret_cast<uint16_t *>(smem + L.hot);
        // DM_FULL stages the slot image (DpiImg::frows), DM_HOT the BFS-ordered table
        const uint16_t *tr = DM == DM_FULL ? reinterpret_cast<const uint16_t *>(P.dpi.frows)
                                           : reinterpret_cast<const uint16_t *>(P.dpi.trans);
        const uint32_t nh = H * P.dpi.ncls;
        if ((nh & 7) == 0) {
            for (uint32_t i = tid; i < nh / 8; i += NT) reinterpret_cast<uint4 *>(hot)[i] = __ldg(reinterpret_cast<const uint4 *>(tr) + i);
        } else {
            for (uint32_t i = tid; i < nh; i += NT) hot[i] = __ldg(tr + i);
        }
        C.dpi.H = H;
        C.dpi.HK2 = H ? 2 * (H * P.dpi.ncls - 1) : 0;
        C.dpi.sp = reinterpret_cast<const uint2 *>(smem + L.sp);
        C.dpi.S = 0;
        if (DM != DM_FULL && !C.dpi.wide) {
            uint2 *sp = reinterpret_cast<uint2 *>(smem + L.sp);
            for (uint32_t i = tid; i < P.dpi.sparse_states; i += NT) sp[i] = __ldg(P.dpi.sparse + H + i);
            C.dpi.S = P.dpi.sparse_states;
        }
        if (P.dpi.meta_smem) {
            uint32_t *mt = reinterpret_cast<uint32_t *>(smem + L.meta);
            if (DM == DM_FULL)
                for (uint32_t i = tid; i < P.dpi.n_acc; i += NT) mt[i] = __ldg(P.dpi.acc_meta + i);
            else
                for (uint32_t i = tid; i < P.dpi.n_states; i += NT) mt[i] = __ldg(P.dpi.out_meta + i);
        }
    }
    if ((SMASK & MASK_IPSEC) && has_esp) {
        uint32_t *te = reinterpret_cast<uint32_t *>(smem + L.te), *mn = reinterpret_cast<uint32_t *>(smem + L.ms_nib);
        for (uint32_t i = tid; i < 256 * 32; i += NT) te[i] = __ldg(P.esp.te + (i >> 5));   // T0 x 32 lanes
        for (uint32_t i = tid; i < 72 * 16; i += NT) mn[i] = __ldg(P.esp.rss_nib + i);
        C.te = te + lane;         // this lane's bank column
        C.ms_nib = mn;
#if NFC_ESP_RK_SMEM
        uint32_t *rk = reinterpret_cast<uint32_t *>(smem + L.rk);
        for (uint32_t i = tid; i < P.esp.n_sa * 44; i += NT) rk[(i / 44) * ESP_RK_STRIDE + i % 44] = __ldg(P.esp.sa[i / 44].rk + i % 44);
#endif
    }
    if ((SMASK & MASK_LPM4) && (mask & MASK_LPM4) && P.l4.nh_smem) {
        uint4 *r = reinterpret_cast<uint4 *>(smem + L.nh4);
        for (uint32_t i = tid; i < P.l4.n_nh; i += NT) {
            const uint2 n = __ldg(P.l4.nh + i);
            const uint32_t pt = n.y >> 16;
            const uint2 m = pt < P.l4.n_ports ? __ldg(P.l4.pmac + pt) : make_uint2(0, 0);
            r[i] = make_uint4(n.x, n.y, m.x, m.y);
        }
    }
    C.nat_nib = nullptr;
    if ((SMASK & MASK_NAT) && (mask & MASK_NAT)) {
        uint32_t *nn = reinterpret_cast<uint32_t *>(smem + L.nat_nib);
        for (uint32_t i = tid; i < 72 * 16; i += NT) nn[i] = __ldg(P.nat.nib + i);
        C.nat_nib = nn;
    }
    if ((SMASK & MASK_LB) && (mask & MASK_LB)) {
        uint32_t *ln = reinterpret_cast<uint32_t *>(smem + L.lb_nib);
        for (uint32_t i = tid; i < 72 * 16; i += NT) ln[i] = __ldg(P.lb.nib + i);
        C.lb_nib = ln;
    }
}

template <uint32_t S, int DM, bool RGV>
__global__ void __launch_bounds__(KCfg<S, DM>::threads, KCfg<S, DM>::minb) sfc_kernel(const KParams P)
{
    constexpr int NT = KCfg<S, DM>::threads, NW = KCfg<S, DM>::nwarp, WS = KCfg<S, DM>::nws;
    uint8_t *smem = nfc_smem;
    __shared__ uint32_t s_tile;
    const uint32_t mask = P.present & sig_mask(S);
    const SmemLayout &L = P.lay;
    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t NP = P.n_pkts;
    unsigned long long *wst = reinterpret_cast<unsigned long long *>(smem + L.wst);
    uint32_t *vst = reinterpret_cast<uint32_t *>(smem + L.vst);
    const uint32_t n_var = P.stats_len - NFIX;
    for (uint32_t i = tid; i < NW * WS; i += NT) wst[i] = 0;
    if (P.smem_stats)
        for (uint32_t i = tid; i < n_var; i += NT) vst[i] = 0;

    const bool has_esp = (sig_mask(S) & MASK_IPSEC) && P.esp_pos < P.n_nf;
    Ctx C;
    setup_ctx<sig_mask(S), DM, NT>(P, smem, L, mask, has_esp, vst, C);
    __syncthreads();
    unsigned long long *ws = wst + warp * WS;

    if (!KCfg<S, DM>::esp || (S == SIG_ANY && !has_esp)) {
        // warp-granular persistent loop: chunks of 32 consecutive packets (NFC_CLAIM
        // chunks per atomic claim), no CTA barriers; the next chunk is claimed and located (off/len loads, header
        // prefetch to L2) before the current one is processed
        uint32_t cbase = 0, cleft = 0;
        auto claim = [&]() {                 // next 32-packet chunk; one atomic per P.claim chunks
            const uint32_t CL = P.claim;
            if (cleft == 0) {
                uint32_t b = 0;
                if (lane == 0) b = atomicAdd(P.tile_counter, 32u * CL);
                cbase = __shfl_sync(0xFFFFFFFFu, b, 0);
                cleft = CL;
            }
            const uint32_t c = cbase;
            cbase += 32;
            cleft--;
            return c;
        };
        // software pipeline over chunks: descriptors (off/len) of chunk c2 are loaded two
        // iterations ahead, the frame of chunk c1 is prefetched into L2 one ahead
        uint32_t c0 = claim(), c1 = claim();
#if NFC_DESC_L1
        // descriptors (off/len) are prefetched into L1 two chunks ahead -- no registers held
        // across a chunk -- and re-loaded (L1 hits) when the frame prefetch and the chunk need them
        auto desc_l1 = [&](uint32_t g) {
            if (g < NP) {
                if (P.n_batches == 1) {   // (multi-batch: chunk records staged in shared memory)
                    asm volatile("prefetch.global.L1 [%0];" ::"l"(P.b0.off + g));
                    asm volatile("prefetch.global.L1 [%0];" ::"l"(P.b0.len + g));
                }
            }
        };
        desc_l1(c0 + lane);
        desc_l1(c1 + lane);
        // the next chunk's descriptors (off/len; multi-batch calls: from its chunk record)
        // are read at the top of the current one and carried into it, so its header loads
        // issue without a descriptor round trip
        uint64_t off0 = 0;
        uint32_t len0 = 0;
        const bool late = NFC_PF_LATE && (P.n_batches == 1 || P.crec != nullptr);                 // warp-uniform
        if (late && c0 + lane < NP) desc_get(P, c0 + lane, off0, len0);
        // multi-batch: chunk records staged two chunks ahead in a per-warp 2-slot ring
        const bool stg = late && P.n_batches > 1;                                                  // warp-uniform
        const uint32_t crs = (uint32_t)__cvta_generic_to_shared(smem) + L.crs + warp * 64;
        uint32_t slot1 = 32;                                                                      // c1's slot
        if (stg) crec_stage(P, c1, crs + slot1, lane);
        // a3: family regrouping.  A chunk mixing IPv4 and IPv6 packets runs the
        // IPv4 speculative block for neither and diverges through every NF.  The RG
        // instantiation (NFC_REGROUP=1 builds) defers such a chunk's IPv6 packets to a per-warp
        // queue in shared memory and runs them later as chunks of their own (a "virtual" chunk
        // once 32 wait, the rest after the last real chunk), so every chunk a warp runs is one
        // family; the launcher picks it while the chain's previous call saw > 1/8 mixed chunks.
        // Measured slower on the dual-stack C5 traffic (the deferred chunks lose the descriptor
        // and header pipelining, and the IPv4 chunks run with their IPv6 lanes idle), so the
        // default build counts mixed chunks (ST_MIXED_CHUNKS) and runs them as they come.
        constexpr bool RG = RGV && rg_sig(S, DM);
        const uint32_t rgq = (uint32_t)__cvta_generic_to_shared(smem) + L.rgq + warp * NFC_RGQ * 4;   // shared address
        const uint32_t rgn = rgq + 4 * (NFC_RGQ - 1);      // the last word: queue length
        if (RG && lane == 0) asm volatile("st.shared.u32 [%0], %1;" ::"r"(rgn), "r"(0u) : "memory");
        __syncwarp();
        for (;;) {
            const uint32_t qn = RG ? lds_u32_v(rgn) : 0u;  // deferred packets queued (warp-uniform)
            const bool virt = RG && (qn >= 32 || (c0 >= NP && qn > 0));          // a deferred chunk
            if (!virt && c0 >= NP) break;
            uint64_t off1 = 0;
            uint32_t len1 = 0, c2 = 0, g;
            bool valid;
            Loc loc;
            if (virt) {
                valid = lane < qn;
                g = valid ? lds_u32_v(rgq + 4 * lane) : 0u;
                loc = pkt_locate(P, g, valid);
            } else {
                if (stg) {
                    asm volatile("cp.async.wait_all;" ::: "memory");
                    __syncwarp();
                }
                if (c1 + lane < NP) {
                    if (late) {
                        if (stg) desc_get_s(P, c1 + lane, off1, len1, crs + slot1);   // consumed after the head part
                        else desc_get(P, c1 + lane, off1, len1);
                    } else {
                        asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(pkt_locate(P, c1 + lane, true).f));
                    }
                }
                c2 = claim();
                desc_l1(c2 + lane);
                if (stg) {
                    __syncwarp();                          // every lane has read c1's slot
                    slot1 ^= 32;                           // c2 goes to the other slot
                    crec_stage(P, c2, crs + slot1, lane);
                }
                g = c0 + lane;
                valid = g < NP;
                loc = late ? Loc{P.b0.arena + off0, len0, g} : pkt_locate(P, g, valid);
            }
            Pkt k;
            pkt_begin(C, loc, valid, k);
            if constexpr (rg_sig(S, DM)) {
                if (!virt) {
                    const uint32_t FULL = 0xFFFFFFFFu;
                    const bool v6 = valid && k.alive && k.v.fam != 4;
                    const uint32_t b6 = __ballot_sync(FULL, v6);
                    if (b6 && b6 != __ballot_sync(FULL, valid && k.alive)) {     // mixed chunk
                        if (lane == 0) ws[ST_MIXED_CHUNKS]++;
                        if constexpr (RG) {                // defer its IPv6 lanes
                            const uint32_t pos = qn + __popc(b6 & ((1u << lane) - 1));
                            if (v6 && pos < NFC_RGQ - 1) { // (a full queue: the rest run here)
                                asm volatile("st.shared.u32 [%0], %1;" ::"r"(rgq + 4 * pos), "r"(g) : "memory");
                                k.alive = false;           // not processed in this chunk
                                valid = false;             // no record, no counters here
                            }
                            __syncwarp();
                            if (lane == 0)
                                asm volatile("st.shared.u32 [%0], %1;" ::"r"(rgn),
                                             "r"(min(qn + __popc(b6), (uint32_t)NFC_RGQ - 1)) : "memory");
                            __syncwarp();
                        }
                    }
                }
            }
            run_part<S, DM, true>(P, C, k);
            if (!virt && late && c1 + lane < NP) asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(P.b0.arena + off1));
            run_part<S, DM, false>(P, C, k);
            pkt_end<S>(P, C, k, valid, g, ws, lane);
            if (virt) {                                     // drop the 32 processed entries
                const uint32_t rest = qn > 32 ? qn - 32 : 0u;
                __syncwarp();
                const uint32_t x = lane < rest ? lds_u32_v(rgq + 4 * (32 + lane)) : 0u;
                __syncwarp();
                if (lane < rest) asm volatile("st.shared.u32 [%0], %1;" ::"r"(rgq + 4 * lane), "r"(x) : "memory");
                if (lane == 0) asm volatile("st.shared.u32 [%0], %1;" ::"r"(rgn), "r"(rest) : "memory");
                __syncwarp();
            } else {
                c0 = c1;
                c1 = c2;
                off0 = off1;
                len0 = len1;
            }
        }
#else
        Loc loc = pkt_locate(P, c0 + lane, c0 + lane < P.n_pkts);
        Raw raw1 = pkt_raw(P, c1 + lane, c1 + lane < P.n_pkts);
#if NFC_HDR_AHEAD
        // the next chunk's header words are loaded at the tail of the current chunk (after
        // its last NF, before the record store and counters), so the L2 read overlaps them
        uint32_t hn[16];
        if (c0 + lane < P.n_pkts) load_header(loc.f, loc.len, hn, C.pol_f);
#endif
        while (c0 < P.n_pkts) {
            // locate chunk c1 (its descriptors arrived during the last chunk) BEFORE issuing
            // the descriptor loads of c2: an address add that consumed a just-issued load's
            // scoreboard slot would wait for that DRAM read and undo the two-ahead pipeline
            const Loc loc1 = pkt_loc(P, raw1, c1 + lane, c1 + lane < P.n_pkts);
            if (c1 + lane < P.n_pkts) asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(loc1.f));
            const uint32_t c2 = claim();
            const Raw raw2 = pkt_raw(P, c2 + lane, c2 + lane < P.n_pkts);
            const uint32_t g = c0 + lane;
            const bool valid = g < P.n_pkts;
            Pkt k;
#if NFC_HDR_AHEAD
            pkt_begin_h(loc, valid, k, hn);
#else
            pkt_begin(C, loc, valid, k);
#endif
            run_part<S, DM, true>(P, C, k);
            run_part<S, DM, false>(P, C, k);
#if NFC_HDR_AHEAD
            if (c1 + lane < P.n_pkts) load_header(loc1.f, loc1.len, hn, C.pol_f);
#endif
            pkt_end<S>(P, C, k, valid, g, ws, lane);
            c0 = c1;
            c1 = c2;
            loc = loc1;
            raw1 = raw2;
        }
#endif
    } else if constexpr (KCfg<S, DM>::esp) {
        // CTA tiles claimed in global order (ESP sequence numbers need the order)
        for (;;) {
            if (tid == 0) s_tile = atomicAdd(P.tile_counter, 1u);
            __syncthreads();
            const uint32_t tile = s_tile;
            __syncthreads();
            if (tile >= P.n_tiles) break;
            const uint32_t g = tile * NT + tid;
            const bool valid = g < P.n_pkts;
            Pkt k;
            pkt_begin(C, pkt_locate(P, g, valid), valid, k);
            run_part<S, DM, true>(P, C, k);
#if NFC_ESP_RK_SMEM
            uint32_t bincl = 0;
            if constexpr (S != SIG_ANY) bincl = esp_blocks_scan<NW>(smem, L, k);
#endif
            esp_assign<NW>(P, C, smem, L, tile, k);
#if NFC_ESP_RK_SMEM
            if constexpr (S != SIG_ANY) esp_ctr_tile<NW>(P, C, smem, L, k, bincl);   // (the generic kernel: fused cipher)
#endif
            run_part<S, DM, false>(P, C, k);
            pkt_end<S>(P, C, k, valid, g, ws, lane);
        }
    }
    // ---- flush CTA counters; derive drop total and per-position in / applied
    __syncthreads();
    if (warp == 0) {
        unsigned long long t[2] = {0, 0};
        const uint32_t i = lane;     // slots 0..31 by lane, 32..NWS-1 by lanes 0..NWS-33
#pragma unroll
        for (int r = 0; r < 2; r++) {
            const uint32_t idx = i + 32 * r;
            if (idx < WS)
                for (int w = 0; w < NW; w++) t[r] += wst[w * WS + idx];
        }
        __syncwarp();
        wst[i] = t[0];
        if (i + 32 < WS) wst[i + 32] = t[1];
        __syncwarp();
        if (lane == 0) {
            unsigned long long in = wst[ST_PKTS] - wst[ST_PARSE_DROP];
            for (uint32_t p = 0; p < P.n_nf; p++) {
                const unsigned long long d = wst[ST_POS_BASE + 4 * p + 1], ps = wst[ST_POS_BASE + 4 * p + 2];
                wst[ST_POS_BASE + 4 * p] = in;
                wst[ST_POS_BASE + 4 * p + 3] = in - d - ps;
                in -= d;
            }
            if (NFC_FWD_DERIVED) wst[ST_FWD] = in;   // survivors of every position
            wst[ST_DROP] = wst[ST_PKTS] - wst[ST_FWD];
        }
        __syncwarp();
        for (uint32_t idx = lane; idx < WS; idx += 32)
            if (wst[idx]) atomicAdd(&P.stats[idx], wst[idx]);
        if (lane == 0 && P.mix && wst[ST_MIXED_CHUNKS]) atomicAdd(P.mix, (uint32_t)wst[ST_MIXED_CHUNKS]);
    }
    if (P.smem_stats)
        for (uint32_t i = tid; i < n_var; i += NT)
            if (vst[i]) atomicAdd(&P.stats[NFIX + i], (unsigned long long)vst[i]);
}

// ---------------------------------------------------------------- host launch
template <uint32_t S, int DM, bool RGV>
int launch_t(const KParams &p, int dev, void *stream, std::string &err, LaunchCfg *cfg, bool query_only)
{
    constexpr int NT = KCfg<S, DM>::threads;
    const size_t smem = smem_layout(p.present & sig_mask(S), KCfg<S, DM>::nwarp, p, KCfg<S, DM>::nws, DM).total;
    static int attr_smem[64] = {0};   // per device: dynamic smem size already granted
    static int per_sm_cache[64] = {0};
    static size_t per_sm_smem[64] = {0};
    const int d = dev & 63;
    if ((int)smem > attr_smem[d]) {
        if (cudaFuncSetAttribute(sfc_kernel<S, DM, RGV>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess) {
            err = "cudaFuncSetAttribute failed (shared memory " + std::to_string(smem) + " B)";
            return NFC_ECUDA;
        }
        attr_smem[d] = (int)smem;
    }
    int per_sm = per_sm_cache[d];
    if (!per_sm || per_sm_smem[d] != smem) {
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, sfc_kernel<S, DM, RGV>, NT, smem);
        if (per_sm < 1) per_sm = 1;
        per_sm_cache[d] = per_sm;
        per_sm_smem[d] = smem;
    }
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int grid = sms * per_sm;
    // chunks per claim: NFC_CLAIM (DM_FULL) when every warp gets many claims, else 1 (large
    // frames or small batches: the tail of the last claims would dominate)
    const uint32_t chunks = (p.n_pkts + 31) / 32;
    uint32_t claim = KCfg<S, DM>::claim;
    if ((uint64_t)chunks < 16ull * claim * (uint64_t)grid * KCfg<S, DM>::nwarp) claim = 1;
    const uint32_t units = KCfg<S, DM>::esp ? p.n_tiles : (chunks + claim - 1) / claim / KCfg<S, DM>::nwarp + 1;
    if (!query_only && (uint32_t)grid > units) grid = (int)units;
    if (grid < 1) grid = 1;
    if (cfg) { cfg->grid = grid; cfg->block = NT; cfg->smem = smem; }
    if (query_only) return NFC_OK;
    KParams q = p;
    q.claim = claim;
    q.lay = smem_layout(p.present & sig_mask(S), KCfg<S, DM>::nwarp, p, KCfg<S, DM>::nws, DM);
    sfc_kernel<S, DM, RGV><<<grid, NT, smem, (cudaStream_t)stream>>>(q);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) { err = std::string("sfc_kernel launch: ") + cudaGetErrorString(e); return NFC_ECUDA; }
    return NFC_OK;
}

// chain signatures with dedicated instantiations (sfc_inst_*.cu)
static constexpr uint32_t SIG_C1 = make_sig(3, NFC_ACL, NFC_DPI, NFC_LPM4);                       // also C5 k=3
static constexpr uint32_t SIG_C2 = make_sig(1, NFC_IPSEC);
static constexpr uint32_t SIG_C3 = make_sig(3, NFC_ACL, NFC_DPI, NFC_LB);
static constexpr uint32_t SIG_C4 = make_sig(5, NFC_ACL, NFC_LPM6, NFC_DPI, NFC_IPSEC, NFC_LB);
static constexpr uint32_t SIG_K1 = make_sig(1, NFC_ACL);
static constexpr uint32_t SIG_K2 = make_sig(2, NFC_ACL, NFC_DPI);
static constexpr uint32_t SIG_K4 = make_sig(4, NFC_ACL, NFC_DPI, NFC_LPM4, NFC_LPM6);
static constexpr uint32_t SIG_K5 = make_sig(5, NFC_ACL, NFC_DPI, NFC_LPM4, NFC_LPM6, NFC_IPSEC);
static constexpr uint32_t SIG_K6 = make_sig(6, NFC_ACL, NFC_DPI, NFC_LPM4, NFC_LPM6, NFC_IPSEC, NFC_LB);
static constexpr uint32_t SIG_N3 = make_sig(3, NFC_ACL, NFC_LPM4, NFC_NAT);                       // NEXT-3

#define NFC_DECLARE_LAUNCH(S, DM)                                                                   \
    extern template int launch_t<S, DM, false>(const KParams &, int, void *, std::string &, LaunchCfg *, bool);
#define NFC_INSTANTIATE_LAUNCH(S, DM)                                                               \
    template int launch_t<S, DM, false>(const KParams &, int, void *, std::string &, LaunchCfg *, bool);
// the a3 regrouping instantiation (rg_sig chains only)
#define NFC_DECLARE_LAUNCH_RG(S, DM)                                                                \
    extern template int launch_t<S, DM, true>(const KParams &, int, void *, std::string &, LaunchCfg *, bool);
#define NFC_INSTANTIATE_LAUNCH_RG(S, DM)                                                            \
    template int launch_t<S, DM, true>(const KParams &, int, void *, std::string &, LaunchCfg *, bool);

} // namespace nfc
