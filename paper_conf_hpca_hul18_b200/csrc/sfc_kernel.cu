// sfc_kernel.cu -- the fused, persistent SFC kernel for sm_100a.
//
// One launch drains all packets of an nfc_process_batch call.  Every thread
// carries one packet through the whole chain in registers:
//   parse once (the de-duplicated header classifier)
//   -> NFs in original SFC order, a dropped packet skipping every later NF
//      (early drop; no batch re-split or per-NF launch)
//   -> one 16 B result record; counters in per-warp private shared memory.
// Scheduling (persistent kernel, P:L112, P:L235 [SIV]): without IPsec each warp
// claims 32-packet chunks from a global atomic counter (no CTA barriers); with
// IPsec each CTA claims TILE-packet tiles in order and assigns per-SA ESP
// sequence numbers in global packet order by a decoupled look-back.
// Tables stay on chip where they fit: the ACL bit-vector image, the hot rows
// of the Aho-Corasick DFA, AES T-tables and Toeplitz nibble tables live in
// shared memory; DIR-24-8 / IPv6 hash levels are read through L2 with an
// evict-last policy while the packet stream is evict-first.  Packet bytes are
// read from HBM once and rewritten in place.  No tensor cores: nothing here is
// a dense contraction.
#include <cuda_runtime.h>
#include <stdint.h>

#include "nfc_internal.h"

namespace nfc {

static constexpr int TILE = 256;        // threads per CTA (== packets per IPsec tile)
static constexpr int NWARP = TILE / 32;
static constexpr int DPI_LIST = 16;     // distinct matches kept in a list before the bitmap path
static constexpr int NFIX = ST_VAR_BASE;

// tuning knobs (compile-time; defaults are the measured best)
#ifndef NFC_PIPE
#define NFC_PIPE 1            // 1: one-chunk lookahead, 3: three-stage pipeline
#endif
#ifndef NFC_EARLY_T24
#define NFC_EARLY_T24 0       // issue the TBL24 read right after parse
#endif
#ifndef NFC_MINB
#define NFC_MINB 3            // min resident CTAs per SM for chains without IPsec
#endif

// ---------------------------------------------------------------- shared memory layout
struct SmemLayout {
    uint32_t wst, vst, te, ms_nib, lb_nib, cls, hot, acl4, acl6, wcnt, prefix, total;
};
__host__ __device__ inline SmemLayout smem_layout(uint32_t mask, const KParams &p)
{
    SmemLayout L{};
    uint32_t o = 0;
    L.wst = o; o += NWARP * NFIX * 8;                              // per-warp private counters (u64)
    L.vst = o; o += (p.smem_stats ? p.stats_len - NFIX : 0) * 4;  // ACL/LB/SA hit counters (u32)
    o = (o + 15) & ~15u;
    if (mask & MASK_IPSEC) { L.te = o; o += 256 * 32 * 4; L.ms_nib = o; o += 72 * 16 * 4; }
    if (mask & MASK_LB) { L.lb_nib = o; o += 72 * 16 * 4; }
    if (mask & MASK_DPI) { L.cls = o; o += 256; L.hot = o; o += (p.dpi.hot_states * p.dpi.ncls * 2 + 15) & ~15u; }
    o = (o + 15) & ~15u;
    if (mask & MASK_ACL) {
        const uint32_t s4 = p.acl.smem_words ? p.acl.words4 : 0, s6 = p.acl.smem_words ? p.acl.words6 : 0;
        L.acl4 = o; o += s4 * 4;
        L.acl6 = o; o += s6 * 4;
    }
    o = (o + 15) & ~15u;
    if (mask & MASK_IPSEC) {
        L.wcnt = o; o += NWARP * 256 * 2;
        L.prefix = o; o += 256 * 4;
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
__device__ __forceinline__ void st_stream16(void *a, uint4 v, uint64_t pol)
{
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.u32 [%0], {%1,%2,%3,%4}, %5;"
                 ::"l"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "l"(pol) : "memory");
}
__device__ __forceinline__ uint32_t ld_tab16(const uint16_t *a, uint64_t pol)
{
    uint16_t v;
    asm("ld.global.nc.L2::cache_hint.u16 %0, [%1], %2;" : "=h"(v) : "l"(a), "l"(pol));
    return v;
}

// byte k (0..63) of the 64 B header cache; k compile-time in hot paths
__device__ __forceinline__ uint32_t hbyte(const uint32_t h[16], uint32_t k) { return (h[k >> 2] >> ((k & 3) * 8)) & 0xFF; }
__device__ __forceinline__ uint32_t hbe16(const uint32_t h[16], uint32_t k) { return hbyte(h, k) << 8 | hbyte(h, k + 1); }
__device__ __forceinline__ uint32_t hbe32(const uint32_t h[16], uint32_t k) { return hbe16(h, k) << 16 | hbe16(h, k + 2); }
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
#pragma unroll
    for (int c = 0; c < 4; c++) {
        uint4 v = c < (int)nch ? ld_stream16(f + 16 * c, pol) : make_uint4(0, 0, 0, 0);
        h[4 * c] = v.x; h[4 * c + 1] = v.y; h[4 * c + 2] = v.z; h[4 * c + 3] = v.w;
    }
}

// Parse (P:L87 validity check): Ethernet -> IPv4/IPv6 -> UDP/TCP.
__device__ __forceinline__ bool parse(const uint32_t h[16], const uint8_t *f, uint32_t flen, PV &v)
{
    if (flen < 14) return false;
    uint32_t et = hbe16(h, 12);
    bool frag = false;
    if (et == 0x0800) {
        if (flen < 34) return false;
        uint32_t vi = hbyte(h, 14);
        if ((vi >> 4) != 4) return false;
        uint32_t ihl = vi & 15;
        if (ihl < 5) return false;
        uint32_t tot = hbe16(h, 16);
        if (tot < 4 * ihl || 14 + tot > flen) return false;
        v.fam = 4;
        v.l4_off = 14 + 4 * ihl;
        v.ip_end = 14 + tot;
        v.proto = hbyte(h, 23);
        v.src[0] = hbe32(h, 26);
        v.dst[0] = hbe32(h, 30);
        v.src[1] = v.src[2] = v.src[3] = v.dst[1] = v.dst[2] = v.dst[3] = 0;
        uint32_t fo = hbe16(h, 20);
        frag = (fo & 0x2000) || (fo & 0x1FFF);       // MF set or non-zero offset
    } else if (et == 0x86DD) {
        if (flen < 54) return false;
        if ((hbyte(h, 14) >> 4) != 6) return false;
        uint32_t pl = hbe16(h, 18);
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
        uint32_t l4 = v.l4_off;
        if (v.proto == 17) {
            if (l4 + 8 > v.ip_end) return false;
            l4len = 8;
        } else {
            if (l4 + 20 > v.ip_end) return false;
            // data offset: byte 46 sits in the header cache; other offsets are rare -> memory
            uint32_t doff = (l4 == 34 ? hbyte(h, 46) : (uint32_t)f[l4 + 12]) >> 4;
            if (doff < 5 || l4 + 4 * doff > v.ip_end) return false;
            l4len = 4 * doff;
        }
        if (l4 == 34) { v.sport = hbe16(h, 34); v.dport = hbe16(h, 36); }
        else if (l4 == 54) { v.sport = hbe16(h, 54); v.dport = hbe16(h, 56); }
        else {
            v.sport = (uint32_t)f[l4] << 8 | f[l4 + 1];      // IPv4 options: rare, from memory
            v.dport = (uint32_t)f[l4 + 2] << 8 | f[l4 + 3];
        }
    }
    v.pl_off = v.l4_off + l4len;
    return true;
}

// ---------------------------------------------------------------- ACL
// Bit-vector first match: five interval lookups (binary search over the
// elementary-interval starts), AND of the five rule bitsets, lowest set bit.
__device__ __forceinline__ uint32_t bsearch32(const uint32_t *B, uint32_t m, uint32_t key)
{
    uint32_t lo = 0;
    while (m > 1) {
        const uint32_t half = m >> 1;
        lo = (B[lo + half] <= key) ? lo + half : lo;
        m -= half;
    }
    return lo;
}
__device__ __forceinline__ bool le128(const uint32_t *b, const uint32_t k[4])
{
    if (b[0] != k[0]) return b[0] < k[0];
    if (b[1] != k[1]) return b[1] < k[1];
    if (b[2] != k[2]) return b[2] < k[2];
    return b[3] <= k[3];
}
__device__ __forceinline__ uint32_t bsearch128(const uint32_t *B, uint32_t m, const uint32_t k[4])
{
    uint32_t lo = 0;
    while (m > 1) {
        const uint32_t half = m >> 1;
        lo = le128(B + 4 * (lo + half), k) ? lo + half : lo;
        m -= half;
    }
    return lo;
}

// interval of key: bucket on the top 8 bits bounds the binary search to [bk[t], bk[t+1]]
__device__ __forceinline__ uint32_t iv32(const uint32_t *A, uint32_t okeys, uint32_t obk, uint32_t key, int kbits)
{
    const uint32_t t = key >> (kbits - 8);
    const uint32_t lo = A[obk + t], hi = A[obk + t + 1];
    return lo + bsearch32(A + okeys + lo, hi - lo + 1, key);
}
__device__ __forceinline__ uint32_t iv128(const uint32_t *A, uint32_t okeys, uint32_t obk, const uint32_t k[4])
{
    const uint32_t t = k[0] >> 24;
    const uint32_t lo = A[obk + t], hi = A[obk + t + 1];
    return lo + bsearch128(A + okeys + 4 * lo, hi - lo + 1, k);
}

// returns global rule index (0xFFFF none) | action << 31
__device__ __forceinline__ uint32_t nf_acl(const uint32_t *A, uint32_t default_action, const PV &v)
{
    const uint32_t n = A[0];
    if (n == 0) return 0xFFFFu | default_action << 31;
    const uint32_t W = A[1];
    uint32_t js, jd;
    if (A[6] == 1) {
        js = iv32(A, A[8], A[18], v.src[0], 32);
        jd = iv32(A, A[10], A[19], v.dst[0], 32);
    } else {
        js = iv128(A, A[8], A[18], v.src);
        jd = iv128(A, A[10], A[19], v.dst);
    }
    const uint32_t jsp = iv32(A, A[12], A[20], v.sport, 16);
    const uint32_t jdp = iv32(A, A[14], A[21], v.dport, 16);
    const uint64_t *vs = reinterpret_cast<const uint64_t *>(A + A[9]) + (size_t)js * W;
    const uint64_t *vd = reinterpret_cast<const uint64_t *>(A + A[11]) + (size_t)jd * W;
    const uint64_t *vsp = reinterpret_cast<const uint64_t *>(A + A[13]) + (size_t)jsp * W;
    const uint64_t *vdp = reinterpret_cast<const uint64_t *>(A + A[15]) + (size_t)jdp * W;
    const uint64_t *vpr = reinterpret_cast<const uint64_t *>(A + A[16]) + (size_t)v.proto * W;
    for (uint32_t w = 0; w < W; w++) {
        const uint64_t x = vs[w] & vd[w] & vsp[w] & vdp[w] & vpr[w];
        if (x) return A[A[17] + 64 * w + (__ffsll((long long)x) - 1)];
    }
    return 0xFFFFu | default_action << 31;
}

// ---------------------------------------------------------------- DPI
// Aho-Corasick DFA walk.  States below hot_states use full 256-byte rows staged
// in shared memory; the rest read the global class-compressed table.
struct DpiCtx {
    const uint8_t *cls;     // smem
    const uint16_t *hot;    // smem
    uint32_t H, ncls, wide, HK1;
    const void *trans;
    const uint32_t *out_off;
    const uint16_t *out_ids;
    const uint8_t *pat_action;
};

// One DFA step.  Hot rows (the first H states in BFS order, class-compressed) are
// staged in shared memory with the same layout as the global table.
__device__ __forceinline__ uint32_t dfa_step(const DpiCtx &c, uint32_t s, uint32_t b, bool &acc)
{
    const uint32_t k = s * c.ncls + c.cls[b];
    uint32_t e;
    if (c.wide) {
        e = __ldg(reinterpret_cast<const uint32_t *>(c.trans) + k);
        acc = e >> 31;
        return e & 0x7FFFFFFFu;
    }
    e = s < c.H ? (uint32_t)c.hot[k] : (uint32_t)__ldg(reinterpret_cast<const uint16_t *>(c.trans) + k);
    acc = (e >> 15) & 1;
    return e & 0x7FFFu;
}

// Fast DFA walk over payload [a, b) that only ORs the accept bits (exact match sets
// are recomputed by dpi_slow for the rare packets that hit an accepting state).
// Branch-free step: class lookup, hot-row lookup at a clamped index (shared memory),
// predicated global load for cold states, predicated state update for bytes outside
// the payload.  Bytes 32..63 come from the header cache (a payload never starts
// before byte 34), the rest from memory in 16-B chunks.
template <bool WIDE>
__device__ __forceinline__ uint32_t dfa_byte(const DpiCtx &c, uint32_t s, uint32_t byte, uint32_t &acc)
{
    const uint32_t k = s * c.ncls + c.cls[byte];
    uint32_t e;
    if (WIDE) {
        e = __ldg(reinterpret_cast<const uint32_t *>(c.trans) + k);
        acc = e >> 31;
        return e & 0x7FFFFFFFu;
    }
    e = c.hot[min(k, c.HK1)];
    if (s >= c.H) e = __ldg(reinterpret_cast<const uint16_t *>(c.trans) + k);
    acc = (e >> 15) & 1;
    return e & 0x7FFFu;
}

// Returns the number of accept events and the state after the last one.  One
// accept event (the common matching case) means the match set is exactly the
// output closure of that state; more need the exact re-walk.
template <bool WIDE>
__device__ __forceinline__ void dfa_log(const DpiCtx &c, uint32_t &s, uint32_t byte, uint32_t &cnt, uint32_t &last)
{
    uint32_t acc;
    s = dfa_byte<WIDE>(c, s, byte, acc);
    if (acc) { cnt++; last = s; }
}

// payload bytes [A, 64) of the header cache, A compile-time: no per-byte guards
template <bool WIDE, int A>
__device__ __forceinline__ void walk_cached(const DpiCtx &c, const uint32_t h[16], uint32_t &s, uint32_t &cnt,
                                            uint32_t &last)
{
#pragma unroll
    for (int idx = A; idx < 64; idx++) dfa_log<WIDE>(c, s, (h[idx >> 2] >> ((idx & 3) * 8)) & 0xFF, cnt, last);
}

template <bool WIDE>
__device__ __forceinline__ uint32_t dpi_fast(const DpiCtx &c, const uint32_t h[16], const uint8_t *f, uint32_t a,
                                             uint32_t b, uint64_t pol, uint32_t &last)
{
    uint32_t s = 0, cnt = 0;
    last = 0;
    if (b >= 64 && a == 42) walk_cached<WIDE, 42>(c, h, s, cnt, last);        // IPv4 UDP
    else if (b >= 64 && a == 62) walk_cached<WIDE, 62>(c, h, s, cnt, last);   // IPv6 UDP
    else if (b >= 64 && a == 54) walk_cached<WIDE, 54>(c, h, s, cnt, last);   // IPv4 TCP
    else {
        const uint32_t n = b - a;
#pragma unroll
        for (int idx = 32; idx < 64; idx++) {
            uint32_t acc;
            const uint32_t ns = dfa_byte<WIDE>(c, s, (h[idx >> 2] >> ((idx & 3) * 8)) & 0xFF, acc);
            if ((uint32_t)idx - a < n) {
                s = ns;
                if (acc) { cnt++; last = ns; }
            }
        }
    }
    for (uint32_t ch = max(64u, a & ~15u); ch < b; ch += 16) {
        const uint4 q = ld_stream16(f + ch, pol);
        const uint32_t w[4] = {q.x, q.y, q.z, q.w};
        if (ch >= a && ch + 16 <= b) {
#pragma unroll
            for (int k = 0; k < 16; k++) dfa_log<WIDE>(c, s, (w[k >> 2] >> ((k & 3) * 8)) & 0xFF, cnt, last);
        } else {
#pragma unroll
            for (int k = 0; k < 16; k++) {
                uint32_t acc;
                const uint32_t ns = dfa_byte<WIDE>(c, s, (w[k >> 2] >> ((k & 3) * 8)) & 0xFF, acc);
                if (ch + k - a < b - a) {
                    s = ns;
                    if (acc) { cnt++; last = ns; }
                }
            }
        }
    }
    return cnt;
}

// Exact match set of a packet whose walk hit an accepting state (rare path, not
// inlined): re-walk the payload from memory collecting distinct pattern ids in a
// register list, or -- beyond DPI_LIST ids -- in a per-thread global bitmap; emit
// the (packet, pattern) pairs.  Returns nmatch | any_drop << 31.
struct DpiOvf {
    uint32_t *bitmap;
    uint32_t words;
    uint32_t *match_count, *match_pkt;
    uint16_t *match_pat;
    uint32_t match_cap;
    unsigned long long *stats;
};
__device__ __noinline__ uint32_t dpi_slow(DpiCtx c, const uint8_t *f, uint32_t a, uint32_t b, uint32_t gtid,
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
        s = dfa_step(c, s, (wd >> ((i & 3) * 8)) & 0xFF, acc);
        if (!acc) continue;
        const uint32_t e = __ldg(c.out_off + s + 1);
        for (uint32_t x = __ldg(c.out_off + s); x < e; x++) {
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
        if (n) {
            const uint32_t slot = atomicAdd(o.match_count, n);
            for (uint32_t q = 0; q < n; q++)
                if (slot + q < o.match_cap) { o.match_pkt[slot + q] = pkt_id; o.match_pat[slot + q] = ids[q]; }
            if (slot + n > o.match_cap)
                atomicAdd(&o.stats[ST_MATCH_OVF], (unsigned long long)(slot + n - max(slot, o.match_cap)));
        }
        return n | drop << 31;
    }
    // more than DPI_LIST distinct ids: exact bitmap pass
    atomicAdd(&o.stats[ST_DPI_OVF_PKTS], 1ull);
    uint32_t *bm = o.bitmap + (size_t)gtid * o.words;
    for (uint32_t k = 0; k < o.words; k++) bm[k] = 0;
    uint32_t cnt = 0;
    s = 0;
    drop = 0;
    for (uint32_t i = a; i < b; i++) {
        if (i == a || (i & 15) == 0) q = *reinterpret_cast<const uint4 *>(f + (i & ~15u));
        const uint32_t wd = (i & 8) ? ((i & 4) ? q.w : q.z) : ((i & 4) ? q.y : q.x);
        bool acc;
        s = dfa_step(c, s, (wd >> ((i & 3) * 8)) & 0xFF, acc);
        if (!acc) continue;
        const uint32_t e = __ldg(c.out_off + s + 1);
        for (uint32_t x = __ldg(c.out_off + s); x < e; x++) {
            const uint32_t id = __ldg(c.out_ids + x);
            drop |= __ldg(c.pat_action + id);
            const uint32_t bit = 1u << (id & 31);
            if (bm[id >> 5] & bit) continue;
            bm[id >> 5] |= bit;
            cnt++;
            const uint32_t slot = atomicAdd(o.match_count, 1u);
            if (slot < o.match_cap) { o.match_pkt[slot] = pkt_id; o.match_pat[slot] = (uint16_t)id; }
            else atomicAdd(&o.stats[ST_MATCH_OVF], 1ull);
        }
    }
    return cnt | drop << 31;
}

// ---------------------------------------------------------------- LPM
// DIR-24-8: at most two dependent table reads ("two memory accesses")
__device__ __forceinline__ uint32_t lpm4_lookup(const Lpm4Img &t, uint32_t dst, uint64_t pol)
{
    uint32_t e = ld_tab16(t.tbl24 + (dst >> 8), pol);
    if (e & 0x8000) e = ld_tab16(t.tbllong + ((e & 0x7FFF) << 8) + (dst & 0xFF), pol);
    return e;
}

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
__device__ __forceinline__ void forward_rewrite(uint8_t *f, uint32_t h[16], const PV &v, uint2 nh, uint2 pm, uint64_t pol)
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
__device__ uint32_t nf_esp(uint8_t *f, const PV &v, const EspSa *sap, uint32_t seq, const uint32_t *te)
{
    const uint32_t l4 = v.l4_off, plen = v.ip_end - l4;
    const uint32_t p = (4 - ((plen + 2) & 3)) & 3;
    const uint32_t clen = plen + p + 2;          // multiple of 4
    const uint32_t nK = clen >> 2;
    uint32_t rk[44];
    {
        const uint4 *q = reinterpret_cast<const uint4 *>(sap->rk);
#pragma unroll
        for (int i = 0; i < 11; i++) { uint4 x = __ldg(q + i); rk[4 * i] = x.x; rk[4 * i + 1] = x.y; rk[4 * i + 2] = x.z; rk[4 * i + 3] = x.w; }
    }
    const uint32_t spi = __ldg(&sap->spi), nonce = __ldg(&sap->nonce);
    // 1. move the header 16 B left and fix up the IP header
    {
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
        // ESP header + IV at [l4-16, l4) of the new frame == [f+l4-32, f+l4-16)?  No:
        // new frame starts at f-16, so its byte l4 is f+l4-16; ESP hdr occupies new
        // bytes [l4, l4+16) == f+[l4-16, l4).
        uint8_t *e = f + l4 - 16;
        const uint32_t hw[4] = {spi, seq, 0u, seq};
#pragma unroll
        for (int i = 0; i < 4; i++) {
            e[4 * i] = (uint8_t)(hw[i] >> 24); e[4 * i + 1] = (uint8_t)(hw[i] >> 16);
            e[4 * i + 2] = (uint8_t)(hw[i] >> 8); e[4 * i + 3] = (uint8_t)hw[i];
        }
    }
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
                    uint32_t o[4];
                    aes128_encrypt(te, rk, nonce, 0u, seq, (k >> 2) + 1, o);
                    ks[0] = bswap32(o[0]); ks[1] = bswap32(o[1]); ks[2] = bswap32(o[2]); ks[3] = bswap32(o[3]);
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
    uint64_t gidx;
    uint32_t h[16];
    PV v;
    uint32_t drop, esp_sa, port, acl_rule, lb_b, nmatch, esp_seq, passmask, esp_bytes, out_len;
    uint32_t t24;             // TBL24 entry read right after parse (0xFFFFFFFF: not read)
    bool alive;
};

struct Ctx {
    const uint32_t *acl4, *acl6;
    DpiCtx dpi;
    const uint32_t *te, *ms_nib, *lb_nib;
    uint32_t *vst;            // smem u32 hit counters (nullptr: global atomics)
    uint64_t pol_f, pol_l;
    uint32_t gtid;
};

__device__ __forceinline__ void var_stat(const KParams &P, const Ctx &C, uint32_t idx)
{
    if (C.vst) atomicAdd(&C.vst[idx - NFIX], 1u);
    else atomicAdd(&P.stats[idx], 1ull);
}

struct Loc { uint8_t *f; uint32_t len; uint64_t gidx; };

// stage 1 of the packet pipeline: find the batch, issue the off/len loads
struct Raw { uint8_t *arena; uint64_t off; uint32_t len; uint64_t gidx; };
__device__ __forceinline__ Raw pkt_raw(const KParams &P, uint32_t g, bool valid)
{
    Raw r{nullptr, 0, 0, 0};
    if (!valid) return r;
    uint32_t bi = 0;
    if (P.n_batches > 1) {
        uint32_t lo = 0, hi = P.n_batches - 1;
        while (lo < hi) {
            const uint32_t mid = (lo + hi + 1) >> 1;
            if (P.batches[mid].start <= g) lo = mid; else hi = mid - 1;
        }
        bi = lo;
    }
    const BatchDev &B = P.batches[bi];
    const uint32_t li = g - B.start;
    r.arena = B.arena;
    r.off = B.off[li];
    r.len = B.len[li];
    r.gidx = B.first + li;
    return r;
}
__device__ __forceinline__ Loc pkt_loc(const Raw &r) { return Loc{r.arena + r.off, r.len, r.gidx}; }
__device__ __forceinline__ Loc pkt_locate(const KParams &P, uint32_t g, bool valid) { return pkt_loc(pkt_raw(P, g, valid)); }

__device__ __forceinline__ void pkt_begin(const Ctx &C, const Loc &l, bool valid, Pkt &k)
{
    k.drop = 0xFF; k.esp_sa = 0xFF; k.port = 0; k.acl_rule = 0xFFFF; k.lb_b = 0xFFFF; k.nmatch = 0;
    k.esp_seq = 0; k.passmask = 0; k.esp_bytes = 0; k.alive = false; k.t24 = 0xFFFFFFFFu;
    k.f = l.f; k.flen = k.orig_len = l.len; k.gidx = l.gidx;
    k.out_len = k.flen;
    if (!valid) return;
    load_header(k.f, k.flen, k.h, C.pol_f);
    k.alive = parse(k.h, k.f, k.flen, k.v);
    if (!k.alive) k.drop = 0xFE;
}

template <uint32_t MASK>
__device__ __forceinline__ void run_nf(const KParams &P, const Ctx &C, Pkt &k, uint32_t pos)
{
    const uint32_t kind = P.kind[pos];
    bool dropped = false;
    if ((MASK & MASK_ACL) && kind == NFC_ACL) {
        const uint32_t r = nf_acl(k.v.fam == 4 ? C.acl4 : C.acl6, P.acl.default_action, k.v);
        const uint32_t rule = r & 0xFFFF;
        k.acl_rule = rule;
        var_stat(P, C, P.st_acl + (rule == 0xFFFF ? P.acl.n_rules : rule));
        dropped = (r >> 31) != 0;
    } else if ((MASK & MASK_DPI) && kind == NFC_DPI) {
        uint32_t first;   // state after the (only) accept event when cnt == 1
        const uint32_t cnt = C.dpi.wide ? dpi_fast<true>(C.dpi, k.h, k.f, k.v.pl_off, k.v.ip_end, C.pol_f, first)
                                        : dpi_fast<false>(C.dpi, k.h, k.f, k.v.pl_off, k.v.ip_end, C.pol_f, first);
        if (cnt == 1) {
            // exactly one accept event: match set = output closure of that state (distinct, sorted)
            const uint32_t o0 = __ldg(P.dpi.out_off + first), o1 = __ldg(P.dpi.out_off + first + 1);
            const uint32_t nm = o1 - o0;
            const uint32_t slot = atomicAdd(P.match_count, nm);
            uint32_t drop = 0;
            for (uint32_t q = 0; q < nm; q++) {
                const uint32_t id = __ldg(P.dpi.out_ids + o0 + q);
                drop |= __ldg(P.dpi.pat_action + id);
                if (slot + q < P.match_cap) { P.match_pkt[slot + q] = (uint32_t)k.gidx; P.match_pat[slot + q] = (uint16_t)id; }
            }
            if (slot + nm > P.match_cap)
                atomicAdd(&P.stats[ST_MATCH_OVF], (unsigned long long)(slot + nm - max(slot, P.match_cap)));
            k.nmatch = nm;
            dropped = drop != 0;
        } else if (cnt > 1) {
            const DpiOvf ov{P.dpi.ovf_bitmap, P.dpi.bitmap_words, P.match_count, P.match_pkt, P.match_pat,
                            P.match_cap, P.stats};
            const uint32_t r = dpi_slow(C.dpi, k.f, k.v.pl_off, k.v.ip_end, C.gtid, ov, (uint32_t)k.gidx);
            k.nmatch = r & 0x7FFFFFFFu;
            dropped = (r >> 31) != 0;
        }
    } else if ((MASK & MASK_LPM4) && kind == NFC_LPM4) {
        if (k.v.fam != 4) { k.passmask |= 1u << pos; return; }
        uint32_t nh = k.t24 != 0xFFFFFFFFu ? k.t24 : ld_tab16(P.l4.tbl24 + (k.v.dst[0] >> 8), C.pol_l);
        if (nh & 0x8000) nh = ld_tab16(P.l4.tbllong + ((nh & 0x7FFF) << 8) + (k.v.dst[0] & 0xFF), C.pol_l);
        if (nh == 0x7FFF || hbyte(k.h, 22) <= 1) dropped = true;
        else {
            const uint2 n = __ldg(P.l4.nh + nh);
            const uint32_t pt = n.y >> 16;
            forward_rewrite(k.f, k.h, k.v, n, __ldg(P.l4.pmac + pt), C.pol_f);
            k.port = pt;
        }
    } else if ((MASK & MASK_LPM6) && kind == NFC_LPM6) {
        if (k.v.fam != 6) { k.passmask |= 1u << pos; return; }
        const uint32_t nh = lpm6_lookup(P.l6, k.v.dst);
        if (nh == 0x7FFF || hbyte(k.h, 21) <= 1) dropped = true;
        else {
            const uint2 n = __ldg(P.l6.nh + nh);
            const uint32_t pt = n.y >> 16;
            forward_rewrite(k.f, k.h, k.v, n, __ldg(P.l6.pmac + pt), C.pol_f);
            k.port = pt;
        }
    } else if ((MASK & MASK_IPSEC) && kind == NFC_IPSEC) {
        const uint32_t nl = nf_esp(k.f, k.v, P.esp.sa + k.esp_sa, k.esp_seq, C.te);
        k.esp_bytes = nl - 28 - k.v.l4_off;      // ciphertext bytes |C|
        k.f -= 16;
        k.flen = nl;
        k.out_len = nl;
        load_header(k.f, k.flen, k.h, C.pol_f);
        parse(k.h, k.f, k.flen, k.v);             // later NFs see proto 50, ports 0
    } else if ((MASK & MASK_LB) && kind == NFC_LB) {
        const uint32_t hsh = toeplitz(C.lb_nib, k.v);
        const uint32_t b = (uint32_t)(((uint64_t)hsh * P.lb.n_backends) >> 32);
        k.lb_b = b;
        k.port = __ldg(P.lb.port + b);
        var_stat(P, C, P.st_lb + b);
    }
    if (dropped) { k.drop = pos; k.alive = false; }
}

// record store + counters of one warp's 32 packets into the warp's private slot
__device__ __forceinline__ void pkt_end(const KParams &P, const Ctx &C, Pkt &k, bool valid, uint32_t g,
                                        unsigned long long *ws, uint32_t lane)
{
    if (valid) {
        if (k.drop != 0xFF) k.port = 0xFFFF;
        const uint4 rec = make_uint4(k.drop | k.esp_sa << 8 | k.port << 16, k.acl_rule | k.lb_b << 16,
                                     k.nmatch | k.out_len << 16, k.esp_seq);
        st_stream16(reinterpret_cast<uint4 *>(P.rec) + g, rec, C.pol_f);
    }
    const uint32_t FULL = 0xFFFFFFFFu;
    const bool esp = k.esp_sa != 0xFF;
    const uint32_t nv = __popc(__ballot_sync(FULL, valid));
    const uint32_t nparse = __popc(__ballot_sync(FULL, valid && k.drop == 0xFE));
    const uint32_t nfwd = __popc(__ballot_sync(FULL, valid && k.drop == 0xFF));
    const uint32_t bin = __reduce_add_sync(FULL, k.orig_len);
    const uint32_t bout = __reduce_add_sync(FULL, (valid && k.drop == 0xFF) ? k.out_len : 0u);
    const uint32_t pairs = __reduce_add_sync(FULL, k.nmatch);
    const uint32_t nesp = __popc(__ballot_sync(FULL, esp));
    const uint32_t eb = __reduce_add_sync(FULL, esp ? k.esp_bytes : 0u);
    const uint32_t eblk = __reduce_add_sync(FULL, esp ? (k.esp_bytes + 15) >> 4 : 0u);
    uint32_t pc[NFC_MAX_CHAIN][3];
#pragma unroll
    for (int p = 0; p < NFC_MAX_CHAIN; p++) {
        const bool reached = valid && k.drop != 0xFE && (k.drop == 0xFF || k.drop >= (uint32_t)p);
        pc[p][0] = __popc(__ballot_sync(FULL, reached));
        pc[p][1] = __popc(__ballot_sync(FULL, valid && k.drop == (uint32_t)p));
        pc[p][2] = __popc(__ballot_sync(FULL, reached && ((k.passmask >> p) & 1)));
    }
    if (lane == 0 && nv) {
        ws[ST_PKTS] += nv;
        ws[ST_FWD] += nfwd;
        ws[ST_DROP] += nv - nfwd;
        ws[ST_PARSE_DROP] += nparse;
        ws[ST_BYTES_IN] += bin;
        ws[ST_BYTES_OUT] += bout;
        ws[ST_DPI_PAIRS] += pairs;
        ws[ST_ESP_PKTS] += nesp;
        ws[ST_ESP_BYTES] += eb;
        ws[ST_ESP_BLOCKS] += eblk;
#pragma unroll
        for (int p = 0; p < NFC_MAX_CHAIN; p++) {
            if ((uint32_t)p >= P.n_nf) break;
            ws[ST_POS_BASE + 4 * p] += pc[p][0];
            ws[ST_POS_BASE + 4 * p + 1] += pc[p][1];
            ws[ST_POS_BASE + 4 * p + 2] += pc[p][2];
            ws[ST_POS_BASE + 4 * p + 3] += pc[p][0] - pc[p][1] - pc[p][2];
        }
    }
}

// ESP sequence numbers for one CTA tile: per SA, global packet order (decoupled look-back)
__device__ __forceinline__ void esp_assign(const KParams &P, const Ctx &C, uint8_t *smem, const SmemLayout &L, uint32_t tile,
                           Pkt &k)
{
    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t nsa = P.esp.n_sa;
    uint16_t *wcnt = reinterpret_cast<uint16_t *>(smem + L.wcnt);
    uint32_t *pref = reinterpret_cast<uint32_t *>(smem + L.prefix);
    for (uint32_t i = tid; i < NWARP * 256; i += TILE) wcnt[i] = 0;
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
            for (int w = 0; w < NWARP; w++) { const uint32_t c = wcnt[w * 256 + s]; wcnt[w * 256 + s] = (uint16_t)run; run += c; }
            vec[s] = run;
            pref[s] = 0;
        }
        __syncwarp();
        if (tile > 0) {
            if (lane == 0) { __threadfence(); st_release(P.tile_flag + tile, P.epoch << 2 | 1u); }
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

template <uint32_t MASK>
__global__ void __launch_bounds__(TILE, (MASK & MASK_IPSEC) ? 2 : NFC_MINB) sfc_kernel(const KParams P)
{
    extern __shared__ __align__(16) uint8_t smem[];
    __shared__ uint32_t s_tile;
    const SmemLayout L = smem_layout(MASK, P);
    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    unsigned long long *wst = reinterpret_cast<unsigned long long *>(smem + L.wst);
    uint32_t *vst = reinterpret_cast<uint32_t *>(smem + L.vst);
    const uint32_t n_var = P.stats_len - NFIX;
    for (uint32_t i = tid; i < NWARP * NFIX; i += TILE) wst[i] = 0;
    if (P.smem_stats)
        for (uint32_t i = tid; i < n_var; i += TILE) vst[i] = 0;

    Ctx C;
    C.gtid = blockIdx.x * TILE + tid;
    C.vst = P.smem_stats ? vst : nullptr;
    C.pol_f = pol_first();
    C.pol_l = pol_last();
    C.acl4 = C.acl6 = nullptr;
    C.te = C.ms_nib = C.lb_nib = nullptr;
    C.dpi.cls = smem + L.cls;
    C.dpi.ncls = P.dpi.ncls;
    C.dpi.wide = P.dpi.wide;
    C.dpi.trans = P.dpi.trans;
    C.dpi.out_off = P.dpi.out_off;
    C.dpi.out_ids = P.dpi.out_ids;
    C.dpi.pat_action = P.dpi.pat_action;
    C.dpi.hot = reinterpret_cast<const uint16_t *>(smem + L.hot);
    C.dpi.H = 0;
    C.dpi.HK1 = 0;
    // NFs compiled into this variant but absent from the chain are skipped at run time
    const bool has_esp = (MASK & MASK_IPSEC) && P.esp_pos < P.n_nf;
    if ((MASK & MASK_ACL) && (P.present & MASK_ACL)) {
        if (P.acl.smem_words) {
            uint4 *d4 = reinterpret_cast<uint4 *>(smem + L.acl4);
            uint4 *d6 = reinterpret_cast<uint4 *>(smem + L.acl6);
            for (uint32_t i = tid; i < P.acl.words4 / 4; i += TILE) d4[i] = __ldg(reinterpret_cast<const uint4 *>(P.acl.bv4) + i);
            for (uint32_t i = tid; i < P.acl.words6 / 4; i += TILE) d6[i] = __ldg(reinterpret_cast<const uint4 *>(P.acl.bv6) + i);
            C.acl4 = reinterpret_cast<const uint32_t *>(d4);
            C.acl6 = reinterpret_cast<const uint32_t *>(d6);
        } else {
            C.acl4 = P.acl.bv4;
            C.acl6 = P.acl.bv6;
        }
    }
    if ((MASK & MASK_DPI) && (P.present & MASK_DPI)) {
        uint8_t *cls = smem + L.cls;
        for (uint32_t i = tid; i < 256; i += TILE) cls[i] = __ldg(P.dpi.cls + i);
        const uint32_t H = P.dpi.wide ? 0 : P.dpi.hot_states;
        uint16_t *hot = reinterpret_cast<uint16_t *>(smem + L.hot);
        const uint16_t *tr = reinterpret_cast<const uint16_t *>(P.dpi.trans);
        for (uint32_t i = tid; i < H * P.dpi.ncls; i += TILE) hot[i] = __ldg(tr + i);
        C.dpi.H = H;
        C.dpi.HK1 = H ? H * P.dpi.ncls - 1 : 0;
    }
    if ((MASK & MASK_IPSEC) && has_esp) {
        uint32_t *te = reinterpret_cast<uint32_t *>(smem + L.te), *mn = reinterpret_cast<uint32_t *>(smem + L.ms_nib);
        for (uint32_t i = tid; i < 256 * 32; i += TILE) te[i] = __ldg(P.esp.te + (i >> 5));   // T0 x 32 lanes
        for (uint32_t i = tid; i < 72 * 16; i += TILE) mn[i] = __ldg(P.esp.rss_nib + i);
        C.te = te + lane;         // this lane's bank column
        C.ms_nib = mn;
    }
    if ((MASK & MASK_LB) && (P.present & MASK_LB)) {
        uint32_t *ln = reinterpret_cast<uint32_t *>(smem + L.lb_nib);
        for (uint32_t i = tid; i < 72 * 16; i += TILE) ln[i] = __ldg(P.lb.nib + i);
        C.lb_nib = ln;
    }
    __syncthreads();
    unsigned long long *ws = wst + warp * NFIX;

    if (!has_esp) {
        // warp-granular persistent loop: 32 consecutive packets per claim, no CTA barriers
        auto claim = [&]() {
            uint32_t b = 0;
            if (lane == 0) b = atomicAdd(P.tile_counter, 32u);
            return __shfl_sync(0xFFFFFFFFu, b, 0);
        };
#if NFC_PIPE == 3
        // three-stage software pipeline, one iteration of distance each:
        // claim chunk c+3 | load off/len of c+2 | locate c+1, prefetch its headers | process c
        uint32_t c0 = claim(), c1 = claim(), c2 = claim();
        Loc loc = pkt_locate(P, c0 + lane, c0 + lane < P.n_pkts);
        Raw raw1 = pkt_raw(P, c1 + lane, c1 + lane < P.n_pkts);
        while (c0 < P.n_pkts) {
            uint32_t c3 = 0;
            if (lane == 0) c3 = atomicAdd(P.tile_counter, 32u);
            const Raw raw2 = pkt_raw(P, c2 + lane, c2 + lane < P.n_pkts);
            const Loc loc1 = pkt_loc(raw1);
            if (c1 + lane < P.n_pkts) asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(loc1.f));
#else
        // next chunk claimed and located before the current one is processed
        uint32_t c0 = claim();
        Loc loc = pkt_locate(P, c0 + lane, c0 + lane < P.n_pkts);
        while (c0 < P.n_pkts) {
            const uint32_t c1 = claim();
            const Loc loc1 = pkt_locate(P, c1 + lane, c1 + lane < P.n_pkts);
            if (c1 + lane < P.n_pkts) asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(loc1.f));
#endif
            const uint32_t g = c0 + lane;
            const bool valid = g < P.n_pkts;
            Pkt k;
            pkt_begin(C, loc, valid, k);
#if NFC_EARLY_T24
            if ((MASK & MASK_LPM4) && (P.present & MASK_LPM4) && k.alive && k.v.fam == 4)
                k.t24 = ld_tab16(P.l4.tbl24 + (k.v.dst[0] >> 8), C.pol_l);   // header-phase lookup, used later
#endif
            for (uint32_t pos = 0; pos < P.n_nf && k.alive; pos++) run_nf<MASK>(P, C, k, pos);
            pkt_end(P, C, k, valid, g, ws, lane);
#if NFC_PIPE == 3
            c0 = c1; c1 = c2; c2 = __shfl_sync(0xFFFFFFFFu, c3, 0);
            loc = loc1;
            raw1 = raw2;
#else
            c0 = c1;
            loc = loc1;
#endif
        }
    } else if constexpr ((MASK & MASK_IPSEC) != 0) {
        // CTA tiles claimed in global order (ESP sequence numbers need the order)
        for (;;) {
            if (tid == 0) s_tile = atomicAdd(P.tile_counter, 1u);
            __syncthreads();
            const uint32_t tile = s_tile;
            __syncthreads();
            if (tile >= P.n_tiles) break;
            const uint32_t g = tile * TILE + tid;
            const bool valid = g < P.n_pkts;
            Pkt k;
            pkt_begin(C, pkt_locate(P, g, valid), valid, k);
            for (uint32_t pos = 0; pos < P.esp_pos && k.alive; pos++) run_nf<MASK>(P, C, k, pos);
            esp_assign(P, C, smem, L, tile, k);
            for (uint32_t pos = P.esp_pos; pos < P.n_nf && k.alive; pos++) run_nf<MASK>(P, C, k, pos);
            pkt_end(P, C, k, valid, g, ws, lane);
        }
    }
    // ---- flush CTA counters
    __syncthreads();
    for (uint32_t i = tid; i < NFIX; i += TILE) {
        unsigned long long s = 0;
#pragma unroll
        for (int w = 0; w < NWARP; w++) s += wst[w * NFIX + i];
        if (s) atomicAdd(&P.stats[i], s);
    }
    if (P.smem_stats)
        for (uint32_t i = tid; i < n_var; i += TILE)
            if (vst[i]) atomicAdd(&P.stats[NFIX + i], (unsigned long long)vst[i]);
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

// ---------------------------------------------------------------- host launch
template <uint32_t M>
static int launch_t(const KParams &p, int dev, void *stream, std::string &err, LaunchCfg *cfg, bool query_only)
{
    const size_t smem = smem_layout(M, p).total;
    if (cudaFuncSetAttribute(sfc_kernel<M>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess) {
        err = "cudaFuncSetAttribute failed";
        return NFC_ECUDA;
    }
    int per_sm = 0, sms = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, sfc_kernel<M>, TILE, smem);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (per_sm < 1) per_sm = 1;
    int grid = sms * per_sm;
    if (!query_only && (uint32_t)grid > p.n_tiles) grid = (int)p.n_tiles;
    if (grid < 1) grid = 1;
    if (cfg) { cfg->grid = grid; cfg->block = TILE; cfg->smem = smem; }
    if (query_only) return NFC_OK;
    sfc_kernel<M><<<grid, TILE, smem, (cudaStream_t)stream>>>(p);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) { err = std::string("sfc_kernel launch: ") + cudaGetErrorString(e); return NFC_ECUDA; }
    return NFC_OK;
}

// Chain signatures with a dedicated instantiation (dead NF code removed at compile
// time); any other chain runs the all-NF variant, which interprets the order at run time.
static constexpr uint32_t M_ALL = MASK_ACL | MASK_DPI | MASK_LPM4 | MASK_LPM6 | MASK_IPSEC | MASK_LB;
static constexpr uint32_t M_C1 = MASK_ACL | MASK_DPI | MASK_LPM4;
static constexpr uint32_t M_C2 = MASK_IPSEC;
static constexpr uint32_t M_C3 = MASK_ACL | MASK_DPI | MASK_LB;
static constexpr uint32_t M_C4 = MASK_ACL | MASK_LPM6 | MASK_DPI | MASK_IPSEC | MASK_LB;

static int dispatch(uint32_t mask, const KParams &p, int dev, void *stream, std::string &err, LaunchCfg *cfg,
                    bool query_only)
{
    switch (mask) {
    case M_C1: return launch_t<M_C1>(p, dev, stream, err, cfg, query_only);
    case M_C2: return launch_t<M_C2>(p, dev, stream, err, cfg, query_only);
    case M_C3: return launch_t<M_C3>(p, dev, stream, err, cfg, query_only);
    case M_C4: return launch_t<M_C4>(p, dev, stream, err, cfg, query_only);
    default: return launch_t<M_ALL>(p, dev, stream, err, cfg, query_only);
    }
}

int sfc_launch(uint32_t mask, const KParams &p, int device, void *stream, std::string &err, LaunchCfg *cfg_out)
{
    return dispatch(mask, p, device, stream, err, cfg_out, false);
}

int sfc_query(uint32_t mask, const KParams &p, int device, LaunchCfg *cfg_out)
{
    std::string err;
    return dispatch(mask, p, device, nullptr, err, cfg_out, true);
}

size_t sfc_smem_bytes(uint32_t mask, const KParams &p) { return smem_layout(mask, p).total; }

} // namespace nfc
