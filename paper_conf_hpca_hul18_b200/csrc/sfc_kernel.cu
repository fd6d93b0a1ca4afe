// sfc_kernel.cu -- the fused, persistent SFC kernel for sm_100a.
//
// One launch drains all packets of an nfc_process_batch call.  Each CTA of
// TILE threads repeatedly claims a tile of TILE consecutive packets from a
// global atomic counter (persistent kernel, P:L112, P:L235 [SIV]) and every
// thread carries one packet through the whole chain in registers:
//   parse once (the de-duplicated header classifier)
//   -> NFs in original SFC order, a dropped packet skipping every later NF
//      (early drop; no batch re-split between NFs)
//   -> ESP sequence numbers per SA in global packet order via a decoupled
//      look-back across tiles (the only cross-packet dependency)
//   -> one 16 B result record, counters aggregated per warp / CTA.
// Packet bytes are read from HBM once and rewritten in place.  No tensor
// cores: nothing here is a dense contraction (integer / table-lookup work).
#include <cuda_runtime.h>
#include <stdint.h>

#include "nfc_internal.h"

namespace nfc {

static constexpr int TILE = 256;        // threads per CTA == packets per tile
static constexpr int NWARP = TILE / 32;
static constexpr int DPI_LIST = 16;     // distinct matches kept in registers before the bitmap path

// ---------------------------------------------------------------- shared memory layout
struct SmemLayout {
    uint32_t te, ms_nib, lb_nib, cls, stats, wcnt, prefix, total;
};
__host__ __device__ inline SmemLayout smem_layout(uint32_t mask, const KParams &p)
{
    SmemLayout L{};
    uint32_t o = 0;
    if (mask & MASK_IPSEC) { L.te = o; o += 5 * 256 * 4; L.ms_nib = o; o += 72 * 16 * 4; }
    if (mask & MASK_LB) { L.lb_nib = o; o += 72 * 16 * 4; }
    if (mask & MASK_DPI) { L.cls = o; o += 256; }
    o = (o + 15) & ~15u;
    L.stats = o;
    o += (p.smem_stats ? p.stats_len : ST_VAR_BASE) * 8;
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

// byte k (0..63) of the 64 B header cache; k compile-time in hot paths
__device__ __forceinline__ uint32_t hbyte(const uint32_t h[16], uint32_t k) { return (h[k >> 2] >> ((k & 3) * 8)) & 0xFF; }
__device__ __forceinline__ uint32_t hbe16(const uint32_t h[16], uint32_t k) { return hbyte(h, k) << 8 | hbyte(h, k + 1); }
__device__ __forceinline__ uint32_t hbe32(const uint32_t h[16], uint32_t k) { return hbe16(h, k) << 16 | hbe16(h, k + 2); }
// dynamic byte index: header cache if < 64 else global memory
__device__ __forceinline__ uint32_t dbyte(const uint32_t h[16], const uint8_t *f, uint32_t k)
{
    if (k < 64) {
        uint32_t w = 0;
#pragma unroll
        for (int j = 0; j < 16; j++) w = (j == (int)(k >> 2)) ? h[j] : w;
        return (w >> ((k & 3) * 8)) & 0xFF;
    }
    return f[k];
}

// ---------------------------------------------------------------- per-packet state
struct PV {
    uint32_t fam;                 // 4 or 6
    uint32_t l4_off, ip_end, pl_off;
    uint32_t proto, sport, dport;
    uint32_t src[4], dst[4];      // big-endian-valued words
};

__device__ __forceinline__ void load_header(const uint8_t *f, uint32_t flen, uint32_t h[16])
{
    const uint4 *q = reinterpret_cast<const uint4 *>(f);
    uint32_t nch = min(4u, (flen + 15) >> 4);
#pragma unroll
    for (int c = 0; c < 4; c++) {
        uint4 v = c < (int)nch ? q[c] : make_uint4(0, 0, 0, 0);
        h[4 * c] = v.x; h[4 * c + 1] = v.y; h[4 * c + 2] = v.z; h[4 * c + 3] = v.w;
    }
}

// Parse (P:L87 validity check): Ethernet -> IPv4/IPv6 -> UDP/TCP.
__device__ bool parse(const uint32_t h[16], const uint8_t *f, uint32_t flen, PV &v)
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
            uint32_t doff = dbyte(h, f, l4 + 12) >> 4;
            if (doff < 5 || l4 + 4 * doff > v.ip_end) return false;
            l4len = 4 * doff;
        }
        if (l4 == 34) { v.sport = hbe16(h, 34); v.dport = hbe16(h, 36); }
        else if (l4 == 54) { v.sport = hbe16(h, 54); v.dport = hbe16(h, 56); }
        else {
            v.sport = dbyte(h, f, l4) << 8 | dbyte(h, f, l4 + 1);
            v.dport = dbyte(h, f, l4 + 2) << 8 | dbyte(h, f, l4 + 3);
        }
    }
    v.pl_off = v.l4_off + l4len;
    return true;
}

// ---------------------------------------------------------------- ACL
// First-match linear scan over the packet's family (rules kept in priority order).
__device__ uint32_t nf_acl(const AclImg &a, const PV &v)
{
    uint32_t ports = v.sport << 16 | v.dport;
    (void)ports;
    if (v.fam == 4) {
        for (uint32_t i = 0; i < a.n4; i++) {
            uint4 r = __ldg(a.r4 + 2 * i);
            if (((v.src[0] & r.y) != r.x) | ((v.dst[0] & r.w) != r.z)) continue;
            uint4 t = __ldg(a.r4 + 2 * i + 1);
            if (v.sport < (t.x & 0xFFFF) || v.sport > (t.x >> 16)) continue;
            if (v.dport < (t.y & 0xFFFF) || v.dport > (t.y >> 16)) continue;
            if (!((t.z >> 8) & 1) && (t.z & 0xFF) != v.proto) continue;
            return t.w | ((t.z >> 16) & 1) << 31;
        }
    } else {
        for (uint32_t i = 0; i < a.n6; i++) {
            const uint4 *r = a.r6 + 5 * i;
            uint4 s = __ldg(r), sm = __ldg(r + 1);
            if (((v.src[0] & sm.x) != s.x) | ((v.src[1] & sm.y) != s.y) | ((v.src[2] & sm.z) != s.z) |
                ((v.src[3] & sm.w) != s.w)) continue;
            uint4 d = __ldg(r + 2), dm = __ldg(r + 3);
            if (((v.dst[0] & dm.x) != d.x) | ((v.dst[1] & dm.y) != d.y) | ((v.dst[2] & dm.z) != d.z) |
                ((v.dst[3] & dm.w) != d.w)) continue;
            uint4 t = __ldg(r + 4);
            if (v.sport < (t.x & 0xFFFF) || v.sport > (t.x >> 16)) continue;
            if (v.dport < (t.y & 0xFFFF) || v.dport > (t.y >> 16)) continue;
            if (!((t.z >> 8) & 1) && (t.z & 0xFF) != v.proto) continue;
            return t.w | ((t.z >> 16) & 1) << 31;
        }
    }
    return 0xFFFFu | a.default_action << 31;   // no match
}

// ---------------------------------------------------------------- DPI
struct DpiOut { uint32_t nmatch; bool drop; uint16_t ids[DPI_LIST]; bool ovf; };

__device__ __forceinline__ uint32_t dfa_step(const DpiImg &d, const uint8_t *cls, uint32_t s, uint32_t b, bool &acc)
{
    uint32_t c = cls[b];
    uint32_t e;
    if (d.wide) { e = __ldg(reinterpret_cast<const uint32_t *>(d.trans) + s * d.ncls + c); acc = e >> 31; e &= 0x7FFFFFFFu; }
    else { e = __ldg(reinterpret_cast<const uint16_t *>(d.trans) + s * d.ncls + c); acc = e >> 15; e &= 0x7FFFu; }
    return e;
}

// Walk the DFA over payload [pl_off, ip_end).  Distinct ids go to a register list;
// more than DPI_LIST distinct ids switch to an exact per-thread bitmap rescan.
template <typename F>
__device__ __forceinline__ void dpi_scan(const uint8_t *f, uint32_t a, uint32_t b, F &&on_byte)
{
    if (a >= b) return;
    uint32_t c0 = a & ~15u;
    for (uint32_t c = c0; c < b; c += 16) {
        uint4 q = *reinterpret_cast<const uint4 *>(f + c);
        uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
        for (int k = 0; k < 16; k++) {
            uint32_t idx = c + k;
            if (idx >= a && idx < b) on_byte((w[k >> 2] >> ((k & 3) * 8)) & 0xFF);
        }
    }
}

__device__ void nf_dpi(const DpiImg &d, const uint8_t *cls, const uint8_t *f, const PV &v, uint32_t gtid,
                       DpiOut &o)
{
    o.nmatch = 0; o.drop = false; o.ovf = false;
    uint32_t s = 0;
    dpi_scan(f, v.pl_off, v.ip_end, [&](uint32_t byte) {
        bool acc;
        s = dfa_step(d, cls, s, byte, acc);
        if (acc) {
            uint32_t e = __ldg(d.out_off + s + 1);
            for (uint32_t x = __ldg(d.out_off + s); x < e; x++) {
                uint32_t id = __ldg(d.out_ids + x);
                o.drop |= __ldg(d.pat_action + id) != 0;
                if (o.ovf) continue;
                bool seen = false;
                for (uint32_t k = 0; k < o.nmatch; k++) seen |= o.ids[k] == id;
                if (!seen) {
                    if (o.nmatch < DPI_LIST) o.ids[o.nmatch++] = (uint16_t)id;
                    else o.ovf = true;
                }
            }
        }
    });
}

// exact distinct set with a per-thread bitmap (rare path), emitting pairs directly
__device__ uint32_t dpi_bitmap_pass(const DpiImg &d, const uint8_t *cls, const uint8_t *f, const PV &v,
                                    uint32_t gtid, const KParams &P, uint32_t pkt_id)
{
    uint32_t *bm = d.ovf_bitmap + (size_t)gtid * d.bitmap_words;
    for (uint32_t k = 0; k < d.bitmap_words; k++) bm[k] = 0;
    uint32_t s = 0, cnt = 0;
    dpi_scan(f, v.pl_off, v.ip_end, [&](uint32_t byte) {
        bool acc;
        s = dfa_step(d, cls, s, byte, acc);
        if (acc) {
            uint32_t e = __ldg(d.out_off + s + 1);
            for (uint32_t x = __ldg(d.out_off + s); x < e; x++) {
                uint32_t id = __ldg(d.out_ids + x);
                uint32_t bit = 1u << (id & 31);
                if (!(bm[id >> 5] & bit)) {
                    bm[id >> 5] |= bit;
                    cnt++;
                    uint32_t slot = atomicAdd(P.match_count, 1u);
                    if (slot < P.match_cap) { P.match_pkt[slot] = pkt_id; P.match_pat[slot] = (uint16_t)id; }
                    else atomicAdd(&P.stats[ST_MATCH_OVF], 1ull);
                }
            }
        }
    });
    return cnt;
}

// ---------------------------------------------------------------- LPM
__device__ __forceinline__ uint32_t lpm4_lookup(const Lpm4Img &t, uint32_t dst)
{
    uint32_t e = __ldg(t.tbl24 + (dst >> 8));
    if (e & 0x8000) e = __ldg(t.tbllong + ((e & 0x7FFF) << 8) + (dst & 0xFF));
    return e;
}

__device__ uint32_t lpm6_lookup(const Lpm6Img &t, const uint32_t dst[4])
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
__device__ void forward_rewrite(uint8_t *f, uint32_t h[16], const PV &v, uint2 nh, uint2 pm)
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
        } else {                              // IPv4 options: header beyond the cache
            sum = (h[3] >> 16);
            for (uint32_t k = 16; k < v.l4_off; k += 2) {
                uint32_t lo = dbyte(h, f, k), hi = dbyte(h, f, k + 1);
                if (k != 24) sum += lo | hi << 8;
            }
        }
        sum = (sum & 0xFFFF) + (sum >> 16);
        sum = (sum & 0xFFFF) + (sum >> 16);
        h[6] |= (~sum) & 0xFFFF;
    } else {
        h[5] -= 1u << 8;                      // hop limit: byte 21
    }
    uint4 *q = reinterpret_cast<uint4 *>(f);
    q[0] = make_uint4(h[0], h[1], h[2], h[3]);
    q[1] = make_uint4(h[4], h[5], h[6], h[7]);
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
__device__ __forceinline__ void aes128_encrypt(const uint32_t *te, const uint32_t rk[44], uint32_t in0, uint32_t in1,
                                               uint32_t in2, uint32_t in3, uint32_t out[4])
{
    const uint32_t *T0 = te, *T1 = te + 256, *T2 = te + 512, *T3 = te + 768, *S = te + 1024;
    uint32_t s0 = in0 ^ rk[0], s1 = in1 ^ rk[1], s2 = in2 ^ rk[2], s3 = in3 ^ rk[3];
#pragma unroll
    for (int r = 1; r < 10; r++) {
        uint32_t t0 = T0[s0 >> 24] ^ T1[(s1 >> 16) & 255] ^ T2[(s2 >> 8) & 255] ^ T3[s3 & 255] ^ rk[4 * r];
        uint32_t t1 = T0[s1 >> 24] ^ T1[(s2 >> 16) & 255] ^ T2[(s3 >> 8) & 255] ^ T3[s0 & 255] ^ rk[4 * r + 1];
        uint32_t t2 = T0[s2 >> 24] ^ T1[(s3 >> 16) & 255] ^ T2[(s0 >> 8) & 255] ^ T3[s1 & 255] ^ rk[4 * r + 2];
        uint32_t t3 = T0[s3 >> 24] ^ T1[(s0 >> 16) & 255] ^ T2[(s1 >> 8) & 255] ^ T3[s2 & 255] ^ rk[4 * r + 3];
        s0 = t0; s1 = t1; s2 = t2; s3 = t3;
    }
    out[0] = (S[s0 >> 24] << 24 | S[(s1 >> 16) & 255] << 16 | S[(s2 >> 8) & 255] << 8 | S[s3 & 255]) ^ rk[40];
    out[1] = (S[s1 >> 24] << 24 | S[(s2 >> 16) & 255] << 16 | S[(s3 >> 8) & 255] << 8 | S[s0 & 255]) ^ rk[41];
    out[2] = (S[s2 >> 24] << 24 | S[(s3 >> 16) & 255] << 16 | S[(s0 >> 8) & 255] << 8 | S[s1 & 255]) ^ rk[42];
    out[3] = (S[s3 >> 24] << 24 | S[(s0 >> 16) & 255] << 16 | S[(s1 >> 8) & 255] << 8 | S[s2 & 255]) ^ rk[43];
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
template <uint32_t MASK>
__global__ void __launch_bounds__(TILE, (MASK & MASK_IPSEC) ? 1 : 2) sfc_kernel(const KParams P)
{
    extern __shared__ __align__(16) uint8_t smem[];
    __shared__ uint32_t s_tile;
    const SmemLayout L = smem_layout(MASK, P);
    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t gtid = blockIdx.x * TILE + tid;
    unsigned long long *sst = reinterpret_cast<unsigned long long *>(smem + L.stats);
    const uint32_t n_sst = P.smem_stats ? P.stats_len : ST_VAR_BASE;
    for (uint32_t i = tid; i < n_sst; i += TILE) sst[i] = 0;
    uint32_t *te = reinterpret_cast<uint32_t *>(smem + L.te);
    uint32_t *ms_nib = reinterpret_cast<uint32_t *>(smem + L.ms_nib);
    uint32_t *lb_nib = reinterpret_cast<uint32_t *>(smem + L.lb_nib);
    uint8_t *cls = smem + L.cls;
    // NFs compiled into this variant but absent from the chain are skipped at run time
    const bool has_esp = (MASK & MASK_IPSEC) && P.esp_pos < P.n_nf;
    if ((MASK & MASK_IPSEC) && has_esp) {
        for (uint32_t i = tid; i < 5 * 256; i += TILE) te[i] = __ldg(P.esp.te + i);
        for (uint32_t i = tid; i < 72 * 16; i += TILE) ms_nib[i] = __ldg(P.esp.rss_nib + i);
    }
    if ((MASK & MASK_LB) && (P.present & MASK_LB))
        for (uint32_t i = tid; i < 72 * 16; i += TILE) lb_nib[i] = __ldg(P.lb.nib + i);
    if ((MASK & MASK_DPI) && (P.present & MASK_DPI))
        for (uint32_t i = tid; i < 256; i += TILE) cls[i] = __ldg(P.dpi.cls + i);
    // variable stats live in smem or go straight to global memory
    auto stat_add = [&](uint32_t idx, unsigned long long v) {
        if (P.smem_stats) atomicAdd(&sst[idx], v);
        else atomicAdd(&P.stats[idx], v);
    };
    __syncthreads();

    for (;;) {
        if (tid == 0) s_tile = atomicAdd(P.tile_counter, 1u);
        __syncthreads();
        const uint32_t tile = s_tile;
        __syncthreads();
        if (tile >= P.n_tiles) break;
        const uint32_t g = tile * TILE + tid;
        const bool valid = g < P.n_pkts;
        // ---- locate the packet
        uint32_t bi = 0;
        if (P.n_batches > 1 && valid) {
            uint32_t lo = 0, hi = P.n_batches - 1;
            while (lo < hi) {
                uint32_t mid = (lo + hi + 1) >> 1;
                if (P.batches[mid].start <= g) lo = mid; else hi = mid - 1;
            }
            bi = lo;
        }
        uint8_t *f = nullptr;
        uint32_t flen = 0;
        uint64_t gidx = 0;
        if (valid) {
            const BatchDev &B = P.batches[bi];
            uint32_t li = g - B.start;
            f = B.arena + B.off[li];
            flen = B.len[li];
            gidx = B.first + li;
        }
        // ---- per-packet state
        uint32_t h[16];
        PV v{};
        uint32_t drop = 0xFF, esp_sa = 0xFF, port = 0, acl_rule = 0xFFFF, lb_b = 0xFFFF, nmatch = 0, esp_seq = 0;
        uint32_t passmask = 0, esp_bytes = 0;
        bool ok = false;
        if (valid) {
            load_header(f, flen, h);
            ok = parse(h, f, flen, v);
            if (!ok) drop = 0xFE;
        }
        bool alive = ok;
        uint32_t out_len = flen;

        auto run_nf = [&](uint32_t pos) {
            const uint32_t kind = P.kind[pos];
            bool dropped = false;
            if ((MASK & MASK_ACL) && kind == NFC_ACL) {
                uint32_t r = nf_acl(P.acl, v);
                uint32_t rule = r & 0xFFFF;
                acl_rule = rule;
                stat_add(P.st_acl + (rule == 0xFFFF ? P.acl.n_rules : rule), 1ull);
                dropped = (r >> 31) != 0;
            } else if ((MASK & MASK_DPI) && kind == NFC_DPI) {
                DpiOut o;
                nf_dpi(P.dpi, cls, f, v, gtid, o);
                const uint32_t pkt_id = (uint32_t)gidx;
                if (!o.ovf) {
                    nmatch = o.nmatch;
                    if (o.nmatch) {
                        uint32_t slot = atomicAdd(P.match_count, o.nmatch);
                        for (uint32_t k = 0; k < o.nmatch; k++)
                            if (slot + k < P.match_cap) { P.match_pkt[slot + k] = pkt_id; P.match_pat[slot + k] = o.ids[k]; }
                        if (slot + o.nmatch > P.match_cap)
                            stat_add(ST_MATCH_OVF, (unsigned long long)(slot + o.nmatch - max(slot, P.match_cap)));
                    }
                } else {
                    nmatch = dpi_bitmap_pass(P.dpi, cls, f, v, gtid, P, pkt_id);
                    stat_add(ST_DPI_OVF_PKTS, 1ull);
                }
                dropped = o.drop;
            } else if ((MASK & MASK_LPM4) && kind == NFC_LPM4) {
                if (v.fam != 4) { passmask |= 1u << pos; return; }
                uint32_t nh = lpm4_lookup(P.l4, v.dst[0]);
                uint32_t ttl = hbyte(h, 22);
                if (nh == 0x7FFF || ttl <= 1) { dropped = true; }
                else {
                    uint2 n = __ldg(P.l4.nh + nh);
                    uint32_t pt = n.y >> 16;
                    forward_rewrite(f, h, v, n, __ldg(P.l4.pmac + pt));
                    port = pt;
                }
            } else if ((MASK & MASK_LPM6) && kind == NFC_LPM6) {
                if (v.fam != 6) { passmask |= 1u << pos; return; }
                uint32_t nh = lpm6_lookup(P.l6, v.dst);
                uint32_t hl = hbyte(h, 21);
                if (nh == 0x7FFF || hl <= 1) { dropped = true; }
                else {
                    uint2 n = __ldg(P.l6.nh + nh);
                    uint32_t pt = n.y >> 16;
                    forward_rewrite(f, h, v, n, __ldg(P.l6.pmac + pt));
                    port = pt;
                }
            } else if ((MASK & MASK_IPSEC) && kind == NFC_IPSEC) {
                uint32_t nl = nf_esp(f, v, P.esp.sa + esp_sa, esp_seq, te);
                esp_bytes = nl - 28 - v.l4_off;          // == clen (ciphertext bytes)
                f -= 16;
                flen = nl;
                out_len = nl;
                load_header(f, flen, h);
                parse(h, f, flen, v);                    // later NFs see proto 50, ports 0
            } else if ((MASK & MASK_LB) && kind == NFC_LB) {
                uint32_t hsh = toeplitz(lb_nib, v);
                uint32_t b = (uint32_t)(((uint64_t)hsh * P.lb.n_backends) >> 32);
                lb_b = b;
                port = __ldg(P.lb.port + b);
                stat_add(P.st_lb + b, 1ull);
            }
            if (dropped) { drop = pos; alive = false; }
        };

        const uint32_t n_pre = has_esp ? P.esp_pos : P.n_nf;
        for (uint32_t pos = 0; pos < n_pre && alive; pos++) run_nf(pos);

        if ((MASK & MASK_IPSEC) && has_esp) {   // uniform across the CTA
            // ---- ESP sequence numbers: per SA, global packet order (decoupled look-back)
            const uint32_t nsa = P.esp.n_sa;
            uint16_t *wcnt = reinterpret_cast<uint16_t *>(smem + L.wcnt);
            uint32_t *pref = reinterpret_cast<uint32_t *>(smem + L.prefix);
            for (uint32_t i = tid; i < NWARP * 256; i += TILE) wcnt[i] = 0;
            uint32_t sa = 0xFFFF;
            if (alive) sa = toeplitz(ms_nib, v) % nsa;
            __syncthreads();
            const uint32_t key = alive ? sa : (0x10000u + lane);
            const uint32_t grp = __match_any_sync(0xFFFFFFFFu, key);
            const uint32_t rank = __popc(grp & ((1u << lane) - 1));
            if (alive && rank == 0) wcnt[warp * 256 + sa] = (uint16_t)__popc(grp);
            __syncthreads();
            if (warp == 0) {
                uint32_t *vec = P.tile_vec + (size_t)tile * 2 * nsa;
                for (uint32_t s = lane; s < nsa; s += 32) {
                    uint32_t run = 0;
#pragma unroll
                    for (int w = 0; w < NWARP; w++) { uint32_t c = wcnt[w * 256 + s]; wcnt[w * 256 + s] = (uint16_t)run; run += c; }
                    vec[s] = run;                                   // aggregate
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
            if (alive) {
                esp_sa = sa;
                esp_seq = __ldg(P.seq_in + sa) + pref[sa] + wcnt[warp * 256 + sa] + rank + 1;
                stat_add(P.st_sa + sa, 1ull);
            }
            for (uint32_t pos = P.esp_pos; pos < P.n_nf && alive; pos++) run_nf(pos);
        }

        // ---- result record + counters (warp-aggregated)
        if (valid) {
            if (drop != 0xFF) port = 0xFFFF;
            uint4 rec;
            rec.x = drop | esp_sa << 8 | port << 16;
            rec.y = acl_rule | lb_b << 16;
            rec.z = nmatch | out_len << 16;
            rec.w = esp_seq;
            reinterpret_cast<uint4 *>(P.rec)[g] = rec;
        }
        const uint32_t FULL = 0xFFFFFFFFu;
        const uint32_t b_valid = __ballot_sync(FULL, valid);
        const uint32_t b_parse = __ballot_sync(FULL, valid && drop == 0xFE);
        const uint32_t b_fwd = __ballot_sync(FULL, valid && drop == 0xFF);
        const uint32_t out_bytes = __reduce_add_sync(FULL, (valid && drop == 0xFF) ? out_len : 0u);
        const uint32_t pairs = __reduce_add_sync(FULL, valid ? nmatch : 0u);
        const uint32_t eb = __reduce_add_sync(FULL, esp_sa != 0xFF ? esp_bytes : 0u);
        const uint32_t eblk = __reduce_add_sync(FULL, esp_sa != 0xFF ? (esp_bytes + 15) >> 4 : 0u);
        const uint32_t ep = __ballot_sync(FULL, esp_sa != 0xFF);
        uint32_t pos_cnt[NFC_MAX_CHAIN][3];
#pragma unroll
        for (int p = 0; p < NFC_MAX_CHAIN; p++) {
            const bool reached = valid && drop != 0xFE && (drop == 0xFF || drop >= (uint32_t)p);
            pos_cnt[p][0] = __popc(__ballot_sync(FULL, reached));
            pos_cnt[p][1] = __popc(__ballot_sync(FULL, valid && drop == (uint32_t)p));
            pos_cnt[p][2] = __popc(__ballot_sync(FULL, reached && ((passmask >> p) & 1)));
        }
        if (lane == 0) {
            const uint32_t nv = __popc(b_valid);
            if (nv) {
                atomicAdd(&sst[ST_PKTS], (unsigned long long)nv);
                atomicAdd(&sst[ST_FWD], (unsigned long long)__popc(b_fwd));
                atomicAdd(&sst[ST_DROP], (unsigned long long)(nv - __popc(b_fwd)));
                atomicAdd(&sst[ST_PARSE_DROP], (unsigned long long)__popc(b_parse));
                atomicAdd(&sst[ST_BYTES_OUT], (unsigned long long)out_bytes);
                atomicAdd(&sst[ST_DPI_PAIRS], (unsigned long long)pairs);
                if (ep) {
                    atomicAdd(&sst[ST_ESP_PKTS], (unsigned long long)__popc(ep));
                    atomicAdd(&sst[ST_ESP_BYTES], (unsigned long long)eb);
                    atomicAdd(&sst[ST_ESP_BLOCKS], (unsigned long long)eblk);
                }
                for (uint32_t p = 0; p < P.n_nf; p++) {
                    const uint32_t base = ST_POS_BASE + 4 * p;
                    atomicAdd(&sst[base], (unsigned long long)pos_cnt[p][0]);
                    atomicAdd(&sst[base + 1], (unsigned long long)pos_cnt[p][1]);
                    atomicAdd(&sst[base + 2], (unsigned long long)pos_cnt[p][2]);
                    atomicAdd(&sst[base + 3], (unsigned long long)(pos_cnt[p][0] - pos_cnt[p][1] - pos_cnt[p][2]));
                }
            }
        }
        // bytes_in: original frame length (before ESP growth)
        {
            uint32_t orig = 0;
            if (valid) {
                const BatchDev &B = P.batches[bi];
                orig = B.len[g - B.start];
            }
            const uint32_t bi_sum = __reduce_add_sync(FULL, orig);
            if (lane == 0 && bi_sum) atomicAdd(&sst[ST_BYTES_IN], (unsigned long long)bi_sum);
        }
    }
    // ---- flush CTA counters
    __syncthreads();
    for (uint32_t i = tid; i < n_sst; i += TILE)
        if (sst[i]) atomicAdd(&P.stats[i], sst[i]);
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
