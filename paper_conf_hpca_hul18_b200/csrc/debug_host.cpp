// debug_host.cpp -- include/nfc_debug.h: the device table images walked on the
// host with the kernel's algorithms, so the builders can be checked without a
// GPU.  Diagnostics only; not on the packet path.
#include <algorithm>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "../../include/nfc_debug.h"
#include "nfc_internal.h"

using namespace nfc;

struct nfc_dbg {
    uint32_t kind = 0;
    std::vector<uint32_t> r4, r6;
    uint32_t n_rules = 0, default_action = 0;
    DpiHost dpi;
    std::vector<uint16_t> tbl24, tbllong;
    std::vector<uint2> nh, pmac;
    Lpm6Host l6;
    NatHost nat;
    // the fused kernel's IPv4 search image (AclImg::f4) and 16-bit first level (AclImg::x4)
    std::vector<uint32_t> f4;
    uint32_t f4_key[4] = {0}, f4_bv[4] = {0}, f4_d3 = 0;
    std::vector<uint16_t> x4;
    uint32_t d16 = 0;
};

static inline uint32_t be32(const uint8_t *p) { return (uint32_t)p[0] << 24 | (uint32_t)p[1] << 16 | (uint32_t)p[2] << 8 | p[3]; }
static inline uint32_t m32(int len) { return len <= 0 ? 0u : len >= 32 ? 0xFFFFFFFFu : 0xFFFFFFFFu << (32 - len); }

extern "C" {

int nfc_dbg_build(uint32_t kind, const void *spec, size_t spec_bytes, nfc_dbg **out)
{
    if (!spec || !out) return NFC_EINVAL;
    nfc_dbg *d = new (std::nothrow) nfc_dbg();
    if (!d) return NFC_ENOMEM;
    d->kind = kind;
    std::string err = "bad kind";
    switch (kind) {
    case NFC_ACL:
        if (spec_bytes != sizeof(nfc_acl_spec)) break;
        err = build_acl(*static_cast<const nfc_acl_spec *>(spec), d->r4, d->r6);
        d->n_rules = static_cast<const nfc_acl_spec *>(spec)->n_rules;
        d->default_action = static_cast<const nfc_acl_spec *>(spec)->default_action;
        if (err.empty()) {
            build_acl4_fast(d->r4, d->f4, d->f4_key, d->f4_bv, d->f4_d3);
            build_acl4_index(d->r4, d->x4, d->d16);
        }
        break;
    case NFC_DPI:
        if (spec_bytes != sizeof(nfc_dpi_spec)) break;
        err = build_dpi(*static_cast<const nfc_dpi_spec *>(spec), d->dpi);
        break;
    case NFC_LPM4:
        if (spec_bytes != sizeof(nfc_lpm4_spec)) break;
        err = build_lpm4(*static_cast<const nfc_lpm4_spec *>(spec), d->tbl24, d->tbllong, d->nh, d->pmac);
        break;
    case NFC_LPM6:
        if (spec_bytes != sizeof(nfc_lpm6_spec)) break;
        err = build_lpm6(*static_cast<const nfc_lpm6_spec *>(spec), d->l6);
        break;
    case NFC_NAT:
        if (spec_bytes != sizeof(nfc_nat_spec)) break;
        err = build_nat(*static_cast<const nfc_nat_spec *>(spec), d->nat);
        break;
    }
    if (!err.empty()) {
        delete d;
        return NFC_EINVAL;
    }
    *out = d;
    return NFC_OK;
}

void nfc_dbg_destroy(nfc_dbg *d) { delete d; }

int nfc_dbg_dpi_shape(nfc_dbg *d, uint32_t *n_states, uint32_t *n_classes, uint32_t *wide)
{
    if (!d || d->kind != NFC_DPI) return NFC_EINVAL;
    *n_states = d->dpi.n_states;
    *n_classes = d->dpi.ncls;
    *wide = d->dpi.wide;
    return NFC_OK;
}

int nfc_dbg_dpi(nfc_dbg *d, const uint8_t *buf, size_t n, uint16_t *ids, uint32_t cap, uint32_t *count,
                uint32_t *drop)
{
    if (!d || d->kind != NFC_DPI) return NFC_EINVAL;
    const DpiHost &D = d->dpi;
    std::vector<uint8_t> seen(D.action.size(), 0);
    std::vector<uint16_t> got;
    uint32_t s = 0, dr = 0;
    for (size_t i = 0; i < n; i++) {
        uint32_t c = D.cls[buf[i]], e;
        bool acc;
        if (D.wide) { uint32_t x; memcpy(&x, &D.trans[((size_t)s * D.ncls + c) * 4], 4); acc = x >> 31; e = x & 0x7FFFFFFFu; }
        else { uint16_t x; memcpy(&x, &D.trans[((size_t)s * D.ncls + c) * 2], 2); acc = x >> 15; e = x & 0x7FFFu; }
        s = e;
        if (acc)
            for (uint32_t k = D.out_off[s]; k < D.out_off[s + 1]; k++) {
                uint16_t id = D.out_ids[k];
                dr |= D.action[id];
                if (!seen[id]) { seen[id] = 1; got.push_back(id); }
            }
    }
    std::sort(got.begin(), got.end());
    for (uint32_t k = 0; k < got.size() && k < cap; k++) ids[k] = got[k];
    *count = (uint32_t)got.size();
    *drop = dr;
    return NFC_OK;
}

int nfc_dbg_dpi_tier(nfc_dbg *d, uint32_t hot, uint32_t sparse, const uint8_t *buf, size_t n, uint16_t *ids,
                     uint32_t cap, uint32_t *count, uint32_t *drop, uint32_t *tier_steps)
{
    if (!d || d->kind != NFC_DPI) return NFC_EINVAL;
    const DpiHost &D = d->dpi;
    if (D.wide || hot == 0 || hot > D.n_states) return NFC_EINVAL;
    std::vector<uint8_t> seen(D.action.size(), 0);
    std::vector<uint16_t> got;
    uint32_t s = 0, dr = 0, ts[3] = {0, 0, 0};
    auto row = [&](uint32_t st, uint32_t c) {
        uint16_t x;
        memcpy(&x, &D.trans[((size_t)st * D.ncls + c) * 2], 2);
        return (uint32_t)x;
    };
    for (size_t i = 0; i < n; i++) {
        // the kernel's DM_HOT step (sfc_kernel.cuh dfa_entry): dense / sparse / cold
        const uint32_t c = D.cls[buf[i]];
        const bool sp = s >= hot;
        uint32_t rx = 0xFFFFFFFFu, ry = 0;
        if (sp && s - hot < sparse) { rx = D.sparse[s].x; ry = D.sparse[s].y; }
        const uint32_t b = sp ? (rx & 0xFFFF) : s;
        uint32_t e = b < hot ? row(b, c) : 0;
        if (sp && c == ((rx >> 16) & 0xFF)) e = ry & 0xFFFF;
        if (sp && c == (rx >> 24)) e = ry >> 16;
        if (b >= hot) e = row(s, c);
        ts[b >= hot ? 2 : sp ? 1 : 0]++;
        s = e & 0x7FFF;
        if (e >> 15)
            for (uint32_t k = D.out_off[s]; k < D.out_off[s + 1]; k++) {
                uint16_t id = D.out_ids[k];
                dr |= D.action[id];
                if (!seen[id]) { seen[id] = 1; got.push_back(id); }
            }
    }
    std::sort(got.begin(), got.end());
    for (uint32_t k = 0; k < got.size() && k < cap; k++) ids[k] = got[k];
    *count = (uint32_t)got.size();
    *drop = dr;
    if (tier_steps) memcpy(tier_steps, ts, sizeof(ts));
    return NFC_OK;
}

int nfc_dbg_dpi_slot(nfc_dbg *d, const uint8_t *buf, size_t n, uint16_t *ids, uint32_t cap, uint32_t *count,
                     uint32_t *drop, uint32_t *events, uint32_t *summary)
{
    if (!d || d->kind != NFC_DPI) return NFC_EINVAL;
    const DpiHost &D = d->dpi;
    if (D.wide || D.frows.empty()) return NFC_EINVAL;
    std::vector<uint8_t> seen(D.action.size(), 0);
    std::vector<uint16_t> got;
    uint32_t s = 0, dr = 0, cnt = 0, mx = 0;
    for (size_t i = 0; i < n; i++) {
        // the kernel's DM_FULL step (sfc_kernel.cuh dfa_entry / dfa_step): the row of slot
        // s is physical row n_acc + s; the entry is the next slot, sign-extended
        const int32_t e = D.frows[(size_t)((int32_t)D.n_acc + (int32_t)s) * D.ncls + D.cls[buf[i]]];
        s = (uint32_t)e;
        cnt += s >> 31;
        mx = std::max(mx, s);
        if (e < 0) {
            const uint32_t st = D.acc_id[~s];
            for (uint32_t k = D.out_off[st]; k < D.out_off[st + 1]; k++) {
                uint16_t id = D.out_ids[k];
                dr |= D.action[id];
                if (!seen[id]) { seen[id] = 1; got.push_back(id); }
            }
        }
    }
    std::sort(got.begin(), got.end());
    for (uint32_t k = 0; k < got.size() && k < cap; k++) ids[k] = got[k];
    *count = (uint32_t)got.size();
    *drop = dr;
    if (events) *events = cnt;
    // the kernel's single-accept summary: acc_meta[~mx] (0 without exactly one event)
    if (summary) *summary = cnt == 1 ? D.acc_meta[~mx] : 0u;
    return NFC_OK;
}

int nfc_dbg_dpi_tier_shape(nfc_dbg *d, uint32_t *n_d1, uint32_t *n_sparse_ok)
{
    if (!d || d->kind != NFC_DPI) return NFC_EINVAL;
    *n_d1 = d->dpi.n_d1;
    uint32_t k = 0;
    for (size_t s = d->dpi.n_d1; s < d->dpi.sparse.size(); s++) k += (d->dpi.sparse[s].x & 0xFFFF) != 0xFFFF;
    *n_sparse_ok = k;
    return NFC_OK;
}

int nfc_dbg_lpm4(nfc_dbg *d, uint32_t dst, uint32_t *nh, uint32_t *reads)
{
    if (!d || d->kind != NFC_LPM4) return NFC_EINVAL;
    uint32_t e = d->tbl24[dst >> 8], r = 1;
    if (e & 0x8000) { e = d->tbllong[((e & 0x7FFF) << 8) + (dst & 0xFF)]; r = 2; }
    *nh = e;
    *reads = r;
    return NFC_OK;
}

int nfc_dbg_lpm6_levels(nfc_dbg *d, uint32_t *n_levels)
{
    if (!d || d->kind != NFC_LPM6) return NFC_EINVAL;
    *n_levels = (uint32_t)d->l6.lens.size();
    return NFC_OK;
}

int nfc_dbg_lpm6(nfc_dbg *d, const uint8_t dst[16], uint32_t *nh, uint32_t *probes, uint32_t *slot_reads)
{
    if (!d || d->kind != NFC_LPM6) return NFC_EINVAL;
    const Lpm6Host &T = d->l6;
    uint32_t w[4] = {be32(dst), be32(dst + 4), be32(dst + 8), be32(dst + 12)};
    uint32_t best = T.def_nh, pr = 0, sr = 0;
    int lo = 0, hi = (int)T.lens.size() - 1;
    while (lo <= hi) {
        int mid = (lo + hi) >> 1, L = T.lens[mid];
        uint32_t k[4] = {w[0] & m32(L), w[1] & m32(L - 32), w[2] & m32(L - 64), w[3] & m32(L - 96)};
        uint32_t m = T.mask[mid], h = l6_hash(k[0], k[1], k[2], k[3]) & m;
        pr++;
        bool found = false;
        uint32_t info = 0;
        for (;;) {
            const Lpm6Entry &e = T.ent[T.base[mid] + h];
            sr++;
            if (!(e.info & L6_VALID)) break;
            if (!memcmp(e.key, k, 16)) { found = true; info = e.info; break; }
            h = (h + 1) & m;
        }
        if (found) {
            if ((info & 0xFFFF) != 0x7FFF) best = info & 0xFFFF;
            lo = mid + 1;
        } else {
            hi = mid - 1;
        }
    }
    *nh = best;
    *probes = pr;
    *slot_reads = sr;
    return NFC_OK;
}

// the kernel's fixed-depth window search (sfc_kernel.cu iv_search): `st` halvings from
// the bucket start, clamped to the last real interval
static uint32_t bs32(const uint32_t *B, uint32_t lo, uint32_t st, uint32_t m, uint32_t key)
{
    for (uint32_t h = (1u << st) >> 1; h; h >>= 1) if (B[lo + h] <= key) lo += h;
    return std::min(lo, m - 1);
}
static bool le128h(const uint32_t *b, const uint32_t *k)
{
    for (int q = 0; q < 3; q++) if (b[q] != k[q]) return b[q] < k[q];
    return b[3] <= k[3];
}
static uint32_t bs128(const uint32_t *B, uint32_t lo, uint32_t st, uint32_t m, const uint32_t *k)
{
    for (uint32_t h = (1u << st) >> 1; h; h >>= 1) if (le128h(B + 4 * (lo + h), k)) lo += h;
    return std::min(lo, m - 1);
}

int nfc_dbg_acl(nfc_dbg *d, uint32_t family, const uint8_t *src, const uint8_t *dst, uint16_t sport,
                uint16_t dport, uint8_t proto, uint32_t *rule, uint32_t *action)
{
    if (!d || d->kind != NFC_ACL) return NFC_EINVAL;
    const uint32_t *A = family == 4 ? d->r4.data() : d->r6.data();
    *rule = 0xFFFF;
    *action = d->default_action;
    if (A[0] == 0) return NFC_OK;
    uint32_t s[4], t[4];
    int nb = family == 4 ? 1 : 4;
    for (int k = 0; k < nb; k++) { s[k] = be32(src + 4 * k); t[k] = be32(dst + 4 * k); }
    const uint32_t W = A[1];
    auto iv32 = [&](int q, uint32_t key, int kbits) {
        return bs32(A + A[8 + 2 * q], reinterpret_cast<const uint16_t *>(A + A[18 + q])[key >> (kbits - 8)], A[23], A[2 + q], key);
    };
    auto iv128 = [&](int q, const uint32_t *k) {
        return bs128(A + A[8 + 2 * q], reinterpret_cast<const uint16_t *>(A + A[18 + q])[k[0] >> 24], A[23], A[2 + q], k);
    };
    uint32_t js = nb == 1 ? iv32(0, s[0], 32) : iv128(0, s);
    uint32_t jd = nb == 1 ? iv32(1, t[0], 32) : iv128(1, t);
    uint32_t jsp = iv32(2, sport, 16), jdp = iv32(3, dport, 16);
    auto bv = [&](uint32_t off, uint32_t j, uint32_t w) {
        uint64_t x;
        memcpy(&x, A + off + 2 * ((size_t)j * W + w), 8);
        return x;
    };
    // as the kernel (acl_match_w): W == 1 directly, else candidate words from the
    // aggregate rows (ABV) in increasing order
    const uint32_t WA = A[29];
    for (uint32_t a = 0; a < (W == 1 ? 1u : WA); a++) {
        uint64_t cand = 1;
        if (W > 1) {   // aggregate rows: WA words per row
            auto ag = [&](uint32_t off, uint32_t j) { uint64_t x; memcpy(&x, A + off + 2 * ((size_t)j * WA + a), 8); return x; };
            cand = ag(A[24], js) & ag(A[25], jd) & ag(A[26], jsp) & ag(A[27], jdp) & ag(A[28], proto);
        }
        while (cand) {
            const uint32_t w = 64 * a + __builtin_ctzll(cand);
            uint64_t x = bv(A[9], js, w) & bv(A[11], jd, w) & bv(A[13], jsp, w) & bv(A[15], jdp, w) & bv(A[16], proto, w);
            if (x) {
                uint32_t e = A[A[17] + 64 * w + __builtin_ctzll(x)];
                *rule = e & 0xFFFF;
                *action = e >> 31;
                return NFC_OK;
            }
            cand &= cand - 1;
        }
    }
    return NFC_OK;
}

// IPv4 lookups through the fused kernel's other ACL images, as the kernel does them:
// which = 0: the search image (acl4_fast: bucket on the top NFC_ACLF_BITS bits, two or
// three halvings over the padded keys, bitsets at the affine image of the key address);
// which = 1: the 16-bit first level (acl_core's x4 path: per-prefix / per-port interval,
// d16 halvings for the addresses), then the bit-vector match.  NFC_EUNSUP if the rule
// set has no such image.
int nfc_dbg_acl4_image(nfc_dbg *d, uint32_t which, uint32_t src, uint32_t dst, uint16_t sport, uint16_t dport,
                       uint8_t proto, uint32_t *rule, uint32_t *action)
{
    if (!d || d->kind != NFC_ACL || !rule || !action) return NFC_EINVAL;
    const uint32_t *A = d->r4.data();
    if (which == 0) {
        if (d->f4.empty()) return NFC_EUNSUP;
        const uint8_t *F = reinterpret_cast<const uint8_t *>(d->f4.data());
        auto u16 = [&](uint32_t o) { uint16_t v; memcpy(&v, F + o, 2); return (uint32_t)v; };
        auto u32 = [&](uint32_t o) { uint32_t v; memcpy(&v, F + o, 4); return v; };
        const uint32_t key[4] = {src, dst, sport, dport};
        uint64_t x = 0;
        memcpy(&x, F + ACLF_PROTO + 8 * proto, 8);
        for (int q = 0; q < 4; q++) {
            const uint32_t kb = q < 2 ? 32 : 16;
            uint32_t a = u16(ACLF_BK + 2 * ACLF_NB * q + 2 * (key[q] >> (kb - NFC_ACLF_BITS)));   // key byte offset
            if (d->f4_d3) a += u32(a + 16) <= key[q] ? 16 : 0;
            a += u32(a + 8) <= key[q] ? 8 : 0;
            a += u32(a + 4) <= key[q] ? 4 : 0;
            uint64_t bv;
            memcpy(&bv, F + d->f4_bv[q] + 2 * (a - d->f4_key[q]), 8);
            x &= bv;
        }
        *rule = 0xFFFF;
        *action = d->default_action;
        if (x) {
            const uint32_t e = u32(ACLF_RULE + 4 * (uint32_t)__builtin_ctzll(x));
            *rule = e & 0xFFFF;
            *action = e >> 31;
        }
        return NFC_OK;
    }
    if (d->x4.empty()) return NFC_EUNSUP;
    uint32_t js = d->x4[src >> 16], jd = d->x4[65536 + (dst >> 16)];
    const uint32_t jsp = d->x4[131072 + sport], jdp = d->x4[196608 + dport];
    for (int i = (int)(d->d16 & 255) - 1; i >= 0; i--) js += A[A[8] + js + (1u << i)] <= src ? 1u << i : 0u;
    for (int i = (int)(d->d16 >> 8) - 1; i >= 0; i--) jd += A[A[10] + jd + (1u << i)] <= dst ? 1u << i : 0u;
    js = std::min(js, A[2] - 1);
    jd = std::min(jd, A[3] - 1);
    const uint32_t W = A[1], WA = A[29];
    auto row = [&](uint32_t off, uint32_t j, uint32_t w, uint32_t stride) { uint64_t v; memcpy(&v, A + off + 2 * ((size_t)j * stride + w), 8); return v; };
    *rule = 0xFFFF;
    *action = d->default_action;
    for (uint32_t a = 0; a < WA; a++) {
        uint64_t cand = row(A[24], js, a, WA) & row(A[25], jd, a, WA) & row(A[26], jsp, a, WA) & row(A[27], jdp, a, WA) &
                        row(A[28], proto, a, WA);
        while (cand) {
            const uint32_t w = 64 * a + (uint32_t)__builtin_ctzll(cand);
            const uint64_t x = row(A[9], js, w, W) & row(A[11], jd, w, W) & row(A[13], jsp, w, W) & row(A[15], jdp, w, W) &
                               row(A[16], proto, w, W);
            if (x) {
                const uint32_t e = A[A[17] + 64 * w + (uint32_t)__builtin_ctzll(x)];
                *rule = e & 0xFFFF;
                *action = e >> 31;
                return NFC_OK;
            }
            cand &= cand - 1;
        }
    }
    return NFC_OK;
}

int nfc_dbg_aes128_block(const uint8_t key[16], const uint8_t in[16], uint8_t out[16])
{
    std::vector<uint32_t> te;
    build_aes_tables(te);
    uint32_t rk[44];
    aes_expand(key, rk);
    const uint32_t *T0 = &te[0], *T1 = &te[256], *T2 = &te[512], *T3 = &te[768], *S = &te[1024];
    uint32_t s0 = be32(in) ^ rk[0], s1 = be32(in + 4) ^ rk[1], s2 = be32(in + 8) ^ rk[2], s3 = be32(in + 12) ^ rk[3];
    for (int r = 1; r < 10; r++) {
        uint32_t t0 = T0[s0 >> 24] ^ T1[(s1 >> 16) & 255] ^ T2[(s2 >> 8) & 255] ^ T3[s3 & 255] ^ rk[4 * r];
        uint32_t t1 = T0[s1 >> 24] ^ T1[(s2 >> 16) & 255] ^ T2[(s3 >> 8) & 255] ^ T3[s0 & 255] ^ rk[4 * r + 1];
        uint32_t t2 = T0[s2 >> 24] ^ T1[(s3 >> 16) & 255] ^ T2[(s0 >> 8) & 255] ^ T3[s1 & 255] ^ rk[4 * r + 2];
        uint32_t t3 = T0[s3 >> 24] ^ T1[(s0 >> 16) & 255] ^ T2[(s1 >> 8) & 255] ^ T3[s2 & 255] ^ rk[4 * r + 3];
        s0 = t0; s1 = t1; s2 = t2; s3 = t3;
    }
    uint32_t o[4];
    o[0] = (S[s0 >> 24] << 24 | S[(s1 >> 16) & 255] << 16 | S[(s2 >> 8) & 255] << 8 | S[s3 & 255]) ^ rk[40];
    o[1] = (S[s1 >> 24] << 24 | S[(s2 >> 16) & 255] << 16 | S[(s3 >> 8) & 255] << 8 | S[s0 & 255]) ^ rk[41];
    o[2] = (S[s2 >> 24] << 24 | S[(s3 >> 16) & 255] << 16 | S[(s0 >> 8) & 255] << 8 | S[s1 & 255]) ^ rk[42];
    o[3] = (S[s3 >> 24] << 24 | S[(s0 >> 16) & 255] << 16 | S[(s1 >> 8) & 255] << 8 | S[s2 & 255]) ^ rk[43];
    for (int i = 0; i < 4; i++) {
        out[4 * i] = (uint8_t)(o[i] >> 24); out[4 * i + 1] = (uint8_t)(o[i] >> 16);
        out[4 * i + 2] = (uint8_t)(o[i] >> 8); out[4 * i + 3] = (uint8_t)o[i];
    }
    return NFC_OK;
}

int nfc_dbg_toeplitz(const uint8_t key[40], const uint8_t *in, size_t n, uint32_t *h)
{
    if (n > 36) return NFC_EINVAL;
    std::vector<uint32_t> nib;
    build_toeplitz_nibbles(key, nib);
    uint32_t x = 0;
    for (size_t i = 0; i < n; i++) x ^= nib[(2 * i) * 16 + (in[i] >> 4)] ^ nib[(2 * i + 1) * 16 + (in[i] & 15)];
    *h = x;
    return NFC_OK;
}

int nfc_dbg_nat(nfc_dbg *d, uint8_t proto, uint32_t src, uint32_t dst, uint16_t sport, uint16_t dport, uint16_t ck,
                uint32_t out[5], uint32_t *probes)
{
    if (!d || d->kind != NFC_NAT || !out) return NFC_EINVAL;
    const NatHost &N = d->nat;
    // the kernel's nat_values (sfc_kernel.cuh): Toeplitz over src|dst|sport|dport by the
    // nibble tables, DNAT open-addressing probe, SNAT by the inside prefixes, RFC 1624
    uint8_t t[12];
    for (int k = 0; k < 4; k++) { t[k] = (uint8_t)(src >> (24 - 8 * k)); t[4 + k] = (uint8_t)(dst >> (24 - 8 * k)); }
    t[8] = (uint8_t)(sport >> 8); t[9] = (uint8_t)sport; t[10] = (uint8_t)(dport >> 8); t[11] = (uint8_t)dport;
    uint32_t h = 0;
    for (int i = 0; i < 12; i++) h ^= N.nib[(2 * i) * 16 + (t[i] >> 4)] ^ N.nib[(2 * i + 1) * 16 + (t[i] & 15)];
    uint32_t nsrc = src, ndst = dst, nsp = sport, ndp = dport, np = 0;
    const uint32_t key1 = (uint32_t)dport | (uint32_t)proto << 16;
    for (uint32_t slot = nat_slot(dst, key1) & N.img.dnat_mask;; slot = (slot + 1) & N.img.dnat_mask) {
        np++;
        const uint4 e = N.dnat[slot];
        if (!(e.y & NAT_VALID)) break;
        if (e.x == dst && (e.y & 0xFFFFFF) == key1) { ndst = e.z; ndp = e.w; break; }
    }
    for (uint32_t q = 0; q < N.img.n_inside; q++)
        if ((src & N.img.in_mask[q]) == N.img.in_pref[q]) {
            nsrc = N.pool[(h & 0xFFFF) % N.img.n_pool];
            nsp = N.img.port_lo + (h >> 16) % N.img.port_range;
            break;
        }
    uint32_t c = ck;
    if (!(proto == 17 && c == 0)) {
        auto upd = [](uint32_t hc, uint32_t m, uint32_t m1) {
            auto add = [](uint32_t a, uint32_t b) { uint32_t x = a + b; return (x & 0xFFFF) + (x >> 16); };
            return m == m1 ? hc : (~add(add(~hc & 0xFFFF, ~m & 0xFFFF), m1) & 0xFFFF);
        };
        c = upd(c, src >> 16, nsrc >> 16);
        c = upd(c, src & 0xFFFF, nsrc & 0xFFFF);
        c = upd(c, dst >> 16, ndst >> 16);
        c = upd(c, dst & 0xFFFF, ndst & 0xFFFF);
        c = upd(c, sport, nsp);
        c = upd(c, dport, ndp);
        if (proto == 17 && c == 0) c = 0xFFFF;
    }
    out[0] = nsrc; out[1] = ndst; out[2] = nsp; out[3] = ndp; out[4] = c;
    if (probes) *probes = np;
    return NFC_OK;
}

int nfc_dbg_hmac_sha1(const uint8_t key[20], const uint8_t *msg, size_t n, uint8_t out[20])
{
    nfc_sa sa{};
    memcpy(sa.auth_key, key, 20);
    nfc_ipsec_spec spec{1, &sa};
    std::vector<EspSa> v;
    if (!build_ipsec(spec, v).empty()) return NFC_EINVAL;
    // inner: ipad state, then msg with padding counting the 64-B ipad block
    uint32_t h[5];
    memcpy(h, v[0].ipad, 20);
    std::vector<uint8_t> m(msg, msg + n);
    m.push_back(0x80);
    while ((m.size() % 64) != 56) m.push_back(0);
    uint64_t bits = (uint64_t)(64 + n) * 8;
    for (int i = 7; i >= 0; i--) m.push_back((uint8_t)(bits >> (8 * i)));
    for (size_t b = 0; b < m.size(); b += 64) sha1_compress(h, &m[b]);
    uint8_t blk[64] = {0};
    for (int i = 0; i < 5; i++) { blk[4 * i] = (uint8_t)(h[i] >> 24); blk[4 * i + 1] = (uint8_t)(h[i] >> 16); blk[4 * i + 2] = (uint8_t)(h[i] >> 8); blk[4 * i + 3] = (uint8_t)h[i]; }
    blk[20] = 0x80;
    uint64_t ob = (64 + 20) * 8;
    for (int i = 0; i < 8; i++) blk[63 - i] = (uint8_t)(ob >> (8 * i));
    uint32_t g[5];
    memcpy(g, v[0].opad, 20);
    sha1_compress(g, blk);
    for (int i = 0; i < 5; i++) { out[4 * i] = (uint8_t)(g[i] >> 24); out[4 * i + 1] = (uint8_t)(g[i] >> 16); out[4 * i + 2] = (uint8_t)(g[i] >> 8); out[4 * i + 3] = (uint8_t)g[i]; }
    return NFC_OK;
}

} // extern "C"
