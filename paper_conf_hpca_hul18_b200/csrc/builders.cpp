// builders.cpp -- host-side table builders: logical specs -> device images.
//
// ACL, Aho-Corasick DFA, IPv4 DIR-24-8
// ("two memory accesses"), IPv6 binary search on prefix lengths over
// per-length hash tables ("hashing ... binary search ... up to 7 memory
// lookups"), AES-128 key schedule + T-tables and HMAC-SHA1 ipad/opad
// precompute, Toeplitz nibble tables for the RSS / LB flow hash
// (P:L87).  Product code: independent of oracle/.
#include <algorithm>
#include <array>
#include <cstring>
#include <map>
#include <unordered_map>

#include "nfc_internal.h"

namespace nfc {

const uint8_t MS_RSS_KEY[40] = {0x6d, 0x5a, 0x56, 0xda, 0x25, 0x5b, 0x0e, 0xc2, 0x41, 0x67,
                                0x25, 0x3d, 0x43, 0xa3, 0x8f, 0xb0, 0xd0, 0xca, 0x2b, 0xcb,
                                0xae, 0x7b, 0x30, 0xb4, 0x77, 0xcb, 0x2d, 0xa3, 0x80, 0x30,
                                0xf2, 0x0c, 0x6a, 0x42, 0xb7, 0x3b, 0xbe, 0xac, 0x01, 0xfa};

static inline uint32_t be32(const uint8_t *p) { return (uint32_t)p[0] << 24 | (uint32_t)p[1] << 16 | (uint32_t)p[2] << 8 | p[3]; }
static inline uint32_t mask32(int len) { return len <= 0 ? 0u : len >= 32 ? 0xFFFFFFFFu : 0xFFFFFFFFu << (32 - len); }
static void mask128(const uint8_t *a, int len, uint32_t w[4])
{
    for (int k = 0; k < 4; k++) w[k] = be32(a + 4 * k) & mask32(len - 32 * k);
}

// ---------------------------------------------------------------- ACL
// Bit-vector classification (Lakshman & Stiliadis style), one image per address
// family.  Each of the fields src, dst, sport, dport is cut into elementary
// intervals at the rule boundaries; interval j carries the bitset of rules whose
// range contains it; proto has a direct 256-entry bitset table.  The lookup ANDs
// the five bitsets and takes the lowest set bit = the first matching rule.
// Blob layout (u32 words): see AclBv in nfc_internal.h.
namespace {
typedef unsigned __int128 u128;
static u128 key128(const uint8_t *a)
{
    u128 k = 0;
    for (int i = 0; i < 16; i++) k = (k << 8) | a[i];
    return k;
}
static u128 mask128v(int len) { return len <= 0 ? (u128)0 : len >= 128 ? ~(u128)0 : ~(u128)0 << (128 - len); }

struct FieldIv {
    std::vector<u128> b;                  // interval starts, b[0] = 0
    std::vector<uint64_t> bv;             // b.size() x W words
};

static void build_field(const std::vector<std::pair<u128, u128>> &rng, u128 maxv, uint32_t W, FieldIv &f)
{
    std::vector<u128> pts{0};
    for (auto &r : rng) {
        pts.push_back(r.first);
        if (r.second != maxv) pts.push_back(r.second + 1);
    }
    std::sort(pts.begin(), pts.end());
    pts.erase(std::unique(pts.begin(), pts.end()), pts.end());
    f.b = pts;
    f.bv.assign(pts.size() * W, 0);
    for (size_t r = 0; r < rng.size(); r++) {
        size_t j0 = std::lower_bound(pts.begin(), pts.end(), rng[r].first) - pts.begin();
        for (size_t j = j0; j < pts.size() && pts[j] <= rng[r].second; j++) f.bv[j * W + r / 64] |= 1ull << (r % 64);
    }
}
} // namespace

std::string build_acl(const nfc_acl_spec &s, std::vector<uint32_t> &blob4, std::vector<uint32_t> &blob6)
{
    if (s.n_rules > 32767) return "acl: too many rules (max 32767)";
    if (s.n_rules && !s.rules) return "acl: rules == NULL";
    if (s.default_action > 1) return "acl: default_action must be 0 or 1";
    for (uint32_t i = 0; i < s.n_rules; i++) {
        const nfc_acl_rule &r = s.rules[i];
        int maxl = r.family == 4 ? 32 : 128;
        if (r.family != 4 && r.family != 6) return "acl: family must be 4 or 6";
        if (r.slen > maxl || r.dlen > maxl) return "acl: prefix length out of range";
        if (r.sp_lo > r.sp_hi || r.dp_lo > r.dp_hi) return "acl: port range lo > hi";
        if (r.action > 1 || r.proto_any > 1) return "acl: bad action/proto_any";
    }
    for (int fam : {4, 6}) {
        std::vector<uint32_t> &blob = fam == 4 ? blob4 : blob6;
        std::vector<uint32_t> gidx;
        for (uint32_t i = 0; i < s.n_rules; i++)
            if (s.rules[i].family == fam) gidx.push_back(i);
        const uint32_t n = (uint32_t)gidx.size(), W = (n + 63) / 64, kw = fam == 4 ? 1 : 4;
        const int bits = fam == 4 ? 32 : 128;
        const u128 amax = fam == 4 ? (u128)0xFFFFFFFFu : ~(u128)0;
        std::vector<std::pair<u128, u128>> rs, rd, rsp, rdp;
        for (uint32_t g : gidx) {
            const nfc_acl_rule &r = s.rules[g];
            u128 sk = fam == 4 ? (u128)be32(r.src) : key128(r.src), dk = fam == 4 ? (u128)be32(r.dst) : key128(r.dst);
            u128 sm = mask128v(r.slen) >> (128 - bits), dm = mask128v(r.dlen) >> (128 - bits);
            if (fam == 4) { sm &= 0xFFFFFFFFu; dm &= 0xFFFFFFFFu; }
            rs.push_back({sk & sm, (sk & sm) | (amax & ~sm)});
            rd.push_back({dk & dm, (dk & dm) | (amax & ~dm)});
            rsp.push_back({r.sp_lo, r.sp_hi});
            rdp.push_back({r.dp_lo, r.dp_hi});
        }
        FieldIv F[4];
        build_field(rs, amax, W ? W : 1, F[0]);
        build_field(rd, amax, W ? W : 1, F[1]);
        build_field(rsp, 0xFFFF, W ? W : 1, F[2]);
        build_field(rdp, 0xFFFF, W ? W : 1, F[3]);
        const uint32_t Wd = W ? W : 1;
        std::vector<uint64_t> vproto(256 * Wd, 0);
        for (uint32_t r = 0; r < n; r++) {
            const nfc_acl_rule &ru = s.rules[gidx[r]];
            for (int p = 0; p < 256; p++)
                if (ru.proto_any || ru.proto == p) vproto[p * Wd + r / 64] |= 1ull << (r % 64);
        }
        blob.assign(ACLBV_HDR, 0);
        blob[0] = n; blob[1] = Wd; blob[2] = (uint32_t)F[0].b.size(); blob[3] = (uint32_t)F[1].b.size();
        blob[4] = (uint32_t)F[2].b.size(); blob[5] = (uint32_t)F[3].b.size(); blob[6] = kw;
        auto align_to = [&](size_t a) { while (blob.size() % a) blob.push_back(0); };
        // 257-entry bucket index per field on the top 8 key bits: bucket[t] = interval
        // containing the first key of bucket t; the answer lies in [bk[t], bk[t+1]]
        auto buckets = [&](const FieldIv &f, int kbits) {
            std::vector<uint32_t> bk(257);
            for (int t = 0; t <= 256; t++) {
                u128 first = t == 256 ? (kbits == 128 ? ~(u128)0 : (((u128)1 << kbits) - 1)) : (u128)t << (kbits - 8);
                bk[t] = (uint32_t)(std::upper_bound(f.b.begin(), f.b.end(), first) - f.b.begin() - 1);
            }
            return bk;
        };
        // fixed-depth search: `steps` halvings cover the widest bucket window, so the
        // device loop has a table-wide (warp-uniform) trip count instead of a per-key one
        auto steps_of = [](const std::vector<uint32_t> &bk) {
            uint32_t mmax = 1, st = 0;
            for (int t = 0; t < 256; t++) mmax = std::max(mmax, bk[t + 1] - bk[t] + 1);
            while ((1u << st) < mmax) st++;
            return st;
        };
        const int fbits[4] = {bits, bits, 16, 16};
        std::vector<uint32_t> BK[4];
        uint32_t steps = 0, maxst = 0;
        for (int q = 0; q < 4; q++) {
            BK[q] = buckets(F[q], fbits[q]);
            steps |= steps_of(BK[q]) << (8 * q);
            maxst = std::max(maxst, steps_of(BK[q]));
        }
        // keys (16-B aligned so an IPv6 key is one 128-bit load), followed by 2^maxst
        // all-ones pad keys: the window may run past the last interval start (the kernel
        // runs the four searches jointly for the largest depth)
        auto put_keys = [&](const FieldIv &f, uint32_t kwords, uint32_t) {
            align_to(4);
            uint32_t o = (uint32_t)blob.size();
            for (u128 k : f.b)
                for (int q = (int)kwords - 1; q >= 0; q--) blob.push_back((uint32_t)(k >> (32 * q)));
            for (uint32_t i = 0; i < (1u << maxst) * kwords; i++) blob.push_back(0xFFFFFFFFu);
            return o;
        };
        auto put_bv = [&](const std::vector<uint64_t> &v) {
            align_to(2);
            uint32_t o = (uint32_t)blob.size();
            for (uint64_t x : v) { blob.push_back((uint32_t)x); blob.push_back((uint32_t)(x >> 32)); }
            return o;
        };
        auto put_bk = [&](const std::vector<uint32_t> &bk) {   // 257 u16 (interval indices < 2^16)
            uint32_t o = (uint32_t)blob.size();
            for (int t = 0; t < 258; t += 2) blob.push_back(bk[t] | (t + 1 < 257 ? bk[t + 1] << 16 : 0u));
            return o;
        };
        uint32_t offs[14];
        offs[0] = put_keys(F[0], kw, steps & 255); offs[1] = put_bv(F[0].bv);
        offs[2] = put_keys(F[1], kw, (steps >> 8) & 255); offs[3] = put_bv(F[1].bv);
        offs[4] = put_keys(F[2], 1, (steps >> 16) & 255);  offs[5] = put_bv(F[2].bv);
        offs[6] = put_keys(F[3], 1, steps >> 24);  offs[7] = put_bv(F[3].bv);
        offs[8] = put_bv(vproto);
        offs[9] = (uint32_t)blob.size();
        for (uint32_t r = 0; r < n; r++) blob.push_back(gidx[r] | (uint32_t)s.rules[gidx[r]].action << 31);
        for (int q = 0; q < 4; q++) offs[10 + q] = put_bk(BK[q]);
        blob[22] = steps;
        blob[23] = maxst;
        // aggregate level (ABV, Baboescu & Varghese): per row, bit w of aggregate word
        // w / 64 is set iff the row's bitset word w is non-zero.  The lookup ANDs the
        // five aggregate rows first and examines only the candidate words, in order
        // (first match = lowest rule index), so large rule sets need not scan W words.
        const uint32_t WA = (Wd + 63) / 64;
        auto put_agg = [&](const std::vector<uint64_t> &v) {
            std::vector<uint64_t> ag(v.size() / Wd * WA, 0);
            for (size_t j = 0; j < v.size() / Wd; j++)
                for (uint32_t w = 0; w < Wd; w++)
                    if (v[j * Wd + w]) ag[j * WA + w / 64] |= 1ull << (w % 64);
            return put_bv(ag);
        };
        blob[24] = put_agg(F[0].bv);
        blob[25] = put_agg(F[1].bv);
        blob[26] = put_agg(F[2].bv);
        blob[27] = put_agg(F[3].bv);
        blob[28] = put_agg(vproto);
        blob[29] = WA;
        while (blob.size() & 3) blob.push_back(0);   // 16-B multiple for staging copies
        for (int k = 0; k < 14; k++) blob[8 + k] = offs[k];
    }
    return "";
}

// 16-bit first level of an IPv4 bit-vector blob with W > 32 (> 2K rules; AclImg::x4): per field the
// interval containing each 16-bit key prefix (addresses: then a window search whose
// depth is the widest 16-bit bucket, usually 0-2 halvings instead of 5-7 after the 8-bit
// buckets) or each port (exact: no search).  Empty if the blob does not qualify.
void build_acl4_index(const std::vector<uint32_t> &b, std::vector<uint16_t> &x, uint32_t &d16)
{
    x.clear();
    d16 = 0;
    // (measured: +15 % at 10K rules, -1.5 % at 1K and -13 % at 200 rules, whose images mostly hit in L1)
    if (b.size() < ACLBV_HDR || b[0] == 0 || b[1] <= 32 || b[6] != 1) return;
    x.assign(4 * 65536, 0);
    for (int q = 0; q < 4; q++) {
        const uint32_t m = b[2 + q], *keys = &b[b[8 + 2 * q]];
        if (m > 65535) { x.clear(); d16 = 0; return; }
        uint32_t j = 0, widest = 1;
        for (uint32_t t = 0; t < 65536; t++) {
            const uint32_t first = q < 2 ? t << 16 : t;        // first key of the bucket / the port
            while (j + 1 < m && keys[j + 1] <= first) j++;
            x[q * 65536 + t] = (uint16_t)j;
            if (q < 2) {                                         // the bucket's window [j, j_last]
                const uint32_t last = first | 0xFFFFu;
                uint32_t e = j;
                while (e + 1 < m && keys[e + 1] <= last) e++;
                widest = std::max(widest, e - j + 1);
            }
        }
        if (q < 2) {
            uint32_t st = 0;
            while ((1u << st) < widest) st++;
            if (st > b[23]) st = b[23];   // never wider than the 8-bit buckets' (the key pad covers those)
            d16 |= st << (8 * q);
        }
    }
}

// Search image of an IPv4 bit-vector blob (AclImg::f4 layout, nfc_internal.h): the
// same intervals, bitsets, buckets and rule words, with bucket entries as key addresses
// and pad entries instead of clamps.  Only for W == 1 (<= 64 rules) and window depth
// <= 3: the kernel always takes three halvings (8-key window).  key_off / bv_off
// receive the per-field array offsets.
void build_acl4_fast(const std::vector<uint32_t> &b, std::vector<uint32_t> &f, uint32_t key_off[4], uint32_t bv_off[4],
                     uint32_t &d3)
{
    f.clear();
    d3 = 0;
    if (b.size() < ACLBV_HDR || b[0] == 0 || b[0] > 64 || b[1] != 1 || b[6] != 1) return;
    const uint32_t m[4] = {b[2], b[3], b[4], b[5]};
    // bucket t of a field: the interval of its first key; the window [bk(t), bk(t+1)]
    // (the interval of the bucket's last key) must fit the kernel's 2 or 3 halvings
    std::vector<uint32_t> bk[4];
    uint32_t widest = 1;
    for (int q = 0; q < 4; q++) {
        const uint32_t *keys = &b[b[8 + 2 * q]], kb = q < 2 ? 32 : 16;
        bk[q].resize(ACLF_NB);
        uint32_t j = 0;
        for (uint32_t t = 0; t < ACLF_NB; t++) {
            const uint32_t first = t << (kb - NFC_ACLF_BITS), last = first | ((1u << (kb - NFC_ACLF_BITS)) - 1);
            while (j + 1 < m[q] && keys[j + 1] <= first) j++;
            uint32_t e = j;
            while (e + 1 < m[q] && keys[e + 1] <= last) e++;
            bk[q][t] = j;
            widest = std::max(widest, e - j + 1);
        }
    }
    if (widest > 8) return;           // more than three halvings: the bit-vector blob path
    d3 = widest > 4 ? 1 : 0;
    size_t bytes = ACLF_REC;
    for (int q = 0; q < 4; q++) {
        key_off[q] = (uint32_t)bytes;
        bytes += (4 * (size_t)(m[q] + 8) + 7) & ~(size_t)7;
        bv_off[q] = (uint32_t)bytes;
        bytes += 8 * (size_t)(m[q] + 8);
    }
    bytes = (bytes + 15) & ~(size_t)15;
    if (bytes > 65535) return;   // bucket entries are u16 byte offsets
    f.assign(bytes / 4, 0);
    uint16_t *bkt = reinterpret_cast<uint16_t *>(f.data());
    for (int q = 0; q < 4; q++) {
        const uint32_t keys = b[8 + 2 * q], bv = b[9 + 2 * q];
        for (uint32_t j = 0; j < m[q] + 8; j++) {
            const uint32_t jj = std::min(j, m[q] - 1);   // the pad entries repeat the last one
            f[key_off[q] / 4 + j] = b[keys + jj];
            f[bv_off[q] / 4 + 2 * j] = b[bv + 2 * jj];
            f[bv_off[q] / 4 + 2 * j + 1] = b[bv + 2 * jj + 1];
        }
        for (uint32_t t = 0; t < ACLF_NB; t++) bkt[q * ACLF_NB + t] = (uint16_t)(key_off[q] + 4 * bk[q][t]);
    }
    for (uint32_t i = 0; i < 512; i++) f[ACLF_PROTO / 4 + i] = b[b[16] + i];
    for (uint32_t r = 0; r < b[0]; r++) f[ACLF_RULE / 4 + r] = b[b[17] + r];
}

// ---------------------------------------------------------------- DPI
// Aho-Corasick (1975) goto/failure construction, converted to a full DFA over
// byte classes (bytes that occur in no pattern share one class: from every
// state they lead to the root).
std::string build_dpi(const nfc_dpi_spec &s, DpiHost &o)
{
    if (s.n_patterns == 0 || s.n_patterns > 65535) return "dpi: n_patterns must be 1..65535";
    o.maxlen = 0;
    if (!s.blob || !s.off || !s.action) return "dpi: NULL pointer";
    // byte classes
    std::array<int, 256> cls{};
    cls.fill(0);
    for (uint32_t j = 0; j < s.n_patterns; j++) {
        if (s.off[j + 1] <= s.off[j]) return "dpi: empty pattern";
        if (s.action[j] > 1) return "dpi: action must be 0 or 1";
        o.maxlen = std::max(o.maxlen, s.off[j + 1] - s.off[j]);
        for (uint32_t k = s.off[j]; k < s.off[j + 1]; k++) cls[s.blob[k]] = 1;
    }
    // used bytes get classes 0..u-1; all unused bytes share class u (if any) -> ncls <= 256
    int ncls = 0;
    for (int b = 0; b < 256; b++) if (cls[b]) cls[b] = ++ncls;   // 1-based for now
    const int other = ncls;
    bool any_unused = false;
    for (int b = 0; b < 256; b++) {
        if (cls[b]) cls[b] -= 1;
        else { cls[b] = other; any_unused = true; }
    }
    if (any_unused) ncls++;
    // trie with sparse children
    std::vector<std::vector<std::pair<int, int>>> kids(1);   // (class, child)
    std::vector<std::vector<uint16_t>> own(1);
    for (uint32_t j = 0; j < s.n_patterns; j++) {
        int st = 0;
        for (uint32_t k = s.off[j]; k < s.off[j + 1]; k++) {
            int c = cls[s.blob[k]], nx = -1;
            for (auto &kc : kids[st]) if (kc.first == c) { nx = kc.second; break; }
            if (nx < 0) {
                nx = (int)kids.size();
                kids.emplace_back();
                own.emplace_back();
                kids[st].push_back({c, nx});
            }
            st = nx;
        }
        own[st].push_back((uint16_t)j);
    }
    size_t n = kids.size();
    // BFS renumbering
    std::vector<int> order, newid(n, -1), fail(n, 0);
    order.reserve(n);
    order.push_back(0);
    newid[0] = 0;
    for (size_t h = 0; h < order.size(); h++) {
        int u = order[h];
        std::sort(kids[u].begin(), kids[u].end());
        for (auto &kc : kids[u]) { newid[kc.second] = (int)order.size(); order.push_back(kc.second); }
    }
    // full DFA (old ids) in BFS order
    std::vector<int> delta(n * ncls, 0);
    std::vector<std::vector<uint16_t>> outc(n);
    for (int u : order) {
        int f = fail[u];
        for (int c = 0; c < ncls; c++) delta[(size_t)u * ncls + c] = (u == 0) ? 0 : delta[(size_t)f * ncls + c];
        for (auto &kc : kids[u]) {
            int v = kc.second;
            fail[v] = (u == 0) ? 0 : delta[(size_t)f * ncls + kc.first];
            delta[(size_t)u * ncls + kc.first] = v;
        }
        // output closure: own(u) U out(fail(u)); fail(u) precedes u in BFS order
        std::vector<uint16_t> oc = own[u];
        if (u != 0) oc.insert(oc.end(), outc[fail[u]].begin(), outc[fail[u]].end());
        std::sort(oc.begin(), oc.end());
        oc.erase(std::unique(oc.begin(), oc.end()), oc.end());
        outc[u] = std::move(oc);
    }
    o.ncls = (uint32_t)ncls;
    o.n_states = (uint32_t)n;
    o.wide = n > 32768 ? 1 : 0;
    o.cls.resize(256);
    for (int b = 0; b < 256; b++) o.cls[b] = (uint8_t)cls[b];
    size_t es = o.wide ? 4 : 2;
    o.trans.assign(n * ncls * es, 0);
    for (size_t u = 0; u < n; u++) {
        for (int c = 0; c < ncls; c++) {
            int v = delta[u * ncls + c];
            uint32_t e = (uint32_t)newid[v];
            if (!outc[v].empty()) e |= o.wide ? 0x80000000u : 0x8000u;
            size_t at = ((size_t)newid[u] * ncls + c) * es;
            if (o.wide) memcpy(&o.trans[at], &e, 4);
            else { uint16_t e16 = (uint16_t)e; memcpy(&o.trans[at], &e16, 2); }
        }
    }
    o.out_off.assign(n + 1, 0);
    o.out_ids.clear();
    for (size_t k = 0; k < n; k++) {
        int u = order[k];
        o.out_off[k] = (uint32_t)o.out_ids.size();
        o.out_ids.insert(o.out_ids.end(), outc[u].begin(), outc[u].end());
    }
    o.out_off[n] = (uint32_t)o.out_ids.size();
    if (o.out_ids.empty()) o.out_ids.push_back(0);
    o.action.assign(s.action, s.action + s.n_patterns);
    // tier records (DpiImg::sparse): base = first depth <= 1 state on the failure chain,
    // exceptions = the classes where the row differs from the base row (at most 2)
    {
        std::vector<int> depth(n, 0);
        for (int u : order)
            for (auto &kc : kids[u]) depth[kc.second] = depth[u] + 1;
        uint32_t nd1 = 0;
        for (size_t u = 0; u < n; u++) nd1 += depth[u] <= 1;
        o.n_d1 = nd1;                      // BFS order: exactly the ids [0, nd1)
        o.sparse.assign(n, make_uint2(0xFFFFFFFFu, 0));
        auto entry = [&](int v) {
            uint32_t e = (uint32_t)newid[v];
            if (!outc[v].empty()) e |= 0x8000u;
            return e;
        };
        if (!o.wide) {
            for (int u : order) {
                if (depth[u] <= 1) continue;
                int b = fail[u];
                while (depth[b] > 1) b = fail[b];
                int ex[3], nx = 0;
                for (int c = 0; c < ncls && nx < 3; c++)
                    if (delta[(size_t)u * ncls + c] != delta[(size_t)b * ncls + c]) ex[nx++] = c;
                if (nx > 2) continue;      // cold
                int c0 = nx ? ex[0] : 0, c1 = nx > 1 ? ex[1] : c0;
                uint32_t e0 = entry(delta[(size_t)u * ncls + c0]), e1 = entry(delta[(size_t)u * ncls + c1]);
                o.sparse[newid[u]] = make_uint2((uint32_t)newid[b] | (uint32_t)c0 << 16 | (uint32_t)c1 << 24,
                                                e0 | e1 << 16);
            }
        }
    }
    // per-state match summary for the kernel's single-accept path: closure offset,
    // size and whether any pattern in it is a DROP pattern
    o.out_meta.assign(n, 0);
    for (size_t k = 0; k < n; k++) {
        const uint32_t o0 = o.out_off[k], nm = o.out_off[k + 1] - o0;
        uint32_t drop = 0;
        for (uint32_t x = o0; x < o0 + nm; x++) drop |= o.action[o.out_ids[x]];
        // a one-pattern closure carries the pattern id itself (no CSR read when emitting)
        const uint32_t lo = nm == 1 ? o.out_ids[o0] : o0;
        o.out_meta[k] = (lo < (1u << 20) && nm < 2047u) ? (lo | nm << 20 | drop << 31) : DPI_META_NONE;
    }
    // slot image (DpiImg::frows): non-accepting states 0.., accepting -1.. (BFS order);
    // physical row of slot x = n_acc + x
    o.frows.clear();
    o.acc_id.clear();
    o.acc_meta.clear();
    o.n_acc = 0;
    if (!o.wide) {
        std::vector<int32_t> slot(n);
        int32_t na = 0, nn = 0;
        for (size_t k = 0; k < n; k++) slot[k] = outc[order[k]].empty() ? nn++ : -(++na);
        o.n_acc = (uint32_t)na;
        o.acc_id.assign(na, 0);
        o.acc_meta.assign(na, 0);
        for (size_t k = 0; k < n; k++)
            if (slot[k] < 0) { o.acc_id[-slot[k] - 1] = (uint32_t)k; o.acc_meta[-slot[k] - 1] = o.out_meta[k]; }
        o.frows.assign(n * ncls, 0);
        for (size_t u = 0; u < n; u++) {
            const size_t row = (size_t)(na + slot[newid[u]]);
            for (int c = 0; c < ncls; c++) o.frows[row * ncls + c] = (int16_t)slot[newid[delta[u * ncls + c]]];
        }
    }
    return "";
}

// ---------------------------------------------------------------- next hops
static std::string build_nh(uint32_t n_nh, const nfc_nexthop *nh, uint32_t n_ports, const uint8_t *pm,
                            std::vector<uint2> &dn, std::vector<uint2> &dp)
{
    if (n_nh == 0 || n_nh > 32767 || !nh) return "lpm: n_nexthops must be 1..32767";
    if (n_ports == 0 || !pm) return "lpm: need port MACs";
    dn.resize(n_nh);
    for (uint32_t i = 0; i < n_nh; i++) {
        if (nh[i].port >= n_ports) return "lpm: next hop port >= n_ports";
        const uint8_t *m = nh[i].mac;
        dn[i] = make_uint2((uint32_t)m[0] | (uint32_t)m[1] << 8 | (uint32_t)m[2] << 16 | (uint32_t)m[3] << 24,
                           (uint32_t)m[4] | (uint32_t)m[5] << 8 | (uint32_t)nh[i].port << 16);
    }
    dp.resize(n_ports);
    for (uint32_t p = 0; p < n_ports; p++) {
        const uint8_t *m = pm + 6 * p;
        dp[p] = make_uint2((uint32_t)m[0] | (uint32_t)m[1] << 8 | (uint32_t)m[2] << 16 | (uint32_t)m[3] << 24,
                           (uint32_t)m[4] | (uint32_t)m[5] << 8);
    }
    return "";
}

// ---------------------------------------------------------------- LPM4: DIR-24-8
std::string build_lpm4(const nfc_lpm4_spec &s, std::vector<uint16_t> &tbl24, std::vector<uint16_t> &tbllong,
                       std::vector<uint2> &nh, std::vector<uint2> &pmac)
{
    std::string e = build_nh(s.n_nexthops, s.nexthops, s.n_ports, s.port_macs, nh, pmac);
    if (!e.empty()) return e;
    if (s.n_routes && !s.routes) return "lpm4: routes == NULL";
    std::vector<uint32_t> idx(s.n_routes);
    std::unordered_map<uint64_t, int> seen;
    for (uint32_t i = 0; i < s.n_routes; i++) {
        const nfc_route4 &r = s.routes[i];
        if (r.len > 32) return "lpm4: len > 32";
        if (r.prefix & ~mask32(r.len)) return "lpm4: host bits set in prefix";
        if (r.nh >= s.n_nexthops) return "lpm4: nh out of range";
        if (!seen.emplace((uint64_t)r.prefix << 8 | r.len, 1).second) return "lpm4: duplicate prefix";
        idx[i] = i;
    }
    std::stable_sort(idx.begin(), idx.end(), [&](uint32_t a, uint32_t b) { return s.routes[a].len < s.routes[b].len; });
    tbl24.assign(1u << 24, 0x7FFF);
    tbllong.clear();
    for (uint32_t i : idx) {
        const nfc_route4 &r = s.routes[i];
        if (r.len <= 24) {
            uint32_t first = r.prefix >> 8, cnt = 1u << (24 - r.len);
            for (uint32_t k = 0; k < cnt; k++) tbl24[first + k] = r.nh;
        } else {
            uint32_t t = r.prefix >> 8;
            if (!(tbl24[t] & 0x8000)) {
                uint32_t g = (uint32_t)(tbllong.size() / 256);
                if (g >= 0x8000) return "lpm4: too many /25+ groups";
                tbllong.insert(tbllong.end(), 256, tbl24[t]);
                tbl24[t] = (uint16_t)(0x8000 | g);
            }
            uint32_t g = tbl24[t] & 0x7FFF, first = r.prefix & 0xFF, cnt = 1u << (32 - r.len);
            for (uint32_t k = 0; k < cnt; k++) tbllong[g * 256 + first + k] = r.nh;
        }
    }
    if (tbllong.empty()) tbllong.assign(256, 0x7FFF);
    return "";
}

// ---------------------------------------------------------------- LPM6: Waldvogel
namespace {
struct BitTrie {
    struct N { int c[2]; int nh; };
    std::vector<N> n{N{{-1, -1}, -1}};
    void insert(const uint32_t w[4], int len, int nh)
    {
        int u = 0;
        for (int i = 0; i < len; i++) {
            int b = (w[i >> 5] >> (31 - (i & 31))) & 1;
            if (n[u].c[b] < 0) { n[u].c[b] = (int)n.size(); n.push_back(N{{-1, -1}, -1}); }
            u = n[u].c[b];
        }
        n[u].nh = nh;
    }
    int best(const uint32_t w[4], int len) const  // longest real prefix of length <= len matching w
    {
        int u = 0, b = n[0].nh;
        for (int i = 0; i < len && u >= 0; i++) {
            u = n[u].c[(w[i >> 5] >> (31 - (i & 31))) & 1];
            if (u >= 0 && n[u].nh >= 0) b = n[u].nh;
        }
        return b;
    }
};
struct K4 {
    uint32_t w[4];
    bool operator==(const K4 &o) const { return memcmp(w, o.w, 16) == 0; }
};
struct K4H { size_t operator()(const K4 &k) const { return l6_hash(k.w[0], k.w[1], k.w[2], k.w[3]); } };
} // namespace

std::string build_lpm6(const nfc_lpm6_spec &s, Lpm6Host &o)
{
    std::string e = build_nh(s.n_nexthops, s.nexthops, s.n_ports, s.port_macs, o.nh, o.pmac);
    if (!e.empty()) return e;
    if (s.n_routes && !s.routes) return "lpm6: routes == NULL";
    BitTrie trie;
    std::vector<int> present(129, 0);
    o.def_nh = 0x7FFF;
    std::unordered_map<K4, int, K4H> dup[129];
    for (uint32_t i = 0; i < s.n_routes; i++) {
        const nfc_route6 &r = s.routes[i];
        if (r.len > 128) return "lpm6: len > 128";
        if (r.nh >= s.n_nexthops) return "lpm6: nh out of range";
        K4 k;
        mask128(r.prefix, r.len, k.w);
        for (int q = 0; q < 4; q++)
            if (be32(r.prefix + 4 * q) != k.w[q]) return "lpm6: host bits set in prefix";
        if (!dup[r.len].emplace(k, 1).second) return "lpm6: duplicate prefix";
        trie.insert(k.w, r.len, r.nh);
        present[r.len] = 1;
        if (r.len == 0) o.def_nh = r.nh;
    }
    o.lens.clear();
    std::vector<int> lvl(129, -1);
    for (int L = 1; L <= 128; L++)
        if (present[L]) { lvl[L] = (int)o.lens.size(); o.lens.push_back((uint8_t)L); }
    int m = (int)o.lens.size();
    std::vector<std::unordered_map<K4, uint32_t, K4H>> tab(m);
    for (uint32_t i = 0; i < s.n_routes; i++) {
        const nfc_route6 &r = s.routes[i];
        if (r.len == 0) continue;
        K4 k;
        mask128(r.prefix, r.len, k.w);
        int t = lvl[r.len];
        tab[t][k] = 0;
        // markers on the binary-search path towards level t
        int lo = 0, hi = m - 1;
        while (lo <= hi) {
            int mid = (lo + hi) >> 1;
            if (mid == t) break;
            if (mid < t) {
                K4 mk;
                for (int q = 0; q < 4; q++) mk.w[q] = k.w[q] & mask32(o.lens[mid] - 32 * q);
                tab[mid].emplace(mk, 0);
                lo = mid + 1;
            } else {
                hi = mid - 1;
            }
        }
    }
    o.base.assign(m, 0);
    o.mask.assign(m, 0);
    o.ent.clear();
    for (int j = 0; j < m; j++) {
        size_t cnt = tab[j].size(), sz = 2;
        while (sz < 2 * cnt) sz <<= 1;
        o.base[j] = (uint32_t)o.ent.size();
        o.mask[j] = (uint32_t)(sz - 1);
        o.ent.resize(o.ent.size() + sz);
        Lpm6Entry *T = &o.ent[o.base[j]];
        memset(T, 0, sz * sizeof(Lpm6Entry));
        for (auto &kv : tab[j]) {
            int b = trie.best(kv.first.w, o.lens[j]);
            uint32_t info = (b < 0 ? 0x7FFFu : (uint32_t)b) | L6_VALID;
            uint32_t h = l6_hash(kv.first.w[0], kv.first.w[1], kv.first.w[2], kv.first.w[3]) & o.mask[j];
            while (T[h].info & L6_VALID) h = (h + 1) & o.mask[j];
            memcpy(T[h].key, kv.first.w, 16);
            T[h].info = info;
        }
    }
    if (o.ent.empty()) o.ent.resize(2);
    if (o.lens.empty()) { o.base.push_back(0); o.mask.push_back(1); }
    return "";
}

// ---------------------------------------------------------------- AES-128 / HMAC-SHA1
// S-box through exp/log tables of generator 3 in GF(2^8) and the FIPS-197
// affine map; Te tables as in the classic 32-bit T-table formulation.
static uint8_t xt(uint8_t x) { return (uint8_t)((x << 1) ^ ((x & 0x80) ? 0x1b : 0)); }
static void sbox_tables(uint8_t sb[256])
{
    uint8_t ex[256], lg[256] = {0};
    uint8_t x = 1;
    for (int i = 0; i < 255; i++) { ex[i] = x; lg[x] = (uint8_t)i; x = (uint8_t)(x ^ xt(x)); }
    for (int v = 0; v < 256; v++) {
        uint8_t inv = v ? ex[(255 - lg[v]) % 255] : 0;
        uint8_t r = inv;
        for (int k = 1; k <= 4; k++) r ^= (uint8_t)((inv << k) | (inv >> (8 - k)));
        sb[v] = (uint8_t)(r ^ 0x63);
    }
}

void build_aes_tables(std::vector<uint32_t> &te)
{
    uint8_t sb[256];
    sbox_tables(sb);
    te.assign(5 * 256, 0);
    for (int v = 0; v < 256; v++) {
        uint8_t s = sb[v], s2 = xt(s), s3 = (uint8_t)(s2 ^ s);
        uint32_t t0 = (uint32_t)s2 << 24 | (uint32_t)s << 16 | (uint32_t)s << 8 | s3;
        te[v] = t0;
        te[256 + v] = (t0 >> 8) | (t0 << 24);
        te[512 + v] = (t0 >> 16) | (t0 << 16);
        te[768 + v] = (t0 >> 24) | (t0 << 8);
        te[1024 + v] = s;
    }
}

void aes_expand(const uint8_t key[16], uint32_t rk[44])
{
    uint8_t sb[256];
    sbox_tables(sb);
    for (int i = 0; i < 4; i++) rk[i] = be32(key + 4 * i);
    uint8_t rc = 1;
    for (int i = 4; i < 44; i++) {
        uint32_t t = rk[i - 1];
        if ((i & 3) == 0) {
            t = (t << 8) | (t >> 24);
            t = (uint32_t)sb[t >> 24] << 24 | (uint32_t)sb[(t >> 16) & 255] << 16 | (uint32_t)sb[(t >> 8) & 255] << 8 | sb[t & 255];
            t ^= (uint32_t)rc << 24;
            rc = xt(rc);
        }
        rk[i] = rk[i - 4] ^ t;
    }
}

static inline uint32_t rol(uint32_t x, int n) { return (x << n) | (x >> (32 - n)); }
void sha1_compress(uint32_t h[5], const uint8_t blk[64])
{
    uint32_t w[80];
    for (int t = 0; t < 16; t++) w[t] = be32(blk + 4 * t);
    for (int t = 16; t < 80; t++) w[t] = rol(w[t - 3] ^ w[t - 8] ^ w[t - 14] ^ w[t - 16], 1);
    uint32_t a = h[0], b = h[1], c = h[2], d = h[3], e = h[4];
    for (int t = 0; t < 80; t++) {
        uint32_t f, k;
        if (t < 20) { f = d ^ (b & (c ^ d)); k = 0x5a827999u; }
        else if (t < 40) { f = b ^ c ^ d; k = 0x6ed9eba1u; }
        else if (t < 60) { f = (b & c) | (d & (b | c)); k = 0x8f1bbcdcu; }
        else { f = b ^ c ^ d; k = 0xca62c1d6u; }
        uint32_t tmp = rol(a, 5) + f + e + k + w[t];
        e = d; d = c; c = rol(b, 30); b = a; a = tmp;
    }
    h[0] += a; h[1] += b; h[2] += c; h[3] += d; h[4] += e;
}

std::string build_ipsec(const nfc_ipsec_spec &s, std::vector<EspSa> &out)
{
    if (s.n_sa == 0 || s.n_sa > 255 || !s.sas) return "ipsec: n_sa must be 1..255";
    out.assign(s.n_sa, EspSa{});
    for (uint32_t i = 0; i < s.n_sa; i++) {
        const nfc_sa &a = s.sas[i];
        EspSa &d = out[i];
        aes_expand(a.aes_key, d.rk);
        d.spi = a.spi;
        d.nonce = be32(a.nonce);
        uint8_t blk[64];
        static const uint32_t IV[5] = {0x67452301u, 0xefcdab89u, 0x98badcfeu, 0x10325476u, 0xc3d2e1f0u};
        for (int pass = 0; pass < 2; pass++) {
            uint8_t pad = pass ? 0x5c : 0x36;
            for (int k = 0; k < 64; k++) blk[k] = (uint8_t)((k < 20 ? a.auth_key[k] : 0) ^ pad);
            uint32_t *st = pass ? d.opad : d.ipad;
            memcpy(st, IV, sizeof IV);
            sha1_compress(st, blk);
        }
    }
    return "";
}

// ---------------------------------------------------------------- Toeplitz
// nib[k*16 + v] = XOR of the 32-bit key windows at input bit positions
// 4k..4k+3 selected by the bits of nibble v (MSB first).
void build_toeplitz_nibbles(const uint8_t key[40], std::vector<uint32_t> &nib)
{
    auto window = [&](int bit) {
        uint32_t w = 0;
        for (int j = 0; j < 32; j++) {
            int kb = bit + j;
            int v = kb < 320 ? (key[kb >> 3] >> (7 - (kb & 7))) & 1 : 0;
            w = (w << 1) | (uint32_t)v;
        }
        return w;
    };
    nib.assign(72 * 16, 0);
    for (int k = 0; k < 72; k++)
        for (int v = 0; v < 16; v++) {
            uint32_t h = 0;
            for (int j = 0; j < 4; j++)
                if ((v >> (3 - j)) & 1) h ^= window(4 * k + j);
            nib[k * 16 + v] = h;
        }
}

// ---------------------------------------------------------------- NAT44 (R#30)
std::string build_nat(const nfc_nat_spec &s, NatHost &o)
{
    if (s.n_inside > NAT_MAX_INSIDE || (s.n_inside && !s.inside)) return "nat: n_inside must be <= 64 (with prefixes)";
    if (s.n_pool == 0 || s.n_pool > 65536 || !s.pool) return "nat: n_pool must be 1..65536";
    if (s.port_lo > s.port_hi || s.port_hi > 65535) return "nat: port range must satisfy lo <= hi <= 65535";
    if (s.n_dnat && !s.dnat) return "nat: dnat == NULL";
    if (!s.key) return "nat: key == NULL";
    o.img = NatImg{};
    o.img.n_inside = s.n_inside;
    for (uint32_t k = 0; k < s.n_inside; k++) {
        if (s.inside[k].len > 32) return "nat: inside prefix length > 32";
        const uint32_t m = s.inside[k].len ? 0xFFFFFFFFu << (32 - s.inside[k].len) : 0u;
        o.img.in_mask[k] = m;
        o.img.in_pref[k] = s.inside[k].prefix & m;
    }
    o.pool.assign(s.pool, s.pool + s.n_pool);
    o.img.n_pool = s.n_pool;
    o.img.port_lo = s.port_lo;
    o.img.port_range = s.port_hi - s.port_lo + 1;
    o.img.ext_ports = s.ext_ports;
    uint32_t cap = 16;
    while (cap < 2 * s.n_dnat) cap <<= 1;
    o.dnat.assign(cap, make_uint4(0, 0, 0, 0));
    for (uint32_t k = 0; k < s.n_dnat; k++) {
        const nfc_nat_dnat &e = s.dnat[k];
        if (e.proto != 6 && e.proto != 17) return "nat: dnat proto must be 6 or 17";
        const uint32_t key1 = (uint32_t)e.ext_port | (uint32_t)e.proto << 16;
        uint32_t h = nat_slot(e.ext_addr, key1) & (cap - 1);
        while (o.dnat[h].y & NAT_VALID) {
            if (o.dnat[h].x == e.ext_addr && (o.dnat[h].y & 0xFFFFFF) == key1) return "nat: duplicate dnat entry";
            h = (h + 1) & (cap - 1);
        }
        o.dnat[h] = make_uint4(e.ext_addr, key1 | NAT_VALID, e.int_addr, e.int_port);
    }
    o.img.dnat_mask = cap - 1;
    build_toeplitz_nibbles(s.key, o.nib);
    return "";
}

} // namespace nfc
