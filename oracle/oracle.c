/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY (see oracle.h).  Not part of the product.
 *
 * A plain, slow, single-threaded C11 implementation of what the NFCompass hot
 * path computes: every packet, independently and in global order, traverses
 * the chain's NFs in their ORIGINAL order until one drops it (the result that
 * NFCompass's re-organization must preserve: "the packet processing path must
 * not be modified ... the alert or log operation should be executed in the
 * same packet state", P:L269 [SIV.B.2]).  Each function below cites the
 * passage it follows.  Where the paper is silent the reading taken is the one
 * listed in DESIGN.md ("R#k").  No SIMD, no AES-NI/SHA-NI, no OpenMP; shares
 * no code with the CUDA path.
 */
#include "oracle.h"
#include <stdlib.h>
#include <string.h>

/* ======================================================================
 * AES-128 (FIPS-197), used by IPsec AES-128-CTR (P:L130 [SIII.A.2]).
 * The S-box is derived from its definition (FIPS-197 S5.1.1: multiplicative
 * inverse in GF(2^8) followed by the affine transform), not typed in.
 * ==================================================================== */
static uint8_t gf_mul(uint8_t a, uint8_t b) /* FIPS-197 S4.2 */
{
    uint8_t p = 0;
    for (int i = 0; i < 8; i++) {
        if (b & 1) p ^= a;
        uint8_t hi = a & 0x80;
        a <<= 1;
        if (hi) a ^= 0x1b; /* m(x) = x^8 + x^4 + x^3 + x + 1 */
        b >>= 1;
    }
    return p;
}

static uint8_t SBOX[256];
static int sbox_ready = 0;

static void sbox_init(void) /* FIPS-197 S5.1.1 */
{
    if (sbox_ready) return;
    for (int x = 0; x < 256; x++) {
        uint8_t inv = 0;
        if (x != 0)
            for (int y = 1; y < 256; y++)
                if (gf_mul((uint8_t)x, (uint8_t)y) == 1) { inv = (uint8_t)y; break; }
        uint8_t s = 0;
        for (int i = 0; i < 8; i++) {
            int bit = ((inv >> i) & 1) ^ ((inv >> ((i + 4) % 8)) & 1) ^ ((inv >> ((i + 5) % 8)) & 1) ^
                      ((inv >> ((i + 6) % 8)) & 1) ^ ((inv >> ((i + 7) % 8)) & 1) ^ ((0x63 >> i) & 1);
            s |= (uint8_t)(bit << i);
        }
        SBOX[x] = s;
    }
    sbox_ready = 1;
}

static void aes_key_expansion(const uint8_t key[16], uint8_t w[176]) /* FIPS-197 S5.2 */
{
    sbox_init();
    memcpy(w, key, 16);
    uint8_t rcon = 1;
    for (int i = 4; i < 44; i++) {
        uint8_t t[4];
        memcpy(t, w + 4 * (i - 1), 4);
        if (i % 4 == 0) {
            uint8_t t0 = t[0]; /* RotWord */
            t[0] = t[1]; t[1] = t[2]; t[2] = t[3]; t[3] = t0;
            for (int j = 0; j < 4; j++) t[j] = SBOX[t[j]]; /* SubWord */
            t[0] ^= rcon;
            rcon = gf_mul(rcon, 2);
        }
        for (int j = 0; j < 4; j++) w[4 * i + j] = w[4 * (i - 4) + j] ^ t[j];
    }
}

static void aes_cipher(const uint8_t w[176], const uint8_t in[16], uint8_t out[16]) /* FIPS-197 S5.1 */
{
    uint8_t s[4][4];
    for (int c = 0; c < 4; c++)
        for (int r = 0; r < 4; r++) s[r][c] = in[r + 4 * c];
    for (int r = 0; r < 4; r++)
        for (int c = 0; c < 4; c++) s[r][c] ^= w[4 * c + r]; /* AddRoundKey(0) */
    for (int round = 1; round <= 10; round++) {
        for (int r = 0; r < 4; r++)
            for (int c = 0; c < 4; c++) s[r][c] = SBOX[s[r][c]]; /* SubBytes */
        uint8_t t[4][4];
        for (int r = 0; r < 4; r++)
            for (int c = 0; c < 4; c++) t[r][c] = s[r][(c + r) % 4]; /* ShiftRows */
        memcpy(s, t, 16);
        if (round != 10) { /* MixColumns, FIPS-197 S5.1.3 */
            for (int c = 0; c < 4; c++) {
                uint8_t a0 = s[0][c], a1 = s[1][c], a2 = s[2][c], a3 = s[3][c];
                s[0][c] = gf_mul(a0, 2) ^ gf_mul(a1, 3) ^ a2 ^ a3;
                s[1][c] = a0 ^ gf_mul(a1, 2) ^ gf_mul(a2, 3) ^ a3;
                s[2][c] = a0 ^ a1 ^ gf_mul(a2, 2) ^ gf_mul(a3, 3);
                s[3][c] = gf_mul(a0, 3) ^ a1 ^ a2 ^ gf_mul(a3, 2);
            }
        }
        for (int r = 0; r < 4; r++)
            for (int c = 0; c < 4; c++) s[r][c] ^= w[16 * round + 4 * c + r]; /* AddRoundKey */
    }
    for (int c = 0; c < 4; c++)
        for (int r = 0; r < 4; r++) out[r + 4 * c] = s[r][c];
}

void or_aes128_encrypt_block(const uint8_t key[16], const uint8_t in[16], uint8_t out[16])
{
    uint8_t w[176];
    aes_key_expansion(key, w);
    aes_cipher(w, in, out);
}

/* CTR mode (NIST SP 800-38A S6.5; RFC 3686 S4): block j uses counter block
 * ctr_block0 with its last 32 bits incremented j times (big-endian). */
void or_aes128_ctr(const uint8_t key[16], const uint8_t ctr_block0[16], const uint8_t *in,
                   uint8_t *out, size_t n)
{
    uint8_t w[176], cb[16], ks[16];
    aes_key_expansion(key, w);
    memcpy(cb, ctr_block0, 16);
    for (size_t off = 0; off < n; off += 16) {
        aes_cipher(w, cb, ks);
        for (size_t j = 0; j < 16 && off + j < n; j++) out[off + j] = in[off + j] ^ ks[j];
        uint32_t ctr = ((uint32_t)cb[12] << 24) | ((uint32_t)cb[13] << 16) | ((uint32_t)cb[14] << 8) | cb[15];
        ctr++;
        cb[12] = (uint8_t)(ctr >> 24); cb[13] = (uint8_t)(ctr >> 16);
        cb[14] = (uint8_t)(ctr >> 8);  cb[15] = (uint8_t)ctr;
    }
}

/* ======================================================================
 * SHA-1 (FIPS 180-4 S6.1) and HMAC (RFC 2104), used by IPsec HMAC-SHA1
 * (P:L130 [SIII.A.2]).
 * ==================================================================== */
static uint32_t rotl(uint32_t x, int n) { return (x << n) | (x >> (32 - n)); }

static void sha1_block(uint32_t H[5], const uint8_t blk[64])
{
    uint32_t W[80];
    for (int t = 0; t < 16; t++)
        W[t] = ((uint32_t)blk[4 * t] << 24) | ((uint32_t)blk[4 * t + 1] << 16) |
               ((uint32_t)blk[4 * t + 2] << 8) | blk[4 * t + 3];
    for (int t = 16; t < 80; t++) W[t] = rotl(W[t - 3] ^ W[t - 8] ^ W[t - 14] ^ W[t - 16], 1);
    uint32_t a = H[0], b = H[1], c = H[2], d = H[3], e = H[4];
    for (int t = 0; t < 80; t++) {
        uint32_t f, K;
        if (t < 20)      { f = (b & c) ^ (~b & d);          K = 0x5a827999u; }
        else if (t < 40) { f = b ^ c ^ d;                   K = 0x6ed9eba1u; }
        else if (t < 60) { f = (b & c) ^ (b & d) ^ (c & d); K = 0x8f1bbcdcu; }
        else             { f = b ^ c ^ d;                   K = 0xca62c1d6u; }
        uint32_t T = rotl(a, 5) + f + e + K + W[t];
        e = d; d = c; c = rotl(b, 30); b = a; a = T;
    }
    H[0] += a; H[1] += b; H[2] += c; H[3] += d; H[4] += e;
}

void or_sha1(const uint8_t *msg, size_t n, uint8_t out[20])
{
    uint32_t H[5] = {0x67452301u, 0xefcdab89u, 0x98badcfeu, 0x10325476u, 0xc3d2e1f0u};
    size_t full = n / 64;
    for (size_t i = 0; i < full; i++) sha1_block(H, msg + 64 * i);
    uint8_t tail[128];
    size_t rem = n - 64 * full;
    memset(tail, 0, sizeof tail);
    memcpy(tail, msg + 64 * full, rem);
    tail[rem] = 0x80; /* FIPS 180-4 S5.1.1 padding */
    size_t tl = (rem + 1 + 8 <= 64) ? 64 : 128;
    uint64_t bits = (uint64_t)n * 8;
    for (int j = 0; j < 8; j++) tail[tl - 1 - j] = (uint8_t)(bits >> (8 * j));
    sha1_block(H, tail);
    if (tl == 128) sha1_block(H, tail + 64);
    for (int i = 0; i < 5; i++) {
        out[4 * i] = (uint8_t)(H[i] >> 24); out[4 * i + 1] = (uint8_t)(H[i] >> 16);
        out[4 * i + 2] = (uint8_t)(H[i] >> 8); out[4 * i + 3] = (uint8_t)H[i];
    }
}

void or_hmac_sha1(const uint8_t *key, size_t klen, const uint8_t *msg, size_t n, uint8_t out[20])
{
    uint8_t k0[64], kh[20];
    memset(k0, 0, 64);
    if (klen > 64) { or_sha1(key, klen, kh); memcpy(k0, kh, 20); }
    else memcpy(k0, key, klen);
    uint8_t *buf = (uint8_t *)malloc(64 + n + 20);
    for (int i = 0; i < 64; i++) buf[i] = k0[i] ^ 0x36;
    memcpy(buf + 64, msg, n);
    uint8_t inner[20];
    or_sha1(buf, 64 + n, inner);
    for (int i = 0; i < 64; i++) buf[i] = k0[i] ^ 0x5c;
    memcpy(buf + 64, inner, 20);
    or_sha1(buf, 84, out);
    free(buf);
}

/* ======================================================================
 * Toeplitz hash (Microsoft RSS), the RSS flow hash of the paper's I/O model
 * (P:L87 [SII.B.1] "Receive Side Steering"); reused for ESP SA selection and
 * the load balancer's flow hash (R#8, R#22).
 * ==================================================================== */
uint32_t or_toeplitz(const uint8_t key[40], const uint8_t *in, size_t n)
{
    uint32_t result = 0;
    uint32_t window = ((uint32_t)key[0] << 24) | ((uint32_t)key[1] << 16) | ((uint32_t)key[2] << 8) | key[3];
    size_t next_bit = 32; /* index of the next key bit to shift into the window */
    for (size_t i = 0; i < n; i++) {
        for (int b = 7; b >= 0; b--) {
            if ((in[i] >> b) & 1) result ^= window;
            int kb = (next_bit < 320) ? (key[next_bit / 8] >> (7 - next_bit % 8)) & 1 : 0;
            window = (window << 1) | (uint32_t)kb;
            next_bit++;
        }
    }
    return result;
}

static const uint8_t MS_RSS_KEY[40] = {
    0x6d, 0x5a, 0x56, 0xda, 0x25, 0x5b, 0x0e, 0xc2, 0x41, 0x67, 0x25, 0x3d, 0x43, 0xa3,
    0x8f, 0xb0, 0xd0, 0xca, 0x2b, 0xcb, 0xae, 0x7b, 0x30, 0xb4, 0x77, 0xcb, 0x2d, 0xa3,
    0x80, 0x30, 0xf2, 0x0c, 0x6a, 0x42, 0xb7, 0x3b, 0xbe, 0xac, 0x01, 0xfa};

/* RFC 1071: one's-complement sum of 16-bit big-endian words, complemented. */
uint16_t or_ipv4_checksum(const uint8_t *hdr, size_t hlen)
{
    uint32_t sum = 0;
    for (size_t i = 0; i + 1 < hlen; i += 2) sum += ((uint32_t)hdr[i] << 8) | hdr[i + 1];
    while (sum >> 16) sum = (sum & 0xffff) + (sum >> 16);
    return (uint16_t)~sum;
}

/* ======================================================================
 * Oracle chain state
 * ==================================================================== */
typedef struct { int32_t child[2]; int32_t nh; } trie_node; /* unibit trie (textbook LPM) */
typedef struct { trie_node *n; size_t cnt, cap; } trie;

typedef struct {
    int32_t *go;     /* go[s*256+a]: goto function, -1 = fail (Aho & Corasick 1975, Alg. 2) */
    int32_t *fail;   /* failure function (Alg. 3) */
    int32_t *out1;   /* first pattern id ending exactly at s, -1 none */
    int32_t *outnx;  /* next pattern id with the same string (duplicates), -1 end */
    size_t n_states;
} acm;

struct or_chain {
    or_spec s;
    trie t4, t6;
    acm ac;
    uint32_t *seq;     /* per-SA sequence counters */
    uint32_t *stamp;   /* DPI distinct-set stamps (per pattern) */
    uint32_t stamp_gen;
    size_t stats_len;
};

static int32_t trie_new(trie *t)
{
    if (t->cnt == t->cap) {
        t->cap = t->cap ? 2 * t->cap : 1024;
        t->n = (trie_node *)realloc(t->n, t->cap * sizeof(trie_node));
    }
    t->n[t->cnt].child[0] = t->n[t->cnt].child[1] = -1;
    t->n[t->cnt].nh = -1;
    return (int32_t)t->cnt++;
}

static int bit_of(const uint8_t *a, int i) { return (a[i / 8] >> (7 - i % 8)) & 1; }

static void trie_insert(trie *t, const uint8_t *addr, int len, int32_t nh)
{
    int32_t cur = 0;
    for (int i = 0; i < len; i++) {
        int b = bit_of(addr, i);
        if (t->n[cur].child[b] < 0) {
            int32_t nn = trie_new(t);
            t->n[cur].child[b] = nn;
        }
        cur = t->n[cur].child[b];
    }
    t->n[cur].nh = nh;
}

static int32_t trie_lookup(const trie *t, const uint8_t *addr, int bits)
{
    int32_t cur = 0, best = t->n[0].nh;
    for (int i = 0; i < bits && cur >= 0; i++) {
        cur = t->n[cur].child[bit_of(addr, i)];
        if (cur >= 0 && t->n[cur].nh >= 0) best = t->n[cur].nh;
    }
    return best;
}

/* Aho-Corasick construction (Aho & Corasick 1975, Algorithms 2 and 3), the
 * string matcher the paper's DPI uses (P:L132 [SIII.A.2]). */
static void ac_build(acm *m, const or_spec *s)
{
    size_t cap = 1;
    for (uint32_t j = 0; j < s->n_pat; j++) cap += s->pat_off[j + 1] - s->pat_off[j];
    m->go = (int32_t *)malloc(cap * 256 * sizeof(int32_t));
    m->fail = (int32_t *)calloc(cap, sizeof(int32_t));
    m->out1 = (int32_t *)malloc(cap * sizeof(int32_t));
    m->outnx = (int32_t *)malloc((s->n_pat + 1) * sizeof(int32_t));
    for (size_t i = 0; i < cap * 256; i++) m->go[i] = -1;
    for (size_t i = 0; i < cap; i++) m->out1[i] = -1;
    m->n_states = 1;
    /* Algorithm 2: goto function (a trie of the patterns) */
    for (uint32_t j = 0; j < s->n_pat; j++) {
        int32_t st = 0;
        for (uint32_t k = s->pat_off[j]; k < s->pat_off[j + 1]; k++) {
            uint8_t a = s->pat_blob[k];
            if (m->go[st * 256 + a] < 0) m->go[st * 256 + a] = (int32_t)m->n_states++;
            st = m->go[st * 256 + a];
        }
        m->outnx[j] = m->out1[st];
        m->out1[st] = (int32_t)j;
    }
    /* Algorithm 3: failure function by breadth-first search */
    int32_t *queue = (int32_t *)malloc(m->n_states * sizeof(int32_t));
    size_t qh = 0, qt = 0;
    for (int a = 0; a < 256; a++) {
        int32_t q = m->go[a];
        if (q > 0) { m->fail[q] = 0; queue[qt++] = q; }
    }
    while (qh < qt) {
        int32_t r = queue[qh++];
        for (int a = 0; a < 256; a++) {
            int32_t q = m->go[r * 256 + a];
            if (q < 0) continue;
            queue[qt++] = q;
            int32_t st = m->fail[r];
            while (st != 0 && m->go[st * 256 + a] < 0) st = m->fail[st];
            int32_t g = m->go[st * 256 + a];
            m->fail[q] = (g >= 0 && g != q) ? g : 0;
        }
    }
    free(queue);
}

/* DPI distinct pattern set M over buf (R#9): Algorithm 1 of Aho & Corasick,
 * output(s) = patterns ending at s or at any state on its failure chain. */
static uint32_t ac_scan(or_chain *c, const uint8_t *buf, size_t n, uint32_t *ids, uint32_t cap, int *any_drop)
{
    acm *m = &c->ac;
    uint32_t cnt = 0;
    c->stamp_gen++;
    if (c->stamp_gen == 0) { memset(c->stamp, 0, c->s.n_pat * sizeof(uint32_t)); c->stamp_gen = 1; }
    int32_t st = 0;
    for (size_t i = 0; i < n; i++) {
        uint8_t a = buf[i];
        while (st != 0 && m->go[st * 256 + a] < 0) st = m->fail[st];
        st = m->go[st * 256 + a] >= 0 ? m->go[st * 256 + a] : 0;
        for (int32_t u = st; u != 0; u = m->fail[u]) {
            for (int32_t j = m->out1[u]; j >= 0; j = m->outnx[j]) {
                if (c->stamp[j] == c->stamp_gen) continue;
                c->stamp[j] = c->stamp_gen;
                if (cnt < cap) ids[cnt] = (uint32_t)j;
                cnt++;
                if (c->s.pat_action[j]) *any_drop = 1;
            }
        }
    }
    return cnt;
}

static int cmp_u32(const void *a, const void *b)
{
    uint32_t x = *(const uint32_t *)a, y = *(const uint32_t *)b;
    return x < y ? -1 : x > y;
}

uint32_t or_ac_match(or_chain *c, const uint8_t *buf, size_t n, uint32_t *ids, uint32_t cap)
{
    int d = 0;
    uint32_t k = ac_scan(c, buf, n, ids, cap, &d);
    qsort(ids, k < cap ? k : cap, sizeof(uint32_t), cmp_u32);
    return k;
}

or_chain *oracle_create(const or_spec *spec)
{
    or_chain *c = (or_chain *)calloc(1, sizeof(or_chain));
    c->s = *spec;
    sbox_init();
    trie_new(&c->t4);
    trie_new(&c->t6);
    for (uint32_t i = 0; i < spec->n_r4; i++) {
        uint8_t a[4] = {(uint8_t)(spec->r4[i].prefix >> 24), (uint8_t)(spec->r4[i].prefix >> 16),
                        (uint8_t)(spec->r4[i].prefix >> 8), (uint8_t)spec->r4[i].prefix};
        trie_insert(&c->t4, a, spec->r4[i].len, spec->r4[i].nh);
    }
    for (uint32_t i = 0; i < spec->n_r6; i++) trie_insert(&c->t6, spec->r6[i].prefix, spec->r6[i].len, spec->r6[i].nh);
    if (spec->n_pat) ac_build(&c->ac, spec);
    c->stamp = (uint32_t *)calloc(spec->n_pat + 1, sizeof(uint32_t));
    c->seq = (uint32_t *)calloc(spec->n_sa + 1, sizeof(uint32_t));
    for (uint32_t i = 0; i < spec->n_sa; i++) c->seq[i] = spec->sa[i].seq0;
    c->stats_len = OR_ST_VAR_BASE + spec->n_acl + 1 + spec->n_lb + spec->n_sa;
    return c;
}

void oracle_destroy(or_chain *c)
{
    if (!c) return;
    free(c->t4.n); free(c->t6.n);
    free(c->ac.go); free(c->ac.fail); free(c->ac.out1); free(c->ac.outnx);
    free(c->stamp); free(c->seq);
    free(c);
}

size_t oracle_stats_len(const or_chain *c) { return c->stats_len; }

int32_t or_lpm4(or_chain *c, uint32_t dst)
{
    uint8_t a[4] = {(uint8_t)(dst >> 24), (uint8_t)(dst >> 16), (uint8_t)(dst >> 8), (uint8_t)dst};
    return trie_lookup(&c->t4, a, 32);
}

int32_t or_lpm6(or_chain *c, const uint8_t dst[16]) { return trie_lookup(&c->t6, dst, 128); }

static int prefix_match(const uint8_t *a, const uint8_t *p, int len)
{
    for (int i = 0; i < len; i++)
        if (bit_of(a, i) != bit_of(p, i)) return 0;
    return 1;
}

/* ACL: first matching rule by linear scan (R: SURVEY 8(c)(i)2). */
int32_t or_acl(or_chain *c, uint8_t family, const uint8_t *src, const uint8_t *dst, uint16_t sport,
               uint16_t dport, uint8_t proto)
{
    for (uint32_t i = 0; i < c->s.n_acl; i++) {
        const or_acl_rule *r = &c->s.acl[i];
        if (r->family != family) continue;
        if (!prefix_match(src, r->src, r->slen)) continue;
        if (!prefix_match(dst, r->dst, r->dlen)) continue;
        if (sport < r->sp_lo || sport > r->sp_hi) continue;
        if (dport < r->dp_lo || dport > r->dp_hi) continue;
        if (!r->proto_any && r->proto != proto) continue;
        return (int32_t)i;
    }
    return -1;
}

/* ======================================================================
 * Packet parse -- the header classifier the paper de-duplicates to run once
 * (P:L267, P:L269 [SIV.B.2]); validity check of the I/O loop.
 * ==================================================================== */
typedef struct {
    int family;            /* 4 or 6 */
    int l4_off, ip_end;    /* byte offsets within the frame */
    int pl_off;            /* payload span [pl_off, ip_end) */
    uint8_t proto;
    uint16_t sport, dport;
    uint8_t src[16], dst[16];
} pview;

static uint16_t be16(const uint8_t *p) { return (uint16_t)((p[0] << 8) | p[1]); }

static int parse(const uint8_t *f, int flen, pview *v)
{
    memset(v, 0, sizeof *v);
    if (flen < 14) return 0;
    uint16_t et = be16(f + 12);
    int frag = 0;
    if (et == 0x0800) {
        if (flen < 34) return 0;
        if ((f[14] >> 4) != 4) return 0;
        int ihl = f[14] & 15;
        if (ihl < 5) return 0;
        int tot = be16(f + 16);
        if (tot < 4 * ihl || 14 + tot > flen) return 0;
        v->family = 4;
        v->l4_off = 14 + 4 * ihl;
        v->ip_end = 14 + tot;
        v->proto = f[23];
        memcpy(v->src, f + 26, 4);
        memcpy(v->dst, f + 30, 4);
        uint16_t fo = be16(f + 20);
        frag = (fo & 0x2000) || (fo & 0x1fff);
    } else if (et == 0x86DD) {
        if (flen < 54) return 0;
        if ((f[14] >> 4) != 6) return 0;
        int pl = be16(f + 18);
        if (54 + pl > flen) return 0;
        v->family = 6;
        v->l4_off = 54;
        v->ip_end = 54 + pl;
        v->proto = f[20];
        memcpy(v->src, f + 22, 16);
        memcpy(v->dst, f + 38, 16);
    } else {
        return 0;
    }
    int l4len = 0;
    if (!frag && v->proto == 17) {
        if (v->l4_off + 8 > v->ip_end) return 0;
        l4len = 8;
    } else if (!frag && v->proto == 6) {
        if (v->l4_off + 20 > v->ip_end) return 0;
        int doff = f[v->l4_off + 12] >> 4;
        if (doff < 5 || v->l4_off + 4 * doff > v->ip_end) return 0;
        l4len = 4 * doff;
    }
    if (l4len) {
        v->sport = be16(f + v->l4_off);
        v->dport = be16(f + v->l4_off + 2);
    }
    v->pl_off = v->l4_off + l4len;
    return 1;
}

/* Test hook: the parse above, exposed so the hand-built-frame pins of SURVEY
 * 8(c)(i) can check every field.  out = {ok, family, l4_off, ip_end, pl_off,
 * proto, sport, dport}. */
int or_parse(const uint8_t *f, int flen, int32_t out[8])
{
    pview v;
    int ok = parse(f, flen, &v);
    out[0] = ok; out[1] = v.family; out[2] = v.l4_off; out[3] = v.ip_end; out[4] = v.pl_off;
    out[5] = v.proto; out[6] = v.sport; out[7] = v.dport;
    return ok;
}

static size_t tuple_bytes(const pview *v, uint8_t *t)
{
    int al = v->family == 4 ? 4 : 16;
    memcpy(t, v->src, al);
    memcpy(t + al, v->dst, al);
    t[2 * al] = (uint8_t)(v->sport >> 8); t[2 * al + 1] = (uint8_t)v->sport;
    t[2 * al + 2] = (uint8_t)(v->dport >> 8); t[2 * al + 3] = (uint8_t)v->dport;
    return (size_t)(2 * al + 4);
}

/* IPsec ESP transport mode (R#8: RFC 4303 + RFC 3686 + RFC 2404).
 * Builds the output frame in a scratch buffer, then writes it at frame-16. */
static int esp_apply(or_chain *c, uint8_t *frame, int flen, const pview *v, uint32_t sa_idx, uint32_t seq,
                     uint64_t *stats)
{
    const or_sa *sa = &c->s.sa[sa_idx];
    int plen = v->ip_end - v->l4_off;
    int p = (4 - ((plen + 2) % 4)) % 4;
    int clen = plen + p + 2;
    int out_len = v->ip_end + 30 + p;
    uint8_t *o = (uint8_t *)malloc((size_t)out_len);
    memcpy(o, frame, (size_t)v->l4_off);
    if (v->family == 4) {
        o[23] = 50;
        int tot = be16(o + 16) + 30 + p;
        o[16] = (uint8_t)(tot >> 8); o[17] = (uint8_t)tot;
        o[24] = o[25] = 0;
        uint16_t ck = or_ipv4_checksum(o + 14, (size_t)(v->l4_off - 14));
        o[24] = (uint8_t)(ck >> 8); o[25] = (uint8_t)ck;
    } else {
        o[20] = 50;
        int pl = be16(o + 18) + 30 + p;
        o[18] = (uint8_t)(pl >> 8); o[19] = (uint8_t)pl;
    }
    uint8_t *esp = o + v->l4_off;
    esp[0] = (uint8_t)(sa->spi >> 24); esp[1] = (uint8_t)(sa->spi >> 16);
    esp[2] = (uint8_t)(sa->spi >> 8);  esp[3] = (uint8_t)sa->spi;
    esp[4] = (uint8_t)(seq >> 24); esp[5] = (uint8_t)(seq >> 16);
    esp[6] = (uint8_t)(seq >> 8);  esp[7] = (uint8_t)seq;
    memset(esp + 8, 0, 4); /* IV = be64(seq) */
    memcpy(esp + 12, esp + 4, 4);
    uint8_t *pt = (uint8_t *)malloc((size_t)clen);
    memcpy(pt, frame + v->l4_off, (size_t)plen);
    for (int i = 0; i < p; i++) pt[plen + i] = (uint8_t)(i + 1); /* RFC 4303 S2.4 default padding */
    pt[plen + p] = (uint8_t)p;
    pt[plen + p + 1] = v->proto;
    uint8_t cb[16]; /* RFC 3686 S4: nonce || IV || be32(1) */
    memcpy(cb, sa->nonce, 4);
    memcpy(cb + 4, esp + 8, 8);
    cb[12] = cb[13] = cb[14] = 0; cb[15] = 1;
    or_aes128_ctr(sa->aes_key, cb, pt, esp + 16, (size_t)clen);
    uint8_t icv[20]; /* RFC 2404: HMAC-SHA1-96 over ESP hdr || IV || C */
    or_hmac_sha1(sa->auth_key, 20, esp, (size_t)(16 + clen), icv);
    memcpy(esp + 16 + clen, icv, 12);
    memcpy(frame - 16, o, (size_t)out_len);
    free(pt);
    free(o);
    stats[OR_ST_ESP_PKTS]++;
    stats[OR_ST_ESP_BYTES] += (uint64_t)clen;
    stats[OR_ST_ESP_BLOCKS] += (uint64_t)((clen + 15) / 16);
    (void)flen;
    return out_len;
}

/* L2/L3 forward after an LPM hit (P:L128 [SIII.A.2]; R#6): eth.dst = nh.mac,
 * eth.src = port_mac[nh.port], TTL/hop limit - 1, IPv4 checksum recomputed. */
static void forward_rewrite(uint8_t *f, const pview *v, const or_nexthop *nh, const uint8_t *pmac, uint32_t n_port)
{
    memcpy(f, nh->mac, 6);
    if (nh->port < n_port) memcpy(f + 6, pmac + 6 * nh->port, 6);
    if (v->family == 4) {
        f[22] -= 1;
        f[24] = f[25] = 0;
        uint16_t ck = or_ipv4_checksum(f + 14, (size_t)(v->l4_off - 14));
        f[24] = (uint8_t)(ck >> 8); f[25] = (uint8_t)ck;
    } else {
        f[21] -= 1;
    }
}

/* RFC 1624 eqn. 3: HC' = ~(~HC + ~m + m'), one's complement 16-bit sums. */
static uint32_t oc_add16(uint32_t a, uint32_t b)
{
    uint32_t x = a + b;
    return (x & 0xFFFF) + (x >> 16);
}
uint16_t or_csum_update(uint16_t hc, uint16_t m, uint16_t m1)
{
    uint32_t x = oc_add16(oc_add16((uint16_t)~hc, (uint16_t)~m), m1);
    return (uint16_t)~x;
}

/* NAT44 ("For traffics to Internet, the NAT network function performs
 * source and destination NAT"; Table II row NAT: header read + write, no drop;
 * reading R#30).  Applies to IPv4 TCP/UDP packets (L4 header parsed) whose
 * egress port, as set by the NFs before it, is marked as Internet-facing.
 *   h    = Toeplitz(nat_key, src | dst | sport | dport) of the packet as it arrives;
 *   DNAT : the first entry with (proto, ext_addr, ext_port) == (proto, dst, dport)
 *          rewrites dst, dport to (int_addr, int_port);
 *   SNAT : if src lies in one of the inside prefixes (first match), src := pool[(h
 *          & 0xFFFF) mod n_pool], sport := port_lo + ((h >> 16) mod (port_hi -
 *          port_lo + 1))  (deterministic NAPT: a pure function of the flow);
 *   the IPv4 header checksum is recomputed (RFC 1071), the TCP / UDP checksum is
 *   updated per changed 16-bit word by RFC 1624 eqn. 3 (pseudo-header addresses
 *   and ports); a UDP checksum of 0 ("none", RFC 768) stays 0, and an updated
 *   UDP checksum of 0 is sent as 0xFFFF.
 * Returns 1 if the NAT applied, 0 for pass-through. */
static uint32_t be32p(const uint8_t *p) { return (uint32_t)p[0] << 24 | (uint32_t)p[1] << 16 | (uint32_t)p[2] << 8 | p[3]; }
static void put32p(uint8_t *p, uint32_t v) { p[0] = (uint8_t)(v >> 24); p[1] = (uint8_t)(v >> 16); p[2] = (uint8_t)(v >> 8); p[3] = (uint8_t)v; }
static int nat_apply(const or_spec *s, uint8_t *f, pview *v, uint32_t port)
{
    if (v->family != 4 || (v->proto != 6 && v->proto != 17) || v->pl_off == v->l4_off) return 0;
    if (port >= 32 || !((s->nat_ext_ports >> port) & 1)) return 0;
    uint8_t t[12];
    tuple_bytes(v, t);
    const uint32_t h = or_toeplitz(s->nat_key, t, 12);
    const uint32_t src = be32p(v->src), dst = be32p(v->dst);
    uint32_t nsrc = src, ndst = dst;
    uint16_t nsp = v->sport, ndp = v->dport;
    for (uint32_t k = 0; k < s->n_nat_dnat; k++) {
        const or_nat_dnat *e = &s->nat_dnat[k];
        if (e->proto == v->proto && e->ext_addr == dst && e->ext_port == v->dport) {
            ndst = e->int_addr;
            ndp = e->int_port;
            break;
        }
    }
    for (uint32_t k = 0; k < s->n_nat_inside; k++) {
        const or_nat_prefix *q = &s->nat_inside[k];
        const uint32_t m = q->len == 0 ? 0u : 0xFFFFFFFFu << (32 - q->len);
        if ((src & m) == (q->prefix & m)) {
            nsrc = s->nat_pool[(h & 0xFFFF) % s->n_nat_pool];
            nsp = (uint16_t)(s->nat_port_lo + (h >> 16) % (s->nat_port_hi - s->nat_port_lo + 1));
            break;
        }
    }
    const int l4 = v->l4_off, ck_at = v->proto == 6 ? l4 + 16 : l4 + 6;
    uint16_t ck = be16(f + ck_at);
    if (!(v->proto == 17 && ck == 0)) {
        const uint16_t m[6] = {(uint16_t)(src >> 16), (uint16_t)src, (uint16_t)(dst >> 16), (uint16_t)dst, v->sport, v->dport};
        const uint16_t m1[6] = {(uint16_t)(nsrc >> 16), (uint16_t)nsrc, (uint16_t)(ndst >> 16), (uint16_t)ndst, nsp, ndp};
        for (int k = 0; k < 6; k++)
            if (m[k] != m1[k]) ck = or_csum_update(ck, m[k], m1[k]);
        if (v->proto == 17 && ck == 0) ck = 0xFFFF;
        f[ck_at] = (uint8_t)(ck >> 8);
        f[ck_at + 1] = (uint8_t)ck;
    }
    put32p(f + 26, nsrc);
    put32p(f + 30, ndst);
    f[l4] = (uint8_t)(nsp >> 8); f[l4 + 1] = (uint8_t)nsp;
    f[l4 + 2] = (uint8_t)(ndp >> 8); f[l4 + 3] = (uint8_t)ndp;
    f[24] = f[25] = 0;
    const uint16_t ipck = or_ipv4_checksum(f + 14, (size_t)(l4 - 14));
    f[24] = (uint8_t)(ipck >> 8); f[25] = (uint8_t)ipck;
    put32p(v->src, nsrc);
    put32p(v->dst, ndst);
    v->sport = nsp;
    v->dport = ndp;
    return 1;
}

uint64_t oracle_run(or_chain *c, uint8_t *arena, const uint64_t *off, const uint16_t *len, uint32_t n,
                    uint64_t first_global, or_result *res, uint32_t *match_pkt, uint16_t *match_pat,
                    uint64_t match_cap, uint64_t *stats, const uint32_t *seq_override)
{
    const or_spec *s = &c->s;
    uint64_t n_pairs = 0;
    uint32_t *ids = (uint32_t *)malloc((s->n_pat + 1) * sizeof(uint32_t));
    uint64_t *acl_hits = stats + OR_ST_VAR_BASE;
    uint64_t *lb_hits = acl_hits + s->n_acl + 1;
    uint64_t *sa_pkts = lb_hits + s->n_lb;
    for (uint32_t i = 0; i < n; i++) {
        uint8_t *f = arena + off[i];
        int flen = len[i];
        or_result r = {0xFF, 0xFF, 0, 0xFFFF, 0xFFFF, 0, (uint16_t)flen, 0};
        stats[OR_ST_PKTS]++;
        stats[OR_ST_BYTES_IN] += (uint64_t)flen;
        pview v;
        int dropped = 0;
        if (!parse(f, flen, &v)) {
            r.drop_nf = 0xFE;
            stats[OR_ST_PARSE_DROP]++;
            dropped = 1;
        }
        for (uint32_t p = 0; !dropped && p < s->n_nf; p++) {
            uint64_t *ps = stats + OR_ST_POS_BASE + 4 * p;
            ps[0]++;
            int pass = 0;
            switch (s->kind[p]) {
            case OR_ACL: {
                int32_t rule = or_acl(c, (uint8_t)v.family, v.src, v.dst, v.sport, v.dport, v.proto);
                uint32_t act;
                if (rule >= 0) { r.acl_rule = (uint16_t)rule; acl_hits[rule]++; act = s->acl[rule].action; }
                else { acl_hits[s->n_acl]++; act = s->acl_default; }
                if (act == 1) dropped = 1;
                break;
            }
            case OR_DPI: {
                int any_drop = 0;
                uint32_t k = s->n_pat ? ac_scan(c, f + v.pl_off, (size_t)(v.ip_end - v.pl_off), ids, s->n_pat, &any_drop) : 0;
                qsort(ids, k, sizeof(uint32_t), cmp_u32);
                r.dpi_nmatch = (uint16_t)k;
                for (uint32_t j = 0; j < k; j++) {
                    if (n_pairs < match_cap) {
                        match_pkt[n_pairs] = (uint32_t)(first_global + i);
                        match_pat[n_pairs] = (uint16_t)ids[j];
                    }
                    n_pairs++;
                }
                stats[OR_ST_DPI_PAIRS] += k;
                if (any_drop) dropped = 1;
                break;
            }
            case OR_LPM4:
            case OR_LPM6: {
                int want = s->kind[p] == OR_LPM4 ? 4 : 6;
                if (v.family != want) { pass = 1; break; }
                int32_t nh;
                const or_nexthop *tab;
                const uint8_t *pm;
                uint32_t np;
                if (want == 4) {
                    uint32_t d = ((uint32_t)v.dst[0] << 24) | ((uint32_t)v.dst[1] << 16) | ((uint32_t)v.dst[2] << 8) | v.dst[3];
                    nh = or_lpm4(c, d); tab = s->nh4; pm = s->pmac4; np = s->n_port4;
                } else {
                    nh = or_lpm6(c, v.dst); tab = s->nh6; pm = s->pmac6; np = s->n_port6;
                }
                int ttl = want == 4 ? f[22] : f[21];
                if (nh < 0 || ttl <= 1) { dropped = 1; break; } /* R#12 */
                forward_rewrite(f, &v, &tab[nh], pm, np);
                r.port = tab[nh].port;
                break;
            }
            case OR_IPSEC: {
                uint8_t t[36];
                size_t tl = tuple_bytes(&v, t);
                uint32_t sa = or_toeplitz(MS_RSS_KEY, t, tl) % s->n_sa;
                uint32_t seq = seq_override ? seq_override[i] : ++c->seq[sa];
                int ol = esp_apply(c, f, flen, &v, sa, seq, stats);
                f -= 16;
                flen = ol;
                r.esp_sa = (uint8_t)sa;
                r.esp_seq = seq;
                r.out_len = (uint16_t)ol;
                sa_pkts[sa]++;
                parse(f, flen, &v); /* NFs after ESP see proto 50, ports 0 */
                break;
            }
            case OR_LB: {
                uint8_t t[36];
                size_t tl = tuple_bytes(&v, t);
                uint32_t h = or_toeplitz(s->lb_key, t, tl);
                uint32_t b = (uint32_t)(((uint64_t)h * s->n_lb) >> 32);
                r.lb_backend = (uint16_t)b;
                r.port = s->lb_port[b];
                lb_hits[b]++;
                break;
            }
            case OR_NAT:
                pass = !nat_apply(s, f, &v, r.port);
                break;
            default:
                break;
            }
            if (dropped) { ps[1]++; r.drop_nf = (uint8_t)p; }
            else if (pass) ps[2]++;
            else ps[3]++;
        }
        if (dropped) {
            r.port = 0xFFFF;
            stats[OR_ST_DROP]++;
        } else {
            stats[OR_ST_FWD]++;
            stats[OR_ST_BYTES_OUT] += r.out_len;
        }
        res[i] = r;
    }
    if (n_pairs > match_cap) stats[OR_ST_MATCH_OVF] += n_pairs - match_cap;
    free(ids);
    return n_pairs;
}

/* ======================================================================
 * SFC parallelization with packet copies and XOR merge (P:L243-263
 * [SIV.B.1]; semantics in oracle.h).  Written independently of oracle_run
 * above (which stays the definition): each NF here acts on a private copy
 * and reports its effects, which the group merge then commits.
 * ==================================================================== */
typedef struct {
    int dropped, pass;              /* verdict of this NF on its copy */
    int set_port; uint16_t port;
    int acl; uint16_t acl_rule; uint32_t acl_hit;
    int lb; uint16_t lb_backend;
    int dpi; uint32_t n_ids; uint32_t *ids;
} nf_eff;

static void nf_on_copy(or_chain *c, uint32_t p, uint8_t *f, const pview *v, nf_eff *e)
{
    const or_spec *s = &c->s;
    switch (s->kind[p]) {
    case OR_ACL: {                       /* first matching rule */
        int32_t rule = or_acl(c, (uint8_t)v->family, v->src, v->dst, v->sport, v->dport, v->proto);
        uint32_t act;
        e->acl = 1;
        if (rule >= 0) { e->acl_rule = (uint16_t)rule; e->acl_hit = (uint32_t)rule; act = s->acl[rule].action; }
        else { e->acl_rule = 0xFFFF; e->acl_hit = s->n_acl; act = s->acl_default; }
        e->dropped = act == 1;
        break;
    }
    case OR_DPI: {                       /* distinct pattern set of the payload */
        int any_drop = 0;
        e->dpi = 1;
        e->n_ids = s->n_pat ? ac_scan(c, f + v->pl_off, (size_t)(v->ip_end - v->pl_off), e->ids, s->n_pat, &any_drop) : 0;
        qsort(e->ids, e->n_ids, sizeof(uint32_t), cmp_u32);
        e->dropped = any_drop;
        break;
    }
    case OR_LPM4:
    case OR_LPM6: {
        int want = s->kind[p] == OR_LPM4 ? 4 : 6;
        if (v->family != want) { e->pass = 1; break; }
        int32_t nh;
        const or_nexthop *tab;
        if (want == 4) {
            uint32_t d = ((uint32_t)v->dst[0] << 24) | ((uint32_t)v->dst[1] << 16) | ((uint32_t)v->dst[2] << 8) | v->dst[3];
            nh = or_lpm4(c, d); tab = s->nh4;
        } else {
            nh = or_lpm6(c, v->dst); tab = s->nh6;
        }
        int ttl = want == 4 ? f[22] : f[21];
        if (nh < 0 || ttl <= 1) { e->dropped = 1; break; }       /* R#12 */
        forward_rewrite(f, v, &tab[nh], want == 4 ? s->pmac4 : s->pmac6, want == 4 ? s->n_port4 : s->n_port6);
        e->set_port = 1;
        e->port = tab[nh].port;
        break;
    }
    case OR_LB: {                        /* flow hash -> backend */
        uint8_t t[36];
        size_t tl = tuple_bytes(v, t);
        uint32_t h = or_toeplitz(s->lb_key, t, tl);
        uint32_t b = (uint32_t)(((uint64_t)h * s->n_lb) >> 32);
        e->lb = 1;
        e->lb_backend = (uint16_t)b;
        e->set_port = 1;
        e->port = s->lb_port[b];
        break;
    }
    default:
        break;
    }
}

uint64_t oracle_run_reorg(or_chain *c, const uint8_t *group, uint8_t *arena, const uint64_t *off,
                          const uint16_t *len, uint32_t n, uint64_t first_global, or_result *res,
                          uint32_t *match_pkt, uint16_t *match_pat, uint64_t match_cap, uint64_t *stats)
{
    const or_spec *s = &c->s;
    /* grouping must be consecutive from 0; IPSEC alone in its group */
    if (s->n_nf == 0 || group[0] != 0) return UINT64_MAX;
    for (uint32_t p = 1; p < s->n_nf; p++)
        if (group[p] != group[p - 1] && group[p] != group[p - 1] + 1) return UINT64_MAX;
    for (uint32_t p = 0; p < s->n_nf; p++)
        if ((s->kind[p] == OR_IPSEC || s->kind[p] == OR_NAT) &&
            ((p > 0 && group[p - 1] == group[p]) || (p + 1 < s->n_nf && group[p + 1] == group[p])))
            return UINT64_MAX;   /* IPSEC and NAT stand alone (R#29, R#30) */
    uint64_t n_pairs = 0;
    uint64_t *acl_hits = stats + OR_ST_VAR_BASE;
    uint64_t *lb_hits = acl_hits + s->n_acl + 1;
    uint64_t *sa_pkts = lb_hits + s->n_lb;
    uint32_t *idbuf = (uint32_t *)malloc((size_t)8 * (s->n_pat + 1) * sizeof(uint32_t));
    uint8_t *orig = (uint8_t *)malloc(65536), *copy = (uint8_t *)malloc((size_t)8 * 65536);
    for (uint32_t i = 0; i < n; i++) {
        uint8_t *f = arena + off[i];
        int flen = len[i];
        or_result r = {0xFF, 0xFF, 0, 0xFFFF, 0xFFFF, 0, (uint16_t)flen, 0};
        stats[OR_ST_PKTS]++;
        stats[OR_ST_BYTES_IN] += (uint64_t)flen;
        pview v;
        int dropped = 0;
        if (!parse(f, flen, &v)) {
            r.drop_nf = 0xFE;
            stats[OR_ST_PARSE_DROP]++;
            dropped = 1;
        }
        uint32_t p0 = 0;
        while (!dropped && p0 < s->n_nf) {
            uint32_t p1 = p0;
            while (p1 + 1 < s->n_nf && group[p1 + 1] == group[p0]) p1++;
            if (s->kind[p0] == OR_NAT) {               /* singleton: applied to the packet itself */
                uint64_t *ps = stats + OR_ST_POS_BASE + 4 * p0;
                ps[0]++;
                if (nat_apply(s, f, &v, r.port)) ps[3]++;
                else ps[2]++;
                p0 = p1 + 1;
                continue;
            }
            if (s->kind[p0] == OR_IPSEC) {             /* singleton: applied to the packet itself */
                uint64_t *ps = stats + OR_ST_POS_BASE + 4 * p0;
                ps[0]++;
                uint8_t t[36];
                size_t tl = tuple_bytes(&v, t);
                uint32_t sa = or_toeplitz(MS_RSS_KEY, t, tl) % s->n_sa;
                uint32_t seq = ++c->seq[sa];
                int ol = esp_apply(c, f, flen, &v, sa, seq, stats);
                f -= 16;
                flen = ol;
                r.esp_sa = (uint8_t)sa;
                r.esp_seq = seq;
                r.out_len = (uint16_t)ol;
                sa_pkts[sa]++;
                ps[3]++;
                parse(f, flen, &v);
                p0 = p1 + 1;
                continue;
            }
            /* duplicate the packet entering the group, run every member on its copy */
            memcpy(orig, f, (size_t)flen);
            nf_eff eff[8];
            uint32_t m = p1 - p0 + 1;
            for (uint32_t j = 0; j < m; j++) {
                memset(&eff[j], 0, sizeof(nf_eff));
                eff[j].ids = idbuf + (size_t)j * (s->n_pat + 1);
                memcpy(copy + (size_t)j * 65536, orig, (size_t)flen);
                nf_on_copy(c, p0 + j, copy + (size_t)j * 65536, &v, &eff[j]);
            }
            /* XOR merge: out = orig ^ OR_j (orig ^ copy_j) */
            for (int k = 0; k < flen; k++) {
                uint8_t acc = 0;
                for (uint32_t j = 0; j < m; j++) acc |= (uint8_t)(orig[k] ^ copy[(size_t)j * 65536 + k]);
                f[k] = (uint8_t)(orig[k] ^ acc);
            }
            /* commit in original order up to the earliest dropper */
            for (uint32_t j = 0; j < m; j++) {
                const uint32_t p = p0 + j;
                uint64_t *ps = stats + OR_ST_POS_BASE + 4 * p;
                nf_eff *e = &eff[j];
                ps[0]++;
                if (e->acl) { r.acl_rule = e->acl_rule; acl_hits[e->acl_hit]++; }
                if (e->dpi) {
                    r.dpi_nmatch = (uint16_t)e->n_ids;
                    for (uint32_t q = 0; q < e->n_ids; q++) {
                        if (n_pairs < match_cap) {
                            match_pkt[n_pairs] = (uint32_t)(first_global + i);
                            match_pat[n_pairs] = (uint16_t)e->ids[q];
                        }
                        n_pairs++;
                    }
                    stats[OR_ST_DPI_PAIRS] += e->n_ids;
                }
                if (e->lb) { r.lb_backend = e->lb_backend; lb_hits[e->lb_backend]++; }
                if (e->set_port) r.port = e->port;
                if (e->dropped) { ps[1]++; r.drop_nf = (uint8_t)p; dropped = 1; break; }
                if (e->pass) ps[2]++;
                else ps[3]++;
            }
            if (!dropped) parse(f, flen, &v);          /* the merged packet enters the next group */
            p0 = p1 + 1;
        }
        if (dropped) {
            r.port = 0xFFFF;
            stats[OR_ST_DROP]++;
        } else {
            stats[OR_ST_FWD]++;
            stats[OR_ST_BYTES_OUT] += r.out_len;
        }
        res[i] = r;
    }
    if (n_pairs > match_cap) stats[OR_ST_MATCH_OVF] += n_pairs - match_cap;
    free(idbuf); free(orig); free(copy);
    return n_pairs;
}
