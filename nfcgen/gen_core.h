/*
 * nfcgen/gen_core.h -- the per-packet body of the seeded synthetic traffic
 * generator, shared by the host generator (gen.c) and the device generator
 * (gen_dev.cu) so both write identical bytes.  Input generator only: no
 * parsing, classification, lookup, checksum, hashing or cryptography -- a
 * counter-based RNG (SplitMix64 finaliser keyed by (seed, stream, index)) and
 * byte assembly.  GEN_FN is `static inline` in C and `__host__ __device__` in CUDA.
 */
#ifndef NFCGEN_GEN_CORE_H
#define NFCGEN_GEN_CORE_H
#include <stdint.h>

#ifdef __CUDACC__
#define GEN_FN static __host__ __device__ inline
#else
#define GEN_FN static inline
#endif

GEN_FN void gen_zero(void *d, unsigned n) { for (unsigned k = 0; k < n; k++) ((uint8_t *)d)[k] = 0; }
GEN_FN void gen_copy(void *d, const void *s, unsigned n) { for (unsigned k = 0; k < n; k++) ((uint8_t *)d)[k] = ((const uint8_t *)s)[k]; }

typedef struct {
    uint64_t seed;
    uint64_t n_flows;
    uint32_t v6_bp;          /* IPv6 share in basis points (0..10000) */
    uint32_t pkt_len;        /* fixed frame length; 0 = IMIX; 1 = uniform 60..1514 */
    uint32_t match_ppm;      /* planted DPI pattern probability, per million packets */
    uint32_t in_acl_pct;     /* % of flows drawn inside a random ACL rule */
    uint32_t tcp_pct;        /* % of non-rule flows that are TCP (rest UDP) */
    uint32_t ttl;            /* TTL / hop limit */
    uint32_t ttl1_ppm;       /* packets with TTL 1 (edge case), per million */
    uint32_t malformed_ppm;  /* malformed frames (edge case), per million */
    uint32_t printable;      /* payload bytes drawn from 0x20..0x7e */
    uint32_t headroom, tailroom;
    uint32_t l4csum;         /* 1: arbitrary (random) TCP/UDP checksum fields, 1/8 of UDP 0 = none */
    /* valid edge-case frames (SURVEY 8(c)(i) parse cases), per million packets */
    uint32_t opt_ppm;        /* IPv4 with options: IHL 6..15 */
    uint32_t frag_ppm;       /* IPv4 fragments: MF set and/or non-zero fragment offset */
    uint32_t tcpopt_ppm;     /* TCP with options: data offset 6..15 */
    uint32_t trailer_ppm;    /* Ethernet trailer: IP length ends 1..46 B before the frame end */
} gen_params;

typedef struct {
    uint32_t n_r4; const uint32_t *r4_prefix; const uint8_t *r4_len;
    uint32_t n_r6; const uint8_t *r6_prefix; const uint8_t *r6_len;   /* 16 B each */
    uint32_t n_acl4; const uint32_t *acl4_idx;                         /* rule indices per family */
    uint32_t n_acl6; const uint32_t *acl6_idx;
    const uint8_t *acl_rules;                                          /* 48 B rules */
    uint32_t n_pat; const uint8_t *pat_blob; const uint32_t *pat_off;
} gen_tables;

enum { S_FLOW = 1, S_FAM, S_INACL, S_RULE, S_SRC, S_DST, S_DST2, S_SP, S_DP, S_ROUTE, S_PROTO, S_LEN,
       S_PAY, S_MATCH, S_PAT, S_POFF, S_TTL, S_BAD, S_BADK, S_SRC2, S_CSUM,
       S_OPT, S_OPTN, S_FRAG, S_FRAGK, S_TOPT, S_TOPTN, S_TRL, S_TRLN, S_OPTB };

GEN_FN uint64_t mix64(uint64_t z)
{
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

GEN_FN uint64_t gen_rnd(uint64_t seed, uint32_t stream, uint64_t idx)
{
    return mix64(mix64(seed * 0xD1B54A32D192ED03ull + stream) ^ idx);
}
#define R(st, i) gen_rnd(p->seed, (st), (i))

/* fill addr bits beyond len with random bits (network order, nbytes 4 or 16) */
GEN_FN uint8_t rnd_byte(uint64_t r0, uint64_t r1, int k) { return (uint8_t)((k < 8 ? r0 : r1) >> (8 * (k & 7))); }
GEN_FN void host_bits(uint8_t *a, const uint8_t *pref, int len, int nbytes, uint64_t r0, uint64_t r1)
{
    for (int k = 0; k < nbytes; k++) {
        const int keep = len - 8 * k; /* prefix bits in this byte */
        const uint32_t m = keep >= 8 ? 0xFFu : keep <= 0 ? 0u : (0xFF00u >> keep) & 0xFFu;
        a[k] = (uint8_t)(((uint32_t)pref[k] & m) | ((uint32_t)rnd_byte(r0, r1, k) & ~m & 0xFFu));
    }
}

typedef struct { int fam; uint8_t src[16], dst[16]; uint16_t sp, dp; uint8_t proto; } flow_t;

GEN_FN void make_flow(const gen_params *p, const gen_tables *t, uint64_t f, flow_t *fl)
{
    gen_zero(fl, sizeof *fl);
    fl->fam = (R(S_FAM, f) % 10000) < p->v6_bp ? 6 : 4;
    int nb = fl->fam == 4 ? 4 : 16;
    uint32_t n_rules = fl->fam == 4 ? t->n_acl4 : t->n_acl6;
    const uint32_t *ridx = fl->fam == 4 ? t->acl4_idx : t->acl6_idx;
    uint8_t zero[16] = {0};
    if (n_rules && (R(S_INACL, f) % 100) < p->in_acl_pct) {
        const uint8_t *rule = t->acl_rules + 48 * (size_t)ridx[R(S_RULE, f) % n_rules];
        host_bits(fl->src, rule + 16, rule[1], nb, R(S_SRC, f), R(S_SRC2, f));
        host_bits(fl->dst, rule + 32, rule[2], nb, R(S_DST, f), R(S_DST2, f));
        uint16_t sl = (uint16_t)(rule[6] | rule[7] << 8), sh = (uint16_t)(rule[8] | rule[9] << 8);
        uint16_t dl = (uint16_t)(rule[10] | rule[11] << 8), dh = (uint16_t)(rule[12] | rule[13] << 8);
        fl->sp = (uint16_t)(sl + R(S_SP, f) % ((uint32_t)sh - sl + 1));
        fl->dp = (uint16_t)(dl + R(S_DP, f) % ((uint32_t)dh - dl + 1));
        fl->proto = rule[4] ? 17 : rule[3];
    } else {
        host_bits(fl->src, zero, 0, nb, R(S_SRC, f), R(S_SRC2, f));
        uint32_t nr = fl->fam == 4 ? t->n_r4 : t->n_r6;
        if (nr) {
            uint64_t k = R(S_ROUTE, f) % nr;
            uint8_t pref[16] = {0};
            int plen;
            if (fl->fam == 4) {
                uint32_t v = t->r4_prefix[k];
                pref[0] = (uint8_t)(v >> 24); pref[1] = (uint8_t)(v >> 16); pref[2] = (uint8_t)(v >> 8); pref[3] = (uint8_t)v;
                plen = t->r4_len[k];
            } else {
                gen_copy(pref, t->r6_prefix + 16 * k, 16);
                plen = t->r6_len[k];
            }
            host_bits(fl->dst, pref, plen, nb, R(S_DST, f), R(S_DST2, f));
        } else {
            host_bits(fl->dst, zero, 0, nb, R(S_DST, f), R(S_DST2, f));
        }
        fl->sp = (uint16_t)R(S_SP, f);
        fl->dp = (uint16_t)R(S_DP, f);
        fl->proto = (R(S_PROTO, f) % 100) < p->tcp_pct ? 6 : 17;
    }
}

/* Shape of packet i: IPv4 header words, TCP data offset, fragment kind, trailer bytes.
 * With every edge ppm at 0 this is IHL 5 / data offset 5 / no fragment / no trailer. */
typedef struct { uint32_t ihl, doff, frag, trailer; } shape_t;

GEN_FN shape_t pkt_shape(const gen_params *p, uint64_t i, int fam, uint8_t proto)
{
    shape_t s = {5, 5, 0, 0};
    if (fam == 4 && (R(S_OPT, i) % 1000000) < p->opt_ppm) s.ihl = 6 + (uint32_t)(R(S_OPTN, i) % 10);
    if (fam == 4 && (R(S_FRAG, i) % 1000000) < p->frag_ppm) s.frag = 1 + (uint32_t)(R(S_FRAGK, i) % 3);
    if (proto == 6 && (R(S_TOPT, i) % 1000000) < p->tcpopt_ppm) s.doff = 6 + (uint32_t)(R(S_TOPTN, i) % 10);
    if ((R(S_TRL, i) % 1000000) < p->trailer_ppm) s.trailer = 1 + (uint32_t)(R(S_TRLN, i) % 46);
    return s;
}

GEN_FN uint32_t frame_len(const gen_params *p, uint64_t i, int fam, uint8_t proto, shape_t *sh)
{
    uint32_t L = p->pkt_len;
    if (L == 0) {
        uint64_t u = R(S_LEN, i) % 10000;
        L = u < 6122 ? 64 : u < 8469 ? 536 : 1360; /* IMIX */
    } else if (L == 1) {
        L = 60 + (uint32_t)(R(S_LEN, i) % (1514 - 60 + 1)); /* uniform ragged lengths (tests) */
    }
    *sh = pkt_shape(p, i, fam, proto);
    uint32_t hdr = (fam == 4 ? 14 + 4 * sh->ihl : 54) + (proto == 6 ? 4 * sh->doff : proto == 17 ? 8 : 0);
    if (L < hdr) L = hdr;
    if (sh->trailer > L - hdr) sh->trailer = L - hdr;   /* the IP packet keeps its L4 header */
    return L;
}

GEN_FN void put16(uint8_t *b, uint32_t v) { b[0] = (uint8_t)(v >> 8); b[1] = (uint8_t)v; }
GEN_FN uint64_t round16(uint64_t x) { return (x + 15) & ~15ull; }

/* Frame length of packet i (and its flow). */
GEN_FN uint32_t gen_len_one(const gen_params *p, const gen_tables *t, uint64_t i)
{
    flow_t fl;
    make_flow(p, t, R(S_FLOW, i) % p->n_flows, &fl);
    shape_t sh;
    return frame_len(p, i, fl.fam, fl.proto, &sh);
}

/* Write packet i (frame length L) at f. */
GEN_FN void gen_fill_one(const gen_params *p, const gen_tables *t, uint64_t i, uint8_t *f, uint32_t L)
{
    const uint8_t mac_d[6] = {0x02, 0, 0, 0, 0, 0x01}, mac_s[6] = {0x02, 0, 0, 0, 0, 0x02};
    flow_t fl;
    make_flow(p, t, R(S_FLOW, i) % p->n_flows, &fl);
    shape_t sh;
    (void)frame_len(p, i, fl.fam, fl.proto, &sh);
    const uint32_t ip_end = L - sh.trailer;
    gen_copy(f, mac_d, 6);
    gen_copy(f + 6, mac_s, 6);
    uint32_t ttl = (R(S_TTL, i) % 1000000) < p->ttl1_ppm ? 1 : p->ttl;
    uint32_t l4;
    if (fl.fam == 4) {
        put16(f + 12, 0x0800);
        f[14] = (uint8_t)(0x40 | sh.ihl); f[15] = 0;
        put16(f + 16, ip_end - 14);
        put16(f + 18, (uint32_t)(i & 0xffff));
        /* DF, not a fragment; or a fragment: MF, a non-zero offset, or both */
        const uint32_t fo = 1 + (uint32_t)(R(S_FRAGK, i) >> 8) % 0x1fff;
        put16(f + 20, sh.frag == 0 ? 0x4000 : sh.frag == 1 ? 0x2000 : sh.frag == 2 ? fo : 0x2000 | fo);
        f[22] = (uint8_t)ttl; f[23] = fl.proto;
        f[24] = f[25] = 0;
        gen_copy(f + 26, fl.src, 4);
        gen_copy(f + 30, fl.dst, 4);
        l4 = 14 + 4 * sh.ihl;
        for (uint32_t j = 34; j < l4; j++) f[j] = (uint8_t)(R(S_OPTB, (i << 6) + j) & 0xff); /* options */
    } else {
        put16(f + 12, 0x86DD);
        f[14] = 0x60; f[15] = 0; f[16] = 0; f[17] = 0;
        put16(f + 18, ip_end - 54);
        f[20] = fl.proto; f[21] = (uint8_t)ttl;
        gen_copy(f + 22, fl.src, 16);
        gen_copy(f + 38, fl.dst, 16);
        l4 = 54;
    }
    uint32_t pl = l4;
    /* checksum fields: 0, or (l4csum) an arbitrary value -- never computed here */
    const uint64_t rc = R(S_CSUM, i);
    const uint32_t ck = p->l4csum ? (uint32_t)(rc & 0xffff) : 0;
    if (fl.proto == 17) {
        put16(f + l4, fl.sp); put16(f + l4 + 2, fl.dp);
        put16(f + l4 + 4, ip_end - l4); put16(f + l4 + 6, ((rc >> 16) & 7) == 0 ? 0 : ck);
        pl = l4 + 8;
    } else if (fl.proto == 6) {
        put16(f + l4, fl.sp); put16(f + l4 + 2, fl.dp);
        uint64_t r = R(S_SP, i);
        for (int b = 0; b < 8; b++) f[l4 + 4 + b] = (uint8_t)(r >> (8 * b));
        f[l4 + 12] = (uint8_t)(sh.doff << 4); f[l4 + 13] = 0x18;
        put16(f + l4 + 14, 0xffff); put16(f + l4 + 16, ck); put16(f + l4 + 18, 0);
        for (uint32_t j = 20; j < 4 * sh.doff; j++) f[l4 + j] = (uint8_t)(R(S_OPTB, (i << 6) + j) >> 8); /* TCP options */
        pl = l4 + 4 * sh.doff;
    }
    /* payload */
    for (uint32_t j = pl; j < L; j++) {
        uint32_t q = j - pl;
        uint64_t r = R(S_PAY, (i << 14) + (q >> 3));
        uint8_t b = (uint8_t)(r >> (8 * (q & 7)));
        f[j] = p->printable ? (uint8_t)(0x20 + b % 95) : b;
    }
    if (t->n_pat && (R(S_MATCH, i) % 1000000) < p->match_ppm) {
        uint64_t pk = R(S_PAT, i) % t->n_pat;
        uint32_t plen = t->pat_off[pk + 1] - t->pat_off[pk];
        if (pl + plen <= ip_end) {
            uint32_t o = pl + (uint32_t)(R(S_POFF, i) % (ip_end - pl - plen + 1));
            gen_copy(f + o, t->pat_blob + t->pat_off[pk], plen);
        }
    }
    if ((R(S_BAD, i) % 1000000) < p->malformed_ppm) {
        switch (R(S_BADK, i) % 5) {
        case 0: put16(f + 12, 0x0806); break;                       /* ARP: not IP */
        case 1: f[14] = (uint8_t)((f[14] & 0x0f) | 0x50); break;    /* bad version */
        case 2: if (fl.fam == 4) put16(f + 16, L); else put16(f + 18, L); break; /* length overrun */
        case 3: if (fl.fam == 4) f[14] = 0x44; else f[14] = 0x40; break;        /* IHL 4 / version 4 in v6 */
        case 4: if (fl.fam == 4) { put16(f + 16, 20 + 4); } else { put16(f + 18, 4); } break; /* L4 truncated */
        }
    }
}

#endif
