/*
 * oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, single-threaded C11 oracle for the NFCompass (Hu & Li, HPCA'18)
 * service-function-chain hot path.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.  The
 * product path (paper_conf_hpca_hul18_b200/) never includes, links or calls it,
 * and this file includes nothing from the product.
 *
 * Citations: "P:Lnn" = /root/reference/PAPER.md line nn (section in brackets);
 * "R#k" = reading k in DESIGN.md section "Readings of the paper".
 *
 * The binary layouts of the logical specs below are the interface both sides
 * read; they are declared here
 * independently of include/nfc.h.
 */
#ifndef NFC_ORACLE_H
#define NFC_ORACLE_H
#include <stdint.h>
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

/* NF kinds, in the numbering of the logical chain spec. */
enum { OR_ACL = 1, OR_DPI = 2, OR_LPM4 = 3, OR_LPM6 = 4, OR_IPSEC = 5, OR_LB = 6, OR_NAT = 7 };

/* 48 B ACL rule (P:L219 firewall; P:L383 ClassBench-style 5-tuple rules). */
typedef struct {
    uint8_t family;     /* 4 or 6 */
    uint8_t slen, dlen; /* prefix lengths */
    uint8_t proto;
    uint8_t proto_any;  /* 1 = wildcard protocol */
    uint8_t action;     /* 0 PERMIT, 1 DENY */
    uint16_t sp_lo, sp_hi, dp_lo, dp_hi;
    uint8_t pad[2];
    uint8_t src[16], dst[16]; /* network byte order; IPv4 uses bytes 0..3 */
} or_acl_rule;

typedef struct { uint32_t prefix; uint8_t len; uint8_t pad; uint16_t nh; } or_route4;      /* 8 B  */
typedef struct { uint8_t prefix[16]; uint16_t nh; uint8_t len; uint8_t pad; } or_route6;   /* 20 B */
typedef struct { uint16_t port; uint8_t mac[6]; } or_nexthop;                              /* 8 B  */
typedef struct {                                                                          /* 48 B */
    uint32_t spi, seq0;
    uint8_t aes_key[16];
    uint8_t nonce[4];
    uint8_t auth_key[20];
} or_sa;

/* NAT44 tables ("the NAT network function performs source and destination
 * NAT"; Table II row NAT: reads and writes the header, never drops; R#30). */
typedef struct { uint32_t prefix; uint8_t len; uint8_t pad[3]; } or_nat_prefix;          /* 8 B  */
typedef struct {                                                                          /* 16 B */
    uint32_t ext_addr; uint16_t ext_port; uint8_t proto; uint8_t pad;
    uint32_t int_addr; uint16_t int_port; uint16_t pad2;
} or_nat_dnat;

typedef struct {
    uint32_t n_nf;
    uint8_t kind[8];           /* kind[p] for chain position p (original SFC order) */
    /* ACL */
    const or_acl_rule *acl; uint32_t n_acl; uint32_t acl_default; /* default action 0/1 */
    /* DPI */
    const uint8_t *pat_blob; const uint32_t *pat_off; const uint8_t *pat_action; uint32_t n_pat;
    /* LPM4 */
    const or_route4 *r4; uint32_t n_r4; const or_nexthop *nh4; uint32_t n_nh4;
    const uint8_t *pmac4; uint32_t n_port4;
    /* LPM6 */
    const or_route6 *r6; uint32_t n_r6; const or_nexthop *nh6; uint32_t n_nh6;
    const uint8_t *pmac6; uint32_t n_port6;
    /* IPSEC */
    const or_sa *sa; uint32_t n_sa;
    /* LB */
    const uint16_t *lb_port; uint32_t n_lb; const uint8_t *lb_key; /* 40 B Toeplitz key */
    /* NAT (R#30): addresses are host-order u32 values */
    const or_nat_prefix *nat_inside; uint32_t n_nat_inside;
    const uint32_t *nat_pool; uint32_t n_nat_pool;
    uint32_t nat_port_lo, nat_port_hi;
    const or_nat_dnat *nat_dnat; uint32_t n_nat_dnat;
    uint32_t nat_ext_ports;    /* bit p: egress port p faces the Internet */
    const uint8_t *nat_key;    /* 40 B Toeplitz key of the translation hash */
} or_spec;

/* 16 B per-packet record (identical layout on both sides). */
typedef struct {
    uint8_t drop_nf;     /* 0xFF forwarded; 0xFE parse failure; else chain position */
    uint8_t esp_sa;      /* 0xFF if ESP not applied */
    uint16_t port;       /* egress port; 0 if none set; 0xFFFF if dropped */
    uint16_t acl_rule;   /* first matching rule; 0xFFFF none / not reached */
    uint16_t lb_backend; /* 0xFFFF if not reached */
    uint16_t dpi_nmatch; /* number of distinct matched pattern IDs */
    uint16_t out_len;    /* frame length after the chain */
    uint32_t esp_seq;    /* ESP sequence number, 0 if not applied */
} or_result;

/* stats vector (u64) layout */
#define OR_ST_PKTS 0
#define OR_ST_BYTES_IN 1
#define OR_ST_FWD 2
#define OR_ST_DROP 3
#define OR_ST_BYTES_OUT 4
#define OR_ST_PARSE_DROP 5
#define OR_ST_DPI_PAIRS 6
#define OR_ST_MATCH_OVF 7
#define OR_ST_ESP_PKTS 8
#define OR_ST_ESP_BYTES 9
#define OR_ST_ESP_BLOCKS 10
#define OR_ST_POS_BASE 16 /* + 4*p + {0 in, 1 drop, 2 pass-through, 3 applied} */
#define OR_ST_VAR_BASE 64 /* acl_hits[n_acl], acl_default_hits, lb_hits[n_lb], sa_pkts[n_sa] */

typedef struct or_chain or_chain;

or_chain *oracle_create(const or_spec *spec);
void oracle_destroy(or_chain *c);
size_t oracle_stats_len(const or_chain *c);

/* Run packets [0,n) in order.  arena is modified in place (frames may grow into
 * tailroom and ESP moves the frame start 16 B left into headroom).  If
 * seq_override != NULL, ESP uses seq_override[i] instead of the per-SA counter
 * (sampled parity at full size).  Returns number of match pairs
 * produced (may exceed match_cap; pairs beyond the cap are not written). */
uint64_t oracle_run(or_chain *c, uint8_t *arena, const uint64_t *off, const uint16_t *len,
                    uint32_t n, uint64_t first_global, or_result *res,
                    uint32_t *match_pkt, uint16_t *match_pat, uint64_t match_cap,
                    uint64_t *stats, const uint32_t *seq_override);

/* SFC parallelization (P:L243-263 [SIV.B.1], Figs. 13-14): the chain is cut into
 * groups of consecutive positions (group[p], non-decreasing from 0, consecutive);
 * every NF of a group receives its own copy of the packet entering the group
 * ("creates the copy of network packets and distributes them"), and the
 * copies are merged by the paper's XOR rule: out = orig ^ OR_f (orig ^
 * f(orig)).  Verdict: dropped iff some member dropped, at the smallest such
 * position; side effects of members after that position are discarded ("the
 * alert or log operation should be executed in the same packet state",
 * P:L269).  Egress port: last setter in original order (R#19).  A group holding
 * IPSEC must hold only IPSEC (it grows the packet, Table II "Add/Rm").
 * Returns the number of match pairs, or UINT64_MAX if the grouping is invalid.
 * Same outputs as oracle_run exactly when every group is parallel-legal. */
uint64_t oracle_run_reorg(or_chain *c, const uint8_t *group, uint8_t *arena, const uint64_t *off,
                          const uint16_t *len, uint32_t n, uint64_t first_global, or_result *res,
                          uint32_t *match_pkt, uint16_t *match_pat, uint64_t match_cap, uint64_t *stats);

/* ---- individual primitives, exported for the pin tests ---- */
void or_aes128_encrypt_block(const uint8_t key[16], const uint8_t in[16], uint8_t out[16]);
void or_aes128_ctr(const uint8_t key[16], const uint8_t ctr_block0[16], const uint8_t *in,
                   uint8_t *out, size_t n);
void or_sha1(const uint8_t *msg, size_t n, uint8_t out[20]);
void or_hmac_sha1(const uint8_t *key, size_t klen, const uint8_t *msg, size_t n, uint8_t out[20]);
uint32_t or_toeplitz(const uint8_t key[40], const uint8_t *in, size_t n);
uint16_t or_ipv4_checksum(const uint8_t *hdr, size_t hlen);
/* RFC 1624 eqn. 3: checksum after one 16-bit field changes from m to m1 */
uint16_t or_csum_update(uint16_t hc, uint16_t m, uint16_t m1);
/* DPI: distinct pattern set of one byte string; returns |M|, writes sorted IDs into ids (cap). */
uint32_t or_ac_match(or_chain *c, const uint8_t *buf, size_t n, uint32_t *ids, uint32_t cap);
/* LPM: next hop index or -1 */
int32_t or_lpm4(or_chain *c, uint32_t dst);
int32_t or_lpm6(or_chain *c, const uint8_t dst[16]);
/* ACL: first matching rule or -1 (family 4 or 6; addresses in network order) */
int32_t or_acl(or_chain *c, uint8_t family, const uint8_t *src, const uint8_t *dst,
               uint16_t sport, uint16_t dport, uint8_t proto);

/* Parse of SURVEY 8(c)(i) 1 (test hook): out = {ok, family, l4_off, ip_end, pl_off, proto, sport, dport}. */
int or_parse(const uint8_t *f, int flen, int32_t out[8]);

#ifdef __cplusplus
}
#endif
#endif
