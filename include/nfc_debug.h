/*
 * nfc_debug.h -- host-side emulation of the device table images (diagnostics).
 *
 * Each handle holds the device image that nfc_load_tables would upload, built
 * by the same host builders, and walks it on the CPU with the same algorithm
 * the fused kernel uses.  This lets the table builders (Aho-Corasick DFA,
 * DIR-24-8, IPv6 binary search on prefix lengths, ACL image, AES T-tables,
 * Toeplitz nibble tables) be checked on a machine without a GPU.  Not part of
 * the packet path.  Status codes as in nfc.h.
 */
#ifndef NFC_DEBUG_H
#define NFC_DEBUG_H
#include "nfc.h"

#ifdef __cplusplus
extern "C" {
#endif

typedef struct nfc_dbg nfc_dbg;

/* Build the image of `kind` from its logical spec (same validation as nfc_load_tables). */
NFC_API int nfc_dbg_build(uint32_t kind, const void *spec, size_t spec_bytes, nfc_dbg **out);
NFC_API void nfc_dbg_destroy(nfc_dbg *d);

/* DPI: distinct matched pattern ids of buf (ascending, up to cap), count, any-DROP flag. */
NFC_API int nfc_dbg_dpi(nfc_dbg *d, const uint8_t *buf, size_t n, uint16_t *ids, uint32_t cap,
                        uint32_t *count, uint32_t *drop);
/* DPI image shape: states, byte classes, 1 if 32-bit entries. */
NFC_API int nfc_dbg_dpi_shape(nfc_dbg *d, uint32_t *n_states, uint32_t *n_classes, uint32_t *wide);
/* DPI, tiered placement as the kernel's DM_HOT mode walks it: rows of states [0, hot) dense,
   states [hot, hot + sparse) by their sparse record (base row + <= 2 exceptions), the rest
   from the full table.  Same outputs as nfc_dbg_dpi; tier_steps (3 u32, may be NULL) counts
   steps taken from dense rows, sparse records and the full table. */
NFC_API int nfc_dbg_dpi_tier(nfc_dbg *d, uint32_t hot, uint32_t sparse, const uint8_t *buf, size_t n,
                             uint16_t *ids, uint32_t cap, uint32_t *count, uint32_t *drop, uint32_t *tier_steps);
/* DPI, slot image as the kernel's DM_FULL mode walks it (DpiImg::frows: signed slots,
   accepting states negative).  Same outputs as nfc_dbg_dpi; events = accept events of the
   walk; summary = the per-slot match summary the kernel reads when events == 1
   (closure offset | size << 20 | DROP << 31), else 0.  events/summary may be NULL. */
NFC_API int nfc_dbg_dpi_slot(nfc_dbg *d, const uint8_t *buf, size_t n, uint16_t *ids, uint32_t cap,
                             uint32_t *count, uint32_t *drop, uint32_t *events, uint32_t *summary);
/* DPI tier shape: states of depth <= 1, states with a representable sparse record. */
NFC_API int nfc_dbg_dpi_tier_shape(nfc_dbg *d, uint32_t *n_d1, uint32_t *n_sparse_ok);
/* NAT44 translation as the kernel computes it from the device image (nat_values):
   out = {src, dst, sport, dport, tcp/udp checksum} for a packet the NAT applies to;
   probes (may be NULL) = DNAT hash-table slots read. */
NFC_API int nfc_dbg_nat(nfc_dbg *d, uint8_t proto, uint32_t src, uint32_t dst, uint16_t sport, uint16_t dport,
                        uint16_t ck, uint32_t out[5], uint32_t *probes);
/* LPM4: next-hop index (0x7FFF = miss) and number of table reads (1 or 2). */
NFC_API int nfc_dbg_lpm4(nfc_dbg *d, uint32_t dst, uint32_t *nh, uint32_t *reads);
/* LPM6: next-hop index (0x7FFF = miss), hash-level probes and hash-slot reads. */
NFC_API int nfc_dbg_lpm6(nfc_dbg *d, const uint8_t dst[16], uint32_t *nh, uint32_t *probes, uint32_t *slot_reads);
NFC_API int nfc_dbg_lpm6_levels(nfc_dbg *d, uint32_t *n_levels);
/* ACL: first matching rule (0xFFFF none) and the resulting action (0 permit / 1 deny). */
NFC_API int nfc_dbg_acl(nfc_dbg *d, uint32_t family, const uint8_t *src, const uint8_t *dst, uint16_t sport,
                        uint16_t dport, uint8_t proto, uint32_t *rule, uint32_t *action);
/* ACL, IPv4, through the fused kernel's other images: which = 0 the search image of <= 64-rule
 * sets (AclImg::f4), 1 the 16-bit first level of > 2K-rule sets (AclImg::x4); addresses as
 * host-order u32.  NFC_EUNSUP if the rule set has no such image. */
NFC_API int nfc_dbg_acl4_image(nfc_dbg *d, uint32_t which, uint32_t src, uint32_t dst, uint16_t sport, uint16_t dport,
                               uint8_t proto, uint32_t *rule, uint32_t *action);
/* Crypto / hash primitives as the kernel computes them (T-tables, nibble tables, ipad/opad states). */
NFC_API int nfc_dbg_aes128_block(const uint8_t key[16], const uint8_t in[16], uint8_t out[16]);
NFC_API int nfc_dbg_toeplitz(const uint8_t key[40], const uint8_t *in, size_t n, uint32_t *h);
NFC_API int nfc_dbg_hmac_sha1(const uint8_t key[20], const uint8_t *msg, size_t n, uint8_t out[20]);

#ifdef __cplusplus
}
#endif
#endif
