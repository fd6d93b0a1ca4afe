/*
 * nfcgen/gen.c -- seeded synthetic traffic generator (input generator only).
 *
 * Serves both the oracle and the CUDA path with identical packet bytes.  It
 * holds none of the method's arithmetic: no parsing, classification, lookup,
 * checksum, hashing or cryptography -- only a counter-based RNG
 * (SplitMix64 finaliser keyed by (seed, stream, index)) and byte assembly.
 * The IPv4 header checksum is left 0 (NIC checksum-offload convention; input
 * checksums are never verified, R#13).
 *
 * Every packet is a pure function of (params, tables, global index), so any
 * index range can be generated independently (sharding, sampled parity).
 * Workload recipe: DESIGN.md "Synthetic inputs"; traffic model P:L136
 * ("randomly generated IP traffic with UDP payloads"), IMIX P:L361.
 */
#include <stdint.h>
#include <string.h>

#include "gen_core.h"

uint64_t nfcgen_rnd(uint64_t seed, uint32_t stream, uint64_t idx) { return gen_rnd(seed, stream, idx); }

/* The 5-tuple of flow f (table generators use it to draw entries real flows hit). */
void nfcgen_flow(const gen_params *p, const gen_tables *t, uint64_t f, uint32_t *fam, uint8_t *src, uint8_t *dst,
                 uint16_t *sp, uint16_t *dp, uint8_t *proto)
{
    flow_t fl;
    make_flow(p, t, f, &fl);
    *fam = (uint32_t)fl.fam;
    memcpy(src, fl.src, 16);
    memcpy(dst, fl.dst, 16);
    *sp = fl.sp;
    *dp = fl.dp;
    *proto = fl.proto;
}

/* Slot size of packet i (headroom + frame + tailroom, 16-B aligned). */
uint64_t nfcgen_layout(const gen_params *p, const gen_tables *t, uint64_t first, uint32_t n, uint64_t base,
                       uint64_t *off, uint16_t *len)
{
    uint64_t pos = base;
    for (uint32_t k = 0; k < n; k++) {
        uint32_t L = gen_len_one(p, t, first + k);
        off[k] = pos + p->headroom;
        len[k] = (uint16_t)L;
        pos += round16((uint64_t)p->headroom + L + p->tailroom);
    }
    return pos;
}

/* Write packets [first, first+n) at the offsets from nfcgen_layout. */
void nfcgen_fill(const gen_params *p, const gen_tables *t, uint64_t first, uint32_t n, uint8_t *arena,
                 const uint64_t *off, const uint16_t *len)
{
    for (uint32_t k = 0; k < n; k++) gen_fill_one(p, t, first + k, arena + off[k], len[k]);
}
