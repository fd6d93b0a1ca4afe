// nfc_internal.h -- device image formats and kernel parameters shared by the
// host table builders (builders.cpp), the C ABI (capi.cu) and the fused
// kernel (sfc_kernel.cu).  Product code only; nothing here is seen by oracle/.
#pragma once
#include <stdint.h>
#include <vector_functions.h>
#include <vector_types.h>
#include <string>
#include <vector>

#include "../../include/nfc.h"

#ifndef NFC_REGROUP
#define NFC_REGROUP 0         // 1: a3 regrouping -- the IPv6 packets of mixed chunks deferred to a per-warp queue
                              //    (family-pure chunks); measured slower than the mixed chunks (DESIGN.md a3)
#endif

namespace nfc {

// ---------------------------------------------------------------- ACL
// Bit-vector image per family (u32 blob):
//   [0] n rules of the family  [1] W = 64-bit words per bitset  [2..5] interval counts
//   m_src, m_dst, m_sport, m_dport  [6] key words per address (1 v4, 4 v6)
//   [8..17] word offsets: keys_src, bv_src, keys_dst, bv_dst, keys_sp, bv_sp, keys_dp, bv_dp,
//   bv_proto (256 x W), ridx (global rule index | action << 31),  [18..21] bucket tables
//   (257 u16 per field) on the top 8 key bits,  [22] search steps per field (8 bits each),
//   [23] max steps.  Key arrays are 16-B aligned and followed by 2^maxsteps all-ones pad keys.  Bitsets are
//   u64 at even offsets.
static const uint32_t ACLBV_HDR = 32;   // [24..28] aggregate-row offsets, [29] WA
struct AclImg {
    const uint32_t *bv4, *bv6;        // device blobs
    uint32_t words4, words6;          // blob sizes (u32 words)
    uint32_t n_rules;
    uint32_t default_action;
    uint32_t smem_words;              // words staged in shared memory (0 = read from global)
    uint32_t hdr4[ACLBV_HDR], hdr6[ACLBV_HDR];   // image headers, read from the constant bank
    // Search image of an IPv4 rule set with W == 1 and window depth <= 3 (build_acl4_fast):
    // what the fused kernel stages in shared memory in place of the IPv4 blob (fast = 1)
    const uint32_t *f4;               // device copy (nullptr: not representable)
    uint32_t words_f4;                // its size (u32 words, 16-B multiple)
    uint32_t fast;                    // per launch: 1 = the fused kernel stages f4 (acl4_fast)
    uint32_t f4_key[4], f4_bv[4];     // byte offsets of the key and bitset arrays per field
    uint32_t f4_d3;                   // 1: some bucket window needs a third halving (else two)
    // 16-bit first level of an IPv4 rule set read from global memory (W > 32: the 10K
    // rule set), build_acl4_index: 4 x 65536 u16 -- the interval of (src >> 16) << 16 and
    // of (dst >> 16) << 16 (window searches of d16 & 255 / d16 >> 8 halvings follow),
    // and the interval of every source / destination port (no search)
    const uint16_t *x4;
    uint32_t d16;
};
// Search image layout (byte offsets): four 256-entry u16 bucket tables (src, dst,
// sport, dport) on the top 8 key bits, each entry the byte offset of the window's
// first key; the proto bitsets (256 x u64); the rule words (<= 64 x u32); then per
// field the interval start keys (u32) and, apart, their bitsets (u64), both followed by
// 8 copies of the last entry, so a 3-halving window search needs no clamp and the
// bitset of key j sits at a fixed affine image of the key's address (bv + 2 (key - k0)).
#ifndef NFC_ACLF_BITS
#define NFC_ACLF_BITS 9       // search image buckets: the top NFC_ACLF_BITS bits of each key (9 and 10: same C1; 9 saves 4 KB)
#endif
static const uint32_t ACLF_NB = 1u << NFC_ACLF_BITS;                 // buckets per field
static const uint32_t ACLF_BK = 0, ACLF_PROTO = 8 * ACLF_NB, ACLF_RULE = ACLF_PROTO + 2048, ACLF_REC = ACLF_RULE + 256;

// ---------------------------------------------------------------- DPI
// Full Aho-Corasick DFA over byte classes, states numbered in BFS order.
// trans[s * ncls + cls[b]] = next | ACCEPT (bit 15 for u16, bit 31 for u32
// entries) where ACCEPT means the next state has a non-empty output set.
// out_off/out_ids: CSR of the output closure (sorted distinct pattern ids).
struct DpiImg {
    const uint8_t *cls;          // 256 byte -> class
    const void *trans;           // u16 or u32 entries
    uint32_t ncls, n_states, wide;
    const uint32_t *out_off;     // n_states + 1
    const uint16_t *out_ids;
    const uint8_t *pat_action;   // n_pat
    uint32_t n_pat;
    uint32_t *ovf_bitmap;        // per resident thread scratch for > DPI_LIST distinct matches
    uint32_t bitmap_words;       // words per thread
    uint32_t hot_states;         // states whose full 256-byte rows are staged in shared memory
    uint32_t row2, hk2;          // per launch: bytes per DFA row (2 ncls); byte offset of the last hot entry
    const uint32_t *out_meta;    // per state: out_off (the pattern id if n_out == 1) | n_out << 20 | any DROP << 31
                                 // (DPI_META_NONE if the closure does not fit the fields)
    uint32_t meta_smem;          // 1: out_meta staged in shared memory
    // Tiered placement (DM_HOT): rows of states [0, hot_states) are dense in shared
    // memory; states [hot_states, hot_states + sparse_states) are sparse records in
    // shared memory; the rest are read from `trans` (cold).  A sparse record describes
    // a state s by a dense base state b (the first state of depth <= 1 on s's failure
    // chain) and the <= 2 classes where s's row differs from b's row:
    //   x = b | c0 << 16 | c1 << 24,  y = e0 | e1 << 16   (b = 0xFFFF: not representable, cold)
    // next(s, c) = c == c0 ? e0 : c == c1 ? e1 : row(b)[c].
    const uint2 *sparse;         // n_states records (entries [0, n_d1) unused)
    uint32_t n_d1;               // states of depth <= 1
    uint32_t maxlen;             // longest pattern (bytes): a walk started maxlen - 1 bytes
                                 // early is in the exact state (warp-split payload walks)
    uint32_t sparse_states;      // per launch: records staged in shared memory
    // Slot image (DM_FULL, the whole DFA in shared memory).  A state is named by a
    // signed slot: non-accepting states 0, 1, 2, ... (root = 0), accepting states
    // -1, -2, ... (both in BFS order).  Rows are stored so that the row of slot x
    // starts x * row2 bytes from the row of slot 0 (accepting rows below it), and an
    // entry is the next state's slot (s16).  A step is then one multiply-add and one
    // sign-extending load, the accept test is the sign bit, and the unique accepting
    // entry of a walk with one accept event is its largest entry as u32.
    const int16_t *frows;        // n_states * ncls entries, physical row order
    const uint32_t *acc_id;      // n_acc: BFS state id of accepting slot -(q+1)
    const uint32_t *acc_meta;    // n_acc: out_meta of accepting slot -(q+1)
    uint32_t n_acc;
};
static const uint32_t DPI_META_NONE = 0x7FFFFFFFu;

// ---------------------------------------------------------------- LPM4 (DIR-24-8)
// tbl24[dst>>8]: bit 15 set -> long group g = v & 0x7FFF, nh = tbllong[g*256 + (dst&255)];
// else nh = v.  nh == 0x7FFF means no route.
struct Lpm4Img {
    const uint16_t *tbl24;
    const uint16_t *tbllong;
    const uint2 *nh;             // {port | mac0<<16 | mac1<<24, mac2..mac5}
    const uint2 *pmac;           // per port: {mac0..3, mac4|mac5<<8}
    uint32_t n_nh, n_ports;
    uint32_t nh_smem;            // per launch: 1 = {nh, pmac[port]} records (16 B) staged in shared memory
};

// ---------------------------------------------------------------- LPM6 (Waldvogel)
// Binary search on the sorted distinct prefix lengths; one hash table per
// length holding real prefixes and markers, each entry carrying the best
// matching real prefix (bmp) of length <= its level.
struct Lpm6Entry { uint32_t key[4]; uint32_t info; uint32_t pad[3]; }; // info: bmp | VALID
static const uint32_t L6_VALID = 0x80000000u;
struct Lpm6Img {
    uint32_t n_levels;
    uint32_t def_nh;             // ::/0 next hop or 0x7FFF
    const uint8_t *lens;         // n_levels
    const uint32_t *base;        // entry offset per level
    const uint32_t *mask;        // table size - 1 per level
    const uint4 *ent;            // 2 x uint4 per entry
    const uint2 *nh;
    const uint2 *pmac;
    uint32_t n_nh, n_ports;
};

// ---------------------------------------------------------------- IPsec
struct EspSa {                   // 256 B
    uint32_t rk[44];             // AES-128 round keys, big-endian words (FIPS-197 w[i])
    uint32_t spi, nonce;         // nonce as big-endian word
    uint32_t ipad[5], opad[5];   // SHA-1 states after the HMAC ipad / opad blocks
    uint32_t pad[8];
};
static_assert(sizeof(EspSa) == 256, "EspSa must stay 16-B aligned in arrays");
// round keys staged in shared memory per SA at an odd word stride (bank spread)
static const uint32_t ESP_RK_STRIDE = 45;
struct EspImg {
    const EspSa *sa;
    uint32_t n_sa;
    const uint32_t *te;          // Te0..Te3 (4 x 256 words) + sbox (256 words)
    const uint32_t *rss_nib;     // Toeplitz nibble table for the MS RSS key (72 x 16)
};

struct LbImg {
    const uint16_t *port;
    uint32_t n_backends;
    const uint32_t *nib;         // Toeplitz nibble table of the LB key (72 x 16)
};

// ---------------------------------------------------------------- NAT44 (R#30)
// Inside prefixes in the constant bank (uniform loop); DNAT entries in an
// open-addressing table: {ext_addr, ext_port | proto << 16 | NAT_VALID, int_addr,
// int_port}, slot = nat_slot(ext_addr, ext_port | proto << 16) & mask, linear probing.
static const uint32_t NAT_MAX_INSIDE = 64, NAT_VALID = 0x80000000u;
__host__ __device__ inline uint32_t nat_slot(uint32_t a, uint32_t b)
{
    uint32_t x = a * 0x9E3779B1u ^ (b + 0x7F4A7C15u) * 0x85EBCA77u;
    x ^= x >> 15;
    x *= 0x2C1B3C6Du;
    return x ^ (x >> 13);
}
struct NatImg {
    uint32_t n_inside;
    uint32_t in_pref[NAT_MAX_INSIDE], in_mask[NAT_MAX_INSIDE];
    const uint32_t *pool;
    uint32_t n_pool, port_lo, port_range;
    const uint4 *dnat;
    uint32_t dnat_mask;
    uint32_t ext_ports;
    const uint32_t *nib;         // Toeplitz nibble table of the NAT key (72 x 16)
};

// ---------------------------------------------------------------- launch
struct BatchDev { uint8_t *arena; const uint64_t *off; const uint16_t *len; uint32_t n; uint32_t start; uint64_t first; };
// Multi-batch calls: one 32-B record per 32-packet chunk (built on the device by
// k_chunk_recs before the fused kernel), for the batch of the chunk's first packet:
// packet g of that batch has off = offp[g], len = lenp[g], bytes at arena + off and
// global index gb + g.  meta = lane where the next batch starts (0: none) | 1<<5 if
// the chunk holds more than one batch boundary (those lanes take the binary search).
struct ChunkRec { const uint64_t *offp; const uint16_t *lenp; uint8_t *arena; uint32_t gb_lo, meta; };  // gb_lo: (first - start) mod 2^32
static_assert(sizeof(ChunkRec) == 32, "ChunkRec is 32 B");

enum { MASK_ACL = 1u << NFC_ACL, MASK_DPI = 1u << NFC_DPI, MASK_LPM4 = 1u << NFC_LPM4,
       MASK_LPM6 = 1u << NFC_LPM6, MASK_IPSEC = 1u << NFC_IPSEC, MASK_LB = 1u << NFC_LB,
       MASK_NAT = 1u << NFC_NAT };

// stats vector layout
enum { ST_PKTS = 0, ST_BYTES_IN, ST_FWD, ST_DROP, ST_BYTES_OUT, ST_PARSE_DROP, ST_DPI_PAIRS,
       ST_MATCH_OVF, ST_ESP_PKTS, ST_ESP_BYTES, ST_ESP_BLOCKS, ST_DPI_OVF_PKTS, ST_MIXED_CHUNKS,
       ST_POS_BASE = 16, ST_VAR_BASE = 64 };

// byte offsets of the kernel's dynamic shared-memory regions (computed on the host per
// launch, read by the kernel from the constant bank)
struct SmemLayout {
    uint32_t wst, vst, te, ms_nib, lb_nib, cls, hot, sp, meta, seg, acl4, acl6, wcnt, prefix, par, total;
    uint32_t frow0;
    uint32_t nat_nib;             // NAT Toeplitz nibbles
    uint32_t nh4;                 // LPM4 next-hop records (Lpm4Img::nh_smem)
    uint32_t rk;                  // ESP: AES round keys of every SA, ESP_RK_STRIDE words each
    uint32_t crs;                 // multi-batch: per-warp chunk-record staging (2 x 32 B, cp.async)
    uint32_t rgq;                 // a3 regrouping: per-warp queue of deferred IPv6 packet indices
};

struct KParams {
    SmemLayout lay;
    uint32_t n_nf;
    uint32_t kind[NFC_MAX_CHAIN];
    uint32_t esp_pos;            // chain position of IPSEC or 0xFF
    uint32_t present;            // MASK_* bits of the NFs in the chain
    // work
    const BatchDev *batches;
    BatchDev b0;                 // batches[0] (constant bank: no descriptor loads for single-batch calls)
    uint32_t n_batches;
    uint32_t n_pkts;
    uint32_t n_tiles;
    uint32_t claim;              // 32-packet chunks per work claim (set by the launcher)
    const ChunkRec *crec;        // n_batches > 1: one record per 32-packet chunk (else nullptr)
    uint32_t *mix;               // a3: mixed IPv4/IPv6 chunks of this launch (device u32, zeroed per launch)
    uint8_t group[NFC_MAX_CHAIN]; // NFC_F_PARALLEL: parallel group of each chain position (runs, in order)
    uint32_t n_groups;
    uint32_t *tile_counter;
    // outputs
    nfc_pkt_result *rec;
    uint32_t *match_pkt;
    uint16_t *match_pat;
    uint32_t match_cap;
    uint32_t *match_count;
    unsigned long long *stats;
    uint32_t stats_len;
    uint32_t st_acl, st_lb, st_sa;  // bases of the variable stats sections
    uint32_t smem_stats;            // 1 = accumulate stats in shared memory
    // ESP sequence look-back
    uint32_t *tile_flag;            // n_tiles flags (epoch << 2 | status)
    uint32_t *tile_vec;             // n_tiles x 2 x n_sa (aggregate, inclusive prefix)
    uint32_t epoch;
    const uint32_t *seq_in;
    uint32_t *seq_out;
    // tables
    AclImg acl;
    DpiImg dpi;
    Lpm4Img l4;
    Lpm6Img l6;
    EspImg esp;
    LbImg lb;
    NatImg nat;
};

// host-side builders (builders.cpp); return "" on success or an error message
int set_fail(int code, const std::string &msg);
// comm.cu: in-place u64 sum across the ranks of an NCCL communicator, on st
int comm_allreduce_u64(void *comm, unsigned long long *dev, size_t n, cudaStream_t st);
struct DpiHost;
std::string build_regex_dfa(const nfc_dpi_spec &s, DpiHost &o, uint32_t max_states);   // regex.cpp   // capi.cu: nfc_last_error + code
struct HostImage { std::vector<uint8_t> bytes; };
std::string build_acl(const nfc_acl_spec &s, std::vector<uint32_t> &blob4, std::vector<uint32_t> &blob6);
// the record image (AclImg::f4) of an IPv4 blob; empty if the blob does not qualify
void build_acl4_index(const std::vector<uint32_t> &blob4, std::vector<uint16_t> &x, uint32_t &d16);
void build_acl4_fast(const std::vector<uint32_t> &blob4, std::vector<uint32_t> &f, uint32_t key_off[4], uint32_t bv_off[4],
                     uint32_t &d3);
struct DpiHost {
    std::vector<uint8_t> cls;
    std::vector<uint8_t> trans;   // raw bytes (u16 or u32 entries)
    uint32_t ncls = 0, n_states = 0, wide = 0;
    std::vector<uint32_t> out_off;
    std::vector<uint16_t> out_ids;
    std::vector<uint8_t> action;
    std::vector<uint32_t> out_meta;
    uint32_t n_d1 = 0;               // states of depth <= 1 (BFS ids [0, n_d1))
    uint32_t maxlen = 0;             // longest pattern
    std::vector<uint2> sparse;       // per state: tier record (see DpiImg::sparse)
    // slot image (DpiImg::frows), u16 DFAs only
    std::vector<int16_t> frows;      // n_states rows of ncls signed slots, physical order
    std::vector<uint32_t> acc_id;    // accept slot q (slot -(q+1)) -> BFS state id
    std::vector<uint32_t> acc_meta;  // out_meta of accept slot q
    uint32_t n_acc = 0;
};
std::string build_dpi(const nfc_dpi_spec &s, DpiHost &out);
std::string build_lpm4(const nfc_lpm4_spec &s, std::vector<uint16_t> &tbl24, std::vector<uint16_t> &tbllong,
                       std::vector<uint2> &nh, std::vector<uint2> &pmac);
struct Lpm6Host {
    std::vector<uint8_t> lens;
    std::vector<uint32_t> base, mask;
    std::vector<Lpm6Entry> ent;
    uint32_t def_nh = 0x7FFF;
    std::vector<uint2> nh, pmac;
};
std::string build_lpm6(const nfc_lpm6_spec &s, Lpm6Host &out);
std::string build_ipsec(const nfc_ipsec_spec &s, std::vector<EspSa> &sa);
void build_aes_tables(std::vector<uint32_t> &te);           // Te0..3 + sbox
void build_toeplitz_nibbles(const uint8_t key[40], std::vector<uint32_t> &nib);
struct NatHost {
    NatImg img{};                    // scalars + inside prefixes (pointers set by the caller)
    std::vector<uint32_t> pool;
    std::vector<uint4> dnat;         // power-of-two open-addressing table
    std::vector<uint32_t> nib;
};
std::string build_nat(const nfc_nat_spec &s, NatHost &out);
extern const uint8_t MS_RSS_KEY[40];
void aes_expand(const uint8_t key[16], uint32_t rk[44]);
void sha1_compress(uint32_t h[5], const uint8_t blk[64]);

// Waldvogel level hash (host and device use the same function)
#ifdef __CUDACC__
__host__ __device__
#endif
inline uint32_t l6_hash(uint32_t k0, uint32_t k1, uint32_t k2, uint32_t k3)
{
    uint32_t h = k0 * 0x9E3779B1u;
    h = (h ^ (h >> 15) ^ k1) * 0x85EBCA77u;
    h = (h ^ (h >> 13) ^ k2) * 0xC2B2AE3Du;
    h = (h ^ (h >> 16) ^ k3) * 0x27D4EB2Fu;
    return h ^ (h >> 15);
}

// kernel launch (sfc_kernel.cu).  The variant is chosen from the chain kinds and
// the DFA placement (dfa_full: the whole DFA is staged in shared memory).
struct LaunchCfg {
    int grid, block;
    size_t smem;
    int launches = 1;            // kernel launches issued
};
// DFA placement: DM_HOT = hot rows in shared memory, the rest read through L2;
// DM_FULL = the whole DFA in shared memory (one CTA per SM).
enum { DM_HOT = 1, DM_FULL = 2 };
struct Variant { uint32_t sig; int dm; int threads; bool esp; bool rg = false; };
Variant sfc_variant(const uint32_t *kinds, uint32_t n, bool dfa_full);
// records of every 32-packet chunk of a multi-batch call (ChunkRec), on `stream`
int chunk_recs_launch(const BatchDev *batches, uint32_t n_batches, uint32_t n_pkts, ChunkRec *out, void *stream,
                      std::string &err);
// planner.cpp: true iff every group of `group` is a run of consecutive positions whose
// members are pairwise parallel-legal (group[0] = 0, steps of 0 or 1)
bool groups_legal(const uint32_t *kinds, uint32_t n, const uint8_t *group);
int sfc_launch(const Variant &v, const KParams &p, int device, void *stream, std::string &err, LaunchCfg *cfg_out);
size_t sfc_smem_bytes(const Variant &v, const KParams &p);
size_t sfc_smem_limit(int device);      // max dynamic shared memory per CTA (opt-in)
int sfc_query(const Variant &v, const KParams &p, int device, LaunchCfg *cfg_out);  // grid for full occupancy
// NFC_F_UNFUSED baseline (unfused.cu): parse stage, one stage kernel per NF, stats stage
int uf_launch(const uint32_t *kinds, uint32_t n_nf, int dm, const KParams &p, uint32_t *list0, uint32_t *list1,
              uint32_t *counts, uint8_t *passmask, int device, void *stream, std::string &err, uint32_t *n_launch);
// NFC_F_PARALLEL (parallel.cu): the chain's NFs on different warps of a team, XOR merge
size_t par_smem_bytes(const KParams &p, uint32_t n_fwd);
int par_launch(const KParams &p, int device, void *stream, std::string &err, LaunchCfg *cfg);
int rss_shard_launch(const uint8_t *arena, const uint64_t *off, const uint16_t *len, uint32_t n, const uint32_t *nib,
                     uint32_t n_shards, uint8_t *out, void *stream, std::string &err);

} // namespace nfc
