/*
 * nfc.h -- C ABI of the B200-native NFCompass SFC hot path.
 *
 * One fused, persistent sm_100a kernel applies a Service Function Chain (SFC)
 * to batches of packets resident in HBM.  The calls follow the paper's problem
 * statement: traffic traverses a sequence of network functions (NFs) in order
 * (PAPER.md P:L27, P:L42, P:L79 [SI]); packets arrive and are processed in
 * batches (P:L87 [SII.B.1]); each NF reads, writes or drops a packet as in
 * Table II (P:L213-223 [SIV]); a forwarder sets the egress port, the
 * load balancer picks a destination, IPsec encrypts and authenticates
 * (P:L130).  NFCompass re-organizes the chain (parallelize, de-duplicate,
 * early drop, P:L243-271 [SIV.B]) without changing the result of applying the
 * NFs sequentially in the original order; that sequential result is
 * what every call below produces.
 *
 * Conventions
 *  - Every call returns an int status: NFC_OK (0) or a negative NFC_E* code.
 *    Nothing throws across the ABI.  nfc_last_error() returns a thread-local
 *    message for the last failing call on this thread.
 *  - "device pointer" = CUDA global memory on the chain's device (e.g. a torch
 *    CUDA tensor's data_ptr()); "host pointer" = ordinary process memory.
 *  - A chain is bound to one device and is not thread-safe; use one chain per
 *    GPU (multi-GPU = one process or thread per GPU, flows sharded by RSS
 *    hash).
 *  - All integer fields are little-endian host order unless stated; packet
 *    bytes and the address fields of specs are network (big-endian) order.
 */
#ifndef NFC_H
#define NFC_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define NFC_API __attribute__((visibility("default")))
#else
#define NFC_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

/* ---------------------------------------------------------------- status */
#define NFC_OK 0
#define NFC_EINVAL (-1)  /* bad argument or malformed spec                        */
#define NFC_ENOMEM (-2)  /* host or device allocation failed                      */
#define NFC_ECUDA (-3)   /* CUDA runtime error (message in nfc_last_error)        */
#define NFC_ESTATE (-4)  /* tables missing for an NF of the chain, or bad state   */
#define NFC_ECAP (-5)    /* match pairs overflowed match_cap since last collect  */
#define NFC_EUNSUP (-6)  /* unsupported chain (length > 6, repeated IPsec / NAT)  */

/* NF kinds (Table II P:L213-223 rows Firewall, IDS/DPI, LB; P:L128 IPv4/IPv6
 * forwarders; P:L130 IPsec gateway). */
#define NFC_ACL 1   /* firewall: 5-tuple first-match classification, DENY drops */
#define NFC_DPI 2   /* Aho-Corasick multi-pattern DPI (IDS: DROP patterns drop)  */
#define NFC_LPM4 3  /* IPv4 forwarder, longest-prefix match (DIR-24-8)            */
#define NFC_LPM6 4  /* IPv6 forwarder, longest-prefix match (Waldvogel levels)    */
#define NFC_IPSEC 5 /* IPsec ESP gateway: AES-128-CTR + HMAC-SHA1-96              */
#define NFC_LB 6    /* load balancer: flow hash -> backend -> egress port         */
#define NFC_NAT 7   /* NAT44: source NAPT + static destination NAT (R#30)  */

#define NFC_MAX_CHAIN 6

typedef struct nfc_chain nfc_chain; /* opaque; owned by the library */

/* nfc_chain_opts.flags */
#define NFC_F_UNFUSED 1u     /* baseline: one kernel per NF with a
                              * device-side re-split of surviving packets between NFs and
                              * a per-NF header re-read/re-parse -- the per-element
                              * pipeline of P:L142-171.  Identical results; chains with
                              * NFC_IPSEC are rejected with NFC_EUNSUP.                  */

#define NFC_F_PARALLEL 2u    /* SFC parallelization: the
                              * chain's NFs (one parallel-legal group, nfc_plan_parallel)
                              * run at once on different warps, each on its own copy of
                              * a 32-packet chunk, merged by XOR with the earliest
                              * dropper's later side effects discarded.  Identical
                              * results; chains with NFC_IPSEC are rejected (NFC_EUNSUP). */

typedef struct {
    int device;              /* CUDA device ordinal                                   */
    uint32_t flags;          /* 0 (fused, the product), NFC_F_UNFUSED or NFC_F_PARALLEL */
    uint32_t max_batch_pkts; /* hint: largest packet count per nfc_process_batch call */
} nfc_chain_opts;

/* Create a chain. kinds[0..n) = NF kinds in ORIGINAL SFC order; 1 <= n <= 6.
 * A kind may repeat (the paper's chains of four identical FW or IDS NFs, P:L318
 * [SV.B.1], Fig. 13): positions of one kind share that kind's tables; NFC_IPSEC
 * and NFC_NAT at most once (else NFC_EUNSUP).  Allocates device state (stats,
 * ESP sequence counters, scheduling scratch) on opts->device.  *out is owned by
 * the caller and released with nfc_destroy_chain. */
NFC_API int nfc_build_chain(const uint32_t *kinds, uint32_t n, const nfc_chain_opts *opts, nfc_chain **out);
NFC_API void nfc_destroy_chain(nfc_chain *c);

/* Bytes the caller must leave before / after every frame in the arena.
 * Chains with IPSEC: headroom 16 (the Ethernet+IP header moves 16 B left to
 * make room for the ESP header and IV, RFC 4303 transport mode), tailroom 32
 * (ESP trailer + ICV grow the frame by 14..17 B).  Otherwise 0 / 0. */
NFC_API int nfc_chain_room(const nfc_chain *c, uint32_t *headroom, uint32_t *tailroom);

/* ---------------------------------------------------------------- logical specs
 * Host structures, copied by nfc_load_tables; the same binary layouts are what
 * the test oracle reads. */
typedef struct {                 /* 48 B */
    uint8_t family;              /* 4 or 6                                        */
    uint8_t slen, dlen;          /* source / destination prefix lengths           */
    uint8_t proto;               /* IP protocol (ignored if proto_any)            */
    uint8_t proto_any;           /* 1 = any protocol                              */
    uint8_t action;              /* 0 PERMIT, 1 DENY                              */
    uint16_t sp_lo, sp_hi;       /* source port range, inclusive                  */
    uint16_t dp_lo, dp_hi;       /* destination port range, inclusive             */
    uint8_t pad[2];
    uint8_t src[16], dst[16];    /* prefixes, network order (IPv4: bytes 0..3)    */
} nfc_acl_rule;

typedef struct {
    uint32_t n_rules;            /* <= 32767                                      */
    uint32_t default_action;     /* action when no rule matches: 0/1              */
    const nfc_acl_rule *rules;   /* host; rule i has priority i (first match)     */
} nfc_acl_spec;

typedef struct {
    uint32_t n_patterns;         /* 1..65535                                      */
    const uint8_t *blob;         /* host; pattern j = blob[off[j] .. off[j+1])    */
    const uint32_t *off;         /* host; n_patterns+1 offsets                    */
    const uint8_t *action;       /* host; 0 ALERT, 1 DROP                         */
} nfc_dpi_spec;

typedef struct { uint32_t prefix; uint8_t len; uint8_t pad; uint16_t nh; } nfc_route4;     /* 8 B  */
typedef struct { uint8_t prefix[16]; uint16_t nh; uint8_t len; uint8_t pad; } nfc_route6;  /* 20 B */
typedef struct { uint16_t port; uint8_t mac[6]; } nfc_nexthop;                            /* 8 B  */

typedef struct {
    uint32_t n_routes;  const nfc_route4 *routes;    /* prefix: host-order u32 value, len 0..32 */
    uint32_t n_nexthops; const nfc_nexthop *nexthops; /* nh < n_nexthops <= 32767              */
    uint32_t n_ports;   const uint8_t *port_macs;    /* n_ports x 6 B source MAC per port       */
} nfc_lpm4_spec;

typedef struct {
    uint32_t n_routes;  const nfc_route6 *routes;    /* len 0..128                              */
    uint32_t n_nexthops; const nfc_nexthop *nexthops;
    uint32_t n_ports;   const uint8_t *port_macs;
} nfc_lpm6_spec;

typedef struct {                 /* 48 B */
    uint32_t spi;                /* ESP SPI                                        */
    uint32_t seq0;               /* initial sequence counter (first packet: seq0+1)*/
    uint8_t aes_key[16];         /* AES-128 key                                    */
    uint8_t nonce[4];            /* RFC 3686 nonce                                 */
    uint8_t auth_key[20];        /* HMAC-SHA1 key                                  */
} nfc_sa;

typedef struct { uint32_t n_sa; const nfc_sa *sas; } nfc_ipsec_spec; /* 1..255 SAs */

typedef struct {
    uint32_t n_backends;         /* 1..65535                                       */
    const uint16_t *backend_port;/* host; egress port per backend                  */
    const uint8_t *key;          /* host; 40 B Toeplitz key                        */
} nfc_lb_spec;

/* NAT44 ("For traffics to Internet, the NAT network
 * function performs source and destination NAT"; Table II: header read+write, no
 * drop; R#30).  Applies to IPv4 TCP/UDP packets whose egress port (set by
 * the NFs before it; 0 if none) has its bit set in ext_ports.  With h =
 * Toeplitz(key, src|dst|sport|dport) of the arriving packet: DNAT rewrites (dst,
 * dport) of the first entry matching (proto, dst, dport); SNAT, for sources inside
 * one of the prefixes, sets src = pool[(h & 0xFFFF) % n_pool] and sport = port_lo +
 * (h >> 16) % (port_hi - port_lo + 1).  The IPv4 header checksum is recomputed and the
 * TCP/UDP checksum updated per RFC 1624 eqn. 3 (a UDP checksum of 0 stays 0; an
 * updated UDP checksum of 0 becomes 0xFFFF).  Addresses are host-order u32 values. */
typedef struct { uint32_t prefix; uint8_t len; uint8_t pad[3]; } nfc_nat_prefix;        /* 8 B  */
typedef struct {                                                                         /* 16 B */
    uint32_t ext_addr; uint16_t ext_port; uint8_t proto; uint8_t pad;
    uint32_t int_addr; uint16_t int_port; uint16_t pad2;
} nfc_nat_dnat;

typedef struct {
    uint32_t n_inside;  const nfc_nat_prefix *inside; /* host; <= 64 prefixes (SNAT sources)     */
    uint32_t n_pool;    const uint32_t *pool;         /* host; 1..65536 public addresses          */
    uint32_t port_lo, port_hi;                        /* SNAT source port range, lo <= hi < 65536 */
    uint32_t n_dnat;    const nfc_nat_dnat *dnat;     /* host; distinct (proto, ext_addr, ext_port) */
    uint32_t ext_ports;                               /* bit p: egress port p faces the Internet   */
    const uint8_t *key;                               /* host; 40 B Toeplitz key                   */
} nfc_nat_spec;

/* Build the device image of one NF's tables on the host and copy it to the
 * device (synchronous).  spec points to the nfc_*_spec matching kind;
 * spec_bytes = sizeof that struct.  Replaces earlier tables of that kind.
 * Every NF of the chain needs its tables before nfc_process_batch
 * (NFC_ESTATE).  Malformed specs -> NFC_EINVAL: duplicate (prefix,len),
 * len > 32/128, host bits set in a prefix, nh >= n_nexthops, empty pattern,
 * lo > hi port range, n_sa == 0 or > 255, n_backends == 0. */
NFC_API int nfc_load_tables(nfc_chain *c, uint32_t kind, const void *spec, size_t spec_bytes);

/* ---------------------------------------------------------------- batches */
typedef struct {
    uint8_t *arena;              /* device; packet bytes, rewritten in place              */
    const uint64_t *off;         /* device; n frame start offsets into arena, each % 16 == 0 */
    const uint16_t *len;         /* device; n frame lengths (14..16383)                   */
    uint32_t n;                  /* packets in this batch                                 */
    uint32_t reserved;
    uint64_t first_global_index; /* global index of packet 0 (match-pair packet ids)      */
} nfc_batch;

typedef struct {                 /* 16 B per packet */
    uint8_t drop_nf;             /* 0xFF forwarded; 0xFE parse failure; else chain position */
    uint8_t esp_sa;              /* SA index if ESP was applied, else 0xFF                */
    uint16_t port;               /* egress port; 0 if none set; 0xFFFF if dropped         */
    uint16_t acl_rule;           /* first matching ACL rule; 0xFFFF none / not reached    */
    uint16_t lb_backend;         /* LB backend; 0xFFFF if not reached                     */
    uint16_t dpi_nmatch;         /* number of distinct matched patterns                  */
    uint16_t out_len;            /* frame length after the chain                          */
    uint32_t esp_seq;            /* ESP sequence number, 0 if ESP not applied             */
} nfc_pkt_result;

typedef struct {
    nfc_pkt_result *rec;         /* device; one record per packet, batches concatenated   */
    uint32_t *match_pkt;         /* device; match pair packet global index                */
    uint16_t *match_pat;         /* device; match pair pattern id                         */
    uint32_t match_cap;          /* capacity of match_pkt / match_pat                     */
    uint32_t reserved;
    uint32_t *match_count;       /* device u32, incremented atomically; caller zeroes it   */
} nfc_result;

/* Apply the chain to n_batches batches (descriptor array in HOST memory),
 * asynchronously on `stream` (a cudaStream_t; NULL = legacy default stream),
 * in one persistent kernel launch.  Packets are processed as one stream in
 * batch order; every per-packet output equals applying the chain's NFs in
 * original order to each packet, with ESP sequence numbers assigned per SA in
 * that global order (so outputs never depend on how packets are split into
 * batches or calls).  Frames are rewritten in place: forwarders rewrite the
 * Ethernet/IP header; ESP moves the frame start to off-16 and grows the frame
 * to rec.out_len.  Match pairs are appended in unspecified order; pairs beyond
 * match_cap are counted in the stats but not written.  Output bytes of
 * dropped packets are unspecified.  Results are valid after the stream syncs. */
NFC_API int nfc_process_batch(nfc_chain *c, const nfc_batch *batches, uint32_t n_batches,
                      const nfc_result *r, void *stream);

/* End-to-end variant with HOST buffers: copies arena[0, arena_bytes) and
 * off/len to chain-owned device staging buffers on `stream`, runs the chain,
 * copies the rewritten arena, the records and the match pairs back, and
 * synchronizes the stream.  Host buffers should be pinned for full PCIe rate.
 * *n_pairs receives the number of pairs found (may exceed match_cap). */
NFC_API int nfc_process_host(nfc_chain *c, uint8_t *arena, uint64_t arena_bytes, const uint64_t *off,
                     const uint16_t *len, uint32_t n, uint64_t first_global_index,
                     nfc_pkt_result *rec, uint32_t *match_pkt, uint16_t *match_pat,
                     uint32_t match_cap, uint32_t *n_pairs, void *stream);

/* ---------------------------------------------------------------- stats
 * u64 counter vector (layout in DESIGN.md "Stats vector"): totals, per chain
 * position in/drop/pass-through/applied, then ACL per-rule hits (+default),
 * LB per-backend hits and per-SA ESP packets.  Same sequential semantics as
 * the per-packet records. */
#define NFC_STATS_RESET 1u
#define NFC_STATS_ALLREDUCE 2u   /* sum the vector over the ranks of the attached comm  */

NFC_API int nfc_stats_len(const nfc_chain *c, size_t *len);
/* Synchronizes the stream of the chain's last nfc_process_batch / nfc_process_host
 * call (not the whole device), copies min(cap, len) counters to out (host) and
 * optionally resets this GPU's counters (NFC_STATS_RESET).  With
 * NFC_STATS_ALLREDUCE the vector written to out is the sum over every rank of the
 * communicator attached with nfc_attach_comm (one ncclAllReduce(ncclUint64,
 * ncclSum) on that stream: flows shard by RSS hash, so the
 * counters are the only exchange); every rank must make the call (collective),
 * and NFC_ESTATE is returned if no communicator is attached.  Returns NFC_ECAP if
 * match pairs were dropped for capacity since the last reset (on any rank, with
 * NFC_STATS_ALLREDUCE). */
NFC_API int nfc_collect_stats(nfc_chain *c, uint64_t *out, size_t cap, uint32_t flags);

/* ---------------------------------------------------------------- multi-GPU
 * One process (or thread) per GPU, one chain per GPU, flows sharded with
 * nfc_rss_shard (below); the library's only collective is the counter sum of
 * nfc_collect_stats.  NCCL (libnccl.so.2) is loaded on first use of these calls;
 * NFC_ESTATE if it cannot be loaded, NFC_ECUDA (message from NCCL) if a call fails. */
#define NFC_COMM_ID_BYTES 128
/* Rank 0 creates the communicator id (ncclGetUniqueId) and hands the 128 bytes to
 * the other ranks out of band (e.g. a torch.distributed broadcast). */
NFC_API int nfc_comm_unique_id(uint8_t *id, size_t id_bytes);
/* ncclCommInitRank on `device` (collective over nranks ranks); *comm receives the
 * ncclComm_t, owned by the caller (nfc_comm_destroy). */
NFC_API int nfc_comm_init(int device, int nranks, int rank, const uint8_t *id, void **comm);
NFC_API int nfc_comm_destroy(void *comm);
/* Attach an ncclComm_t (from nfc_comm_init or the caller's own NCCL) to the chain
 * for NFC_STATS_ALLREDUCE; NULL detaches.  The chain does not own it. */
NFC_API int nfc_attach_comm(nfc_chain *c, void *nccl_comm);

/* Receive Side Steering for multi-GPU sharding (P:L87 RSS model): shard[i] =
 * RETA[Toeplitz(MS default key, src|dst|sport|dport of frame i) & 127], RETA[j] =
 * j mod n_shards (1..128); frames that fail to parse go to shard 0.  With n_shards
 * dividing 64 and 64 ESP SAs, every SA lives on exactly one shard, so per-SA ESP
 * sequence numbers of a sharded run equal the single-GPU run.  b and shard (u8 x n)
 * are device pointers on `device`; asynchronous on `stream`. */
NFC_API int nfc_rss_shard(int device, const nfc_batch *b, uint32_t n_shards, uint8_t *shard, void *stream);

/* SFC parallelization plan (Tables II-III): cuts
 * the chain kinds[0..n) into groups of consecutive NFs that may run on copies of
 * the same packet and be merged by XOR with a result identical to the
 * sequential chain.  group[p] (n bytes, host memory) receives the group index of
 * position p (0, 1, ... non-decreasing).  Greedy maximal groups under the
 * field-level rule of DESIGN.md R#16 (no read-after-write, no write-after-write on
 * a packet field, per packet family); IPsec always stands alone.  NFC_EINVAL for
 * NULL pointers, n outside 1..6 or an unknown kind. */
NFC_API int nfc_plan_parallel(const uint32_t *kinds, uint32_t n, uint8_t *group);
/* The grouping an NFC_F_PARALLEL chain runs (default: nfc_plan_parallel's maximal
 * groups).  group[p] (n bytes, host) = group of position p: group[0] = 0, each next
 * position the same group or the next, every group pairwise parallel-legal (R#16);
 * else NFC_EINVAL.  Groups run one after another, the members of a group at once on
 * copies of the packet entering it, merged by XOR -- e.g. the paper's
 * configuration (c) of four identical NFs = groups {0,0,1,1} (Fig. 13). */
NFC_API int nfc_set_groups(nfc_chain *c, const uint8_t *group);
NFC_API int nfc_get_groups(const nfc_chain *c, uint8_t *group);

/* ---------------------------------------------------------------- stateful DPI
 * stateful, cross-packet DPI (PAPER.md P:L161 [SIII.B.b]
 * "in-order processing of packet in the same connection ... resembled as traffic
 * stream"; P:L132 [SIII.A.2] Aho-Corasick for string matching; R#32).
 * A flow is the exact (family, proto, src, dst, sport, dport) of a frame that
 * parses under R#24 (ports 0 for fragments and non-TCP/UDP).  The payloads
 * [pl_off, ip_end) of a flow's packets, in global order (calls in order, packets
 * of a call in index order), form one byte stream; every occurrence of a pattern
 * in that stream (case-sensitive, overlapping) is reported against the packet
 * holding its LAST byte.  Flow state (the Aho-Corasick DFA state) persists in a
 * device flow table across calls until nfc_dpi_stream_reset.  Standalone NF: it
 * is not part of a fused chain. */
typedef struct nfc_dpi_stream nfc_dpi_stream; /* opaque; owned by the library */

typedef struct {
    uint32_t *nocc;              /* device; n: occurrences ending in packet i (0 if not inspected) */
    uint8_t *drop;               /* device; n: 1 iff a DROP pattern occurrence ends in packet i   */
    uint32_t *occ_pkt;           /* device; occurrence: packet global index                     */
    uint16_t *occ_pat;           /* device; occurrence: pattern id                              */
    uint16_t *occ_end;           /* device; occurrence: offset of its last byte in the payload  */
    uint32_t occ_cap;            /* capacity of occ_*; occurrences beyond it are counted only   */
    uint32_t reserved;
    uint32_t *occ_count;         /* device u32, incremented atomically; caller zeroes it        */
} nfc_stream_result;

/* Builds the Aho-Corasick DFA of `spec` (NFC_EINVAL as nfc_load_tables for a
 * malformed spec) and a device flow table of the next power of two >= 2 x
 * max_flows slots (1..2^28) on `device`.  NFC_ENOMEM / NFC_ECUDA on failure. */
NFC_API int nfc_dpi_stream_create(int device, const nfc_dpi_spec *spec, uint32_t max_flows, nfc_dpi_stream **out);
/* Regular-expression variant ("for the regular expression we use a DFA";
 * DESIGN.md R#33): spec->blob[off[j] .. off[j+1]) is expression j (not NUL-
 * terminated) over bytes: literals, \xHH, \<punct>, '.', [..] classes with ranges
 * and '^', (..), '|', '?', '*', '+', {m}, {m,n} with n <= 64 and {m,} with m <= 64.
 * An occurrence of expression j ends at byte x iff a non-empty substring of the
 * flow stream ending at x is in its language (unanchored search); it is reported
 * like a pattern occurrence.  A set whose longest match is at most 1 024 bytes is
 * walked per packet (a bounded re-walk of the flow's preceding bytes); a longer or
 * unbounded one is walked flow-serially from the carried state.  NFC_EINVAL for a
 * syntax error, an expression that matches the empty string, or a DFA over
 * max_states states (0 = 2^20); NFC_EUNSUP for anchors ('^' / '$' outside a class)
 * or repeats that expand the NFA beyond 2^16 states; NFC_ENOMEM if the host
 * compiler runs out of memory. */
NFC_API int nfc_dpi_stream_create_regex(int device, const nfc_dpi_spec *spec, uint32_t max_flows,
                                        uint32_t max_states, nfc_dpi_stream **out);
NFC_API int nfc_dpi_stream_destroy(nfc_dpi_stream *s);
/* Forgets every flow (asynchronous on `stream`). */
NFC_API int nfc_dpi_stream_reset(nfc_dpi_stream *s, void *stream);
/* Inspects one batch (frames are only read) asynchronously on `stream`; results are
 * valid after the stream syncs.  Occurrences are appended in unspecified order.  A
 * packet of a new flow that finds the flow table full is not inspected (counted by
 * nfc_dpi_stream_flows).  Calls on one object must be ordered on one stream. */
NFC_API int nfc_dpi_stream_process(nfc_dpi_stream *s, const nfc_batch *b, const nfc_stream_result *r, void *stream);
/* Synchronizes the device; flows in the table and packets not placed (table full). */
NFC_API int nfc_dpi_stream_flows(nfc_dpi_stream *s, uint64_t *n_flows, uint64_t *n_unplaced);

/* Measured device peaks, the denominators of the integer-bound rooflines (SURVEY
 * 8(d): "a repo microbenchmark measures them on the box"): 32-bit ALU-pipe ops/s
 * (independent LOP3/IADD3/SHF/PRMT chains), integer issue ops/s (the same chains
 * interleaved with IMAD: ALU + FMA pipes), conflict-free 32-bit shared-memory
 * lookups/s, and random 32-B L2 sectors/s (64 MiB L2-resident buffer).  Runs ~four
 * short kernels on `device` (synchronous, about 50 ms); clocks are whatever the
 * device runs at (sm_clock_mhz is the nominal maximum). */
typedef struct {
    double alu_tops, issue_tops, smem_glookups, l2_gsectors;
    uint32_t sm_count, sm_clock_mhz;
} nfc_peaks;
NFC_API int nfc_measure_peaks(int device, nfc_peaks *out);

/* Number of kernel launches the library issued on this chain so far. */
NFC_API int nfc_launch_count(const nfc_chain *c, uint64_t *count);

/* Shape of the chain's last fused-kernel launch (diagnostics; all zero before the first
   nfc_process_batch): grid and block size, dynamic shared memory (bytes), DFA placement
   (0 none, 1 tiered: dense rows + sparse records + global, 2 every row in shared memory),
   DFA states with dense rows and with sparse records in shared memory, 1 if the per-state
   match summary is in shared memory, bytes of the ACL images in shared memory. */
typedef struct {
    uint32_t grid, block, smem, dfa_mode, dfa_dense, dfa_sparse, dfa_meta_smem, acl_smem;
} nfc_launch_info;
NFC_API int nfc_last_launch(const nfc_chain *c, nfc_launch_info *out);

NFC_API const char *nfc_last_error(void);
NFC_API const char *nfc_version(void);

#ifdef __cplusplus
}
#endif
#endif /* NFC_H */
