// dpi_stream.cu -- stateful (cross-packet) DPI, SURVEY 8(f) NEXT-4 (include/nfc.h
// "Stateful DPI"; PAPER.md P:L161 [SIII.B.b] in-order processing of the packets of
// a connection, P:L132 [SIII.A.2] Aho-Corasick DPI; R#32, section 16).
//
// Three launches per call, all on the caller's stream:
//   k_flow  -- one thread per packet: R#24 parse, flow key -> slot of a device
//              open-addressing flow table (lock-free insert), payload span;
//   cub radix sort of (slot, packet index) pairs (stable: a flow's packets stay
//              in index order, i.e. stream order);
//   k_walk  -- one thread per packet: rebuilds the packet's start state by
//              re-walking the last maxlen - 1 bytes of its flow's stream (or from
//              the state carried from earlier calls), walks its payload through the
//              Aho-Corasick DFA (the image builders.cpp makes for the fused kernel)
//              and appends every occurrence ending in it;
//   k_commit -- stores each flow's final state for the next call.
// The flow table and the per-flow DFA states persist across calls.
#include <cuda_runtime.h>
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "nfc_internal.h"

using namespace nfc;

namespace {

constexpr uint32_t KW = 10;   // key words: src[4], dst[4], sport<<16|dport, proto | family<<8
constexpr uint32_t KS = 12;   // key words per table slot (48 B: three 16-B loads)
constexpr size_t DFA_SMEM_MAX = 200 * 1024;   // DFA bytes staged in shared memory (k_walk<2>)
#ifndef WALK_SMEM_THREADS
#define WALK_SMEM_THREADS 768   // k_walk<2> CTA size (1024 spills at the 64-register cap)
#endif
constexpr uint32_t HB = 96;   // header bytes staged per packet (IPv4 IHL 15 + TCP data offset: 88)

struct StreamDfa {
    const uint8_t *cls;
    const void *trans;
    const uint32_t *out_off;
    const uint16_t *out_ids;
    const uint8_t *action;
    uint32_t ncls, wide, n_states;
};

__device__ __forceinline__ uint32_t be16d(const uint8_t *p) { return (uint32_t)p[0] << 8 | p[1]; }

// R#24 parse: returns false if the frame is not inspected; key[KW], payload [a, b)
// f holds the frame's first `have` bytes (have = min(flen, HB): every byte the parse
// reads lies below 88, and each read is guarded by a bound that implies < flen).
__device__ bool parse_flow(const uint8_t *f, uint32_t have, uint32_t flen, uint32_t key[KW], uint32_t &a, uint32_t &b)
{
    (void)have;
    if (flen < 14) return false;
    const uint32_t et = be16d(f + 12);
    uint32_t l4, ip_end, proto, fam;
    bool frag = false;
    for (int k = 0; k < (int)KW; k++) key[k] = 0;
    if (et == 0x0800) {
        if (flen < 34 || (f[14] >> 4) != 4) return false;
        const uint32_t ihl = f[14] & 15, tot = be16d(f + 16);
        if (ihl < 5 || tot < 4 * ihl || 14 + tot > flen) return false;
        fam = 4; l4 = 14 + 4 * ihl; ip_end = 14 + tot; proto = f[23];
        key[0] = (uint32_t)f[26] << 24 | (uint32_t)f[27] << 16 | (uint32_t)f[28] << 8 | f[29];
        key[4] = (uint32_t)f[30] << 24 | (uint32_t)f[31] << 16 | (uint32_t)f[32] << 8 | f[33];
        const uint32_t fo = be16d(f + 20);
        frag = (fo & 0x3FFF) != 0;
    } else if (et == 0x86DD) {
        if (flen < 54 || (f[14] >> 4) != 6) return false;
        const uint32_t pl = be16d(f + 18);
        if (54 + pl > flen) return false;
        fam = 6; l4 = 54; ip_end = 54 + pl; proto = f[20];
        for (int w = 0; w < 4; w++) {
            const uint8_t *s = f + 22 + 4 * w, *d = f + 38 + 4 * w;
            key[w] = (uint32_t)s[0] << 24 | (uint32_t)s[1] << 16 | (uint32_t)s[2] << 8 | s[3];
            key[4 + w] = (uint32_t)d[0] << 24 | (uint32_t)d[1] << 16 | (uint32_t)d[2] << 8 | d[3];
        }
    } else {
        return false;
    }
    uint32_t hl = 0;
    if (!frag && proto == 17) {
        if (l4 + 8 > ip_end) return false;
        hl = 8;
    } else if (!frag && proto == 6) {
        if (l4 + 20 > ip_end) return false;
        const uint32_t doff = f[l4 + 12] >> 4;
        if (doff < 5 || l4 + 4 * doff > ip_end) return false;
        hl = 4 * doff;
    }
    if (hl) key[8] = be16d(f + l4) << 16 | be16d(f + l4 + 2);
    key[9] = proto | fam << 8 | 1u << 16;          // bit 16: never an all-zero key
    a = l4 + hl;
    b = ip_end;
    return true;
}

__device__ __forceinline__ uint32_t key_hash(const uint32_t key[KW])
{
    uint32_t h = 0x9E3779B9u;
    for (int k = 0; k < (int)KW; k++) {
        uint32_t x = key[k] * 0xCC9E2D51u;
        x = (x << 15) | (x >> 17);
        h ^= x * 0x1B873593u;
        h = ((h << 13) | (h >> 19)) * 5u + 0xE6546B64u;
    }
    h ^= h >> 16; h *= 0x85EBCA6Bu; h ^= h >> 13; h *= 0xC2B2AE35u; h ^= h >> 16;
    return h;
}

__device__ __forceinline__ uint32_t ld_acquire(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// Flow table slot of `key` (inserted if new); 0xFFFFFFFF if the flow is not in the
// table and cannot be placed: max_flows flows are already placed (so the load factor
// stays <= 1/2), or no free slot within PROBE_MAX probes (a bounded probe: a SYN flood
// of new 5-tuples cannot turn every later miss into a full-table scan).
// lock[s]: 0 empty, 1 key being written, 2 key published, 3 dead (claimed when the
// table was already at max_flows: skipped by every probe).  The capacity is counted
// after the claim, so concurrent packets of one new flow do not over-reserve it.
constexpr uint32_t PROBE_MAX = 64;
__device__ uint32_t flow_slot(uint32_t *lock, uint32_t *keys, uint32_t mask, uint32_t *n_flows, uint32_t max_flows,
                              const uint32_t key[KW])
{
    uint32_t s = key_hash(key) & mask;
    const uint32_t probes = min(mask + 1, PROBE_MAX);
    for (uint32_t probe = 0; probe < probes; probe++, s = (s + 1) & mask) {
        uint32_t l = ld_acquire(&lock[s]);           // published slots need no atomic
        if (l == 0) {
            l = atomicCAS(&lock[s], 0u, 1u);
            if (l == 0) {
                if (atomicAdd(n_flows, 1u) >= max_flows) {   // table at capacity: no new flow
                    atomicSub(n_flows, 1u);
                    __threadfence();
                    atomicExch(&lock[s], 3u);
                    return 0xFFFFFFFFu;
                }
                uint4 *kp = reinterpret_cast<uint4 *>(keys + (size_t)s * KS);
                kp[0] = make_uint4(key[0], key[1], key[2], key[3]);
                kp[1] = make_uint4(key[4], key[5], key[6], key[7]);
                kp[2] = make_uint4(key[8], key[9], 0, 0);
                __threadfence();
                atomicExch(&lock[s], 2u);
                return s;
            }
            l = ld_acquire(&lock[s]);                // the CAS is relaxed: re-read with acquire
        }
        while (l == 1) {                             // acquire: the published key is visible
            __nanosleep(64);                         // yield: the writer may be a lane of this warp
            l = ld_acquire(&lock[s]);
        }
        if (l == 3) continue;                        // dead slot
        const uint4 *kp = reinterpret_cast<const uint4 *>(keys + (size_t)s * KS);
        const uint4 k0 = __ldcg(kp), k1 = __ldcg(kp + 1), k2 = __ldcg(kp + 2);
        if (k0.x == key[0] && k0.y == key[1] && k0.z == key[2] && k0.w == key[3] && k1.x == key[4] &&
            k1.y == key[5] && k1.z == key[6] && k1.w == key[7] && k2.x == key[8] && k2.y == key[9])
            return s;
    }
    return 0xFFFFFFFFu;
}

__global__ void k_flow(nfc_batch b, uint32_t *lock, uint32_t *keys, uint32_t mask, uint32_t max_flows, uint32_t none,
                       uint32_t *ctr, uint32_t *fkey, uint32_t *fidx, uint32_t *span,
                       uint32_t *nocc, uint8_t *drop)
{
    // the first HB bytes of each frame are staged in shared memory with 16-B loads
    // (frames are 16-B aligned; no load starts beyond the frame), then parsed there
    __shared__ uint4 hdr[256 * HB / 16];
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= b.n) return;
    nocc[i] = 0;
    drop[i] = 0;
    fidx[i] = i;
    const uint32_t flen = b.len[i];
    const uint4 *src = reinterpret_cast<const uint4 *>(b.arena + b.off[i]);
    uint4 *h = hdr + threadIdx.x * (HB / 16);
#pragma unroll
    for (uint32_t k = 0; k < HB / 16; k++)
        if (16 * k < flen) h[k] = __ldg(src + k);
    uint32_t key[KW], a, e;
    uint32_t slot = none;
    if (parse_flow(reinterpret_cast<const uint8_t *>(h), min(flen, HB), flen, key, a, e)) {
        slot = flow_slot(lock, keys, mask, &ctr[0], max_flows, key);
        if (slot == 0xFFFFFFFFu) { atomicAdd(&ctr[1], 1u); slot = none; }
        span[i] = a | e << 16;
    }
    fkey[i] = slot;
}

// M: 0 = u16 entries read through L1/L2, 1 = u32 entries (> 32768 states), 2 = u16
// entries staged in shared memory (d.trans points there)
template <int M>
__device__ __forceinline__ uint32_t dfa_step(const StreamDfa &d, const uint8_t *cls, uint32_t s, uint32_t byte,
                                             bool &acc)
{
    const size_t at = (size_t)s * d.ncls + cls[byte];
    uint32_t nx;
    if (M == 1) { nx = __ldg((const uint32_t *)d.trans + at); acc = nx >> 31; return nx & 0x7FFFFFFFu; }
    nx = M == 2 ? ((const uint16_t *)d.trans)[at] : __ldg((const uint16_t *)d.trans + at);
    acc = nx >> 15;
    return nx & 0x7FFFu;
}

// Walks payload bytes [x0, x1) of the frame at p (16-B aligned) from state s.  The
// bytes are fetched as aligned 16-B words, so a payload costs ceil(len/16) + 1 loads
// issued ahead of the dependent DFA steps instead of one byte load per step.
struct Emit {
    nfc_stream_result r;
    uint32_t pkt, a, cnt, dr;
};

template <int M, bool EMIT>
__device__ __forceinline__ uint32_t walk(const StreamDfa &d, const uint8_t *cls, const uint8_t *p, uint32_t x0,
                                         uint32_t x1, uint32_t s, Emit &em)
{
    uint32_t x = x0;
    while (x < x1) {
        const uint32_t base = x & ~15u;
        const uint4 v = __ldg(reinterpret_cast<const uint4 *>(p + base));
        const uint32_t hi = min(x1, base + 16);
        for (; x < hi; x++) {
            const uint32_t q = (x >> 2) & 3;
            const uint32_t wd = q == 0 ? v.x : q == 1 ? v.y : q == 2 ? v.z : v.w;
            bool hit;
            s = dfa_step<M>(d, cls, s, (wd >> (8 * (x & 3))) & 0xFF, hit);
            if (EMIT && hit) {
                const uint32_t o0 = __ldg(d.out_off + s), o1 = __ldg(d.out_off + s + 1);
                for (uint32_t k = o0; k < o1; k++) {
                    const uint32_t pat = __ldg(d.out_ids + k);
                    const uint32_t w = atomicAdd(em.r.occ_count, 1u);
                    if (w < em.r.occ_cap) {
                        em.r.occ_pkt[w] = em.pkt;
                        em.r.occ_pat[w] = (uint16_t)pat;
                        em.r.occ_end[w] = (uint16_t)(x - em.a);
                    }
                    em.dr |= __ldg(d.action + pat);
                }
                em.cnt += o1 - o0;
            }
        }
    }
    return s;
}

// One thread per packet in flow-sorted order (position u).  The packet's start
// state is rebuilt from the flow's stream: a walk from the root that starts
// maxlen - 1 bytes before the payload sees every occurrence ending in the payload
// (an occurrence is at most maxlen bytes long), so the thread re-walks the tail of
// its predecessors in this batch; if the flow's bytes in this batch are shorter than
// that, it starts from the state carried from earlier calls.  The flow's last packet
// leaves its final state in fin[u] (committed by k_commit: readers of fstate and
// its writer never race).
template <int M>
__global__ void __launch_bounds__(M == 2 ? WALK_SMEM_THREADS : 256) k_walk(nfc_batch b, StreamDfa d, uint32_t none, uint32_t need,
                                                          const uint32_t *fkey, const uint32_t *fidx,
                                                          const uint32_t *span, const unsigned long long *cumx,
                                                          const uint32_t *fstate, uint32_t *fin, nfc_stream_result r)
{
    __shared__ uint8_t cls[256];
    extern __shared__ uint4 dyn[];
    for (int k = threadIdx.x; k < 256; k += blockDim.x) cls[k] = d.cls[k];
    if (M == 2) {   // persistent CTAs: the whole DFA in shared memory, copied once per CTA
        const uint32_t n16 = (d.ncls * d.n_states * 2 + 15) / 16;
        for (uint32_t k = threadIdx.x; k < n16; k += blockDim.x) dyn[k] = __ldg((const uint4 *)d.trans + k);
        d.trans = dyn;
    }
    __syncthreads();
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < b.n; u += gridDim.x * blockDim.x) {
        const uint32_t f = fkey[u];
        if (f == none) continue;
        // warm-up start: packet v, byte skip within its payload, start state s.  v is the
        // last position before u of the same flow with payload bytes [v, u) >= need
        // (cumx: exclusive prefix sum of payload lengths in sorted order), found by a
        // galloping search -- O(log distance), so runs of empty payloads (pure ACKs)
        // cost no quadratic walk-back; if the flow's bytes before u in this call are
        // fewer, v is the flow's first packet of the call and s its carried state.
        const unsigned long long cu = cumx[u];
        auto stop = [&](uint32_t d) {                // position u - d (d <= u)
            const uint32_t v = u - d;
            return fkey[v] != f || cu - cumx[v] >= need;
        };
        uint32_t lo = 0, hi = 1;                     // stop(lo) false (lo = 0: none tested), answer in (lo, hi]
        while (hi <= u && !stop(hi)) { lo = hi; hi *= 2; }
        if (hi > u) hi = u + 1;                      // position -1: before the call
        while (hi - lo > 1) {
            const uint32_t mid = lo + (hi - lo) / 2;
            if (stop(mid)) hi = mid; else lo = mid;
        }
        uint32_t v, skip = 0, s = 0;
        if (hi <= u && fkey[u - hi] == f) {
            v = u - hi;
            skip = (uint32_t)(cu - cumx[v] - need);
        } else {
            v = u - lo;                              // the flow's first packet of this call
            s = fstate[f];
        }
        Emit em{r, (uint32_t)b.first_global_index, 0, 0, 0};
        // warm-up walk over [v, u): packets with empty payloads are jumped over by a binary
        // search on cumx (at most `need` non-empty packets lie in the window)
        for (uint32_t w = v; w < u;) {
            if (cumx[w + 1] == cumx[w]) {                    // empty payload: next non-empty position
                const unsigned long long t = cumx[w];
                if (cumx[u] == t) break;                     // no payload byte left before u
                uint32_t a = w + 1, z = u;                   // smallest q in (w, u] with cumx[q] > t
                while (a < z) {
                    const uint32_t m = a + (z - a) / 2;
                    if (cumx[m] > t) z = m; else a = m + 1;
                }
                w = a - 1;
            }
            const uint32_t i = fidx[w], sp = span[i];
            s = walk<M, false>(d, cls, b.arena + b.off[i], (sp & 0xFFFF) + (w == v ? skip : 0), sp >> 16, s, em);
            w++;
        }
        const uint32_t i = fidx[u], sp = span[i];
        em.pkt += i;
        em.a = sp & 0xFFFF;
        s = walk<M, true>(d, cls, b.arena + b.off[i], sp & 0xFFFF, sp >> 16, s, em);
        r.nocc[i] = em.cnt;
        r.drop[i] = (uint8_t)em.dr;
        if (u + 1 == b.n || fkey[u + 1] != f) fin[u] = s;
    }
}

// payload bytes of each position in flow-sorted order (0 for packets not inspected)
__global__ void k_plen(uint32_t n, uint32_t none, const uint32_t *fkey, const uint32_t *fidx, const uint32_t *span,
                       unsigned long long *plen)
{
    const uint32_t u = blockIdx.x * blockDim.x + threadIdx.x;
    if (u >= n) return;
    uint32_t l = 0;
    if (fkey[u] != none) {
        const uint32_t sp = span[fidx[u]];
        l = (sp >> 16) - (sp & 0xFFFF);
    }
    plen[u] = l;
}

// Flow-serial walk (regex sets with unbounded or > 1 024-byte matches: no bounded
// re-walk reconstructs a packet's start state): one thread per flow segment of the
// sorted batch walks the flow's packets in stream order from the carried state.
template <int M>
__global__ void __launch_bounds__(256) k_walk_serial(nfc_batch b, StreamDfa d, uint32_t none, const uint32_t *fkey,
                                                     const uint32_t *fidx, const uint32_t *span,
                                                     const uint32_t *fstate, uint32_t *fin, nfc_stream_result r)
{
    __shared__ uint8_t cls[256];
    for (int k = threadIdx.x; k < 256; k += blockDim.x) cls[k] = d.cls[k];
    __syncthreads();
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < b.n; u += gridDim.x * blockDim.x) {
        const uint32_t f = fkey[u];
        if (f == none || (u > 0 && fkey[u - 1] == f)) continue;   // segment heads only
        uint32_t s = fstate[f], w = u;
        for (; w < b.n && fkey[w] == f; w++) {
            const uint32_t i = fidx[w], sp = span[i];
            Emit em{r, (uint32_t)b.first_global_index + i, sp & 0xFFFF, 0, 0};
            s = walk<M, true>(d, cls, b.arena + b.off[i], sp & 0xFFFF, sp >> 16, s, em);
            r.nocc[i] = em.cnt;
            r.drop[i] = (uint8_t)em.dr;
        }
        fin[w - 1] = s;
    }
}

__global__ void k_commit(uint32_t n, uint32_t none, const uint32_t *fkey, const uint32_t *fin, uint32_t *fstate)
{
    const uint32_t u = blockIdx.x * blockDim.x + threadIdx.x;
    if (u >= n) return;
    const uint32_t f = fkey[u];
    if (f != none && (u + 1 == n || fkey[u + 1] != f)) fstate[f] = fin[u];
}

}  // namespace

struct nfc_dpi_stream {
    int device = 0;
    uint32_t n_slots = 0, mask = 0, key_bits = 0;
    uint32_t *lock = nullptr, *keys = nullptr, *fstate = nullptr, *ctr = nullptr;
    // DFA (device)
    uint8_t *cls = nullptr, *trans = nullptr, *action = nullptr;
    uint32_t *out_off = nullptr;
    uint16_t *out_ids = nullptr;
    uint32_t ncls = 0, wide = 0, n_states = 0, maxlen = 0;
    uint32_t n_sm = 148, smem_ok = 0;   // k_walk<2>: the DFA fits the opt-in shared memory
    // per-call scratch
    uint32_t cap_pkts = 0;
    uint32_t *fkey = nullptr, *fkey2 = nullptr, *fidx = nullptr, *fidx2 = nullptr, *span = nullptr;
    unsigned long long *cumx = nullptr;
    uint32_t max_flows = 0;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    uint64_t launches = 0;
};

#define SCK(call)                                                                                  \
    do {                                                                                           \
        cudaError_t e_ = (call);                                                                   \
        if (e_ != cudaSuccess) return set_fail(NFC_ECUDA, std::string(#call ": ") + cudaGetErrorString(e_)); \
    } while (0)

template <class T>
static cudaError_t dev_copy(T **dst, const T *src, size_t n)
{
    cudaError_t e = cudaMalloc((void **)dst, std::max<size_t>(1, n) * sizeof(T));
    if (e != cudaSuccess) return e;
    return n ? cudaMemcpy(*dst, src, n * sizeof(T), cudaMemcpyHostToDevice) : cudaSuccess;
}

static void free_scratch(nfc_dpi_stream *s)
{
    cudaFree(s->fkey); cudaFree(s->fkey2); cudaFree(s->fidx); cudaFree(s->fidx2); cudaFree(s->span);
    cudaFree(s->cumx);
    cudaFree(s->tmp);
    s->fkey = s->fkey2 = s->fidx = s->fidx2 = s->span = nullptr;
    s->cumx = nullptr;
    s->tmp = nullptr;
    s->cap_pkts = 0;
    s->tmp_bytes = 0;
}

int nfc_dpi_stream_destroy(nfc_dpi_stream *s)
{
    if (!s) return NFC_OK;
    cudaSetDevice(s->device);
    free_scratch(s);
    cudaFree(s->lock); cudaFree(s->keys); cudaFree(s->fstate); cudaFree(s->ctr);
    cudaFree(s->cls); cudaFree(s->trans); cudaFree(s->action); cudaFree(s->out_off); cudaFree(s->out_ids);
    delete s;
    return NFC_OK;
}

static int create_from_host(int device, const DpiHost &h, uint32_t max_flows, nfc_dpi_stream **out);

int nfc_dpi_stream_create(int device, const nfc_dpi_spec *spec, uint32_t max_flows, nfc_dpi_stream **out)
{
    if (!spec || !out) return set_fail(NFC_EINVAL, "dpi_stream_create: NULL pointer");
    if (max_flows == 0 || max_flows > (1u << 28)) return set_fail(NFC_EINVAL, "dpi_stream_create: max_flows must be 1..2^28");
    *out = nullptr;
    DpiHost h;
    std::string e = build_dpi(*spec, h);
    if (!e.empty()) return set_fail(NFC_EINVAL, e);
    return create_from_host(device, h, max_flows, out);
}

int nfc_dpi_stream_create_regex(int device, const nfc_dpi_spec *spec, uint32_t max_flows, uint32_t max_states,
                                nfc_dpi_stream **out)
{
    if (!spec || !out) return set_fail(NFC_EINVAL, "dpi_stream_create_regex: NULL pointer");
    if (max_flows == 0 || max_flows > (1u << 28)) return set_fail(NFC_EINVAL, "dpi_stream_create_regex: max_flows must be 1..2^28");
    *out = nullptr;
    DpiHost h;
    std::string e = build_regex_dfa(*spec, h, max_states ? max_states : (1u << 20));
    if (!e.empty())
        return set_fail(e.find("out of host memory") != std::string::npos ? NFC_ENOMEM
                        : (e.find("unbounded") != std::string::npos || e.find("not supported") != std::string::npos)
                            ? NFC_EUNSUP : NFC_EINVAL, e);
    return create_from_host(device, h, max_flows, out);
}

static int create_from_host(int device, const DpiHost &h, uint32_t max_flows, nfc_dpi_stream **out)
{
    SCK(cudaSetDevice(device));
    nfc_dpi_stream *s = new nfc_dpi_stream;
    s->device = device;
    uint32_t lg = 1;
    while ((1u << lg) < 2 * max_flows) lg++;           // load factor <= 1/2
    s->n_slots = 1u << lg;
    s->max_flows = max_flows;
    s->mask = s->n_slots - 1;
    s->key_bits = lg + 1;                              // slot ids and the "none" key n_slots
    s->ncls = h.ncls;
    s->wide = h.wide;
    s->n_states = h.n_states;
    s->maxlen = h.maxlen;
    cudaError_t ce = cudaSuccess;
    auto ok = [&](cudaError_t x) { if (ce == cudaSuccess) ce = x; };
    ok(cudaMalloc((void **)&s->lock, (size_t)s->n_slots * 4));
    ok(cudaMalloc((void **)&s->keys, (size_t)s->n_slots * KS * 4));
    ok(cudaMalloc((void **)&s->fstate, (size_t)s->n_slots * 4));
    ok(cudaMalloc((void **)&s->ctr, 4 * 4));
    ok(dev_copy(&s->cls, h.cls.data(), h.cls.size()));
    ok(dev_copy(&s->trans, h.trans.data(), h.trans.size()));
    ok(dev_copy(&s->action, h.action.data(), h.action.size()));
    ok(dev_copy(&s->out_off, h.out_off.data(), h.out_off.size()));
    ok(dev_copy(&s->out_ids, h.out_ids.data(), h.out_ids.size()));
    if (ce == cudaSuccess) {
        ok(cudaMemset(s->lock, 0, (size_t)s->n_slots * 4));
        ok(cudaMemset(s->fstate, 0, (size_t)s->n_slots * 4));
        ok(cudaMemset(s->ctr, 0, 16));
        ok(cudaDeviceSynchronize());
    }
    if (ce == cudaSuccess && !s->wide && (size_t)s->ncls * s->n_states * 2 <= DFA_SMEM_MAX) {
        int nsm = 0;
        ok(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, device));
        ok(cudaFuncSetAttribute(k_walk<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)DFA_SMEM_MAX + 16));
        s->n_sm = nsm > 0 ? (uint32_t)nsm : 148;
        s->smem_ok = ce == cudaSuccess;
        // measured slower (one 768-thread CTA per SM: 491 vs 402 us per 4 M packets with
        // the rows in L1), so opt-in only
        if (!getenv("NFC_STREAM_SMEM")) s->smem_ok = 0;
    }
    if (ce != cudaSuccess) {
        nfc_dpi_stream_destroy(s);
        return set_fail(ce == cudaErrorMemoryAllocation ? NFC_ENOMEM : NFC_ECUDA,
                        std::string("dpi_stream_create: ") + cudaGetErrorString(ce));
    }
    *out = s;
    return NFC_OK;
}

int nfc_dpi_stream_reset(nfc_dpi_stream *s, void *stream)
{
    if (!s) return set_fail(NFC_EINVAL, "dpi_stream_reset: NULL stream object");
    SCK(cudaSetDevice(s->device));
    cudaStream_t st = (cudaStream_t)stream;
    SCK(cudaMemsetAsync(s->lock, 0, (size_t)s->n_slots * 4, st));
    SCK(cudaMemsetAsync(s->fstate, 0, (size_t)s->n_slots * 4, st));
    SCK(cudaMemsetAsync(s->ctr, 0, 16, st));
    return NFC_OK;
}

int nfc_dpi_stream_process(nfc_dpi_stream *s, const nfc_batch *b, const nfc_stream_result *r, void *stream)
{
    if (!s || !b || !r) return set_fail(NFC_EINVAL, "dpi_stream_process: NULL pointer");
    if (b->n == 0) return NFC_OK;
    if (!b->arena || !b->off || !b->len || !r->nocc || !r->drop || !r->occ_count ||
        (r->occ_cap && (!r->occ_pkt || !r->occ_pat || !r->occ_end)))
        return set_fail(NFC_EINVAL, "dpi_stream_process: NULL device buffer");
    SCK(cudaSetDevice(s->device));
    cudaStream_t st = (cudaStream_t)stream;
    if (b->n > s->cap_pkts) {
        SCK(cudaStreamSynchronize(st));
        free_scratch(s);
        const size_t n = b->n;
        SCK(cudaMalloc((void **)&s->fkey, n * 4));
        SCK(cudaMalloc((void **)&s->fkey2, n * 4));
        SCK(cudaMalloc((void **)&s->fidx, n * 4));
        SCK(cudaMalloc((void **)&s->fidx2, n * 4));
        SCK(cudaMalloc((void **)&s->span, n * 4));
        SCK(cudaMalloc((void **)&s->cumx, (n + 1) * 8));
        SCK(cub::DeviceRadixSort::SortPairs(nullptr, s->tmp_bytes, s->fkey, s->fkey2, s->fidx, s->fidx2,
                                            (int)n, 0, (int)s->key_bits, st));
        size_t scan_bytes = 0;
        SCK(cub::DeviceScan::ExclusiveSum(nullptr, scan_bytes, s->cumx, s->cumx, (int)n, st));
        s->tmp_bytes = std::max(s->tmp_bytes, scan_bytes);
        SCK(cudaMalloc(&s->tmp, std::max<size_t>(16, s->tmp_bytes)));
        s->cap_pkts = b->n;
    }
    const uint32_t none = s->n_slots;
    const uint32_t blocks = (b->n + 255) / 256;
    k_flow<<<blocks, 256, 0, st>>>(*b, s->lock, s->keys, s->mask, s->max_flows, none, s->ctr, s->fkey, s->fidx, s->span,
                                   r->nocc, r->drop);
    SCK(cudaGetLastError());
    size_t tb = s->tmp_bytes;
    SCK(cub::DeviceRadixSort::SortPairs(s->tmp, tb, s->fkey, s->fkey2, s->fidx, s->fidx2, (int)b->n, 0,
                                        (int)s->key_bits, st));
    k_plen<<<blocks, 256, 0, st>>>(b->n, none, s->fkey2, s->fidx2, s->span, s->cumx);
    SCK(cudaGetLastError());
    tb = s->tmp_bytes;
    SCK(cub::DeviceScan::ExclusiveSum(s->tmp, tb, s->cumx, s->cumx, (int)b->n, st));
    StreamDfa d{s->cls, s->trans, s->out_off, s->out_ids, s->action, s->ncls, s->wide, s->n_states};
    const uint32_t wb = (b->n + 255) / 256, need = s->maxlen - 1;
    // s->fkey (unsorted keys) is dead after the sort: it holds the flows' final states
    const size_t tbytes = (size_t)s->ncls * s->n_states * 2;
    if (s->maxlen == 0xFFFFFFFFu) {          // unbounded / very long matches: flow-serial
        if (s->wide) k_walk_serial<1><<<wb, 256, 0, st>>>(*b, d, none, s->fkey2, s->fidx2, s->span, s->fstate, s->fkey, *r);
        else k_walk_serial<0><<<wb, 256, 0, st>>>(*b, d, none, s->fkey2, s->fidx2, s->span, s->fstate, s->fkey, *r);
    } else if (s->wide) {
        k_walk<1><<<wb, 256, 0, st>>>(*b, d, none, need, s->fkey2, s->fidx2, s->span, s->cumx, s->fstate, s->fkey, *r);
    } else if (s->smem_ok && tbytes <= DFA_SMEM_MAX) {
        k_walk<2><<<s->n_sm, WALK_SMEM_THREADS, (tbytes + 15) / 16 * 16, st>>>(*b, d, none, need, s->fkey2, s->fidx2, s->span,
                                                                s->cumx, s->fstate, s->fkey, *r);
    } else {
        k_walk<0><<<wb, 256, 0, st>>>(*b, d, none, need, s->fkey2, s->fidx2, s->span, s->cumx, s->fstate, s->fkey, *r);
    }
    SCK(cudaGetLastError());
    k_commit<<<blocks, 256, 0, st>>>(b->n, none, s->fkey2, s->fkey, s->fstate);
    SCK(cudaGetLastError());
    s->launches += 4;   // k_flow + k_plen + k_walk + k_commit (the cub sort and scan launch their own kernels)
    return NFC_OK;
}

int nfc_dpi_stream_flows(nfc_dpi_stream *s, uint64_t *n_flows, uint64_t *n_unplaced)
{
    if (!s || !n_flows || !n_unplaced) return set_fail(NFC_EINVAL, "dpi_stream_flows: NULL pointer");
    SCK(cudaSetDevice(s->device));
    SCK(cudaDeviceSynchronize());
    uint32_t c[4];
    SCK(cudaMemcpy(c, s->ctr, 16, cudaMemcpyDeviceToHost));
    *n_flows = c[0];
    *n_unplaced = c[1];
    return NFC_OK;
}
