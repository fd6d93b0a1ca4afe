// parallel.cu -- NEXT-2: SFC parallelization on B200 with packet
// duplication and XOR merge (P:L243-263 [SIV.B.1], Figs. 13-14).
//
// The chain's NFs form parallel-legal groups (nfc_plan_parallel; R#16).
// Every chain this mode accepts (no IPsec) is one group: ACL, DPI, the two
// forwarders (family-disjoint writes) and the load balancer neither read what
// another writes nor write the same field.  So all NFs of the chain run at once:
// a team of n warps (n = chain length) takes a 32-packet chunk, warp j applies NF
// j to ITS OWN copy of the 32 packets (each warp reads and parses the headers
// itself: the duplication of P:L256), and publishes its effects in shared
// memory.  After a team barrier the leader warp merges: header bytes
// out = orig ^ OR_j (orig ^ copy_j) (only the forwarders' copies differ), verdict
// = the earliest dropper in original order, whose later members' side effects
// (alerts = match pairs, per-rule and per-backend hits) are discarded;
// egress port = last setter in original order (R#19).  Results are identical to
// the sequential chain (reorg oracle invariant, tests/test_reorg.py).
//
// The DFA uses the tiered placement (DM_HOT) so the effect slots fit next to it.
// Selected by nfc_chain_opts.flags & NFC_F_PARALLEL.
#include "sfc_kernel.cuh"

namespace nfc {

static constexpr int PAR_NT = 768;

// per (member, lane) effect record, 16 B
//   x: port | dropped << 16 | pass << 17 | set_port << 18
//   y: acl_rule | lb_backend << 16      z: DPI accept events   w: DPI largest entry
__device__ __forceinline__ void bar_team(uint32_t id, uint32_t threads)
{
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(threads) : "memory");
}

// teams per CTA: named barriers 1..15 (0 is __syncthreads)
__host__ __device__ inline uint32_t par_teams(uint32_t n_nf) { return min((uint32_t)(PAR_NT / 32) / n_nf, 15u); }

size_t par_region_bytes(uint32_t n_nf, uint32_t n_fwd)
{
    const uint32_t teams = par_teams(n_nf);
    return (size_t)teams * (n_nf * 32 * 16 + n_fwd * 32 * 32 + 16 + 32 * 4);
}

__global__ void __launch_bounds__(PAR_NT, 1) par_kernel(const KParams P, uint32_t n_fwd)
{
    uint8_t *smem = nfc_smem;
    const SmemLayout &L = P.lay;
    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t n = P.n_nf, teams = par_teams(n);
    const uint32_t team = warp / n, j = warp % n;
    unsigned long long *wst = reinterpret_cast<unsigned long long *>(smem + L.wst);
    uint32_t *vst = reinterpret_cast<uint32_t *>(smem + L.vst);
    const uint32_t n_var = P.stats_len - NFIX;
    for (uint32_t i = tid; i < (PAR_NT / 32) * NWS; i += PAR_NT) wst[i] = 0;
    if (P.smem_stats)
        for (uint32_t i = tid; i < n_var; i += PAR_NT) vst[i] = 0;
    Ctx C;
    setup_ctx<MASK_ACL | MASK_DPI | MASK_LPM4 | MASK_LPM6 | MASK_LB, DM_HOT, PAR_NT>(P, smem, L, P.present, false, vst, C);
    __syncthreads();

    if (team < teams) {
        uint8_t *tb = smem + L.par + team * (n * 32 * 16 + n_fwd * 32 * 32 + 16 + 32 * 4);
        uint4 *eff = reinterpret_cast<uint4 *>(tb);                        // [n][32]
        uint32_t *hcopy = reinterpret_cast<uint32_t *>(tb + n * 32 * 16);  // [n_fwd][8 words][32]
        uint32_t *s_chunk = reinterpret_cast<uint32_t *>(tb + n * 32 * 16 + n_fwd * 32 * 32);
        uint32_t *s_alive = s_chunk + 4;                                   // [32]: packet alive after a group
        unsigned long long *ws = wst + warp * NWS;
        // slot of this member's header copy (forwarders only)
        uint32_t fslot = 0;
        for (uint32_t q = 0; q < j; q++) fslot += (P.kind[q] == NFC_LPM4 || P.kind[q] == NFC_LPM6);
        const uint32_t kind = P.kind[j];
        const uint32_t bar = 1 + team, bthreads = n * 32;
        for (;;) {
            if (j == 0 && lane == 0) *s_chunk = atomicAdd(P.tile_counter, 32u);
            bar_team(bar, bthreads);
            const uint32_t c0 = *s_chunk;
            if (c0 >= P.n_pkts) break;
            const uint32_t g = c0 + lane;
            const bool valid = g < P.n_pkts;
            const Loc loc = pkt_locate(P, g, valid);
            Pkt k;
            pkt_begin(C, loc, valid, k);                                  // this member's copy
            // groups in order (configuration (c) of Fig. 13 has two): the members
            // of group gi run on copies of the packet that enters gi (the merge of the groups
            // before it, re-read from memory), the leader merges them, and the next group starts
            for (uint32_t gi = 0; gi < P.n_groups; gi++) {
                const bool mem = P.group[j] == gi;
                if (gi > 0) {
                    bar_team(bar, bthreads);                               // the leader's merge of gi-1 is out
                    if (mem) {
                        pkt_begin(C, loc, valid, k);                       // the packet entering gi
                        if (!s_alive[lane]) k.alive = false;
                    }
                }
                // ---- member j of group gi: NF j on its copy, no side effects outside the team
                if (mem) {
                    uint32_t x = 0, y = 0xFFFFFFFFu, z = 0, w = 0;
                    if (valid && k.alive) {
                        if (kind == NFC_ACL) {
                            const uint32_t r = nf_acl(C.acl4, C.acl6, P.acl, k.v);
                            y = (r & 0xFFFF) | 0xFFFF0000u;
                            x = (r >> 31) << 16;
                        } else if (kind == NFC_DPI) {
                            const Walk wk = dpi_walk<DM_HOT>(P, C.dpi, k.h, k.f, k.v.pl_off, k.v.ip_end, C.pol_f);
                            z = wk.cnt;
                            w = wk.mx;
                            bool drop = false;
                            const uint32_t st = C.dpi.wide ? (wk.mx & 0x7FFFFFFFu) : (wk.mx & 0x7FFFu);
                            const uint32_t meta = wk.cnt == 1 ? C.meta[st] : 0u;
                            if (wk.cnt == 1 && meta != DPI_META_NONE) {
                                drop = (meta >> 31) != 0;
                            } else if (wk.cnt >= 1) {                     // exact set: DROP flag only
                                const DpiOvf ov{P.dpi.ovf_bitmap, P.dpi.bitmap_words, P.match_count, P.match_pkt,
                                                P.match_pat, P.match_cap, P.stats, 0u};
                                drop = (dpi_slow<DM_HOT>(C.dpi, k.f, k.v.pl_off, k.v.ip_end, C.gtid, ov, pkt_gidx(P, k.g)) >> 31) != 0;
                            }
                            x = (uint32_t)drop << 16;
                        } else if (kind == NFC_LPM4 || kind == NFC_LPM6) {
                            const uint32_t fam = kind == NFC_LPM4 ? 4 : 6;
                            if (k.v.fam != fam) {
                                x = 1u << 17;                              // passes the other family
                            } else {
                                uint32_t nh;
                                if (fam == 4) {
                                    nh = ld_tab16(P.l4.tbl24 + (k.v.dst[0] >> 8), C.pol_l);
                                    if (nh & 0x8000) nh = ld_tab16(P.l4.tbllong + ((nh & 0x7FFF) << 8) + (k.v.dst[0] & 0xFF), C.pol_l);
                                } else {
                                    nh = lpm6_lookup(P.l6, k.v.dst);
                                }
                                if (nh == 0x7FFF || hbyte(k.h, fam == 4 ? 22 : 21) <= 1) {
                                    x = 1u << 16;
                                } else {
                                    const uint2 e = __ldg((fam == 4 ? P.l4.nh : P.l6.nh) + nh);
                                    const uint32_t pt = e.y >> 16;
                                    forward_words(k.f, k.h, k.v, e, __ldg((fam == 4 ? P.l4.pmac : P.l6.pmac) + pt));
                                    x = pt | 1u << 18;
                                }
                            }
                        } else if (kind == NFC_LB) {
                            const uint32_t b = (uint32_t)(((uint64_t)toeplitz(C.lb_nib, k.v) * P.lb.n_backends) >> 32);
                            y = 0xFFFFu | b << 16;
                            x = __ldg(P.lb.port + b) | 1u << 18;
                        }
                    }
                    eff[j * 32 + lane] = make_uint4(x, y, z, w);
                    if (kind == NFC_LPM4 || kind == NFC_LPM6) {
#pragma unroll
                        for (int q = 0; q < 8; q++) hcopy[(fslot * 8 + q) * 32 + lane] = k.h[q];
                        if (j == 0 && valid) load_header(k.f, k.flen, k.h, C.pol_f);   // the leader merges against the original
                    }
                }
                bar_team(bar, bthreads);
                // ---- leader: merge group gi and commit
                if (j == 0) {
                    if (valid && k.alive) {
                        uint32_t acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
                        uint32_t fs = 0;
                        for (uint32_t p = 0; p < n; p++) {
                            const uint32_t kd = P.kind[p];
                            const bool fwd = kd == NFC_LPM4 || kd == NFC_LPM6;
                            if (P.group[p] != gi) { fs += fwd; continue; }
                            const uint4 e = eff[p * 32 + lane];
                            if (fwd) {
#pragma unroll
                                for (int q = 0; q < 8; q++) acc[q] |= k.h[q] ^ hcopy[(fs * 8 + q) * 32 + lane];
                                fs++;
                            }
                            if (kd == NFC_ACL) {
                                k.acl_rule = e.y & 0xFFFF;
                                var_stat(P, C, P.st_acl + (k.acl_rule == 0xFFFF ? P.acl.n_rules : k.acl_rule));
                            } else if (kd == NFC_DPI) {
                                k.nmatch = 0;
                                if (e.z) {
                                    const Walk wk{0, e.z, e.w};
                                    dpi_finish<DM_HOT>(P, C, k, wk);       // emits the pairs, sets nmatch
                                    k.npairs += k.nmatch;
                                }
                            } else if (kd == NFC_LB) {
                                k.lb_b = e.y >> 16;
                                var_stat(P, C, P.st_lb + k.lb_b);
                            }
                            if ((e.x >> 18) & 1) k.port = e.x & 0xFFFF;
                            if ((e.x >> 17) & 1) k.passmask |= 1u << p;
                            if ((e.x >> 16) & 1) { k.drop = p; k.alive = false; break; }
                        }
                        if (k.alive) {                                     // merged header bytes
                            uint32_t any = 0;
#pragma unroll
                            for (int q = 0; q < 8; q++) { k.h[q] ^= acc[q]; any |= acc[q]; }
                            if (any) {
                                st_stream16(k.f, make_uint4(k.h[0], k.h[1], k.h[2], k.h[3]), C.pol_f);
                                st_stream16(k.f + 16, make_uint4(k.h[4], k.h[5], k.h[6], k.h[7]), C.pol_f);
                            }
                        }
                    }
                    if (gi + 1 < P.n_groups) s_alive[lane] = valid && k.alive;
                }
            }
            if (j == 0) pkt_end<SIG_ANY>(P, C, k, valid, g, ws, lane);
        }
    }
    // ---- flush CTA counters (as sfc_kernel)
    __syncthreads();
    constexpr int NW = PAR_NT / 32;
    if (warp == 0) {
        unsigned long long t[2] = {0, 0};
#pragma unroll
        for (int r = 0; r < 2; r++) {
            const uint32_t idx = lane + 32 * r;
            if (idx < NWS)
                for (int q = 0; q < NW; q++) t[r] += wst[q * NWS + idx];
        }
        __syncwarp();
        wst[lane] = t[0];
        if (lane + 32 < NWS) wst[lane + 32] = t[1];
        __syncwarp();
        if (lane == 0) {
            unsigned long long in = wst[ST_PKTS] - wst[ST_PARSE_DROP];
            for (uint32_t p = 0; p < P.n_nf; p++) {
                const unsigned long long d = wst[ST_POS_BASE + 4 * p + 1], ps = wst[ST_POS_BASE + 4 * p + 2];
                wst[ST_POS_BASE + 4 * p] = in;
                wst[ST_POS_BASE + 4 * p + 3] = in - d - ps;
                in -= d;
            }
            if (NFC_FWD_DERIVED) wst[ST_FWD] = in;   // survivors of every position
            wst[ST_DROP] = wst[ST_PKTS] - wst[ST_FWD];
        }
        __syncwarp();
        for (uint32_t idx = lane; idx < NWS; idx += 32)
            if (wst[idx]) atomicAdd(&P.stats[idx], wst[idx]);
    }
    if (P.smem_stats)
        for (uint32_t i = tid; i < n_var; i += PAR_NT)
            if (vst[i]) atomicAdd(&P.stats[NFIX + i], (unsigned long long)vst[i]);
}

size_t par_smem_bytes(const KParams &p, uint32_t n_fwd)
{
    return smem_layout(p.present, PAR_NT / 32, p, NWS, DM_HOT).total + par_region_bytes(p.n_nf, n_fwd);
}

int par_launch(const KParams &p, int device, void *stream, std::string &err, LaunchCfg *cfg)
{
    uint32_t n_fwd = 0;
    for (uint32_t q = 0; q < p.n_nf; q++) n_fwd += (p.kind[q] == NFC_LPM4 || p.kind[q] == NFC_LPM6);
    KParams q = p;
    q.lay = smem_layout(p.present, PAR_NT / 32, p, NWS, DM_HOT);
    q.lay.par = (q.lay.total + 15) & ~15u;
    const size_t smem = q.lay.par + par_region_bytes(p.n_nf, n_fwd);
    if (cudaFuncSetAttribute(par_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess) {
        err = "cudaFuncSetAttribute (parallel) failed: shared memory " + std::to_string(smem) + " B";
        return NFC_ECUDA;
    }
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    const uint32_t teams = par_teams(p.n_nf);
    const uint32_t chunks = (p.n_pkts + 31) / 32;
    const int grid = (int)std::max<uint32_t>(1, std::min<uint32_t>((uint32_t)sms, (chunks + teams - 1) / teams));
    if (cfg) { cfg->grid = grid; cfg->block = PAR_NT; cfg->smem = smem; }
    par_kernel<<<grid, PAR_NT, smem, (cudaStream_t)stream>>>(q, n_fwd);
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) { err = std::string("parallel kernel: ") + cudaGetErrorString(e); return NFC_ECUDA; }
    return NFC_OK;
}

} // namespace nfc
