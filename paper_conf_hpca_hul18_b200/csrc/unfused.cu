// unfused.cu -- the NEXT-1 baseline: the same chain run as one
// kernel per NF with a device-side re-split of the surviving packets between
// NFs -- the per-NF element pipeline NFCompass replaces (Figs. 5
// and 7; "the batch is split ... 36.5 -> 15.8 Gbps").  Every stage
// re-reads the packet header from memory and re-parses it (the redundant
// per-NF classifier of P:L267), re-loads and re-stores the per-packet record,
// and appends its survivors to the next stage's index list.  Results are
// identical to the fused kernel (same device functions); chains with IPsec are
// not offered here (NFC_EUNSUP).  Selected by nfc_chain_opts.flags & NFC_F_UNFUSED.
#include "sfc_kernel.cuh"

namespace nfc {

static constexpr int UF_NT = 256;

// warp-aggregated append of `take` lanes' packet ids to a list (order is irrelevant:
// the chains offered here are per-packet stateless)
__device__ __forceinline__ void uf_append(bool take, uint32_t g, uint32_t *list, uint32_t *count, uint32_t lane)
{
    const uint32_t m = __ballot_sync(0xFFFFFFFFu, take);
    if (!m) return;
    uint32_t base = 0;
    if (lane == 0) base = atomicAdd(count, (uint32_t)__popc(m));
    base = __shfl_sync(0xFFFFFFFFu, base, 0);
    if (take) list[base + __popc(m & ((1u << lane) - 1))] = g;
}

__device__ __forceinline__ uint4 uf_pack(const Pkt &k)
{
    const uint32_t port = k.drop != 0xFF ? 0xFFFFu : k.port;
    return make_uint4(k.drop | k.esp_sa << 8 | port << 16, k.acl_rule | k.lb_b << 16, k.nmatch | k.out_len << 16,
                      k.esp_seq);
}

// stage 0: initial records, parse ("FromDevice + Classifier"), list of parsed packets
__global__ void __launch_bounds__(UF_NT) uf_parse_kernel(const KParams P, uint32_t *out_list, uint32_t *out_count,
                                                         uint8_t *passmask)
{
    const uint32_t lane = threadIdx.x & 31;
    Ctx C{};
    C.pol_f = pol_first();
    for (uint32_t g0 = blockIdx.x * UF_NT; g0 < P.n_pkts; g0 += gridDim.x * UF_NT) {
        const uint32_t g = g0 + threadIdx.x;
        const bool valid = g < P.n_pkts;
        Pkt k;
        pkt_begin(C, pkt_locate(P, g, valid), valid, k);
        if (valid) {
            reinterpret_cast<uint4 *>(P.rec)[g] = uf_pack(k);
            passmask[g] = 0;
        }
        uf_append(valid && k.alive, g, out_list, out_count, lane);
    }
}

// one NF over the packets that survived the previous stages
template <uint32_t KIND, int DM, int NT>
__global__ void __launch_bounds__(NT, DM == DM_FULL ? 1 : 2)
    uf_nf_kernel(const KParams P, uint32_t pos, const uint32_t *in_list, const uint32_t *in_count, uint32_t *out_list,
                 uint32_t *out_count, uint8_t *passmask)
{
    uint8_t *smem = nfc_smem;
    const uint32_t mask = 1u << KIND;
    const SmemLayout &L = P.lay;
    const uint32_t tid = threadIdx.x, lane = tid & 31;
    uint32_t *vst = reinterpret_cast<uint32_t *>(smem + L.vst);
    const uint32_t n_var = P.stats_len - NFIX;
    if (P.smem_stats)
        for (uint32_t i = tid; i < n_var; i += NT) vst[i] = 0;
    Ctx C;
    setup_ctx<1u << KIND, DM, NT>(P, smem, L, mask, false, vst, C);
    C.gtid = blockIdx.x * NT + tid;
    __syncthreads();
    const uint32_t n = *in_count;
    for (uint32_t i0 = blockIdx.x * NT; i0 < n; i0 += gridDim.x * NT) {
        const uint32_t i = i0 + tid;
        const bool valid = i < n;
        const uint32_t g = valid ? in_list[i] : 0;
        Pkt k;
        pkt_begin(C, pkt_locate(P, g, valid), valid, k);     // header re-read + re-parse
        if (valid) {                                          // the packet's state so far
            const uint4 r = reinterpret_cast<const uint4 *>(P.rec)[g];
            k.port = r.x >> 16;
            k.acl_rule = r.y & 0xFFFF;
            k.lb_b = r.y >> 16;
            k.nmatch = r.z & 0xFFFF;
            k.out_len = r.z >> 16;
        }
        const bool ran = valid && k.alive;
        if (ran) nf_apply<KIND, DM>(P, C, k, pos);
        if constexpr (KIND == NFC_DPI) {                      // pairs of this DPI stage (a chain may repeat DPI)
            const uint32_t pr = __reduce_add_sync(0xFFFFFFFFu, ran ? k.nmatch : 0u);
            if (lane == 0 && pr) atomicAdd(&P.stats[ST_DPI_PAIRS], (unsigned long long)pr);
        }
        if (valid) {
            reinterpret_cast<uint4 *>(P.rec)[g] = uf_pack(k);
            if (k.passmask) passmask[g] |= (uint8_t)k.passmask;
        }
        uf_append(valid && k.alive, g, out_list, out_count, lane);
    }
    __syncthreads();
    if (P.smem_stats)
        for (uint32_t i = tid; i < n_var; i += NT)
            if (vst[i]) atomicAdd(&P.stats[NFIX + i], (unsigned long long)vst[i]);
}

// final stage: the fixed and per-position counters from the records (per-rule /
// per-backend hits were counted by the NF stages)
__global__ void __launch_bounds__(UF_NT) uf_stats_kernel(const KParams P, const uint8_t *passmask)
{
    __shared__ unsigned long long cnt[NWS];
    const uint32_t tid = threadIdx.x, lane = tid & 31;
    for (uint32_t i = tid; i < NWS; i += UF_NT) cnt[i] = 0;
    __syncthreads();
    const uint32_t FULL = 0xFFFFFFFFu;
    for (uint32_t g0 = blockIdx.x * UF_NT; g0 < P.n_pkts; g0 += gridDim.x * UF_NT) {
        const uint32_t g = g0 + tid;
        const bool valid = g < P.n_pkts;
        uint4 r = make_uint4(0xFF, 0, 0, 0);
        uint32_t len = 0, pm = 0;
        if (valid) {
            r = reinterpret_cast<const uint4 *>(P.rec)[g];
            len = pkt_locate(P, g, true).len;
            pm = passmask[g];
        }
        const uint32_t drop = r.x & 0xFF, nm = r.z & 0xFFFF, olen = r.z >> 16;
        const bool fwd = valid && drop == 0xFF;
        const uint32_t v[6] = {(uint32_t)__popc(__ballot_sync(FULL, valid)), (uint32_t)__popc(__ballot_sync(FULL, fwd)),
                               (uint32_t)__popc(__ballot_sync(FULL, valid && drop == 0xFE)),
                               __reduce_add_sync(FULL, len), __reduce_add_sync(FULL, fwd ? olen : 0u),
                               __reduce_add_sync(FULL, valid ? nm : 0u)};
        uint32_t nd[NFC_MAX_CHAIN], np[NFC_MAX_CHAIN];
#pragma unroll
        for (int p = 0; p < NFC_MAX_CHAIN; p++) {
            nd[p] = __popc(__ballot_sync(FULL, valid && drop == (uint32_t)p));
            np[p] = __popc(__ballot_sync(FULL, valid && ((pm >> p) & 1)));
        }
        if (lane == 0) {
            atomicAdd(&cnt[ST_PKTS], (unsigned long long)v[0]);
            atomicAdd(&cnt[ST_FWD], (unsigned long long)v[1]);
            atomicAdd(&cnt[ST_PARSE_DROP], (unsigned long long)v[2]);
            atomicAdd(&cnt[ST_BYTES_IN], (unsigned long long)v[3]);
            atomicAdd(&cnt[ST_BYTES_OUT], (unsigned long long)v[4]);
            for (int p = 0; p < NFC_MAX_CHAIN; p++) {
                atomicAdd(&cnt[ST_POS_BASE + 4 * p + 1], (unsigned long long)nd[p]);
                atomicAdd(&cnt[ST_POS_BASE + 4 * p + 2], (unsigned long long)np[p]);
            }
        }
    }
    __syncthreads();
    if (tid == 0) {
        cnt[ST_DROP] = cnt[ST_PKTS] - cnt[ST_FWD];
        unsigned long long in = cnt[ST_PKTS] - cnt[ST_PARSE_DROP];
        for (uint32_t p = 0; p < P.n_nf; p++) {
            const unsigned long long d = cnt[ST_POS_BASE + 4 * p + 1], ps = cnt[ST_POS_BASE + 4 * p + 2];
            cnt[ST_POS_BASE + 4 * p] = in;
            cnt[ST_POS_BASE + 4 * p + 3] = in - d - ps;
            in -= d;
        }
        for (uint32_t p = P.n_nf; p < NFC_MAX_CHAIN; p++) cnt[ST_POS_BASE + 4 * p + 1] = cnt[ST_POS_BASE + 4 * p + 2] = 0;
    }
    __syncthreads();
    for (uint32_t i = tid; i < NWS; i += UF_NT)
        if (cnt[i]) atomicAdd(&P.stats[i], cnt[i]);
}

template <uint32_t KIND, int DM>
static int uf_stage(const KParams &p, uint32_t pos, const uint32_t *in, const uint32_t *in_n, uint32_t *out,
                    uint32_t *out_n, uint8_t *pm, int sms, cudaStream_t st, std::string &err)
{
    constexpr int NT = DM == DM_FULL ? 768 : 256;
    const size_t smem = smem_layout(1u << KIND, NT / 32, p, NWS, DM).total;
    if (cudaFuncSetAttribute(uf_nf_kernel<KIND, DM, NT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
        cudaSuccess) {
        err = "cudaFuncSetAttribute (unfused stage) failed";
        return NFC_ECUDA;
    }
    int per_sm = 1;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, uf_nf_kernel<KIND, DM, NT>, NT, smem);
    if (per_sm < 1) per_sm = 1;
    KParams q = p;
    q.lay = smem_layout(1u << KIND, NT / 32, p, NWS, DM);
    uf_nf_kernel<KIND, DM, NT><<<sms * per_sm, NT, smem, st>>>(q, pos, in, in_n, out, out_n, pm);
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) { err = std::string("unfused stage: ") + cudaGetErrorString(e); return NFC_ECUDA; }
    return NFC_OK;
}

int uf_launch(const uint32_t *kinds, uint32_t n_nf, int dm, const KParams &p, uint32_t *list0, uint32_t *list1,
              uint32_t *counts, uint8_t *passmask, int device, void *stream, std::string &err, uint32_t *n_launch)
{
    cudaStream_t st = (cudaStream_t)stream;
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    *n_launch = 0;
    const uint32_t grid = std::min<uint32_t>((p.n_pkts + UF_NT - 1) / UF_NT, (uint32_t)sms * 8);
    uf_parse_kernel<<<grid, UF_NT, 0, st>>>(p, list0, counts, passmask);
    ++*n_launch;
    uint32_t *lists[2] = {list0, list1};
    for (uint32_t pos = 0; pos < n_nf; pos++) {
        const uint32_t *in = lists[pos & 1], *in_n = counts + pos;
        uint32_t *out = lists[(pos + 1) & 1], *out_n = counts + pos + 1;
        int rc = NFC_OK;
        switch (kinds[pos]) {
        case NFC_ACL: rc = uf_stage<NFC_ACL, DM_HOT>(p, pos, in, in_n, out, out_n, passmask, sms, st, err); break;
        case NFC_DPI:
            rc = dm == DM_FULL ? uf_stage<NFC_DPI, DM_FULL>(p, pos, in, in_n, out, out_n, passmask, sms, st, err)
                               : uf_stage<NFC_DPI, DM_HOT>(p, pos, in, in_n, out, out_n, passmask, sms, st, err);
            break;
        case NFC_LPM4: rc = uf_stage<NFC_LPM4, DM_HOT>(p, pos, in, in_n, out, out_n, passmask, sms, st, err); break;
        case NFC_LPM6: rc = uf_stage<NFC_LPM6, DM_HOT>(p, pos, in, in_n, out, out_n, passmask, sms, st, err); break;
        case NFC_LB: rc = uf_stage<NFC_LB, DM_HOT>(p, pos, in, in_n, out, out_n, passmask, sms, st, err); break;
        case NFC_NAT: rc = uf_stage<NFC_NAT, DM_HOT>(p, pos, in, in_n, out, out_n, passmask, sms, st, err); break;
        default: err = "unfused mode does not run IPsec"; return NFC_EUNSUP;
        }
        if (rc) return rc;
        ++*n_launch;
    }
    uf_stats_kernel<<<grid, UF_NT, 0, st>>>(p, passmask);
    ++*n_launch;
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) { err = std::string("unfused: ") + cudaGetErrorString(e); return NFC_ECUDA; }
    return NFC_OK;
}

} // namespace nfc
