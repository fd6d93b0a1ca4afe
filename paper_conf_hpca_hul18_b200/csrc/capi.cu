// capi.cu -- the C ABI (include/nfc.h): chain object, table upload, launch,
// stats.  Host runtime around the fused kernel; no compute happens here
// beyond building table images (builders.cpp).
#include <cuda_runtime.h>

#include <cstdio>
#include <algorithm>
#include <cstring>
#include <string>
#include <vector>

#include "nfc_internal.h"

using namespace nfc;

static thread_local std::string g_err;

static int fail(int code, const std::string &msg)
{
    g_err = msg;
    return code;
}

int nfc::set_fail(int code, const std::string &msg) { return fail(code, msg); }

#define CK(call)                                                                                   \
    do {                                                                                           \
        cudaError_t e_ = (call);                                                                   \
        if (e_ != cudaSuccess) return fail(NFC_ECUDA, std::string(#call ": ") + cudaGetErrorString(e_)); \
    } while (0)

namespace {
struct DBuf {
    void *p = nullptr;
    size_t n = 0;
    void release()
    {
        if (p) cudaFree(p);
        p = nullptr;
        n = 0;
    }
    cudaError_t reserve(size_t bytes)
    {
        if (bytes <= n && p) return cudaSuccess;
        release();
        cudaError_t e = cudaMalloc(&p, bytes ? bytes : 16);
        if (e == cudaSuccess) n = bytes;
        return e;
    }
    template <typename T> cudaError_t upload(const std::vector<T> &v)
    {
        cudaError_t e = reserve(v.size() * sizeof(T));
        if (e != cudaSuccess) return e;
        return v.empty() ? cudaSuccess : cudaMemcpy(p, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice);
    }
    template <typename T> T *as() const { return reinterpret_cast<T *>(p); }
};
} // namespace

struct nfc_chain {
    int device = 0;
    uint32_t n_nf = 0;
    uint32_t kind[NFC_MAX_CHAIN] = {0};
    uint32_t mask = 0;
    uint32_t esp_pos = 0xFF;
    uint32_t flags = 0;
    uint8_t group[NFC_MAX_CHAIN] = {0};   // NFC_F_PARALLEL groups (default: nfc_plan_parallel)
    nfc_launch_info last{};               // shape of the last fused launch
    DBuf uf_list[2], uf_cnt, uf_pass;     // NFC_F_UNFUSED scratch
    bool loaded[8] = {false};
    // tables
    DBuf acl_r4, acl_r6, acl_f4, acl_x4;
    AclImg acl{};
    DBuf dpi_cls, dpi_trans, dpi_off, dpi_ids, dpi_act, dpi_bitmap, dpi_meta, dpi_sparse, dpi_frows, dpi_accid, dpi_accmeta;
    DpiImg dpi{};
    DBuf l4_tbl24, l4_long, l4_nh, l4_pmac;
    Lpm4Img l4{};
    DBuf l6_lens, l6_base, l6_mask, l6_ent, l6_nh, l6_pmac;
    Lpm6Img l6{};
    DBuf esp_sa, esp_te, esp_nib, esp_seq[2];
    EspImg esp{};
    uint32_t seq_parity = 0;
    DBuf lb_port, lb_nib;
    LbImg lb{};
    NatImg nat{};
    DBuf nat_pool, nat_dnat, nat_nib;
    // stats
    DBuf stats;
    uint32_t stats_len = ST_VAR_BASE;
    uint32_t n_acl_rules = 0, n_lb = 0, n_sa = 0;
    // scheduling
    DBuf counter, tile_flag, tile_vec, batches, crec;
    uint32_t tile_cap = 0;
    uint32_t epoch = 0;
    // host e2e staging
    DBuf h_arena, h_off, h_len, h_rec, h_mp, h_mq, h_mc;
    uint64_t launches = 0;
    cudaStream_t last_stream = nullptr;
    void *comm = nullptr;                 // attached ncclComm_t (NFC_STATS_ALLREDUCE)
    static constexpr int NXS = 4;
    cudaStream_t xs[NXS] = {nullptr, nullptr, nullptr, nullptr};   // nfc_process_host copy/compute streams
    // a3 regrouping: mixed IPv4/IPv6 chunks of the last launch, read back asynchronously; the
    // regrouping kernel variant runs while more than 1/8 of the chunks were mixed
    DBuf mix_dev;
    uint32_t *mix_host = nullptr;         // pinned
    cudaEvent_t mix_ev = nullptr;
    uint32_t mix_chunks = 0;
    bool mix_pending = false, rg_on = false;
    cudaEvent_t xk = nullptr;
    DBuf stats_red;                       // all-reduce destination
};

static int set_device(const nfc_chain *c)
{
    CK(cudaSetDevice(c->device));
    return NFC_OK;
}

static int realloc_stats(nfc_chain *c)
{
    c->stats_len = ST_VAR_BASE + (c->n_acl_rules + 1) + c->n_lb + c->n_sa;
    CK(c->stats.reserve((size_t)c->stats_len * 8));
    CK(cudaMemset(c->stats.p, 0, (size_t)c->stats_len * 8));
    return NFC_OK;
}

extern "C" {

const char *nfc_last_error(void) { return g_err.c_str(); }
const char *nfc_version(void) { return "nfc-b200 0.1 (sm_100a)"; }

int nfc_build_chain(const uint32_t *kinds, uint32_t n, const nfc_chain_opts *opts, nfc_chain **out)
{
    if (!kinds || !out) return fail(NFC_EINVAL, "kinds/out is NULL");
    if (n < 1 || n > NFC_MAX_CHAIN) return fail(NFC_EUNSUP, "chain length must be 1..6");
    uint32_t mask = 0;
    for (uint32_t i = 0; i < n; i++) {
        if (kinds[i] < NFC_ACL || kinds[i] > NFC_NAT) return fail(NFC_EINVAL, "unknown NF kind");
        // repeated kinds (the paper's four identical FW / IDS NFs, Fig. 13)
        // share the kind's tables; IPsec and NAT keep per-chain state or decide on metadata
        // of one position (the ESP sequence look-back, the NAT's egress-port test): once each
        if ((mask & (1u << kinds[i])) && (kinds[i] == NFC_IPSEC || kinds[i] == NFC_NAT))
            return fail(NFC_EUNSUP, "IPsec / NAT at most once per chain");
        mask |= 1u << kinds[i];
    }
    const uint32_t flags = opts ? opts->flags : 0;
    if (flags & ~(NFC_F_UNFUSED | NFC_F_PARALLEL)) return fail(NFC_EINVAL, "opts->flags: unknown bits");
    if ((flags & NFC_F_UNFUSED) && (flags & NFC_F_PARALLEL)) return fail(NFC_EINVAL, "opts->flags: UNFUSED and PARALLEL are exclusive");
    if ((flags & NFC_F_UNFUSED) && (mask & (1u << NFC_IPSEC))) return fail(NFC_EUNSUP, "NFC_F_UNFUSED: IPsec chains are not offered");
    if ((flags & NFC_F_PARALLEL) && (mask & ((1u << NFC_IPSEC) | (1u << NFC_NAT))))
        return fail(NFC_EUNSUP, "NFC_F_PARALLEL: IPsec and NAT chains are not offered");
    nfc_chain *c = new (std::nothrow) nfc_chain();
    if (!c) return fail(NFC_ENOMEM, "out of host memory");
    c->device = opts ? opts->device : 0;
    c->flags = flags;
    c->n_nf = n;
    c->mask = mask;
    for (uint32_t i = 0; i < n; i++) {
        c->kind[i] = kinds[i];
        if (kinds[i] == NFC_IPSEC) c->esp_pos = i;
    }
    nfc_plan_parallel(kinds, n, c->group);             // NFC_F_PARALLEL grouping (nfc_set_groups)
    int rc = set_device(c);
    if (rc == NFC_OK) {
        cudaError_t e = c->counter.reserve(16);
        if (e == cudaSuccess) e = cudaMemset(c->counter.p, 0, 16);
        if (e != cudaSuccess) rc = fail(NFC_ECUDA, cudaGetErrorString(e));
    }
    if (rc == NFC_OK) rc = realloc_stats(c);
    if (rc != NFC_OK) {
        nfc_destroy_chain(c);
        return rc;
    }
    *out = c;
    return NFC_OK;
}

void nfc_destroy_chain(nfc_chain *c)
{
    if (!c) return;
    cudaSetDevice(c->device);
    cudaDeviceSynchronize();
    DBuf *all[] = {&c->acl_r4, &c->acl_r6, &c->acl_f4, &c->acl_x4, &c->dpi_cls, &c->dpi_trans, &c->dpi_off, &c->dpi_ids, &c->dpi_act,
                   &c->dpi_bitmap, &c->dpi_meta, &c->dpi_sparse, &c->dpi_frows, &c->dpi_accid, &c->dpi_accmeta, &c->uf_list[0], &c->uf_list[1], &c->uf_cnt, &c->uf_pass, &c->l4_tbl24, &c->l4_long, &c->l4_nh, &c->l4_pmac, &c->l6_lens, &c->l6_base,
                   &c->l6_mask, &c->l6_ent, &c->l6_nh, &c->l6_pmac, &c->esp_sa, &c->esp_te, &c->esp_nib,
                   &c->esp_seq[0], &c->esp_seq[1], &c->lb_port, &c->lb_nib, &c->nat_pool, &c->nat_dnat, &c->nat_nib,
                   &c->stats, &c->counter,
                   &c->tile_flag, &c->tile_vec, &c->batches, &c->h_arena, &c->h_off, &c->h_len, &c->h_rec,
                   &c->h_mp, &c->h_mq, &c->h_mc, &c->stats_red, &c->crec};
    for (DBuf *b : all) b->release();
    for (int i = 0; i < nfc_chain::NXS; i++)
        if (c->xs[i]) cudaStreamDestroy(c->xs[i]);
    if (c->xk) cudaEventDestroy(c->xk);
    if (c->mix_ev) cudaEventDestroy(c->mix_ev);
    if (c->mix_host) cudaFreeHost(c->mix_host);
    c->mix_dev.release();
    delete c;
}

int nfc_chain_room(const nfc_chain *c, uint32_t *headroom, uint32_t *tailroom)
{
    if (!c || !headroom || !tailroom) return fail(NFC_EINVAL, "NULL argument");
    bool esp = (c->mask & MASK_IPSEC) != 0;
    *headroom = esp ? 16 : 0;
    *tailroom = esp ? 32 : 0;
    return NFC_OK;
}

int nfc_load_tables(nfc_chain *c, uint32_t kind, const void *spec, size_t spec_bytes)
{
    if (!c || !spec) return fail(NFC_EINVAL, "NULL argument");
    if (kind < NFC_ACL || kind > NFC_NAT) return fail(NFC_EINVAL, "unknown NF kind");
    int rc = set_device(c);
    if (rc) return rc;
    cudaDeviceSynchronize();   // tables are replaced atomically w.r.t. later launches
    std::string err;
    switch (kind) {
    case NFC_ACL: {
        if (spec_bytes != sizeof(nfc_acl_spec)) return fail(NFC_EINVAL, "spec_bytes != sizeof(nfc_acl_spec)");
        const nfc_acl_spec &s = *static_cast<const nfc_acl_spec *>(spec);
        std::vector<uint32_t> b4, b6;
        err = build_acl(s, b4, b6);
        if (!err.empty()) return fail(NFC_EINVAL, err);
        CK(c->acl_r4.upload(b4));
        CK(c->acl_r6.upload(b6));
        c->acl = AclImg{c->acl_r4.as<uint32_t>(), c->acl_r6.as<uint32_t>(), (uint32_t)b4.size(),
                        (uint32_t)b6.size(), s.n_rules, s.default_action, 0, {}, {}};
        std::copy(b4.begin(), b4.begin() + ACLBV_HDR, c->acl.hdr4);
        std::copy(b6.begin(), b6.begin() + ACLBV_HDR, c->acl.hdr6);
        std::vector<uint16_t> x4;
        build_acl4_index(b4, x4, c->acl.d16);
        if (!x4.empty()) {
            CK(c->acl_x4.upload(x4));
            c->acl.x4 = c->acl_x4.as<uint16_t>();
        }
        std::vector<uint32_t> f4;
        build_acl4_fast(b4, f4, c->acl.f4_key, c->acl.f4_bv, c->acl.f4_d3);
        if (!f4.empty()) {
            CK(c->acl_f4.upload(f4));
            c->acl.f4 = c->acl_f4.as<uint32_t>();
            c->acl.words_f4 = (uint32_t)f4.size();
        }
        c->n_acl_rules = s.n_rules;
        break;
    }
    case NFC_DPI: {
        if (spec_bytes != sizeof(nfc_dpi_spec)) return fail(NFC_EINVAL, "spec_bytes != sizeof(nfc_dpi_spec)");
        DpiHost d;
        err = build_dpi(*static_cast<const nfc_dpi_spec *>(spec), d);
        if (!err.empty()) return fail(NFC_EINVAL, err);
        CK(c->dpi_cls.upload(d.cls));
        CK(c->dpi_trans.upload(d.trans));
        CK(c->dpi_off.upload(d.out_off));
        CK(c->dpi_ids.upload(d.out_ids));
        CK(c->dpi_act.upload(d.action));
        CK(c->dpi_meta.upload(d.out_meta));
        CK(c->dpi_sparse.upload(d.sparse));
        CK(c->dpi_frows.upload(d.frows));
        CK(c->dpi_accid.upload(d.acc_id));
        CK(c->dpi_accmeta.upload(d.acc_meta));
        c->dpi = DpiImg{};
        c->dpi.frows = c->dpi_frows.as<int16_t>();
        c->dpi.acc_id = c->dpi_accid.as<uint32_t>();
        c->dpi.acc_meta = c->dpi_accmeta.as<uint32_t>();
        c->dpi.n_acc = d.n_acc;
        c->dpi.out_meta = c->dpi_meta.as<uint32_t>();
        c->dpi.sparse = c->dpi_sparse.as<uint2>();
        c->dpi.n_d1 = d.n_d1;
        c->dpi.maxlen = d.maxlen;
        c->dpi.cls = c->dpi_cls.as<uint8_t>();
        c->dpi.trans = c->dpi_trans.p;
        c->dpi.ncls = d.ncls;
        c->dpi.n_states = d.n_states;
        c->dpi.wide = d.wide;
        c->dpi.out_off = c->dpi_off.as<uint32_t>();
        c->dpi.out_ids = c->dpi_ids.as<uint16_t>();
        c->dpi.pat_action = c->dpi_act.as<uint8_t>();
        c->dpi.n_pat = (uint32_t)d.action.size();
        c->dpi.bitmap_words = (c->dpi.n_pat + 31) / 32;
        break;
    }
    case NFC_LPM4: {
        if (spec_bytes != sizeof(nfc_lpm4_spec)) return fail(NFC_EINVAL, "spec_bytes != sizeof(nfc_lpm4_spec)");
        std::vector<uint16_t> t24, tl;
        std::vector<uint2> nh, pm;
        err = build_lpm4(*static_cast<const nfc_lpm4_spec *>(spec), t24, tl, nh, pm);
        if (!err.empty()) return fail(NFC_EINVAL, err);
        CK(c->l4_tbl24.upload(t24));
        CK(c->l4_long.upload(tl));
        CK(c->l4_nh.upload(nh));
        CK(c->l4_pmac.upload(pm));
        c->l4 = Lpm4Img{c->l4_tbl24.as<uint16_t>(), c->l4_long.as<uint16_t>(), c->l4_nh.as<uint2>(),
                        c->l4_pmac.as<uint2>(), (uint32_t)nh.size(), (uint32_t)pm.size()};
        break;
    }
    case NFC_LPM6: {
        if (spec_bytes != sizeof(nfc_lpm6_spec)) return fail(NFC_EINVAL, "spec_bytes != sizeof(nfc_lpm6_spec)");
        Lpm6Host h;
        err = build_lpm6(*static_cast<const nfc_lpm6_spec *>(spec), h);
        if (!err.empty()) return fail(NFC_EINVAL, err);
        CK(c->l6_lens.upload(h.lens));
        CK(c->l6_base.upload(h.base));
        CK(c->l6_mask.upload(h.mask));
        CK(c->l6_ent.upload(h.ent));
        CK(c->l6_nh.upload(h.nh));
        CK(c->l6_pmac.upload(h.pmac));
        c->l6 = Lpm6Img{(uint32_t)h.lens.size(), h.def_nh, c->l6_lens.as<uint8_t>(), c->l6_base.as<uint32_t>(),
                        c->l6_mask.as<uint32_t>(), c->l6_ent.as<uint4>(), c->l6_nh.as<uint2>(),
                        c->l6_pmac.as<uint2>(), (uint32_t)h.nh.size(), (uint32_t)h.pmac.size()};
        break;
    }
    case NFC_IPSEC: {
        if (spec_bytes != sizeof(nfc_ipsec_spec)) return fail(NFC_EINVAL, "spec_bytes != sizeof(nfc_ipsec_spec)");
        const nfc_ipsec_spec &s = *static_cast<const nfc_ipsec_spec *>(spec);
        std::vector<EspSa> sa;
        err = build_ipsec(s, sa);
        if (!err.empty()) return fail(NFC_EINVAL, err);
        std::vector<uint32_t> te, nib, seq(s.n_sa);
        build_aes_tables(te);
        build_toeplitz_nibbles(MS_RSS_KEY, nib);
        for (uint32_t i = 0; i < s.n_sa; i++) seq[i] = s.sas[i].seq0;
        CK(c->esp_sa.upload(sa));
        CK(c->esp_te.upload(te));
        CK(c->esp_nib.upload(nib));
        CK(c->esp_seq[0].upload(seq));
        CK(c->esp_seq[1].upload(seq));
        c->seq_parity = 0;
        c->esp = EspImg{c->esp_sa.as<EspSa>(), s.n_sa, c->esp_te.as<uint32_t>(), c->esp_nib.as<uint32_t>()};
        c->n_sa = s.n_sa;
        break;
    }
    case NFC_LB: {
        if (spec_bytes != sizeof(nfc_lb_spec)) return fail(NFC_EINVAL, "spec_bytes != sizeof(nfc_lb_spec)");
        const nfc_lb_spec &s = *static_cast<const nfc_lb_spec *>(spec);
        if (s.n_backends == 0 || s.n_backends > 65535 || !s.backend_port || !s.key)
            return fail(NFC_EINVAL, "lb: n_backends must be 1..65535 with ports and key");
        std::vector<uint16_t> ports(s.backend_port, s.backend_port + s.n_backends);
        std::vector<uint32_t> nib;
        build_toeplitz_nibbles(s.key, nib);
        CK(c->lb_port.upload(ports));
        CK(c->lb_nib.upload(nib));
        c->lb = LbImg{c->lb_port.as<uint16_t>(), s.n_backends, c->lb_nib.as<uint32_t>()};
        c->n_lb = s.n_backends;
        break;
    }
    case NFC_NAT: {
        if (spec_bytes != sizeof(nfc_nat_spec)) return fail(NFC_EINVAL, "spec_bytes != sizeof(nfc_nat_spec)");
        NatHost h;
        err = build_nat(*static_cast<const nfc_nat_spec *>(spec), h);
        if (!err.empty()) return fail(NFC_EINVAL, err);
        CK(c->nat_pool.upload(h.pool));
        CK(c->nat_dnat.upload(h.dnat));
        CK(c->nat_nib.upload(h.nib));
        c->nat = h.img;
        c->nat.pool = c->nat_pool.as<uint32_t>();
        c->nat.dnat = c->nat_dnat.as<uint4>();
        c->nat.nib = c->nat_nib.as<uint32_t>();
        break;
    }
    }
    c->loaded[kind] = true;
    return realloc_stats(c);
}

static int process_impl(nfc_chain *c, const nfc_batch *bs, uint32_t nb, const nfc_result *r, cudaStream_t st)
{
    for (uint32_t i = 0; i < c->n_nf; i++)
        if (!c->loaded[c->kind[i]]) return fail(NFC_ESTATE, "tables not loaded for an NF of the chain");
    if (!r || !r->rec) return fail(NFC_EINVAL, "result buffers missing");
    if ((c->mask & MASK_DPI) && !r->match_count) return fail(NFC_EINVAL, "match_count is required for DPI chains");
    if (nb && !bs) return fail(NFC_EINVAL, "batches is NULL");
    std::vector<BatchDev> hb(nb);
    uint64_t total = 0;
    for (uint32_t i = 0; i < nb; i++) {
        if (bs[i].n && (!bs[i].arena || !bs[i].off || !bs[i].len)) return fail(NFC_EINVAL, "batch pointers NULL");
        hb[i] = BatchDev{bs[i].arena, bs[i].off, bs[i].len, bs[i].n, (uint32_t)total, bs[i].first_global_index};
        total += bs[i].n;
    }
    if (total > 0xFFFFFFFFull - 1024) return fail(NFC_EINVAL, "too many packets in one call");
    // batches that are consecutive slices of one descriptor run (one arena, off/len arrays
    // and global indices continuing batch to batch -- a NIC RX ring) are one batch to the
    // kernel: the per-packet results are the same by definition, and the warp loop reads
    // the descriptors straight from the kernel parameters instead of chunk records
    if (nb > 1) {
        bool run = true;
        for (uint32_t i = 1; i < nb && run; i++)
            run = hb[i].n == 0 || (hb[i].arena == hb[0].arena && hb[i].off == hb[0].off + hb[i].start &&
                                   hb[i].len == hb[0].len + hb[i].start && hb[i].first == hb[0].first + hb[i].start);
        if (run) {
            hb[0].n = (uint32_t)total;
            hb.resize(1);
            nb = 1;
        }
    }
    c->last_stream = st;
    if (total == 0) return NFC_OK;
    int rc = set_device(c);
    if (rc) return rc;
    const uint32_t TILE_N = 256;
    uint32_t n_tiles = (uint32_t)((total + TILE_N - 1) / TILE_N);
    CK(c->batches.reserve(hb.size() * sizeof(BatchDev)));
    // one batch travels in the kernel parameters (KParams::b0); only multi-batch calls need
    // the descriptor array in device memory (a pageable copy: staged by the driver)
    if (nb > 1) CK(cudaMemcpyAsync(c->batches.p, hb.data(), hb.size() * sizeof(BatchDev), cudaMemcpyHostToDevice, st));
    CK(cudaMemsetAsync(c->counter.p, 0, 4, st));

    KParams p{};
    p.n_nf = c->n_nf;
    for (uint32_t i = 0; i < c->n_nf; i++) p.kind[i] = c->kind[i];
    for (uint32_t i = 0; i < c->n_nf; i++) p.group[i] = c->group[i];
    p.n_groups = (uint32_t)c->group[c->n_nf - 1] + 1;
    p.esp_pos = c->esp_pos;
    p.present = c->mask;
    p.batches = c->batches.as<BatchDev>();
    p.b0 = hb[0];
    p.n_batches = nb;
    p.n_pkts = (uint32_t)total;
    p.n_tiles = n_tiles;
    p.tile_counter = c->counter.as<uint32_t>();
    p.rec = r->rec;
    p.match_pkt = r->match_pkt;
    p.match_pat = r->match_pat;
    p.match_cap = r->match_pkt && r->match_pat ? r->match_cap : 0;
    p.match_count = r->match_count;
    p.stats = c->stats.as<unsigned long long>();
    p.stats_len = c->stats_len;
    p.st_acl = ST_VAR_BASE;
    p.st_lb = ST_VAR_BASE + c->n_acl_rules + 1;
    p.st_sa = p.st_lb + c->n_lb;
    p.smem_stats = c->stats_len <= 4096 ? 1 : 0;
    p.acl = c->acl;
    p.dpi = c->dpi;
    p.l4 = c->l4;
    p.l6 = c->l6;
    p.esp = c->esp;
    p.lb = c->lb;
    p.nat = c->nat;
    if (c->mask & MASK_IPSEC) {
        if (n_tiles > c->tile_cap) {
            uint32_t cap = n_tiles + n_tiles / 4 + 64;
            CK(c->tile_flag.reserve((size_t)cap * 4));
            CK(cudaMemset(c->tile_flag.p, 0, (size_t)cap * 4));
            CK(c->tile_vec.reserve((size_t)cap * 2 * c->n_sa * 4));
            c->tile_cap = cap;
            c->epoch = 0;
        }
        c->epoch = (c->epoch + 1) & 0x3FFFFFFF;
        if (c->epoch == 0) {
            CK(cudaMemsetAsync(c->tile_flag.p, 0, (size_t)c->tile_cap * 4, st));
            c->epoch = 1;
        }
        p.tile_flag = c->tile_flag.as<uint32_t>();
        p.tile_vec = c->tile_vec.as<uint32_t>();
        p.epoch = c->epoch;
        p.seq_in = c->esp_seq[c->seq_parity].as<uint32_t>();
        p.seq_out = c->esp_seq[c->seq_parity ^ 1].as<uint32_t>();
    }
    // Shared memory: with a DM_FULL variant the whole DFA is staged per CTA (one CTA
    // per SM) when it fits next to the rest; otherwise a budget per CTA for the
    // target occupancy stages the ACL image and gives the rest to hot DFA rows.
    Variant v = sfc_variant(c->kind, c->n_nf, false);
    const bool par = (c->flags & NFC_F_PARALLEL) != 0;
    uint32_t n_fwd = 0;
    for (uint32_t q = 0; q < c->n_nf; q++) n_fwd += (c->kind[q] == NFC_LPM4 || c->kind[q] == NFC_LPM6);
    if (par) { v.sig = 0; v.dm = DM_HOT; v.threads = 768; }
    {
        const size_t limit = sfc_smem_limit(c->device);
        p.acl.smem_words = (c->mask & MASK_ACL) ? 1 : 0;
        // the fused kernel stages the IPv4 record image when there is one (the unfused
        // and parallel kernels read the bit-vector blob)
        p.acl.fast = !par && !(c->flags & NFC_F_UNFUSED) && c->acl.f4 != nullptr ? 1u : 0u;
        p.dpi.hot_states = 0;
        p.dpi.sparse_states = 0;
        bool full = false;
        if (!par && (c->mask & MASK_DPI) && !c->dpi.wide && c->dpi.ncls <= 128) {
            Variant vf = sfc_variant(c->kind, c->n_nf, true);
            if (vf.dm == DM_FULL) {
                p.dpi.hot_states = c->dpi.n_states;
                p.dpi.meta_smem = 1;
                if (sfc_smem_bytes(vf, p) + 1024 > limit) p.dpi.meta_smem = 0;
                if (sfc_smem_bytes(vf, p) + 1024 <= limit) { v = vf; full = true; }
                else p.dpi.hot_states = 0;
            }
        }
        if (!full) {
            int smem_sm = 0;
            cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, c->device);
            // CTAs resident per SM: 1 for the big-CTA DPI variants, else the launch-bounds target
            const int target = v.threads > 256 ? 1 : (c->mask & MASK_IPSEC) ? 2 : 4;
            const size_t budget = std::min((size_t)smem_sm / target - 1024 - 64, limit - 1024);
            if (c->mask & MASK_ACL)
                if (sfc_smem_bytes(v, p) > budget / 2) p.acl.smem_words = 0;
            if ((c->mask & MASK_DPI) && !c->dpi.wide) {
                // tiered DFA: every row dense if it fits; else the depth <= 1 rows dense
                // and as many sparse records (8 B) as fit after them (DpiImg::sparse)
                p.dpi.sparse_states = 0;
                const size_t base = par ? par_smem_bytes(p, n_fwd) + 16 : sfc_smem_bytes(v, p), row = 2 * c->dpi.ncls;
                const size_t room = base < budget ? budget - base : 0;
                if ((size_t)c->dpi.n_states * row <= room) {
                    p.dpi.hot_states = c->dpi.n_states;
                } else {
                    const size_t h = std::min<size_t>(c->dpi.n_d1, room / row);
                    p.dpi.hot_states = (uint32_t)h;
                    const size_t left = room - h * row;
                    p.dpi.sparse_states = (uint32_t)std::min<size_t>(c->dpi.n_states - h, left / 8);
                }
            }
        }
    }
    // LPM4 next-hop records in shared memory when they fit beside everything else
    p.l4.nh_smem = 0;
    if (!par && (c->mask & MASK_LPM4) && c->l4.n_nh * 16 <= 8192) {
        p.l4.nh_smem = 1;
        int smem_sm = 0;
        cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, c->device);
        const int per = v.threads > 256 ? 1 : (c->mask & MASK_IPSEC) ? 2 : 4;
        const size_t cap = std::min(sfc_smem_limit(c->device), (size_t)smem_sm / per) - 1024;
        if (sfc_smem_bytes(v, p) > cap) p.l4.nh_smem = 0;
    }
    p.dpi.row2 = 2 * c->dpi.ncls;
    p.dpi.hk2 = p.dpi.hot_states ? 2 * (p.dpi.hot_states * c->dpi.ncls - 1) : 0;
    if (c->mask & MASK_DPI) {
        LaunchCfg q{};
        if (sfc_query(v, p, c->device, &q) != NFC_OK) return fail(NFC_ECUDA, "occupancy query failed");
        size_t threads = (size_t)q.grid * q.block;
        if (c->flags & (NFC_F_UNFUSED | NFC_F_PARALLEL)) {   // other kernels may keep more threads resident
            int sms = 0;
            cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, c->device);
            threads = std::max(threads, (size_t)sms * 2048);
        }
        size_t need = threads * c->dpi.bitmap_words * 4;
        CK(c->dpi_bitmap.reserve(need));
        c->dpi.ovf_bitmap = c->dpi_bitmap.as<uint32_t>();
        p.dpi.ovf_bitmap = c->dpi.ovf_bitmap;
    }
    std::string err;
    if (c->flags & NFC_F_UNFUSED) {
        CK(c->uf_list[0].reserve((size_t)total * 4));
        CK(c->uf_list[1].reserve((size_t)total * 4));
        CK(c->uf_cnt.reserve((NFC_MAX_CHAIN + 1) * 4));
        CK(c->uf_pass.reserve((size_t)total));
        CK(cudaMemsetAsync(c->uf_cnt.p, 0, (NFC_MAX_CHAIN + 1) * 4, st));
        uint32_t nl = 0;
        rc = uf_launch(c->kind, c->n_nf, v.dm, p, c->uf_list[0].as<uint32_t>(), c->uf_list[1].as<uint32_t>(),
                       c->uf_cnt.as<uint32_t>(), c->uf_pass.as<uint8_t>(), c->device, st, err, &nl);
        if (rc) return fail(rc, err);
        c->launches += nl;
        return NFC_OK;
    }
    // IPsec tiles are one CTA each: a variant with bigger CTAs takes fewer, bigger tiles
    if ((c->mask & MASK_IPSEC) && !par && v.threads > (int)TILE_N) p.n_tiles = (uint32_t)((total + v.threads - 1) / v.threads);
    LaunchCfg lc{};
    if (!par && nb > 1 && !(c->mask & MASK_IPSEC)) {
        // multi-batch call: per-chunk descriptor records for the pipelined warp loop
        CK(c->crec.reserve((size_t)((total + 31) / 32) * sizeof(ChunkRec)));
        rc = chunk_recs_launch(p.batches, nb, (uint32_t)total, c->crec.as<ChunkRec>(), st, err);
        if (rc) return fail(rc, err);
        p.crec = c->crec.as<ChunkRec>();
        c->launches++;
    }
    const bool rg_cap = NFC_REGROUP && !par && v.dm == DM_FULL && (c->mask & MASK_ACL) && (c->mask & MASK_DPI) &&
                        c->kind[0] == NFC_ACL && c->kind[1] == NFC_DPI && !(c->mask & MASK_IPSEC);
    if (rg_cap) {
        if (!c->mix_ev) {
            CK(c->mix_dev.reserve(4));
            CK(cudaMallocHost(&c->mix_host, 4));
            CK(cudaEventCreateWithFlags(&c->mix_ev, cudaEventDisableTiming));
            *c->mix_host = 0;
        }
        if (c->mix_pending && cudaEventQuery(c->mix_ev) == cudaSuccess) {   // the last launch's count
            c->rg_on = (uint64_t)*c->mix_host * 8 > c->mix_chunks;
            c->mix_pending = false;
        }
        v.rg = c->rg_on;
        p.mix = c->mix_dev.as<uint32_t>();
        CK(cudaMemsetAsync(p.mix, 0, 4, st));
    }
    rc = par ? par_launch(p, c->device, st, err, &lc) : sfc_launch(v, p, c->device, st, err, &lc);
    if (!rc && rg_cap && !c->mix_pending) {
        CK(cudaMemcpyAsync(c->mix_host, p.mix, 4, cudaMemcpyDeviceToHost, st));
        CK(cudaEventRecord(c->mix_ev, st));
        c->mix_chunks = (uint32_t)((total + 31) / 32);
        c->mix_pending = true;
    }
    if (rc) return fail(rc, err);
    c->last = nfc_launch_info{(uint32_t)lc.grid, (uint32_t)lc.block, (uint32_t)lc.smem,
                              (c->mask & MASK_DPI) ? (uint32_t)v.dm : 0u, p.dpi.hot_states, p.dpi.sparse_states,
                              p.dpi.meta_smem, p.acl.smem_words ? 4 * ((p.acl.fast ? p.acl.words_f4 : p.acl.words4) + p.acl.words6) : 0u};
    c->launches += lc.launches;
    if (c->mask & MASK_IPSEC) c->seq_parity ^= 1;
    return NFC_OK;
}

int nfc_process_batch(nfc_chain *c, const nfc_batch *batches, uint32_t n_batches, const nfc_result *r, void *stream)
{
    if (!c) return fail(NFC_EINVAL, "chain is NULL");
    return process_impl(c, batches, n_batches, r, static_cast<cudaStream_t>(stream));
}

// End-to-end host path, pipelined: the packets are cut into chunks of consecutive
// indices; chunk k's bytes [min off - headroom, max off+len + tailroom) go to the same
// offsets of a device mirror of the arena, its descriptors alongside; copies of chunk
// k+1 (H2D) and chunk k-1 (D2H) run on the other copy stream while chunk k's kernel
// runs, so both PCIe directions stay busy.  Kernels run strictly in chunk order (ESP
// sequence numbers follow global order; the chain's scratch is reused per launch).
int nfc_process_host(nfc_chain *c, uint8_t *arena, uint64_t arena_bytes, const uint64_t *off, const uint16_t *len,
                     uint32_t n, uint64_t first_global_index, nfc_pkt_result *rec, uint32_t *match_pkt,
                     uint16_t *match_pat, uint32_t match_cap, uint32_t *n_pairs, void *stream)
{
    if (!c || (n && (!arena || !off || !len || !rec))) return fail(NFC_EINVAL, "NULL argument");
    int rc = set_device(c);
    if (rc) return rc;
    cudaStream_t user = static_cast<cudaStream_t>(stream);
    uint32_t hr = 0, tr = 0;
    nfc_chain_room(c, &hr, &tr);
    CK(c->h_arena.reserve(arena_bytes + 64));
    CK(c->h_off.reserve((size_t)n * 8 + 8));
    CK(c->h_len.reserve((size_t)n * 2 + 8));
    CK(c->h_rec.reserve((size_t)n * sizeof(nfc_pkt_result) + 16));
    CK(c->h_mp.reserve((size_t)match_cap * 4 + 4));
    CK(c->h_mq.reserve((size_t)match_cap * 2 + 4));
    CK(c->h_mc.reserve(4));
    if (!c->xs[0]) {
        for (int i = 0; i < nfc_chain::NXS; i++) CK(cudaStreamCreateWithFlags(&c->xs[i], cudaStreamNonBlocking));
        CK(cudaEventCreateWithFlags(&c->xk, cudaEventDisableTiming));
    }
    // the copy streams start after the caller's prior work
    CK(cudaEventRecord(c->xk, user));
    for (int i = 0; i < nfc_chain::NXS; i++) CK(cudaStreamWaitEvent(c->xs[i], c->xk, 0));
    CK(cudaMemsetAsync(c->h_mc.p, 0, 4, c->xs[0]));
    CK(cudaEventRecord(c->xk, c->xs[0]));          // "previous kernel done" starts as: counter zeroed
    // chunks: about 32 per call, at least 64 K packets each, round-robin over NXS streams.  A chunk's byte range is
    // scanned while the previous chunks' copies and kernels run; a chunk whose range
    // overlaps an earlier chunk's (frames not laid out in index order) first waits for
    // everything issued before it, so it reads the rewritten bytes back consistently.
    const uint32_t per = std::max<uint32_t>(65536, (n + 31) / 32);
    uint8_t *darena = c->h_arena.as<uint8_t>();
    uint64_t *doff = c->h_off.as<uint64_t>();
    uint16_t *dlen = c->h_len.as<uint16_t>();
    uint64_t max_hi = 0;
    uint32_t k = 0;
    for (uint32_t a0 = 0; a0 < n; a0 += per, k++) {
        const uint32_t cnt = std::min(per, n - a0);
        cudaStream_t st = c->xs[k % nfc_chain::NXS];
        uint64_t lo = ~0ull, hi = 0;
        const uint64_t *o = off + a0;
        const uint16_t *l = len + a0;
        for (uint32_t i = 0; i < cnt; i++) {
            const uint64_t x = o[i], e = x + l[i];
            lo = x < lo ? x : lo;
            hi = e > hi ? e : hi;
        }
        lo = lo >= hr ? lo - hr : 0;
        hi = std::min<uint64_t>(hi + tr, arena_bytes);
        if (lo > arena_bytes || hi < lo) return fail(NFC_EINVAL, "frame outside the arena");
        if (lo < max_hi)
            for (int i = 0; i < nfc_chain::NXS; i++) CK(cudaStreamSynchronize(c->xs[i]));
        max_hi = std::max(max_hi, hi);
        CK(cudaMemcpyAsync(darena + lo, arena + lo, hi - lo, cudaMemcpyHostToDevice, st));
        CK(cudaMemcpyAsync(doff + a0, off + a0, (size_t)cnt * 8, cudaMemcpyHostToDevice, st));
        CK(cudaMemcpyAsync(dlen + a0, len + a0, (size_t)cnt * 2, cudaMemcpyHostToDevice, st));
        CK(cudaStreamWaitEvent(st, c->xk, 0));      // kernels in chunk order
        nfc_batch b{darena, doff + a0, dlen + a0, cnt, 0, first_global_index + a0};
        nfc_result r{c->h_rec.as<nfc_pkt_result>() + a0, c->h_mp.as<uint32_t>(), c->h_mq.as<uint16_t>(), match_cap, 0,
                     c->h_mc.as<uint32_t>()};
        rc = process_impl(c, &b, 1, &r, st);
        if (rc) return rc;
        CK(cudaEventRecord(c->xk, st));
        CK(cudaMemcpyAsync(arena + lo, darena + lo, hi - lo, cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(rec + a0, c->h_rec.as<nfc_pkt_result>() + a0, (size_t)cnt * sizeof(nfc_pkt_result),
                           cudaMemcpyDeviceToHost, st));
    }
    uint32_t cnt = 0;
    CK(cudaStreamWaitEvent(c->xs[0], c->xk, 0));
    CK(cudaMemcpyAsync(&cnt, c->h_mc.p, 4, cudaMemcpyDeviceToHost, c->xs[0]));
    for (int i = 0; i < nfc_chain::NXS; i++) CK(cudaStreamSynchronize(c->xs[i]));
    uint32_t m = cnt < match_cap ? cnt : match_cap;
    if (m && match_pkt && match_pat) {
        CK(cudaMemcpyAsync(match_pkt, c->h_mp.p, (size_t)m * 4, cudaMemcpyDeviceToHost, c->xs[0]));
        CK(cudaMemcpyAsync(match_pat, c->h_mq.p, (size_t)m * 2, cudaMemcpyDeviceToHost, c->xs[0]));
        CK(cudaStreamSynchronize(c->xs[0]));
    }
    c->last_stream = c->xs[0];
    if (n_pairs) *n_pairs = cnt;
    return NFC_OK;
}

int nfc_stats_len(const nfc_chain *c, size_t *len)
{
    if (!c || !len) return fail(NFC_EINVAL, "NULL argument");
    *len = c->stats_len;
    return NFC_OK;
}

int nfc_collect_stats(nfc_chain *c, uint64_t *out, size_t cap, uint32_t flags)
{
    if (!c || (!out && cap)) return fail(NFC_EINVAL, "NULL argument");
    if (flags & ~(NFC_STATS_RESET | NFC_STATS_ALLREDUCE)) return fail(NFC_EINVAL, "unknown stats flags");
    if ((flags & NFC_STATS_ALLREDUCE) && !c->comm) return fail(NFC_ESTATE, "NFC_STATS_ALLREDUCE without an attached comm");
    int rc = set_device(c);
    if (rc) return rc;
    cudaStream_t st = c->last_stream;
    const size_t bytes = (size_t)c->stats_len * 8;
    const void *src = c->stats.p;
    if (flags & NFC_STATS_ALLREDUCE) {
        CK(c->stats_red.reserve(bytes));
        CK(cudaMemcpyAsync(c->stats_red.p, c->stats.p, bytes, cudaMemcpyDeviceToDevice, st));
        rc = comm_allreduce_u64(c->comm, c->stats_red.as<unsigned long long>(), c->stats_len, st);
        if (rc) return rc;
        src = c->stats_red.p;
    }
    std::vector<uint64_t> h(c->stats_len);
    CK(cudaMemcpyAsync(h.data(), src, bytes, cudaMemcpyDeviceToHost, st));
    if (flags & NFC_STATS_RESET) CK(cudaMemsetAsync(c->stats.p, 0, bytes, st));
    CK(cudaStreamSynchronize(st));
    size_t k = cap < h.size() ? cap : h.size();
    if (k) memcpy(out, h.data(), k * 8);
    if (h[ST_MATCH_OVF]) return fail(NFC_ECAP, "match pairs exceeded match_cap");
    return NFC_OK;
}

int nfc_set_groups(nfc_chain *c, const uint8_t *group)
{
    if (!c || !group) return fail(NFC_EINVAL, "NULL argument");
    if (!groups_legal(c->kind, c->n_nf, group))
        return fail(NFC_EINVAL, "groups must be runs of consecutive, pairwise parallel-legal NFs (nfc_plan_parallel)");
    for (uint32_t i = 0; i < c->n_nf && i < NFC_MAX_CHAIN; i++) c->group[i] = group[i];
    return NFC_OK;
}

int nfc_get_groups(const nfc_chain *c, uint8_t *group)
{
    if (!c || !group) return fail(NFC_EINVAL, "NULL argument");
    for (uint32_t i = 0; i < c->n_nf; i++) group[i] = c->group[i];
    return NFC_OK;
}

int nfc_attach_comm(nfc_chain *c, void *nccl_comm)
{
    if (!c) return fail(NFC_EINVAL, "chain is NULL");
    c->comm = nccl_comm;
    return NFC_OK;
}

int nfc_rss_shard(int device, const nfc_batch *b, uint32_t n_shards, uint8_t *shard, void *stream)
{
    if (!b || !shard || n_shards == 0 || n_shards > 128) return fail(NFC_EINVAL, "bad rss_shard arguments");
    if (b->n && (!b->arena || !b->off || !b->len)) return fail(NFC_EINVAL, "batch pointers NULL");
    CK(cudaSetDevice(device));
    static thread_local DBuf nib_dev[16];
    DBuf &nb = nib_dev[device & 15];
    if (!nb.p) {
        std::vector<uint32_t> nib;
        build_toeplitz_nibbles(MS_RSS_KEY, nib);
        CK(nb.upload(nib));
    }
    std::string err;
    int rc = rss_shard_launch(b->arena, b->off, b->len, b->n, nb.as<uint32_t>(), n_shards, shard, stream, err);
    return rc ? fail(rc, err) : NFC_OK;
}

int nfc_last_launch(const nfc_chain *c, nfc_launch_info *out)
{
    if (!c || !out) return fail(NFC_EINVAL, "NULL argument");
    *out = c->last;
    return NFC_OK;
}

int nfc_launch_count(const nfc_chain *c, uint64_t *count)
{
    if (!c || !count) return fail(NFC_EINVAL, "NULL argument");
    *count = c->launches;
    return NFC_OK;
}

} // extern "C"
