// planner.cpp -- SFC parallelization planner (P:L243-263
// [SIV.B.1], Tables II-III).  Host code of the product.
//
// Two NFs of a chain are parallel-legal when running the later one on a copy of
// the packet that entered the earlier one gives the same result as running them
// in sequence: no read-after-write and no write-after-write on the same packet
// field (Table III with the field-level refinement of the "*" cases,
// DESIGN.md R#16).  Read/write sets are per packet family: the IPv4 forwarder
// touches only IPv4 packets, the IPv6 forwarder only IPv6 ones.  Drops and the
// egress port are metadata, resolved by the merge (earliest dropper in original
// order wins and discards the later members' side effects; the last
// setter of the port wins, R#19).  IPsec reads and rewrites the whole packet and
// grows it (Table II "Add/Rm"), so it always stands alone.
#include <stdint.h>

#include <initializer_list>

#include "../../include/nfc.h"

namespace {
enum : uint32_t {
    F_ETH_DST = 1u << 0, F_ETH_SRC = 1u << 1, F_TTL = 1u << 2, F_CSUM = 1u << 3, F_SRC = 1u << 4,
    F_DST = 1u << 5, F_PORTS = 1u << 6, F_PROTO = 1u << 7, F_PAYLOAD = 1u << 8, F_LEN = 1u << 9,
    F_ALL = (1u << 10) - 1
};
struct RW { uint32_t r, w; };

// fields read / written by NF `kind` on a packet of family fam (4 or 6)
RW rw_of(uint32_t kind, int fam)
{
    switch (kind) {
    case NFC_ACL: return {F_SRC | F_DST | F_PORTS | F_PROTO, 0};           // 5-tuple classifier
    case NFC_DPI: return {F_PAYLOAD | F_PROTO | F_LEN, 0};                // payload inspection
    case NFC_LPM4:                                                         // P:L128 forwarder (R#6)
        return fam == 4 ? RW{F_DST | F_TTL, F_ETH_DST | F_ETH_SRC | F_TTL | F_CSUM} : RW{0, 0};
    case NFC_LPM6:
        return fam == 6 ? RW{F_DST | F_TTL, F_ETH_DST | F_ETH_SRC | F_TTL} : RW{0, 0};
    case NFC_IPSEC: return {F_ALL, F_ALL};                                 // encrypts, adds bytes
    case NFC_LB: return {F_SRC | F_DST | F_PORTS | F_PROTO, 0};            // flow hash
    case NFC_NAT:                                                          // P:L383, Table II: NAT44 (R#30)
        return fam == 4 ? RW{F_SRC | F_DST | F_PORTS | F_PROTO, F_SRC | F_DST | F_PORTS | F_CSUM} : RW{0, 0};
    }
    return {F_ALL, F_ALL};
}

// earlier NF a, later NF b: legal in one group (no RAW, no WAW on any family)
bool legal_pair(uint32_t a, uint32_t b)
{
    // IPsec rewrites everything; NAT decides on the egress port an earlier forwarder set
    // (a read of merge-resolved metadata) and rewrites the 5-tuple: both stand alone (R#30)
    if (a == NFC_IPSEC || b == NFC_IPSEC || a == NFC_NAT || b == NFC_NAT) return false;
    for (int fam : {4, 6}) {
        const RW x = rw_of(a, fam), y = rw_of(b, fam);
        if (x.w & y.r) return false;     // read after write
        if (x.w & y.w) return false;     // write after write
    }
    return true;
}
} // namespace

namespace nfc {
bool groups_legal(const uint32_t *kinds, uint32_t n, const uint8_t *group)
{
    if (!kinds || !group || n == 0 || n > NFC_MAX_CHAIN || group[0] != 0) return false;
    for (uint32_t p = 1; p < n; p++)
        if (group[p] != group[p - 1] && group[p] != group[p - 1] + 1) return false;
    for (uint32_t p = 0; p < n; p++)
        for (uint32_t q = p + 1; q < n && group[q] == group[p]; q++)
            if (!legal_pair(kinds[p], kinds[q])) return false;
    return true;
}
} // namespace nfc

extern "C" NFC_API int nfc_plan_parallel(const uint32_t *kinds, uint32_t n, uint8_t *group)
{
    if (!kinds || !group || n == 0 || n > NFC_MAX_CHAIN) return NFC_EINVAL;
    for (uint32_t p = 0; p < n; p++)
        if (kinds[p] < NFC_ACL || kinds[p] > NFC_NAT) return NFC_EINVAL;
    // greedy: extend the current group while the next NF is legal with every member
    uint32_t g = 0, start = 0;
    group[0] = 0;
    for (uint32_t p = 1; p < n; p++) {
        bool ok = true;
        for (uint32_t q = start; q < p && ok; q++) ok = legal_pair(kinds[q], kinds[p]);
        if (!ok) { g++; start = p; }
        group[p] = (uint8_t)g;
    }
    return NFC_OK;
}
