// comm.cu -- NCCL plumbing for multi-GPU runs (DESIGN.md
// "Multi-GPU").  Flows shard by RSS hash (P:L87 [SII.B.1] Receive Side
// Steering), so the data path has no collective; the only exchange is one
// ncclAllReduce(u64, sum) of the per-GPU counter vector at nfc_collect_stats.
//
// NCCL is loaded with dlopen on first use (libnccl.so.2: the copy torch already
// loaded, if any, else the system one), so libnfc.so has no link-time
// dependency on it and the single-GPU path never touches it.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>

#include "nfc_internal.h"

namespace nfc {

namespace {
struct NcclApi {
    ncclResult_t (*get_unique_id)(ncclUniqueId *) = nullptr;
    ncclResult_t (*comm_init_rank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*comm_destroy)(ncclComm_t) = nullptr;
    ncclResult_t (*all_reduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                               cudaStream_t) = nullptr;
    const char *(*error_string)(ncclResult_t) = nullptr;
    std::string why;
    bool ok = false;
};

NcclApi &api()
{
    static NcclApi a;
    static std::once_flag once;
    std::call_once(once, [] {
        const char *env = std::getenv("NFC_NCCL_LIB");
        void *h = nullptr;
        if (env && *env) h = dlopen(env, RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        if (!h) {
            const char *e = dlerror();
            a.why = std::string("cannot load libnccl.so.2: ") + (e ? e : "?");
            return;
        }
        a.get_unique_id = reinterpret_cast<decltype(a.get_unique_id)>(dlsym(h, "ncclGetUniqueId"));
        a.comm_init_rank = reinterpret_cast<decltype(a.comm_init_rank)>(dlsym(h, "ncclCommInitRank"));
        a.comm_destroy = reinterpret_cast<decltype(a.comm_destroy)>(dlsym(h, "ncclCommDestroy"));
        a.all_reduce = reinterpret_cast<decltype(a.all_reduce)>(dlsym(h, "ncclAllReduce"));
        a.error_string = reinterpret_cast<decltype(a.error_string)>(dlsym(h, "ncclGetErrorString"));
        a.ok = a.get_unique_id && a.comm_init_rank && a.comm_destroy && a.all_reduce && a.error_string;
        if (!a.ok) a.why = "libnccl.so.2 lacks an expected symbol";
    });
    return a;
}

int nccl_fail(const NcclApi &a, ncclResult_t r, const char *what)
{
    return set_fail(NFC_ECUDA, std::string(what) + ": " + (a.error_string ? a.error_string(r) : "nccl error"));
}
} // namespace

// Sum `n` u64 counters across the ranks of `comm` (in place on the device) on `st`.
int comm_allreduce_u64(void *comm, unsigned long long *dev, size_t n, cudaStream_t st)
{
    NcclApi &a = api();
    if (!a.ok) return set_fail(NFC_ESTATE, a.why);
    const ncclResult_t r = a.all_reduce(dev, dev, n, ncclUint64, ncclSum, static_cast<ncclComm_t>(comm), st);
    return r == ncclSuccess ? NFC_OK : nccl_fail(a, r, "ncclAllReduce");
}

} // namespace nfc

using namespace nfc;

extern "C" {

int nfc_comm_unique_id(uint8_t *id, size_t id_bytes)
{
    if (!id || id_bytes < NFC_COMM_ID_BYTES) return set_fail(NFC_EINVAL, "id buffer smaller than NFC_COMM_ID_BYTES");
    static_assert(NFC_COMM_ID_BYTES == NCCL_UNIQUE_ID_BYTES, "NFC_COMM_ID_BYTES must equal NCCL_UNIQUE_ID_BYTES");
    NcclApi &a = api();
    if (!a.ok) return set_fail(NFC_ESTATE, a.why);
    ncclUniqueId u;
    const ncclResult_t r = a.get_unique_id(&u);
    if (r != ncclSuccess) return nccl_fail(a, r, "ncclGetUniqueId");
    std::memcpy(id, u.internal, NCCL_UNIQUE_ID_BYTES);
    return NFC_OK;
}

int nfc_comm_init(int device, int nranks, int rank, const uint8_t *id, void **comm)
{
    if (!id || !comm || nranks < 1 || rank < 0 || rank >= nranks) return set_fail(NFC_EINVAL, "bad comm_init arguments");
    NcclApi &a = api();
    if (!a.ok) return set_fail(NFC_ESTATE, a.why);
    if (cudaSetDevice(device) != cudaSuccess) return set_fail(NFC_ECUDA, "cudaSetDevice failed");
    ncclUniqueId u;
    std::memcpy(u.internal, id, NCCL_UNIQUE_ID_BYTES);
    ncclComm_t c = nullptr;
    const ncclResult_t r = a.comm_init_rank(&c, nranks, u, rank);
    if (r != ncclSuccess) return nccl_fail(a, r, "ncclCommInitRank");
    *comm = c;
    return NFC_OK;
}

int nfc_comm_destroy(void *comm)
{
    if (!comm) return NFC_OK;
    NcclApi &a = api();
    if (!a.ok) return set_fail(NFC_ESTATE, a.why);
    const ncclResult_t r = a.comm_destroy(static_cast<ncclComm_t>(comm));
    return r == ncclSuccess ? NFC_OK : nccl_fail(a, r, "ncclCommDestroy");
}

} // extern "C"
