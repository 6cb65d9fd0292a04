// Cross-GPU min-loc through NCCL: every rank
// projects its shard with the fused best kernel, the ranks' 48-byte results
// are all-gathered on the compute stream (NCCL has no MINLOC reduction), and
// the combine kernel takes the lexicographic min of (t, global index) on
// every rank — exact and order-independent.
//
// NCCL is resolved at run time (dlopen of libnccl.so.2 — in a PyTorch process
// the one torch already loaded — or GROPHECY_NCCL_LIB), so the library has no
// link-time NCCL dependency; calls return GROPHECY_ENCCL if it is missing.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <stdint.h>

#include <cstring>
#include <mutex>
#include <string>

#include "grophecy.h"
#include "internal.h"

namespace grophecy {
namespace {

typedef struct { char internal[128]; } NcclUniqueId;   // ncclUniqueId
typedef int (*GetUniqueIdFn)(NcclUniqueId *);
typedef int (*CommInitRankFn)(void **, int, NcclUniqueId, int);
typedef int (*AllGatherFn)(const void *, void *, size_t, int, void *, cudaStream_t);
typedef int (*CommDestroyFn)(void *);
typedef int (*CommCountFn)(const void *, int *);
typedef const char *(*ErrorStringFn)(int);

struct Nccl {
    bool tried = false, ok = false;
    GetUniqueIdFn get_unique_id = nullptr;
    CommInitRankFn comm_init_rank = nullptr;
    AllGatherFn all_gather = nullptr;
    CommDestroyFn comm_destroy = nullptr;
    CommCountFn comm_count = nullptr;
    ErrorStringFn error_string = nullptr;
};
Nccl g_nccl;
std::mutex g_nccl_mu;

const Nccl *nccl()
{
    std::lock_guard<std::mutex> lock(g_nccl_mu);
    if (g_nccl.tried) return g_nccl.ok ? &g_nccl : nullptr;
    g_nccl.tried = true;
    const char *env = getenv("GROPHECY_NCCL_LIB");
    void *h = dlopen(env ? env : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return nullptr;
    g_nccl.get_unique_id = (GetUniqueIdFn)dlsym(h, "ncclGetUniqueId");
    g_nccl.comm_init_rank = (CommInitRankFn)dlsym(h, "ncclCommInitRank");
    g_nccl.all_gather = (AllGatherFn)dlsym(h, "ncclAllGather");
    g_nccl.comm_destroy = (CommDestroyFn)dlsym(h, "ncclCommDestroy");
    g_nccl.comm_count = (CommCountFn)dlsym(h, "ncclCommCount");
    g_nccl.error_string = (ErrorStringFn)dlsym(h, "ncclGetErrorString");
    g_nccl.ok = g_nccl.get_unique_id && g_nccl.comm_init_rank && g_nccl.all_gather &&
                g_nccl.comm_destroy && g_nccl.comm_count;
    return g_nccl.ok ? &g_nccl : nullptr;
}

int nccl_fail(const Nccl *n, int r, const char *what)
{
    std::string m = std::string(what) + ": NCCL error " + std::to_string(r);
    if (n && n->error_string) m += std::string(" (") + n->error_string(r) + ")";
    set_error(m);
    return GROPHECY_ENCCL;
}

constexpr int NCCL_INT8 = 0;   // ncclInt8: the results are moved as bytes

}  // namespace
}  // namespace grophecy

using namespace grophecy;

extern "C" {

int grophecy_nccl_unique_id(void *id_out)
{
    if (!id_out) {
        set_error("null id");
        return GROPHECY_EINVAL;
    }
    const Nccl *n = nccl();
    if (!n) {
        set_error("NCCL (libnccl.so.2) not available");
        return GROPHECY_ENCCL;
    }
    NcclUniqueId id;
    int r = n->get_unique_id(&id);
    if (r) return nccl_fail(n, r, "ncclGetUniqueId");
    std::memcpy(id_out, &id, sizeof id);
    return GROPHECY_OK;
}

int grophecy_nccl_comm_init(int nranks, int rank, const void *id, int device, void **comm_out)
{
    if (!id || !comm_out || nranks < 1 || rank < 0 || rank >= nranks) {
        set_error("grophecy_nccl_comm_init: bad arguments");
        return GROPHECY_EINVAL;
    }
    const Nccl *n = nccl();
    if (!n) {
        set_error("NCCL (libnccl.so.2) not available");
        return GROPHECY_ENCCL;
    }
    DeviceGuard guard(device);
    NcclUniqueId uid;
    std::memcpy(&uid, id, sizeof uid);
    int r = n->comm_init_rank(comm_out, nranks, uid, rank);
    if (r) return nccl_fail(n, r, "ncclCommInitRank");
    return GROPHECY_OK;
}

int grophecy_nccl_comm_destroy(void *comm)
{
    const Nccl *n = nccl();
    if (!n || !comm) return GROPHECY_OK;
    int r = n->comm_destroy(comm);
    if (r) return nccl_fail(n, r, "ncclCommDestroy");
    return GROPHECY_OK;
}

// All-gather of the ranks' device results + combine + D2H (every rank gets
// the global best).  The shared tail of both allreduce entry points.
static int allreduce_device(grophecy_space *s, const Nccl *n, const grophecy_best_result *local,
                            void *nccl_comm, grophecy_best_result *host_out, cudaStream_t st)
{
    int nranks = 0;
    int r = n->comm_count(nccl_comm, &nranks);
    if (r) return nccl_fail(n, r, "ncclCommCount");
    cudaError_t e;
    const size_t need = sizeof(grophecy_best_result) * ((size_t)nranks + 1);
    if (s->mscratch_bytes < need) {   // gathered results + the combined one
        if (s->mscratch) cudaFree(s->mscratch);
        s->mscratch = nullptr;
        s->mscratch_bytes = 0;
        if ((e = cudaMalloc(&s->mscratch, need)) != cudaSuccess) return cuda_fail(e, "cudaMalloc(minloc)");
        s->mscratch_bytes = need;
    }
    grophecy_best_result *gathered = (grophecy_best_result *)s->mscratch;
    grophecy_best_result *result = gathered + nranks;
    r = n->all_gather(local, gathered, sizeof(grophecy_best_result), NCCL_INT8, nccl_comm, st);
    if (r) return nccl_fail(n, r, "ncclAllGather");
    int rc = grophecy_best_combine(gathered, (uint32_t)nranks, result, st);
    if (rc) return rc;
    e = cudaMemcpyAsync(host_out, result, sizeof *host_out, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_fail(e, "grophecy_best_allreduce");
    if (host_out->index == ~0ull) {
        set_error("no valid candidate with finite projected time");
        return GROPHECY_ENOFEASIBLE;
    }
    if (host_out->n_invalid) {
        set_error("batch contains invalid records");
        return GROPHECY_EBADCAND;
    }
    return GROPHECY_OK;
}

int grophecy_best_allreduce(grophecy_space *s, const grophecy_pcie *pc, const grophecy_batch *b,
                            void *nccl_comm, grophecy_best_result *host_out, void *stream)
{
    if (!s || !pc || !b || !nccl_comm || !host_out) {
        set_error("grophecy_best_allreduce: null argument");
        return GROPHECY_EINVAL;
    }
    const Nccl *n = nccl();
    if (!n) {
        set_error("NCCL (libnccl.so.2) not available");
        return GROPHECY_ENCCL;
    }
    DeviceGuard guard(s->device);
    cudaStream_t st = (cudaStream_t)stream;
    grophecy_best_result *local = s->partials + (s->max_partials - 1);
    const int rc = launch_best(s, pc, b, local, 0, st);
    if (rc) return rc;
    return allreduce_device(s, n, local, nccl_comm, host_out, st);
}

int grophecy_best_allreduce_result(grophecy_space *s, const grophecy_best_result *device_in,
                                   void *nccl_comm, grophecy_best_result *host_out, void *stream)
{
    if (!s || !device_in || !nccl_comm || !host_out) {
        set_error("grophecy_best_allreduce_result: null argument");
        return GROPHECY_EINVAL;
    }
    const Nccl *n = nccl();
    if (!n) {
        set_error("NCCL (libnccl.so.2) not available");
        return GROPHECY_ENCCL;
    }
    DeviceGuard guard(s->device);
    return allreduce_device(s, n, device_in, nccl_comm, host_out, (cudaStream_t)stream);
}

}  // extern "C"
