// shard.cu -- SURVEY §8(b)/(e): the z-slab pass with a library-owned NCCL
// communicator (safara_get_unique_id / safara_shard_init / safara_rhs_sharded
// / safara_shard_rms / safara_shard_finalize, include/safara.h).
//
// Per pass (SURVEY §3 call stack 5, §8(e)): the caller's stream forks to the
// shard's comm stream, which runs ONE grouped NCCL exchange of the two owned
// planes next to each slab end with the neighbouring ranks (ncclSend /
// ncclRecv into the ghost planes of u_local), while the caller's stream runs
// the ghost-independent planes (PART_INTERIOR, which also writes the boundary
// faces); the caller's stream then waits for the exchange and runs the <= 4
// planes next to the ghosts (PART_EDGE).  No host synchronisation.  The only
// collective is the optional 5-double all-reduce of the rhs norm (f1).
//
// NCCL is resolved at run time (dlopen of libnccl.so.2 -- in a PyTorch
// process the copy torch already loaded), so loading the library needs no
// NCCL and a missing one is an error code (SAFARA_ERR_NCCL), never a fallback.
#include <dlfcn.h>
#include <nccl.h>

#include <cstdint>
#include <cstring>
#include <mutex>
#include <new>

#include "safara_internal.h"

namespace {

struct Nccl {
    bool tried = false, ok = false;
    ncclResult_t (*GetUniqueId)(ncclUniqueId *) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*CommAbort)(ncclComm_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    ncclResult_t (*Send)(const void *, size_t, ncclDataType_t, int, ncclComm_t,
                         cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*AllReduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t,
                              ncclComm_t, cudaStream_t) = nullptr;
};
Nccl g_nccl;
std::mutex g_nccl_mutex;

template <typename F>
bool sym(void *h, const char *name, F &f) {
    f = reinterpret_cast<F>(dlsym(h, name));
    return f != nullptr;
}

bool nccl_load() {
    std::lock_guard<std::mutex> lock(g_nccl_mutex);
    if (g_nccl.tried) return g_nccl.ok;
    g_nccl.tried = true;
    // the process's NCCL if one is loaded (torch's), else the loader's search
    void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return false;
    Nccl &n = g_nccl;
    n.ok = sym(h, "ncclGetUniqueId", n.GetUniqueId) && sym(h, "ncclCommInitRank", n.CommInitRank) &&
           sym(h, "ncclCommDestroy", n.CommDestroy) && sym(h, "ncclCommAbort", n.CommAbort) &&
           sym(h, "ncclGroupStart", n.GroupStart) && sym(h, "ncclGroupEnd", n.GroupEnd) &&
           sym(h, "ncclSend", n.Send) && sym(h, "ncclRecv", n.Recv) &&
           sym(h, "ncclAllReduce", n.AllReduce);
    return n.ok;
}

constexpr uint32_t kShardMagic = 0x5AFA5A4Du;

struct Shard {
    uint32_t magic = kShardMagic;
    int rank = 0, nranks = 1, device = 0;
    ncclComm_t comm = nullptr;
    cudaStream_t comm_stream = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_halo = nullptr;
};

Shard *as_shard(void *p) {
    Shard *s = static_cast<Shard *>(p);
    return (s && s->magic == kShardMagic) ? s : nullptr;
}

// The caller's device must be the shard's (the communicator is bound to it).
int check_device(const Shard *s) {
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess) return SAFARA_ERR_CUDA;
    return dev == s->device ? SAFARA_OK : SAFARA_ERR_ARG;
}

}  // namespace

extern "C" {

int safara_get_unique_id(void *id128) {
    if (!id128) return SAFARA_ERR_ARG;
    if (!nccl_load()) return SAFARA_ERR_NCCL;
    ncclUniqueId id;
    if (g_nccl.GetUniqueId(&id) != ncclSuccess) return SAFARA_ERR_NCCL;
    static_assert(sizeof(id) == SAFARA_UNIQUE_ID_BYTES, "ncclUniqueId size");
    std::memcpy(id128, &id, sizeof(id));
    return SAFARA_OK;
}

int safara_shard_init(const void *id128, int rank, int nranks, int device, void **shard) {
    if (!id128 || !shard) return SAFARA_ERR_ARG;
    *shard = nullptr;
    if (nranks < 1 || rank < 0 || rank >= nranks) return SAFARA_ERR_ARG;
    int rc = safara_rhs_init(device);  // sm_100 check, kernels set up
    if (rc) return rc;
    if (!nccl_load()) return SAFARA_ERR_NCCL;
    int prev = 0;
    if (cudaGetDevice(&prev) != cudaSuccess) return SAFARA_ERR_CUDA;
    if (cudaSetDevice(device) != cudaSuccess) return SAFARA_ERR_CUDA;
    Shard *s = new (std::nothrow) Shard;
    if (!s) {
        cudaSetDevice(prev);
        return SAFARA_ERR_ARG;
    }
    s->rank = rank;
    s->nranks = nranks;
    s->device = device;
    rc = SAFARA_OK;
    if (cudaStreamCreateWithFlags(&s->comm_stream, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&s->ev_fork, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&s->ev_halo, cudaEventDisableTiming) != cudaSuccess)
        rc = SAFARA_ERR_CUDA;
    if (rc == SAFARA_OK) {
        ncclUniqueId id;
        std::memcpy(&id, id128, sizeof(id));
        if (g_nccl.CommInitRank(&s->comm, nranks, id, rank) != ncclSuccess) {
            s->comm = nullptr;
            rc = SAFARA_ERR_NCCL;
        }
    }
    cudaSetDevice(prev);
    if (rc != SAFARA_OK) {
        safara_shard_finalize(s);
        return rc;
    }
    *shard = s;
    return SAFARA_OK;
}

int safara_shard_finalize(void *shard) {
    Shard *s = as_shard(shard);
    if (!s) return SAFARA_ERR_ARG;
    int prev = 0;
    cudaGetDevice(&prev);
    cudaSetDevice(s->device);
    int rc = SAFARA_OK;
    if (s->comm && g_nccl.CommDestroy(s->comm) != ncclSuccess) rc = SAFARA_ERR_NCCL;
    if (s->comm_stream) cudaStreamDestroy(s->comm_stream);
    if (s->ev_fork) cudaEventDestroy(s->ev_fork);
    if (s->ev_halo) cudaEventDestroy(s->ev_halo);
    cudaSetDevice(prev);
    s->magic = 0;
    delete s;
    return rc;
}

int safara_shard_rank(void *shard, int *rank, int *nranks) {
    Shard *s = as_shard(shard);
    if (!s || !rank || !nranks) return SAFARA_ERR_ARG;
    *rank = s->rank;
    *nranks = s->nranks;
    return SAFARA_OK;
}

int safara_rhs_sharded_ex(void *shard, const double *u_local, const double *forcing_local,
                          double *rhs_local, const safara_dims_t *dims, int k0, int nz_local,
                          const safara_coeffs_t *coeffs, int flags, void *stream) {
    Shard *s = as_shard(shard);
    if (!s || !dims) return SAFARA_ERR_ARG;
    int rc = check_device(s);
    if (rc) return rc;
    if (nz_local < 2 || k0 < 0 || k0 + nz_local > dims->nz) return SAFARA_ERR_SHAPE;
    // rank r's neighbours are r-1 (owning the planes below k0) and r+1 (from
    // k0 + nz_local): the grid ends are exactly the first and last rank
    if ((k0 == 0) != (s->rank == 0) || (k0 + nz_local == dims->nz) != (s->rank == s->nranks - 1))
        return SAFARA_ERR_SHAPE;
    rc = safara_validate_dims(dims, nz_local + 4);
    if (rc) return rc;
    cudaStream_t cs = (cudaStream_t)stream;
    if (s->nranks == 1)
        return safara_rhs_slab(u_local, forcing_local, rhs_local, dims, k0, nz_local, coeffs,
                               flags, SAFARA_PART_ALL, stream);
    // u planes: local p = global k0 - 2 + p; owned [2, nzl+2), ghosts 0-1 and
    // nzl+2, nzl+3.  Two planes per side = 2*sk doubles, contiguous.
    const size_t nplane2 = 2 * (size_t)dims->sk;
    double *u = const_cast<double *>(u_local);
    if (cudaEventRecord(s->ev_fork, cs) != cudaSuccess ||
        cudaStreamWaitEvent(s->comm_stream, s->ev_fork, 0) != cudaSuccess)
        return SAFARA_ERR_CUDA;
    bool ok = g_nccl.GroupStart() == ncclSuccess;
    if (ok && s->rank > 0)
        ok = g_nccl.Send(u + 2 * (size_t)dims->sk, nplane2, ncclFloat64, s->rank - 1, s->comm,
                         s->comm_stream) == ncclSuccess &&
             g_nccl.Recv(u, nplane2, ncclFloat64, s->rank - 1, s->comm, s->comm_stream) ==
                 ncclSuccess;
    if (ok && s->rank < s->nranks - 1)
        ok = g_nccl.Send(u + (size_t)nz_local * dims->sk, nplane2, ncclFloat64, s->rank + 1,
                         s->comm, s->comm_stream) == ncclSuccess &&
             g_nccl.Recv(u + (size_t)(nz_local + 2) * dims->sk, nplane2, ncclFloat64,
                         s->rank + 1, s->comm, s->comm_stream) == ncclSuccess;
    if (g_nccl.GroupEnd() != ncclSuccess) ok = false;
    if (!ok) return SAFARA_ERR_NCCL;
    if (cudaEventRecord(s->ev_halo, s->comm_stream) != cudaSuccess) return SAFARA_ERR_CUDA;
    // ghost-independent planes (and the boundary faces) while the halo flies
    rc = safara_rhs_slab(u_local, forcing_local, rhs_local, dims, k0, nz_local, coeffs, flags,
                         SAFARA_PART_INTERIOR, stream);
    if (rc) {
        cudaStreamWaitEvent(cs, s->ev_halo, 0);  // keep stream order with the exchange
        return rc;
    }
    if (cudaStreamWaitEvent(cs, s->ev_halo, 0) != cudaSuccess) return SAFARA_ERR_CUDA;
    return safara_rhs_slab(u_local, forcing_local, rhs_local, dims, k0, nz_local, coeffs, flags,
                           SAFARA_PART_EDGE, stream);
}

int safara_rhs_sharded(void *shard, const double *u_local, const double *forcing_local,
                       double *rhs_local, int nx, int ny, int nz_global, int k0, int nz_local,
                       const safara_coeffs_t *coeffs, void *stream) {
    safara_dims_t d;
    int rc = safara_dims_canonical(nx, ny, nz_global, &d);
    if (rc) return rc;
    return safara_rhs_sharded_ex(shard, u_local, forcing_local, rhs_local, &d, k0, nz_local,
                                 coeffs, 0, stream);
}

int safara_shard_rms(void *shard, const double *rhs_local, const safara_dims_t *dims, int k0,
                     int nz_local, double *work, double *rms, void *stream) {
    Shard *s = as_shard(shard);
    if (!s || !dims || !rms) return SAFARA_ERR_ARG;
    int rc = check_device(s);
    if (rc) return rc;
    // per-slab sums of squares (interior points of the global grid only)
    rc = safara_rhs_sumsq(rhs_local, dims, k0, nz_local, work, rms, stream);
    if (rc) return rc;
    if (s->nranks > 1 && g_nccl.AllReduce(rms, rms, 5, ncclFloat64, ncclSum, s->comm,
                                          (cudaStream_t)stream) != ncclSuccess)
        return SAFARA_ERR_NCCL;
    const double npts = (double)(dims->nx - 2) * (double)(dims->ny - 2) * (double)(dims->nz - 2);
    if (safara::launch_rms_finish(rms, npts, (cudaStream_t)stream) != cudaSuccess)
        return SAFARA_ERR_CUDA;
    safara::count_launches(1);
    return SAFARA_OK;
}

}  // extern "C"
