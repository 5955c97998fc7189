// kcore_mg.cu -- multi-GPU entry points (include/kcore.h).  Placeholder
// returning KCORE_EUNSUPPORTED until the owner-routed protocol lands; the
// NCCL plumbing helpers are live.
#include "kcore.h"

#include <cstring>
#include <nccl.h>

extern "C" int kcore_nccl_unique_id(void *id_out)
{
    if (!id_out) return KCORE_EINVAL;
    ncclUniqueId id;
    if (ncclGetUniqueId(&id) != ncclSuccess) return KCORE_ENCCL;
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    memcpy(id_out, &id, sizeof(id));
    return KCORE_OK;
}

extern "C" int kcore_nccl_comm_init(void **comm_out, int32_t nranks, const void *id_in, int32_t rank)
{
    if (!comm_out || !id_in || nranks < 1 || rank < 0 || rank >= nranks) return KCORE_EINVAL;
    ncclUniqueId id;
    memcpy(&id, id_in, sizeof(id));
    ncclComm_t c = nullptr;
    if (ncclCommInitRank(&c, nranks, id, rank) != ncclSuccess) return KCORE_ENCCL;
    *comm_out = (void *)c;
    return KCORE_OK;
}

extern "C" int kcore_nccl_comm_destroy(void *comm)
{
    if (!comm) return KCORE_EINVAL;
    return ncclCommDestroy((ncclComm_t)comm) == ncclSuccess ? KCORE_OK : KCORE_ENCCL;
}

extern "C" int kcore_decompose_mg(const int64_t *, const int32_t *, int64_t, int64_t, int64_t,
                                  int64_t, int32_t *, void *, void *, kcore_stats *)
{
    return KCORE_EUNSUPPORTED;
}

extern "C" int kcore_decompose_mg_virtual(const int64_t *, const int32_t *, int64_t, int64_t,
                                          int32_t, int32_t *, void *, kcore_stats *)
{
    return KCORE_EUNSUPPORTED;
}
