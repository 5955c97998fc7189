// kcore_testhooks.cu -- unit-test hooks (include/kcore_test.h): one device
// primitive of the hot path per entry, launched in isolation.
#include "kcore.h"
#include "kcore_test.h"
#include "kc_common.cuh"

namespace {

__global__ void k_test_ballot(const int32_t *vid, const int32_t *pred, int32_t n, int32_t *prefix, int32_t *buf,
                              int32_t *e)
{
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    const bool in = i < n;
    const bool p = in && pred[i] != 0;
    unsigned bits;
    const int a = kc::ballot_excl(p, bits);
    if (in) prefix[i] = a;
    kc::warp_append(p, in ? vid[i] : -1, buf, e);
}

} // namespace

extern "C" int kcore_test_ballot_compact(const int32_t *vid, const int32_t *pred, int32_t n, int32_t *prefix,
                                         int32_t *buf, int32_t *e, void *stream)
{
    if (n < 0 || n > (1 << 20)) return KCORE_EINVAL;
    if (n == 0) return KCORE_OK;
    if (!vid || !pred || !prefix || !buf || !e) return KCORE_EINVAL;
    cudaStream_t st = (cudaStream_t)stream;
    k_test_ballot<<<(n + 255) / 256, 256, 0, st>>>(vid, pred, n, prefix, buf, e);
    if (cudaGetLastError() != cudaSuccess) return KCORE_ECUDA;
    if (cudaStreamSynchronize(st) != cudaSuccess) return KCORE_ECUDA;
    return KCORE_OK;
}
