// kc_common.cuh -- PTX helpers and launch constants shared by the sm_100a
// kernels of the k-core hot path.  (Product code; shares nothing with oracle/.)
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace kc {

constexpr unsigned kFull = 0xffffffffu;

// 64-bit queue tail packs (#vertices appended << 33) | (#arcs appended) so one
// atomicAdd reserves frontier slots and their arc range together.
constexpr int kArcBits = 33;
constexpr unsigned long long kArcMask = (1ULL << kArcBits) - 1ULL;
constexpr unsigned long long kCntOne = 1ULL << kArcBits;

__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void red_release_add_u32(uint32_t *p, uint32_t v)
{
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// fire-and-forget OR (no return value awaited)
__device__ __forceinline__ void red_or_u32(uint32_t *p, uint32_t v)
{
    asm volatile("red.relaxed.gpu.global.or.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// CTA-scope acquire / release on a shared-memory flag
__device__ __forceinline__ int ld_acquire_cta_shared(const int *p)
{
    int v;
    const unsigned a = (unsigned)__cvta_generic_to_shared(p);
    asm volatile("ld.acquire.cta.shared.b32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
    return v;
}

__device__ __forceinline__ void st_release_cta_shared(int *p, int v)
{
    const unsigned a = (unsigned)__cvta_generic_to_shared(p);
    asm volatile("st.release.cta.shared.b32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}

__device__ __forceinline__ void st_release_u32(uint32_t *p, uint32_t v)
{
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ uint32_t atom_add_release_u32(uint32_t *p, uint32_t v)
{
    uint32_t old;
    asm volatile("atom.release.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
    return old;
}

__device__ __forceinline__ uint32_t atom_add_acq_rel_u32(uint32_t *p, uint32_t v)
{
    uint32_t old;
    asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
    return old;
}

__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long *p)
{
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_relaxed_u64(unsigned long long *p, unsigned long long v)
{
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void fence_acq_rel_gpu()
{
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
}

__device__ __forceinline__ int32_t ld_relaxed_i32(const int32_t *p)
{
    int32_t v;
    asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// streaming read-only loads of the CSR (never written during a call)
#ifdef KC_COLIDX_EVICT_FIRST
// L2 evict-first: the adjacency stream must not push deg / code out of L2
__device__ __forceinline__ uint64_t l2_evict_first_policy()
{
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ int32_t ld_stream_i32(const int32_t *p)
{
    int32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;"
                 : "=r"(v) : "l"(p), "l"(l2_evict_first_policy()));
    return v;
}
#else
__device__ __forceinline__ int32_t ld_stream_i32(const int32_t *p)
{
    int32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
#endif

__device__ __forceinline__ int64_t ld_ro_i64(const int64_t *p) { return __ldg(p); }

// L2 residency of the scattered working set (deg, claim bits): the 4 GB
// adjacency stream of a big level must not evict it, or every scattered
// atomic becomes an HBM read-modify-write.
#ifndef KC_DEG_EVICT_LAST
#define KC_DEG_EVICT_LAST 0
#endif
__device__ __forceinline__ uint64_t l2_evict_last_policy()
{
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ int32_t atom_dec_deg(int32_t *p, uint64_t pol)
{
#if KC_DEG_EVICT_LAST
    int32_t old;
    asm volatile("atom.global.L2::cache_hint.add.s32 %0, [%1], -1, %2;" : "=r"(old) : "l"(p), "l"(pol) : "memory");
    return old;
#else
    (void)pol;
    return atomicSub(p, 1);
#endif
}
__device__ __forceinline__ int32_t ld_deg(const int32_t *p, uint64_t pol)
{
#if KC_DEG_EVICT_LAST
    int32_t v;
    asm volatile("ld.global.cg.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
#else
    (void)pol;
    return __ldcg(p);
#endif
}
__device__ __forceinline__ uint32_t atom_or_claim(uint32_t *p, uint32_t bit, uint64_t pol)
{
#if KC_DEG_EVICT_LAST
    uint32_t old;
    asm volatile("atom.global.L2::cache_hint.or.b32 %0, [%1], %2, %3;" : "=r"(old) : "l"(p), "r"(bit), "l"(pol) : "memory");
    return old;
#else
    (void)pol;
    return atomicOr(p, bit);
#endif
}

// L2-coherent loads of data other CTAs write during the call (deg, queue)
__device__ __forceinline__ int32_t ld_cg_i32(const int32_t *p) { return __ldcg(p); }
__device__ __forceinline__ int64_t ld_cg_i64(const int64_t *p) { return __ldcg(p); }

// Optionally warm L2 with the adjacency row [b, e) of a vertex that was just
// claimed (measured: no gain on B200, off by default -- DESIGN.md §8), so
// the next hop's colidx gathers hit L2: one TMA bulk prefetch of the whole
// row (16-byte aligned, capped at KC_BULK_PF bytes), or the first line only.
#ifndef KC_BULK_PF
#define KC_BULK_PF -1
#endif
__device__ __forceinline__ void prefetch_row(const int32_t *colidx, int64_t b, int64_t e)
{
#if KC_BULK_PF > 0
    const uintptr_t lo = reinterpret_cast<uintptr_t>(colidx + b) & ~(uintptr_t)15;
    uintptr_t hi = (reinterpret_cast<uintptr_t>(colidx + e) + 15) & ~(uintptr_t)15;
    if (hi - lo > (uintptr_t)KC_BULK_PF) hi = lo + KC_BULK_PF;
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(lo), "r"((uint32_t)(hi - lo)) : "memory");
#elif KC_BULK_PF < 0
    (void)colidx; (void)b; (void)e;  // no prefetch (measurement variant)
#else
    (void)e;
    asm volatile("prefetch.global.L2 [%0];" ::"l"(colidx + b));
#endif
}

__device__ __forceinline__ unsigned lanemask_lt()
{
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// Ballot scan of Fig. 8(c): every lane of the warp
// contributes a 0/1 predicate; `bits` = __ballot_sync of them, the return value
// = the lane's EXCLUSIVE prefix count (the number of set predicates in lower
// lanes, Fig. 8's a[j]).  The warp's total is __popc(bits), by which one lane
// advances the append cursor e (Fig. 8, Lines 3-5).
__device__ __forceinline__ int ballot_excl(bool p, unsigned &bits)
{
    bits = __ballot_sync(0xffffffffu, p);
    return __popc(bits & lanemask_lt());
}

// Warp-aggregated append (Fig. 8, Lines 1-8): lanes with p write v to
// buf[e_old + a[j]]; the lowest active lane advances *e by the warp's count in
// ONE atomicAdd and broadcasts e_old.  Returns the warp's count.
__device__ __forceinline__ int warp_append(bool p, int32_t v, int32_t *buf, int *e)
{
    unsigned bits;
    const int a = ballot_excl(p, bits);
    if (bits == 0u) return 0;
    const int lead = __ffs(bits) - 1;
    int base = 0;
    if ((int)(threadIdx.x & 31) == lead) base = atomicAdd(e, __popc(bits));
    base = __shfl_sync(0xffffffffu, base, lead);
    if (p) buf[base + a] = v;
    return __popc(bits);
}

} // namespace kc
