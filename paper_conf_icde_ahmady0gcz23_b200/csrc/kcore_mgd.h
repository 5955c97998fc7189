// kcore_mgd.h -- internal: the device-initiated multi-GPU peel (kcore_mgd.cu),
// reached through kcore_decompose_mg_ex / kcore_decompose_mg_virtual(_ex).
#pragma once
#include <cstdint>
#include "kcore.h"

// P virtual ranks on the current GPU (global CSR in, global core out).
int mgd_virtual(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m, int32_t nranks,
                int32_t *core_out, void *stream, kcore_stats *stats);
// One rank per process over NCCL symmetric memory (collective).
int mgd_nccl(const int64_t *rowptr_local, const int32_t *colidx_local, int64_t n_global, int64_t v_begin,
             int64_t v_end, int64_t m_local, int32_t *core_out_local, void *stream, void *nccl_comm,
             kcore_stats *stats);
