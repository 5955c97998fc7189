/*
 * kcore_test.h -- unit-test hooks of libkcore.so (NOT part of the product API
 * in include/kcore.h).  Each hook runs ONE device primitive of the hot path in
 * isolation so a test can pin it against a value the paper prints.
 */
#ifndef KCORE_TEST_H
#define KCORE_TEST_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Warp-level compaction of Fig. 8 (Sec. IV-C "Reducing
 * Contention for Buffer Appending"): the device primitive the scan and the
 * peel use to append claimed vertices (kc::ballot_excl / kc::warp_append).
 * One warp per 32 consecutive entries.  DEVICE pointers:
 *   vid[n]     vertex ids examined by the lanes,
 *   pred[n]    0/1 predicate p[j] (1 = append),
 *   prefix[n]  out: a[j], the exclusive ballot-scan prefix within the warp,
 *   buf[n]     out: appended ids (buf[e_old + a[j]] = vid[j] for p[j] = 1),
 *   e          in/out: the append cursor (int32, advanced once per warp).
 * n in [0, 2^20].  Synchronises `stream`.  Returns a kcore_status. */
int kcore_test_ballot_compact(const int32_t *vid, const int32_t *pred, int32_t n, int32_t *prefix,
                              int32_t *buf, int32_t *e, void *stream);

/* Watchdog of the device-initiated multi-GPU kernel: every wait longer than
 * `ns` nanoseconds aborts the call with KCORE_ECUDA instead of hanging
 * (default 60 s; ns <= 0 restores it).  Tests shorten it to exercise the path. */
int kcore_test_mgd_timeout(int64_t ns);

/* Phase trace of the next kcore_decompose_mg_virtual call (device-initiated
 * protocol; development aid): DEVICE int64[cap][4] records {globaltimer ns,
 * phase (-1 start, 0 init, 1 scan, 2 sub-round), k, removed so far} at every
 * device barrier.  NULL disables. */
int kcore_test_mgd_trace(int64_t *trace, int64_t cap);

#ifdef __cplusplus
}
#endif
#endif
