/*
 * atfgen_test.h — test hooks of libatfgen (not part of the product API).
 *
 * atf_test_exclusive_scan_u32: the decoupled look-back exclusive scan used by the
 * fused expand kernel, exposed alone so it can be checked
 * against std::exclusive_scan on adversarial count arrays.
 *   d_in:  device uint32[n]; d_out: device uint64[n + 1]; d_out[n] = total.
 *   Scratch is allocated internally (cudaMallocAsync on `stream`).  Synchronous.
 */
#ifndef ATFGEN_TEST_H
#define ATFGEN_TEST_H
#include "atfgen.h"
#ifdef __cplusplus
extern "C" {
#endif
atf_status atf_test_exclusive_scan_u32(const uint32_t* d_in, uint64_t* d_out, int64_t n, void* stream);
#ifdef __cplusplus
}
#endif
#endif
