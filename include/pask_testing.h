/*
 * pask_testing.h -- test-only hooks of libpask.so (not part of the product ABI
 * a model server uses).  They let the host logic of the loader / issuer
 * (SURVEY.md §4 tier T2: interleaving, load ordering, error propagation,
 * no deadlock) be exercised on a machine without a GPU, by swapping the CUDA
 * driver table for an in-library fake.
 *
 * The fake driver:
 *   - succeeds every call except the programmed failure;
 *   - cuLibraryLoadData / cuKernelGetFunction sleep load_us microseconds each
 *     (a code upload's host cost);
 *   - cuLaunchKernelEx records the launched kernel id (the catalog id whose
 *     code object was loaded) and whether that kernel had been loaded before
 *     the launch;
 *   - stream capture is unsupported (CUDA_ERROR_NOT_SUPPORTED).
 */
#ifndef PASK_TESTING_H
#define PASK_TESTING_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* enable = 1: route every driver call of newly created contexts to the fake;
 * 0: restore the real driver.  fail_kernel >= 0: loading that catalog kernel
 * fails with CUDA_ERROR_INVALID_IMAGE. */
int pask_test_fake_driver(int32_t enable, int32_t load_us, int32_t fail_kernel);

/* The fake driver's event log since the last enable: out[i] = kernel id of
 * the i-th event, kinds[i] = 0 for a completed load, 1 for a launch on the
 * caller's stream, 3 for a launch on another stream (pask_config.branches), 2
 * for a launch of a kernel that was not yet loaded (must never happen).  Under
 * packaging 2 the `pask_mem` family entry logs as id PASK_MAX_KERNELS - 1 and
 * the contraction family as PASK_K_CONV_IGEMM.  Returns the number of events
 * (writes at most cap). */
int32_t pask_test_fake_log(int32_t *out, int32_t *kinds, int32_t cap);

#ifdef __cplusplus
}
#endif

#endif /* PASK_TESTING_H */
