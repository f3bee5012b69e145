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
 *   - stream capture logs the captured launches; a graph replay launches nothing;
 *   - device memory (only the timeline buffer) is host memory;
 *   - it is compiled only into libpask_testing.so, never into libpask.so.
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

/* Knobs of the fake driver (reset by pask_test_fake_driver):
 *   PASK_FAKE_OCCUPANCY            set what cuOccupancyMaxActiveClusters reports
 *                                  for a 16-CTA cluster (default 1; 0 = cannot
 *                                  co-schedule one); returns 0
 *   PASK_FAKE_CURRENT_DEVICE       make device `value`'s primary context current
 *                                  (default 0); returns 0
 *   PASK_FAKE_MAX_CLUSTER_LAUNCHED returns the largest cluster size (z) launched
 *                                  since the last reset; value ignored
 *   PASK_FAKE_PRIMER_LOADS         returns how many times pask_create's driver
 *                                  primer was uploaded (it is not logged)
 * Unknown knob: -1. */
enum {
  PASK_FAKE_OCCUPANCY = 1,
  PASK_FAKE_CURRENT_DEVICE = 2,
  PASK_FAKE_MAX_CLUSTER_LAUNCHED = 3,
  PASK_FAKE_PRIMER_LOADS = 4
};
int32_t pask_test_fake_knob(int32_t knob, int32_t value);

#ifdef __cplusplus
}
#endif

#endif /* PASK_TESTING_H */
