/*
 * glp_tracker.h — C ABI of libglp_tracker.so, the paper's CUPTI resource tracker (SURVEY §8(f)
 * NEXT-4).
 *
 * GLP4NN profiles each kernel once with a CUPTI-based "resource tracker" (§3.1 P165,
 * Fig. 6 P173: "profile once, execute many") to obtain the kernel analyzer's per-kernel input --
 * grid and block dimensions, registers, shared memory (Table 2 "profiling input", P194-200) -- and
 * the durations behind Eq. 7's launch term ceil(T_K / T_launch) (P243-245).  This library records,
 * between glp_tracker_start and glp_tracker_stop, every kernel the process runs (CUPTI
 * concurrent-kernel activity) and every kernel-launch API call (CUPTI runtime and driver activity
 * of cudaLaunchKernel(ExC) / cuLaunchKernel(Ex)).  Host only; no GPU memory is touched.
 *
 * Ownership: records are copied out into caller structs.  Errors: 0 = OK, non-zero = failure
 * (glp_tracker_last_error() has the CUPTI message; e.g. no device or a CUPTI-incompatible driver).
 * Not thread safe across start/stop; the record accessors are.  Timestamps are CUPTI's (ns).
 * It is a separate library so that the product path (libglp.so) never loads CUPTI.
 */
#ifndef GLP_TRACKER_H_
#define GLP_TRACKER_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  char name[128];          /* mangled kernel name (truncated)                        */
  int grid[3], block[3];   /* #beta (grid) and tau (block) of Table 2                */
  int cluster[3];          /* thread-block cluster dims (CTA pairs: 2,1,1)           */
  int regs;                /* registers per thread                                   */
  int static_smem, dynamic_smem; /* sm_K of Table 2 (bytes per block)                */
  uint64_t queued_ns, submitted_ns, start_ns, end_ns;   /* T_K = end - start           */
  uint32_t stream_id, correlation_id;
} glp_kernel_record_t;

typedef struct {
  uint64_t start_ns, end_ns; /* one kernel-launch API call: T_launch = end - start     */
  uint32_t correlation_id;
  int driver;                /* 1: driver API record, 0: runtime API record            */
} glp_launch_record_t;

int glp_tracker_start(void);            /* enable the activity kinds (idempotent)       */
int glp_tracker_stop(void);             /* flush every buffer and disable               */
void glp_tracker_clear(void);           /* drop the collected records                   */
int glp_tracker_kernel_count(void);
int glp_tracker_kernel(int i, glp_kernel_record_t *rec);
int glp_tracker_launch_count(void);
int glp_tracker_launch(int i, glp_launch_record_t *rec);
const char *glp_tracker_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* GLP_TRACKER_H_ */
