// tracker.cpp — libglp_tracker.so: the paper's CUPTI resource tracker.
//
// GLP4NN profiles every kernel once through a "resource tracker" built on CUPTI (§3.1
// P165, Fig. 6 "profile once, execute many" P173): grid and block shape, registers, shared
// memory and duration of each kernel instance feed the kernel analyzer (Table 2 "profiling input"
// P194-200; T_K of Eq. 7, P245).  Here the tracker is a CUPTI Activity-API collector of
//   * kernel records (CUPTI_ACTIVITY_KIND_CONCURRENT_KERNEL): name, grid, block, cluster,
//     registers, static + dynamic shared memory, queued / submitted / start / end timestamps;
//   * launch-API records (CUPTI_ACTIVITY_KIND_RUNTIME / DRIVER, the kernel-launch entry points):
//     the host-side launch cost, the paper's T_launch.
// The library sits beside libglp.so (its own .so so that the product path never loads CUPTI) and
// is driven by paper_conf_icpp_futhys18_b200.tracker; the stream-pool comparator uses it to put
// the measured T_K / T_launch term into its Eq. 7 bound (glp_pool_set_launch_term).
#include <cupti.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/glp_tracker.h"

namespace {

std::mutex g_mu;
std::vector<glp_kernel_record_t> g_kernels;
std::vector<glp_launch_record_t> g_launches;
bool g_on = false, g_registered = false;
std::string g_err;

constexpr size_t kBuf = 8u << 20;

void CUPTIAPI buffer_requested(uint8_t **buffer, size_t *size, size_t *max_records) {
  *buffer = static_cast<uint8_t *>(aligned_alloc(8, kBuf));
  *size = kBuf;
  *max_records = 0;
}

bool is_launch_cbid(CUpti_ActivityKind kind, CUpti_CallbackId cbid) {
  if (kind == CUPTI_ACTIVITY_KIND_RUNTIME)
    return cbid == CUPTI_RUNTIME_TRACE_CBID_cudaLaunchKernel_v7000 ||
           cbid == CUPTI_RUNTIME_TRACE_CBID_cudaLaunchKernelExC_v11060;
  return cbid == CUPTI_DRIVER_TRACE_CBID_cuLaunchKernel || cbid == CUPTI_DRIVER_TRACE_CBID_cuLaunchKernelEx;
}

void CUPTIAPI buffer_completed(CUcontext, uint32_t, uint8_t *buffer, size_t, size_t valid) {
  CUpti_Activity *rec = nullptr;
  std::lock_guard<std::mutex> lk(g_mu);
  while (cuptiActivityGetNextRecord(buffer, valid, &rec) == CUPTI_SUCCESS) {
    if (rec->kind == CUPTI_ACTIVITY_KIND_CONCURRENT_KERNEL || rec->kind == CUPTI_ACTIVITY_KIND_KERNEL) {
      const auto *k = reinterpret_cast<const CUpti_ActivityKernel9 *>(rec);
      glp_kernel_record_t r;
      memset(&r, 0, sizeof(r));
      if (k->name) strncpy(r.name, k->name, sizeof(r.name) - 1);
      r.grid[0] = k->gridX;
      r.grid[1] = k->gridY;
      r.grid[2] = k->gridZ;
      r.block[0] = k->blockX;
      r.block[1] = k->blockY;
      r.block[2] = k->blockZ;
      r.cluster[0] = (int)k->clusterX;
      r.cluster[1] = (int)k->clusterY;
      r.cluster[2] = (int)k->clusterZ;
      r.regs = k->registersPerThread;
      r.static_smem = k->staticSharedMemory;
      r.dynamic_smem = k->dynamicSharedMemory;
      r.queued_ns = k->queued;
      r.submitted_ns = k->submitted;
      r.start_ns = k->start;
      r.end_ns = k->end;
      r.stream_id = k->streamId;
      r.correlation_id = k->correlationId;
      g_kernels.push_back(r);
    } else if (rec->kind == CUPTI_ACTIVITY_KIND_RUNTIME || rec->kind == CUPTI_ACTIVITY_KIND_DRIVER) {
      const auto *a = reinterpret_cast<const CUpti_ActivityAPI *>(rec);
      if (!is_launch_cbid(rec->kind, a->cbid)) continue;
      glp_launch_record_t r;
      r.start_ns = a->start;
      r.end_ns = a->end;
      r.correlation_id = a->correlationId;
      r.driver = rec->kind == CUPTI_ACTIVITY_KIND_DRIVER ? 1 : 0;
      g_launches.push_back(r);
    }
  }
  free(buffer);
}

int check(CUptiResult r, const char *what) {
  if (r == CUPTI_SUCCESS) return 0;
  const char *s = nullptr;
  cuptiGetResultString(r, &s);
  g_err = std::string(what) + ": " + (s ? s : "unknown CUPTI error");
  return 1;
}

const CUpti_ActivityKind kKinds[] = {CUPTI_ACTIVITY_KIND_CONCURRENT_KERNEL,
                                     CUPTI_ACTIVITY_KIND_RUNTIME, CUPTI_ACTIVITY_KIND_DRIVER};

}  // namespace

extern "C" {

int glp_tracker_start(void) {
  if (g_on) return 0;
  if (!g_registered) {
    if (check(cuptiActivityRegisterCallbacks(buffer_requested, buffer_completed),
              "cuptiActivityRegisterCallbacks"))
      return 1;
    g_registered = true;
  }
  for (CUpti_ActivityKind k : kKinds)
    if (check(cuptiActivityEnable(k), "cuptiActivityEnable")) return 1;
  g_on = true;
  return 0;
}

int glp_tracker_stop(void) {
  if (!g_on) return 0;
  int rc = check(cuptiActivityFlushAll(1), "cuptiActivityFlushAll");
  for (CUpti_ActivityKind k : kKinds) rc |= check(cuptiActivityDisable(k), "cuptiActivityDisable");
  g_on = false;
  return rc;
}

void glp_tracker_clear(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_kernels.clear();
  g_launches.clear();
}

int glp_tracker_kernel_count(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  return (int)g_kernels.size();
}

int glp_tracker_kernel(int i, glp_kernel_record_t *out) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!out || i < 0 || i >= (int)g_kernels.size()) return 1;
  *out = g_kernels[(size_t)i];
  return 0;
}

int glp_tracker_launch_count(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  return (int)g_launches.size();
}

int glp_tracker_launch(int i, glp_launch_record_t *out) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!out || i < 0 || i >= (int)g_launches.size()) return 1;
  *out = g_launches[(size_t)i];
  return 0;
}

const char *glp_tracker_last_error(void) { return g_err.c_str(); }

}  // extern "C"
