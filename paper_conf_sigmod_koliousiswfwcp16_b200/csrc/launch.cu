// launch.cu -- the kernel sequence of one query task (host side).
#include <cuda_runtime.h>

#include "kernels.h"
#include "launch_internal.h"

namespace sb {

cudaError_t set_kernel_attributes(const Plan &p) {
  cudaError_t e = cudaSuccess;
  if (p.nagg == 0) return cudaFuncSetAttribute(sel_kernel(p), cudaFuncAttributeMaxDynamicSharedMemorySize, sel_smem_bytes());
  if (p.bucket_mode) return bk_set_attributes(p);
  if (p.nagg > 0) {
    e = p1_set_attributes(p);
    if (e) return e;
    if (p.p2_smem > 0) e = cudaFuncSetAttribute(p2_kernel(p), cudaFuncAttributeMaxDynamicSharedMemorySize, p.p2_smem);
    if (e) return e;
    if (p.win_block && (e = wb_set_attributes(p))) return e;
    if (p.key_mode == KM_HASH) {
      e = cudaFuncSetAttribute(p2_kernel_count(p), cudaFuncAttributeMaxDynamicSharedMemorySize, p.p2_smem);
      if (e) return e;
    }
    if (p.slab_mode) {
      e = cudaFuncSetAttribute(slab_kernel(false), cudaFuncAttributeMaxDynamicSharedMemorySize, p.p2_smem);
      if (e) return e;
      e = cudaFuncSetAttribute(slab_kernel(true), cudaFuncAttributeMaxDynamicSharedMemorySize, p.p2_smem);
    }
  }
  return e;
}

int p2_blocks_per_sm(const Plan &p) {
  int b = 0;
  if (p.bucket_mode) return 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, p.slab_mode ? slab_kernel(true) : p2_kernel(p), 256, p.p2_smem);
  return b > 0 ? b : 1;
}
int sel_blocks_per_sm(const Plan &p) {
  int b = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, sel_kernel(p), 256, sel_smem_bytes());
  return b > 0 ? b : 1;
}

cudaError_t launch_agg_task(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples, int64_t n,
                            int final_, int has_wm, int64_t wm, int emit_on_finish, int p1_grid, int p2_grid,
                            int win_chunk, cudaStream_t st, cudaEvent_t *evs, int *launches) {
  cudaError_t e;
  if ((e = launch_task_begin(p, q, s, tuples, n, final_, has_wm, wm, emit_on_finish, st))) return e;
  if ((e = launch_zero_panes(p, q, st))) return e;
  *launches = 2;
  if (evs) cudaEventRecord(evs[0], st);
  if (n > 0) {
    if (p.bucket_mode) e = launch_bucket_scan(p, q, tuples, n, p1_grid, st);
    else e = launch_pane_agg(p, q, tuples, n, p1_grid, st);
    if (e) return e;
    *launches += 1;
  }
  if (evs) cudaEventRecord(evs[1], st);
  if (p.bucket_mode) {
    if ((e = launch_bucket_windows(p, q, s, p2_grid, st))) return e;
    *launches += 3;
  } else if (p.slab_mode) {
    if ((e = launch_windows_slab(p, q, s, false, p2_grid, win_chunk, st))) return e;
    if ((e = launch_win_scan(p, q, s, st))) return e;
    if ((e = launch_windows_slab(p, q, s, true, p2_grid, win_chunk, st))) return e;
    *launches += 1;
  } else if (p.key_mode == KM_HASH) {
    if ((e = launch_windows(p, q, s, false, p2_grid, win_chunk, st))) return e;
    if ((e = launch_win_scan(p, q, s, st))) return e;
    if ((e = launch_windows(p, q, s, true, p2_grid, win_chunk, st))) return e;
  } else if (p.win_block) {
    if ((e = launch_windows_block(p, q, s, p.wb_grid, st))) return e;
  } else {
    if ((e = launch_windows_fused(p, q, s, p2_grid, st))) return e;
  }
  if ((e = launch_task_end(p, q, s, st))) return e;
  *launches += p.bucket_mode ? 1 : p.key_mode == KM_HASH ? 4 : 3;
  if (evs) cudaEventRecord(evs[2], st);
  return cudaGetLastError();
}

cudaError_t launch_select_task(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples, int64_t n,
                               int final_, int has_wm, int64_t wm, int emit_on_finish, int sel_grid, cudaStream_t st,
                               cudaEvent_t *evs, int *launches) {
  cudaError_t e;
  if ((e = launch_task_begin(p, q, s, tuples, n, final_, has_wm, wm, emit_on_finish, st))) return e;
  if (evs) cudaEventRecord(evs[0], st);
  if ((e = launch_select(p, q, s, tuples, sel_grid, st))) return e;
  if (evs) cudaEventRecord(evs[1], st);
  if ((e = launch_carry(p, q, tuples, st))) return e;
  if ((e = launch_task_end(p, q, s, st))) return e;
  *launches = 5;
  if (evs) cudaEventRecord(evs[2], st);
  return cudaGetLastError();
}

}  // namespace sb
