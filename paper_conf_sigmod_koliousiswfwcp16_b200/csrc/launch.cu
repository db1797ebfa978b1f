// launch.cu -- the kernel sequence of one query task (host side).
#include <cuda_runtime.h>

#include "kernels.h"
#include "launch_internal.h"

namespace sb {

cudaError_t launch_agg_round(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples, int64_t n,
                             int final_, int has_wm, int64_t wm, int emit_on_finish, int p1_grid, int p2_grid,
                             int win_chunk, cudaStream_t st, cudaEvent_t *evs, int *launches, int round);

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
    if (p.win_wide && (e = ww_set_attributes(p))) return e;
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
  // rounds (State::round_off): every round re-runs the kernel sequence on the next
  // sub-range of the task that k_task_begin chose; the last round applies finish()
  if (p.rounds > 1) {
    int total = 0;
    for (int r = 0; r < p.rounds; ++r) {
      int l = 0;
      const bool last = r == p.rounds - 1;
      cudaError_t e = launch_agg_round(p, q, s, tuples, n, last ? final_ : 0, has_wm, wm, emit_on_finish, p1_grid,
                                       p2_grid, win_chunk, st, r == 0 ? evs : nullptr, &l, r);
      if (e) return e;
      total += l;
    }
    if (evs) cudaEventRecord(evs[2], st);
    *launches = total;
    return cudaSuccess;
  }
  return launch_agg_round(p, q, s, tuples, n, final_, has_wm, wm, emit_on_finish, p1_grid, p2_grid, win_chunk, st,
                          evs, launches, 0);
}

cudaError_t launch_agg_round(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples, int64_t n,
                             int final_, int has_wm, int64_t wm, int emit_on_finish, int p1_grid, int p2_grid,
                             int win_chunk, cudaStream_t st, cudaEvent_t *evs, int *launches, int round) {
  cudaError_t e;
  if ((e = launch_task_begin(p, q, s, tuples, n, final_, has_wm, wm, emit_on_finish, st, round))) return e;
  // a count-window task without tuples (finish() after the last one) closes no
  // window (they close by position, reading A3) and touches no pane: bookkeeping only
  if (n == 0 && p.win_kind == WK_COUNT) {
    if (evs) { cudaEventRecord(evs[0], st); cudaEventRecord(evs[1], st); }
    if ((e = launch_task_end(p, q, s, st))) return e;
    *launches = 2;
    if (evs) cudaEventRecord(evs[2], st);
    return cudaGetLastError();
  }
  if ((e = launch_zero_panes(p, q, st, p.bucket_mode ? 0 : n, p1_grid))) return e;
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
    *launches += 4;     // k_bkt_count, k_win_scan, k_bkt_emit (clean items), k_bkt_emit (dirty items)
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
  *launches += p.bucket_mode ? 1 : p.key_mode == KM_HASH ? 4 : p.win_wide && !p.nhave ? 5 : p.win_block && wb_prepass(p) ? 4 : 3;   // k_win_wide: + count + scan; k_win_block_reg: + k_wb_rows
  if (evs) cudaEventRecord(evs[2], st);
  return cudaGetLastError();
}

// Overlap plans (dense/global pane tables, see Plan::overlap).  On `cs`: task
// prologue, pane-slot initialisation, the scan, a snapshot of State into the
// slot (the window kernels' J0/J1/epoch) and the task epilogue, which advances
// J0 so the next task's prologue can run at once.  On `ws`, after `scan_done`:
// the window phase on the snapshot with the slot's own ticket counter, then
// k_win_end (row count, window-phase errors).  The caller keeps `cs` at most one
// task ahead of `ws` (the pane ring keeps [live_J0·L, ...) intact for that).
cudaError_t launch_agg_task_overlap(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples,
                                    int64_t n, int final_, int has_wm, int64_t wm, int emit_on_finish,
                                    int p1_grid, int p2_grid, cudaStream_t cs, cudaStream_t ws,
                                    cudaEvent_t scan_done, cudaEvent_t *evs, int *launches) {
  cudaError_t e;
  if ((e = launch_task_begin(p, q, s, tuples, n, final_, has_wm, wm, emit_on_finish, cs))) return e;
  if ((e = launch_zero_panes(p, q, cs, 0, p1_grid))) return e;
  *launches = 2;
  if (evs) cudaEventRecord(evs[0], cs);
  if (n > 0) {
    if ((e = launch_pane_agg(p, q, tuples, n, p1_grid, cs))) return e;
    *launches += 1;
  }
  if (evs) cudaEventRecord(evs[1], cs);
  if ((e = cudaMemcpyAsync(s.wst, q.st, sizeof(State), cudaMemcpyDeviceToDevice, cs))) return e;
  if ((e = cudaMemsetAsync(s.ticket, 0, 2 * sizeof(int), cs))) return e;
  if ((e = launch_task_end(p, q, s, cs))) return e;
  if ((e = cudaEventRecord(scan_done, cs))) return e;
  if ((e = cudaStreamWaitEvent(ws, scan_done, 0))) return e;
  QueryDev qw = q;
  qw.st = s.wst;
  qw.tile_ctr = s.ticket;
  if (p.win_block) e = launch_windows_block(p, qw, s, p.wb_grid, ws);
  else e = launch_windows_fused(p, qw, s, p2_grid, ws);
  if (e) return e;
  if ((e = launch_win_end(q, s, ws))) return e;
  *launches += p.win_block ? (wb_prepass(p) ? 4 : 3) : p.win_wide && !p.nhave ? 6 : 4;
  if (evs) cudaEventRecord(evs[2], ws);
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
  *launches = 6;     // k_task_begin, k_select, k_select_fix, k_sel_hdr, k_carry, k_task_end
  if (evs) cudaEventRecord(evs[2], st);
  return cudaGetLastError();
}

}  // namespace sb
