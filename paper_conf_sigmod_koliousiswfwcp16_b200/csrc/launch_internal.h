// launch_internal.h -- per-translation-unit launchers (host side), used by launch.cu.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"
#include "plan.h"

namespace sb {
// k_task.cu
cudaError_t launch_task_begin(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples, int64_t n,
                              int final_, int has_wm, int64_t wm, int emit_on_finish, cudaStream_t st, int round = 0);
cudaError_t launch_zero_panes(const Plan &p, const QueryDev &q, cudaStream_t st, int64_t n, int scan_grid);
// k_pane_cnt initialises the pane slots wholly inside one CTA's tuples: its tuples per CTA (0: other kernels)
int64_t p1_selfzero_per(const Plan &p, int64_t n, int grid, int *g);
bool p1_cnt_fx_plan(const Plan &p);   // the count scan runs k_pane_cnt's FX tables (12 B per entry)
cudaError_t launch_win_scan(const Plan &p, const QueryDev &q, const SlotDev &s, cudaStream_t st);
cudaError_t launch_win_end(const QueryDev &q, const SlotDev &s, cudaStream_t st);
cudaError_t launch_task_end(const Plan &p, const QueryDev &q, const SlotDev &s, cudaStream_t st);
cudaError_t launch_carry(const Plan &p, const QueryDev &q, const void *tuples, cudaStream_t st);
// k_pane.cu
void *p1_kernel(const Plan &p);
cudaError_t p1_set_attributes(const Plan &p);
cudaError_t launch_pane_agg(const Plan &p, const QueryDev &q, const void *tuples, int64_t n, int grid,
                            cudaStream_t st);
// k_window.cu
void *p2_kernel(const Plan &p);
void *p2_kernel_count(const Plan &p);
cudaError_t launch_windows(const Plan &p, const QueryDev &q, const SlotDev &s, bool emit, int grid, int win_chunk,
                           cudaStream_t st);
cudaError_t launch_windows_fused(const Plan &p, const QueryDev &q, const SlotDev &s, int grid, cudaStream_t st);
cudaError_t launch_windows_slab(const Plan &p, const QueryDev &q, const SlotDev &s, bool emit, int grid, int W,
                                cudaStream_t st);
void *slab_kernel(bool emit);
// k_bucket.cu
cudaError_t bk_set_attributes(const Plan &p);
int bk_scan_blocks_per_sm(const Plan &p);
cudaError_t launch_bucket_scan(const Plan &p, const QueryDev &q, const void *tuples, int64_t n, int grid,
                               cudaStream_t st);
cudaError_t launch_bucket_windows(const Plan &p, const QueryDev &q, const SlotDev &s, int nsm, cudaStream_t st);
// k_winblock.cu
bool wb_usable(const Plan &p);
bool wb_prepass(const Plan &p);   // k_win_block_reg: k_wb_rows runs first
cudaError_t wb_set_attributes(const Plan &p);
int wb_blocks_per_sm(const Plan &p);
cudaError_t launch_windows_block(const Plan &p, const QueryDev &q, const SlotDev &s, int grid, cudaStream_t st);
// k_winwide.cu
bool ww_usable(const Plan &p);
cudaError_t ww_set_attributes(const Plan &p);
int ww_blocks_per_sm(const Plan &p);
cudaError_t launch_windows_wide(const Plan &p, const QueryDev &q, const SlotDev &s, int grid, cudaStream_t st);
// k_select.cu
void *sel_kernel(const Plan &p);
int sel_smem_bytes();
cudaError_t launch_select(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples, int grid,
                          cudaStream_t st);
}  // namespace sb
