// kernels.h -- host-side launchers of the sm_100a kernels (kernels.cu).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "plan.h"

namespace sb {

struct SlotDev {
  unsigned char *rows;      // aggregation columns / IStream rows
  void *hdr;                // saber_win_hdr[win_cap]
  int64_t *counts;          // per (window, slab) row counts → offsets
  SlotMeta *meta;
  State *wst;               // overlap: State snapshot the slot's window kernels run on
  int *ticket;              // overlap: the slot's work-ticket counter
};

struct QueryDev {
  State *st;
  uint64_t *table;          // pane ring: R slots × slot_words
  uint64_t *vh_pre;         // van Herk block-prefix arrays (DENSE/GLOBAL), same geometry
  uint64_t *vh_suf;         // van Herk block-suffix arrays
  uint64_t *clist;          // slab mode: per pane slot, entries bucketed by key range
  int32_t *coff;            // slab mode: per pane slot, S+1 bucket offsets
  unsigned char *sel_stage; // σ/π: per-CTA compacted rows before the final placement
  int64_t *cta_cnt;         // σ/π: rows per CTA
  int64_t *pane_ts;         // R
  uint64_t *tile_status;    // IStream look-back
  int64_t tile_status_cap;
  unsigned char *carry[2];  // IStream raw tail
  int64_t carry_cap;        // tuples
  int *tile_ctr;
  // σ/π (IStream) window headers: per closed window the (CTA, CTA-relative row
  // rank) of its first new tuple, each CTA's global row base, and τ at window
  // starts j·l (count windows; ring of ts_mask+1 entries indexed by j)
  int64_t *ihdr_tmp;
  int64_t *cta_base;
  int64_t *win_ts;
  int64_t ts_mask;
  unsigned char *bkt;       // bucket mode: [R][S][g] u16 key offsets, then [R][S][nf][g] f32 values
};

// one task of an aggregation (RStream) query
cudaError_t launch_agg_task(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples,
                            int64_t n, int final_, int has_wm, int64_t wm, int emit_on_finish,
                            int p1_grid, int p2_grid, int win_chunk, cudaStream_t st,
                            cudaEvent_t *evs /* 3 events or nullptr */, int *launches);
// one task of a σ/π (IStream) query
cudaError_t launch_select_task(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples,
                               int64_t n, int final_, int has_wm, int64_t wm, int emit_on_finish,
                               int sel_grid, cudaStream_t st, cudaEvent_t *evs, int *launches);
// overlap plans: the task's scan on `cs`, its window phase on `ws` (after
// `scan_done`, which the caller's next tasks order against)
cudaError_t launch_agg_task_overlap(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples,
                                    int64_t n, int final_, int has_wm, int64_t wm, int emit_on_finish,
                                    int p1_grid, int p2_grid, cudaStream_t cs, cudaStream_t ws,
                                    cudaEvent_t scan_done, cudaEvent_t *evs, int *launches);
cudaError_t launch_init_state(const Plan &p, const QueryDev &q, int64_t base_index, int64_t epoch0, cudaStream_t st);
cudaError_t launch_partition_plan(int ts_word, int tuple_words, int win_kind, int64_t s, int64_t l,
                                  int64_t T0, const void *tuples, int64_t begin, int64_t n,
                                  int64_t *dev_out2, cudaStream_t st);
// occupancy helpers
int p1_smem_bytes(const Plan &p);
int p1_blocks_per_sm(const Plan &p);
int p2_blocks_per_sm(const Plan &p);
int sel_blocks_per_sm(const Plan &p);
int bk_scan_blocks_per_sm(const Plan &p);
bool wb_usable(const Plan &p);
bool wb_prepass(const Plan &p);
bool ww_usable(const Plan &p);
int ww_blocks_per_sm(const Plan &p);
bool p1_is_cnt(const Plan &p);
bool p1_cnt_fx_plan(const Plan &p);
int wb_blocks_per_sm(const Plan &p);
cudaError_t set_kernel_attributes(const Plan &p);

}  // namespace sb
