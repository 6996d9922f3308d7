// sw_menu.h — the compiled kernel configurations (lane, G, R_s, R_l); one sw_inst_<i>.cu per
// entry so nvcc builds them in parallel.  Keep in sync with menu_table in sw_menu.cu.
#pragma once
#include "sw_internal.h"
namespace swb {
#define SWB_MENU_SIZE 12
#define SWB_RECOMPUTE_INDEX 11
#define SWB_DECL(I)                                                                          \
  cudaError_t launch_menu_##I(const SearchParams& p, int grid, int smem, cudaStream_t st); \
  cudaError_t configure_menu_##I(int smem, int* bps);
SWB_DECL(0) SWB_DECL(1) SWB_DECL(2) SWB_DECL(3) SWB_DECL(4) SWB_DECL(5)
SWB_DECL(6) SWB_DECL(7) SWB_DECL(8) SWB_DECL(9) SWB_DECL(10) SWB_DECL(11)
#undef SWB_DECL
}  // namespace swb
