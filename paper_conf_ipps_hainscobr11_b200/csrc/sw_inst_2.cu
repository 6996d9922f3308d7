// Menu entry 2: LaneS16x2, G=8 lanes x R_s=32 rows (group mode), 32 lanes x R_l=8 rows (team mode).
#include "sw_engine.cuh"
#include "sw_menu.h"
namespace swb {
cudaError_t launch_menu_2(const SearchParams& p, int grid, int smem, cudaStream_t st) {
  return launch_search_t<LaneS16x2, 8, 32, 8>(p, grid, smem, st);
}
cudaError_t configure_menu_2(int smem, int* bps) { return configure_t<LaneS16x2, 8, 32, 8>(smem, bps); }
}  // namespace swb
