// Menu entry 0: LaneS16x2, G=4 lanes x R_s=36 rows (group mode), 32 lanes x R_l=8 rows (team mode).
#include "sw_engine.cuh"
#include "sw_menu.h"
namespace swb {
cudaError_t launch_menu_0(const SearchParams& p, int grid, int smem, cudaStream_t st) {
  return launch_search_t<LaneS16x2, 4, 36, 8>(p, grid, smem, st);
}
cudaError_t configure_menu_0(int smem, int* bps) { return configure_t<LaneS16x2, 4, 36, 8>(smem, bps); }
}  // namespace swb
