// Menu entry 10: LaneS16x2, G=1 lanes x R_s=16 rows (group mode), 32 lanes x R_l=4 rows (team mode).
#include "sw_engine.cuh"
#include "sw_menu.h"
namespace swb {
cudaError_t launch_menu_10(const SearchParams& p, int grid, int smem, cudaStream_t st) {
  return launch_search_t<LaneS16x2, 1, 16, 4>(p, grid, smem, st);
}
cudaError_t configure_menu_10(int smem, int* bps) { return configure_t<LaneS16x2, 1, 16, 4>(smem, bps); }
}  // namespace swb
