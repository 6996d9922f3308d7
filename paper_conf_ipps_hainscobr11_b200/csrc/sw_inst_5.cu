// Menu entry 5: LaneS16x2, G=32 lanes x R_s=24 rows (group mode), 32 lanes x R_l=24 rows (team mode).
#include "sw_engine.cuh"
#include "sw_menu.h"
namespace swb {
cudaError_t launch_menu_5(const SearchParams& p, int grid, int smem, cudaStream_t st) {
  return launch_search_t<LaneS16x2, 32, 24, 24>(p, grid, smem, st);
}
cudaError_t configure_menu_5(int smem, int* bps) { return configure_t<LaneS16x2, 32, 24, 24>(smem, bps); }
}  // namespace swb
