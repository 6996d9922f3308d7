// Menu entry 7: LaneS16x2, G=32 lanes x R_s=20 rows (group mode), 32 lanes x R_l=20 rows (team mode).
#include "sw_engine.cuh"
#include "sw_menu.h"
namespace swb {
cudaError_t launch_menu_7(const SearchParams& p, int grid, int smem, cudaStream_t st) {
  return launch_search_t<LaneS16x2, 32, 20, 20>(p, grid, smem, st);
}
cudaError_t configure_menu_7(int smem, int* bps) { return configure_t<LaneS16x2, 32, 20, 20>(smem, bps); }
}  // namespace swb
