// Menu entry 6: LaneS16x2, G=32 lanes x R_s=32 rows (group mode), 32 lanes x R_l=32 rows (team mode).
#include "sw_engine.cuh"
#include "sw_menu.h"
namespace swb {
cudaError_t launch_menu_6(const SearchParams& p, int grid, int smem, cudaStream_t st) {
  return launch_search_t<LaneS16x2, 32, 32, 32>(p, grid, smem, st);
}
cudaError_t configure_menu_6(int smem, int* bps) { return configure_t<LaneS16x2, 32, 32, 32>(smem, bps); }
}  // namespace swb
