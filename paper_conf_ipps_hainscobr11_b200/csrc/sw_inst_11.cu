// Menu entry 11: LaneS32, G=32 lanes x R_s=16 rows (group mode), 32 lanes x R_l=16 rows (team mode).
#include "sw_engine.cuh"
#include "sw_menu.h"
namespace swb {
cudaError_t launch_menu_11(const SearchParams& p, int grid, int smem, cudaStream_t st) {
  return launch_search_t<LaneS32, 32, 16, 16>(p, grid, smem, st);
}
cudaError_t configure_menu_11(int smem, int* bps) { return configure_t<LaneS32, 32, 16, 16>(smem, bps); }
}  // namespace swb
