// sw_menu.cu — table of compiled configurations (see sw_menu.h).
#include "sw_menu.h"

namespace swb {

namespace {
struct Entry {
  KernelConfig cfg;
  cudaError_t (*launch)(const SearchParams&, int, int, cudaStream_t);
  cudaError_t (*configure)(int, int*);
};
#define E(I, LANE, G, RS, RL) {{LANE, G, RS, RL}, launch_menu_##I, configure_menu_##I}
const Entry kMenu[SWB_MENU_SIZE] = {
    E(0, 0, 4, 36, 8),   E(1, 0, 8, 24, 8),    E(2, 0, 8, 32, 8),    E(3, 0, 16, 24, 12),
    E(4, 0, 16, 32, 16), E(5, 0, 32, 24, 24),  E(6, 0, 32, 32, 32),  E(7, 0, 32, 20, 20),
    E(8, 0, 32, 16, 16), E(9, 0, 4, 16, 4),    E(10, 0, 1, 16, 4),   E(11, 1, 32, 16, 16),
};
#undef E

int find(const KernelConfig& c) {
  for (int i = 0; i < SWB_MENU_SIZE; ++i) {
    const KernelConfig& k = kMenu[i].cfg;
    if (k.lane == c.lane && k.G == c.G && k.Rs == c.Rs && k.Rl == c.Rl) return i;
  }
  return -1;
}
}  // namespace

int menu_size() { return SWB_MENU_SIZE; }
KernelConfig menu_entry(int i) { return kMenu[i].cfg; }
KernelConfig recompute_config() { return kMenu[SWB_RECOMPUTE_INDEX].cfg; }

cudaError_t launch_search(const KernelConfig& cfg, const SearchParams& p, int grid, int smem_bytes,
                          cudaStream_t st) {
  const int i = find(cfg);
  if (i < 0) return cudaErrorInvalidValue;
  return kMenu[i].launch(p, grid, smem_bytes, st);
}

cudaError_t configure_kernel(const KernelConfig& cfg, int smem_bytes, int* blocks_per_sm) {
  const int i = find(cfg);
  if (i < 0) return cudaErrorInvalidValue;
  return kMenu[i].configure(smem_bytes, blocks_per_sm);
}

}  // namespace swb
