// regular.cu — placeholder until the regular tree lands.
#include "hbt_internal.cuh"
namespace hbt {
int regular_build(hbt_tree*, const void*, const void*, uint64_t, cudaStream_t) { set_error("regular tree not built yet"); return HBT_EUNSUPPORTED; }
int regular_search(const hbt_tree*, const void*, uint64_t, uint64_t*, void*, cudaStream_t) { return HBT_EUNSUPPORTED; }
int regular_update(hbt_tree*, const hbt_batch*, cudaStream_t) { return HBT_EUNSUPPORTED; }
void regular_free(hbt_tree*) {}
uint32_t regular_smem_levels(const hbt_tree*, uint32_t) { return 0; }
}
