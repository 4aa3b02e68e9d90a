// tri_tiled.cu -- warp-per-instance triangulation with 4x4 register tiles
// (placeholder until the blocked kernel lands; resolve_tri_variant never
// selects it while tiled_supported() returns 0).
#include "common.cuh"

namespace bo {

int tiled_supported(int64_t n) {
    (void)n;
    return 0;
}

int launch_tri_tiled(const void *, void *, int64_t, int64_t, int, int, cudaStream_t) {
    return fail(BO_EUNSUPPORTED, "triangulation TILED not built");
}

}  // namespace bo
