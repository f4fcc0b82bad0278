// sf_frag_r64.cu - frag3 kernel instantiations for rank R = 64 (see sf_frag3.cuh).
#include "sf_frag3.cuh"

namespace sf {
SF_DEFINE_FRAG3_R(64)
}  // namespace sf
