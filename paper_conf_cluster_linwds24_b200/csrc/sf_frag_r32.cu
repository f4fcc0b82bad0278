// sf_frag_r32.cu - frag3 kernel instantiations for rank R = 32 (see sf_frag3.cuh).
#include "sf_frag3.cuh"

namespace sf {
SF_DEFINE_FRAG3_R(32)
}  // namespace sf
