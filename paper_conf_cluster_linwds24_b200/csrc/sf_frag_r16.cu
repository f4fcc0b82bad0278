// sf_frag_r16.cu - frag3 kernel instantiations for rank R = 16 (see sf_frag3.cuh).
#include "sf_frag3.cuh"

namespace sf {
SF_DEFINE_FRAG3_R(16)
}  // namespace sf
