// sf_frag_r16.cu - fragment-kernel instantiations for rank R = 16 (see sf_frag.cuh).
#include "sf_frag.cuh"
#include "sf_frag3.cuh"

namespace sf {
SF_DEFINE_FRAG_R(16)
SF_DEFINE_FRAG3_R(16)
}  // namespace sf
