// sf_frag_r16.cu - fragment-kernel instantiations for rank R = 16 (see sf_frag.cuh).
#include "sf_frag.cuh"

namespace sf {
SF_DEFINE_FRAG_R(16)
}  // namespace sf
