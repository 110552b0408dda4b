// decode_kernel<B> instantiation(s) for B = 3, 4
#include "decode_impl.cuh"

MX_DECODE_INSTANTIATE(3)
MX_DECODE_INSTANTIATE(4)
