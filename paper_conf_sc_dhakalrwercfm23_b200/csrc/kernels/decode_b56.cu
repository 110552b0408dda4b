// decode_kernel<B> instantiation(s) for B = 5, 6
#include "decode_impl.cuh"

MX_DECODE_INSTANTIATE(5)
MX_DECODE_INSTANTIATE(6)
