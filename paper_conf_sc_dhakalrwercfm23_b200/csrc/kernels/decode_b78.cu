// decode_kernel<B> instantiation(s) for B = 7, 8
#include "decode_impl.cuh"

MX_DECODE_INSTANTIATE(7)
MX_DECODE_INSTANTIATE(8)
