// decode_kernel<B> instantiation(s) for B = 2
#include "decode_impl.cuh"

MX_DECODE_INSTANTIATE(2)
