// decode_kernel<B> instantiation(s) for B = 1
#include "decode_impl.cuh"

MX_DECODE_INSTANTIATE(1)
