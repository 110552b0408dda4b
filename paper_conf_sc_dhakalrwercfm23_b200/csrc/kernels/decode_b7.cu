// decode_kernel<B> instantiation for B = 7
#include "decode_impl.cuh"

MX_DECODE_INSTANTIATE(7)
