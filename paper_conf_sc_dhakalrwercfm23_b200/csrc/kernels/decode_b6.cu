// decode_kernel<B> instantiation for B = 6
#include "decode_impl.cuh"

MX_DECODE_INSTANTIATE(6)
