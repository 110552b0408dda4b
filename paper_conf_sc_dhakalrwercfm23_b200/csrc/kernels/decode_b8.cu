// decode_kernel<B> instantiation for B = 8
#include "decode_impl.cuh"

MX_DECODE_INSTANTIATE(8)
