// launch_nch1.cu — instantiates the search kernels for rows of up to 128 floats.
#include "launch.cuh"

namespace song {
template int launch_m<1>(song_index* ix, const SearchArgs& a, int metric, int vk, int qr,
                          int warps, int bps, int sms, cudaStream_t st);
}  // namespace song
