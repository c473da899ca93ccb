// tc_sage.cu — placeholder until the tcgen05 kernels land.
#include "tc_sage.cuh"

namespace buffalo {

int64_t tc_packed_bytes(int64_t d_in, int64_t d_out) {
  return R(round_up(d_out, 16) * 2 * round_up(d_in, 64) * 2);
}
buffalo_status tc_pack_weights(const float*, int, int, void*, cudaStream_t) { return BUFFALO_OK; }
bool tc_fwd_supported(const FwdArgs&) { return false; }
buffalo_status tc_sage_fwd(const FwdArgs&, cudaStream_t) { return BUFFALO_ERR_UNSUPPORTED; }

}  // namespace buffalo
